# ncu full capture (source-level) of one kernel: KREG (regex), ARGS (bench args)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"${KREG:-k_scatter}" -s ${SKIP:-2} -c 1 \
    -o gpurun_out/prof_${TAG:-scatter} -f python bench.py --steps 1 --warmup 1 --profile $ARGS > gpurun_out/prof_${TAG:-scatter}.log 2>&1
echo "full capture rc=$?"
tail -3 gpurun_out/prof_${TAG:-scatter}.log
