# One ncu --set full capture of kernels matching $K (regex), 1 launch after skipping $S.
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
timeout 800 ncu --set full --clock-control none --import-source on -k regex:"$K" -s ${S:-1} -c ${C:-1} \
  -o gpurun_out/prof1 -f python bench.py --steps 1 --warmup 1 --profile --no-cpu-baseline --no-e2e ${ARGS} > gpurun_out/prof.log 2>&1
echo rc=$?
