# Round-2 evidence: launch list (ncu, serialised) + full captures of the hot kernels + bench JSON
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv \
    python bench.py --steps 2 --warmup 1 --profile > gpurun_out/launch_bench_${TAG}.log 2>&1
echo "launch list rc=$?"
python tools/launch_table.py gpurun_out/launches_${TAG}.csv ${TAG} | head -20
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:'k_(hist|scatter|local|probe)' -s 5 -c 4 \
    -o gpurun_out/full_${TAG} -f python bench.py --steps 1 --warmup 1 --profile > gpurun_out/full_${TAG}.log 2>&1
echo "full capture rc=$?"
