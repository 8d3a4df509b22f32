# Round-2 baseline: build, GPU tests, bench.
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -rf 2>&1 | tail -15
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_base.json 2> gpurun_out/bench_base.err; echo "bench rc=$?"
tail -c 1500 gpurun_out/bench_base.json
