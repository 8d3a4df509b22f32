# Full measurement session: tests, bench (all keys), reference arm, ncu launch list + full capture.
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 1200 python -m pytest tests -m gpu -q --timeout 300 -rf 2>&1 | tail -6
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference --steps 5 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo "ref rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 1 --profile > gpurun_out/launch_bench.log 2>&1; echo "launch list rc=$?"
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:'k_(hist|scatter|local|probe)' -s 6 -c 6 \
    -o gpurun_out/prof -f python bench.py --steps 1 --warmup 1 --profile > gpurun_out/prof.log 2>&1; echo "full rc=$?"
cat gpurun_out/bench_full.json | head -c 600; echo
cat gpurun_out/bench_ref.json | head -c 300; echo
