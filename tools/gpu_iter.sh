# GPU iteration: build, GPU tests, bench, launch list.
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -q --timeout 120 -rf -x ${PYTEST_ARGS} 2>&1 | tail -25
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
tail -3 gpurun_out/bench.err
python - <<'PY'
import json
try:
    d = json.load(open("gpurun_out/bench.json"))
    print("value %.3e ms/step %.3f correct %s" % (d["value"], d["ms_per_step"], d["correct"]))
    for k, v in d["phases"].items(): print(k, v)
except Exception as e:
    print("no bench json", e)
PY
if [ -n "$LAUNCHES" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 1 --profile > gpurun_out/launch_bench.log 2>&1; echo "launch list rc=$?"
fi
if [ -n "$FULL" ]; then
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"$FULL" -s 4 -c 4 \
    -o gpurun_out/prof -f python bench.py --steps 1 --warmup 1 --profile > gpurun_out/prof.log 2>&1
echo "full capture rc=$?"
fi
