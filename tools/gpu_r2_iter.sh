# Round-2 iteration: build, GPU tests (PYTEST_ARGS), smoke, bench.
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 1800 python -m pytest tests -m gpu -q --timeout 600 -rf ${PYTEST_ARGS} 2>&1 | tail -25
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 600 python bench.py --steps 10 --warmup 3 ${BENCH_ARGS} > gpurun_out/bench_iter.json 2> gpurun_out/bench_iter.err; echo "bench rc=$?"
tail -3 gpurun_out/bench_iter.err
python - <<'PY'
import json
try:
    d = json.load(open("gpurun_out/bench_iter.json"))
    print("value %.4e ms/step %.3f correct %s digest %s" % (d["value"], d["ms_per_step"], d["correct"], d.get("pair_digest")))
    for k, v in d["phases"].items(): print(k, round(v["ms"], 3), round(v.get("frac_hbm", 0), 3))
    print("launches", d["gpu_launches"], "e2e", d["e2e"] and d["e2e"]["value"])
except Exception as e:
    print("no bench json", e)
PY
