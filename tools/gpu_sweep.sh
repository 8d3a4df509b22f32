cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
for args in $SWEEP; do
  a=$(echo $args | tr ',' ' ')
  timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e $a > gpurun_out/sweep.json 2>gpurun_out/sweep.err
  python - "$a" <<'PY'
import json, sys
try:
    d = json.load(open("gpurun_out/sweep.json"))
    ph = d["phases"]
    print(sys.argv[1], "ms %.2f" % d["ms_per_step"], "ok", d["correct"], " ".join("%s=%.2f" % (k, v["ms"]) for k, v in ph.items()), "B2=%d" % d["config"]["radix_bits_local"])
except Exception as e:
    print(sys.argv[1], "FAILED", e, open("gpurun_out/sweep.err").read()[-300:])
PY
done
