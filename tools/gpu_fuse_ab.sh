# A/B of the fused local pass + probe experiment (tools/experiments/fused_local_probe.patch applied) against the sequential path, M2 at N=1
cd $GRAFT_REPO_ROOT
if [ -n "$RUN_TESTS" ]; then timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 2>&1 | tail -4 > gpurun_out/pt_fuse.txt; fi
for rep in 1 2; do
for cfg in ${CFGS:-off: auto:40 auto:49}; do
  mode=${cfg%%:*}; ps=${cfg#*:}
  if [ -n "$ps" ]; then export MGJ_FUSE_PSMS=$ps; else unset MGJ_FUSE_PSMS; fi
  timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --probe-fuse $mode $ARGS > gpurun_out/ab.json 2>gpurun_out/ab.err
  python - "$cfg" <<'PY'
import json, sys
try:
    d = json.load(open("gpurun_out/ab.json"))
    print(sys.argv[1], "ms %.3f" % d["ms_per_step"], "ok", d["correct"], " ".join("%s=%.3f" % (k, v["ms"]) for k, v in d["phases"].items()))
    if d.get("timeline_us"): print("   ", d["timeline_us"])
except Exception as e:
    print(sys.argv[1], "FAILED", e, open("gpurun_out/ab.err").read()[-500:])
PY
done; done
