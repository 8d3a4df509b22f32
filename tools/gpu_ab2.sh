# tests subset + A/B of library variants (LIBS) for the default and extra configs (ARGS_LIST, ';'-separated)
cd $GRAFT_REPO_ROOT
if [ -n "$PYTEST_K" ]; then timeout 1200 python -m pytest tests -m gpu -q --timeout 600 -rf -k "$PYTEST_K" 2>&1 | tail -6; fi
IFS=';' read -ra AL <<< "${ARGS_LIST:- }"
for args in "${AL[@]}"; do
for rep in 1 2; do
for lib in $LIBS; do
  MGJ_LIB=$GRAFT_REPO_ROOT/paper_conf_sigmod_paullhl21_b200/$lib timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e $args > gpurun_out/ab.json 2>gpurun_out/ab.err
  python - "$lib" "$args" <<'PY'
import json, sys
try:
    d = json.load(open("gpurun_out/ab.json"))
    print(sys.argv[1], sys.argv[2], "ms %.3f" % d["ms_per_step"], "ok", d["correct"], " ".join("%s=%.3f" % (k, v["ms"]) for k, v in d["phases"].items()))
except Exception as e:
    print(sys.argv[1], "FAILED", e, open("gpurun_out/ab.err").read()[-300:])
PY
done
done
done
