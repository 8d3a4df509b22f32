# A/B of prebuilt library variants: LIBS="libmgj_base.so libmgj.so ..." (in the package dir),
# ARGS = extra bench args; each variant runs twice, interleaved.
cd $GRAFT_REPO_ROOT
for rep in 1 2; do
for lib in $LIBS; do
  MGJ_LIB=$GRAFT_REPO_ROOT/paper_conf_sigmod_paullhl21_b200/$lib timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e $ARGS > gpurun_out/ab.json 2>gpurun_out/ab.err
  python - "$lib" <<'PY'
import json, sys
try:
    d = json.load(open("gpurun_out/ab.json"))
    print(sys.argv[1], "ms %.3f" % d["ms_per_step"], "ok", d["correct"], " ".join("%s=%.3f" % (k, v["ms"]) for k, v in d["phases"].items()))
except Exception as e:
    print(sys.argv[1], "FAILED", e, open("gpurun_out/ab.err").read()[-300:])
PY
done
done
