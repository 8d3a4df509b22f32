# Materialisation / wide / zipf bench lines (short).
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -q --timeout 120 -rf -x 2>&1 | tail -3
for cfg in "mat --log2-per-gpu 29 --materialize" "wide --workload wide --log2-per-gpu 28 --materialize" "widenm --workload wide --log2-per-gpu 28" "zipf1 --workload zipf --z 1.0 --log2-per-gpu 29" ${EXTRA_CFG}; do
  set -- $cfg; name=$1; shift
  timeout 600 python bench.py "$@" --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_$name.json 2>gpurun_out/bench_$name.err
  python -c "
import json
try:
  d=json.load(open('gpurun_out/bench_$name.json')); print('$name', 'ms %.2f'%d['ms_per_step'], 'val %.3e'%d['value'], 'ok' if d['correct'] else 'CHECK', {k:round(v['ms'],2) for k,v in d['phases'].items()})
except Exception as e: print('$name', 'FAILED', e, open('gpurun_out/bench_$name.err').read()[-400:])
"
done
