# Bench lines for named configurations: CFGS="name:args;name:args" (args space-separated).
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
[ -n "$TESTS" ] && timeout 900 python -m pytest tests -m gpu -q --timeout 120 -rf -x 2>&1 | tail -3
IFS=';' read -ra LIST <<< "$CFGS"
for item in "${LIST[@]}"; do
  name="${item%%:*}"; args="${item#*:}"
  timeout 600 python bench.py $args --steps ${STEPS:-5} --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_$name.json 2>gpurun_out/bench_$name.err
  python -c "
import json
try:
  d=json.load(open('gpurun_out/bench_$name.json')); print('$name', 'ms %.2f'%d['ms_per_step'], 'val %.3e'%d['value'], 'ok' if d['correct'] else 'CHECK', {k:round(v['ms'],2) for k,v in d['phases'].items()}, 'B2', d['config'].get('radix_bits_local'))
except Exception as e: print('$name', 'FAILED', e, open('gpurun_out/bench_$name.err').read()[-400:])
"
done
