cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python tools/sanitize.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; tail -4 gpurun_out/sanitize_$tool.log
done
timeout 600 python bench.py --workload zipf --z 1.0 --log2-per-gpu 29 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_zipf1.json 2>gpurun_out/bench_zipf1.err; echo "zipf1 rc=$?"
timeout 600 python bench.py --workload zipf --z 0.5 --log2-per-gpu 29 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_zipf05.json 2>gpurun_out/bench_zipf05.err; echo "zipf05 rc=$?"
timeout 600 python bench.py --workload wide --log2-per-gpu 28 --materialize --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_wide.json 2>gpurun_out/bench_wide.err; echo "wide rc=$?"
timeout 600 python bench.py --log2-per-gpu 29 --materialize --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_mat.json 2>gpurun_out/bench_mat.err; echo "mat rc=$?"
for f in zipf1 zipf05 wide mat; do python -c "
import json,sys
try:
  d=json.load(open('gpurun_out/bench_$f.json')); print('$f', 'ms %.2f'%d['ms_per_step'], 'val %.3e'%d['value'], 'status ok' if d['correct'] else 'check', d['match_count'], d['checksum'], {k:round(v['ms'],2) for k,v in d['phases'].items()})
except Exception as e: print('$f', 'FAILED', e, open('gpurun_out/bench_$f.err').read()[-400:])
"; done
