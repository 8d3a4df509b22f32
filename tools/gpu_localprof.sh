# Profile k_local for several cluster sizes (CLS="1 2"), print hot SASS lines.
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
for cl in ${CLS:-1 2}; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --local-cluster $cl > gpurun_out/lb$cl.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/lb$cl.json')); print('CL=$cl grid', d['config']['local_grid'], 'local %.2f probe %.2f' % (d['phases']['local_part']['ms'], d['phases']['probe']['ms']))"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_local' -s 2 -c 1 \
    -o gpurun_out/lprof$cl -f python bench.py --steps 1 --warmup 1 --profile --local-cluster $cl > gpurun_out/lprof$cl.log 2>&1
  echo "capture rc=$?"
  python tools/ncu_hot.py gpurun_out/lprof$cl.ncu-rep k_local 25
done
