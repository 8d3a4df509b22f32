cd $GRAFT_REPO_ROOT
for args in "--overlap stream --compress" "--overlap stream --workload zipf --z 1" "--overlap stream --workload wide --log2-per-gpu 28" "--overlap stream --materialize"; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e $args 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$args', round(d['ms_per_step'],3), d['correct'], {k: round(v['ms'],3) for k,v in d['phases'].items()})"
done
MGJ_SYMM_ARENA=1 timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29655 bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --overlap stream 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('torchrun symm stream', round(d['ms_per_step'],3), d['correct'])"
