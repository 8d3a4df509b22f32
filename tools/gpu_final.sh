# End-of-round evidence: torchrun symmetric-memory N=1 (both shuffle modes), sanitizers, per-config benches.
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
for mode in p2p nccl; do
  MGJ_SYMM_ARENA=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 1 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --shuffle $mode > gpurun_out/torchrun_$mode.json 2> gpurun_out/torchrun_$mode.err
  echo "torchrun $mode rc=$?"
done
bash tools/gpu_extra.sh 2>&1 | grep -v " rc=0$"
timeout 600 python bench.py --scaling strong --log2-total 30 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_strong30.json 2>gpurun_out/bench_strong30.err; echo "strong rc=$?"
timeout 600 python bench.py --radix-bits-global 7 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_n8emul.json 2>gpurun_out/bench_n8emul.err; echo "n8emul rc=$?"
for f in torchrun_p2p torchrun_nccl bench_strong30 bench_n8emul; do python -c "
import json
d=json.load(open('gpurun_out/$f.json')); print('$f', 'ms %.2f'%d['ms_per_step'], 'G/s %.1f'%(d['value']/1e9), d['correct'], {k:round(v['ms'],2) for k,v in d['phases'].items()})"; done
