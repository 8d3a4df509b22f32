cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/cfg
for mode in p2p nccl; do
  MGJ_SYMM_ARENA=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29521 bench.py --gpus 1 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --shuffle $mode > gpurun_out/cfg/torchrun_$mode.json 2> gpurun_out/cfg/torchrun_$mode.err
  python -c "
import json; d=json.load(open('gpurun_out/cfg/torchrun_$mode.json')); print('torchrun_$mode', round(d['ms_per_step'],3), round(d['value']/1e9,1), d['correct'], {k:round(v['ms'],3) for k,v in d['phases'].items()})" || tail -3 gpurun_out/cfg/torchrun_$mode.err
done
