# Round-1 evidence refresh: size sweep (NEXT-4), B1 sweep, torchrun symmetric-memory N=1 (both shuffle modes), extra configs.
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
SWEEP="--log2-per-gpu,22 --log2-per-gpu,24 --log2-per-gpu,26 --log2-per-gpu,27 --log2-per-gpu,28 --log2-per-gpu,29 --log2-per-gpu,30 --radix-bits-global,9 --radix-bits-global,11 --radix-bits-local,6 --radix-bits-local,8" bash tools/gpu_sweep.sh 2>&1 | grep -v "^\[" > gpurun_out/sweep_r1b.txt
cat gpurun_out/sweep_r1b.txt
for mode in p2p nccl; do
  MGJ_SYMM_ARENA=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 1 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --shuffle $mode > gpurun_out/torchrun_$mode.json 2> gpurun_out/torchrun_$mode.err
  echo "torchrun $mode rc=$?"; head -c 400 gpurun_out/torchrun_$mode.json; echo
done
timeout 600 python bench.py --workload zipf --z 0.5 --log2-per-gpu 29 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_zipf05.json 2>gpurun_out/bench_zipf05.err; echo "zipf05 rc=$?"
timeout 600 python bench.py --scaling strong --log2-total 30 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_strong30.json 2>gpurun_out/bench_strong30.err; echo "strong rc=$?"
