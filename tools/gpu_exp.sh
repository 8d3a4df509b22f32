cd $GRAFT_REPO_ROOT
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -Xcompiler -fPIC -shared -I include $EXTRA -o paper_conf_sigmod_paullhl21_b200/libmgj.so paper_conf_sigmod_paullhl21_b200/csrc/mgj.cu
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e $ARGS > gpurun_out/exp.json 2>gpurun_out/exp.err
python -c "
import json; d=json.load(open('gpurun_out/exp.json')); print('ms %.2f'%d['ms_per_step'], {k:round(v['ms'],2) for k,v in d['phases'].items()})" || tail -3 gpurun_out/exp.err
