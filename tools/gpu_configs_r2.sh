# Every BASELINE configuration that fits one GPU, timed like the headline (W=3, K=10), plus variants.
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
mkdir -p gpurun_out/cfg
run() {  # name, args
  timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e $2 > gpurun_out/cfg/$1.json 2> gpurun_out/cfg/$1.err
  python - "$1" <<'PY'
import json, sys
n = sys.argv[1]
try:
    d = json.load(open(f"gpurun_out/cfg/{n}.json"))
    print(f"{n:22s} {d['ms_per_step']:8.3f} ms {d['value']/1e9:7.1f} G/s correct={d['correct']} " +
          " ".join(f"{k}={v['ms']:.3f}" for k, v in d['phases'].items()) + f" B2={d['config']['radix_bits_local']}")
except Exception as e:
    print(n, "FAILED", e, open(f"gpurun_out/cfg/{n}.err").read()[-400:])
PY
}
run m2 ""
run m2_mat "--materialize"
run m4_z1 "--workload zipf --z 1"
run m4_z05 "--workload zipf --z 0.5"
run m5_mat "--workload wide --log2-per-gpu 28 --materialize"
run m5 "--workload wide --log2-per-gpu 28"
run m3_n2size "--log2-per-gpu 30"
run m2_b1_7 "--radix-bits-global 7"
run m2_compress "--compress"
run m2_overlap "--overlap on"
run m2_stream "--overlap stream"
run m2_b1_7_mat "--radix-bits-global 7 --materialize"
for k in 24 26 28; do run size_2p$k "--log2-per-gpu $k"; done
run m2_b1_9 "--radix-bits-global 9"
run m2_b2_6 "--radix-bits-local 6"
run m2_b2_8 "--radix-bits-local 8"
