# Round-2 evidence: full GPU tests, smoke, bench (default + overlap/trace + reference arm),
# ncu launch list and full captures of the hot kernels.  Outputs in gpurun_out/${TAG}/.
cd $GRAFT_REPO_ROOT
O=gpurun_out/${TAG:-r2ev}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 2400 python -m pytest tests -m gpu -q --timeout 900 -rf > $O/pytest_gpu.txt 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.txt
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference > $O/bench_reference.json 2> $O/bench_reference.err; echo "reference rc=$?"
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --overlap on --trace > $O/bench_overlap_trace.json 2>/dev/null; echo "overlap rc=$?"
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --overlap stream --trace > $O/bench_stream_trace.json 2>/dev/null; echo "stream rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv \
    python bench.py --steps 2 --warmup 1 --profile > $O/launch_bench.log 2>&1; echo "launch list rc=$?"
timeout 1800 ncu --set full --clock-control none --import-source on --kernel-name-base function \
    -k regex:'^k_(hist|scatter|local|probe)$' -s 4 -c 4 -o $O/full -f python bench.py --steps 1 --warmup 1 --profile > $O/full.log 2>&1
echo "full capture rc=$?"
python - <<PY
import json
d = json.load(open("$O/bench.json"))
print("bench", round(d["ms_per_step"], 3), "ms", "%.4g" % d["value"], d["correct"], {k: round(v["ms"], 3) for k, v in d["phases"].items()})
print("roofline", d["roofline"]["kernel"], round(d["roofline"]["frac"], 3), "clocks", d["clocks"])
PY
