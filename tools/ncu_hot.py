"""Summarise an ncu report: top SASS instructions by warp-stall samples per kernel.
usage: python tools/ncu_hot.py report.ncu-rep kernel_regex [N]"""
import csv, io, subprocess, sys
rep, kern = sys.argv[1], sys.argv[2]
N = int(sys.argv[3]) if len(sys.argv) > 3 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--kernel-name", f"regex:{kern}",
                      "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
data = [r for r in rows[2:] if len(r) == len(hdr) and r != hdr and r[0] != "Kernel Name"]
ci = {h: i for i, h in enumerate(hdr)}
def num(x):
    try: return int(x)
    except ValueError: return 0
stall_cols = [h for h in hdr if h.startswith("stall_")]
tot = sum(num(r[ci["Warp Stall Sampling (All Samples)"]]) for r in data)
agg = {h: sum(num(r[ci[h]]) for r in data) for h in stall_cols}
print(f"total samples {tot}; stall breakdown:", ", ".join(f"{k[6:]}={v*100/tot:.1f}%" for k, v in sorted(agg.items(), key=lambda x: -x[1])[:10] if v))
ins = sum(num(r[ci["Instructions Executed"]]) for r in data)
print(f"warp instructions executed {ins}")
top = sorted(data, key=lambda r: -num(r[ci["Warp Stall Sampling (All Samples)"]]))[:N]
for r in top:
    s = num(r[ci["Warp Stall Sampling (All Samples)"]])
    st = sorted(((num(r[ci[h]]), h[6:]) for h in stall_cols), reverse=True)[:2]
    print(f"{s*100/tot:5.1f}% {r[ci['Address']][-5:]} {r[ci['Source']].strip()[:60]:60s} ex={r[ci['Instructions Executed']]:>10s} " +
          " ".join(f"{n}={v}" for v, n in st if v))
