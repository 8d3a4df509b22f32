"""Summarise ncu artefacts into markdown for profiles/.
usage: python tools/ncu_summary.py <launches.csv> <full.ncu-rep> <title>"""
import csv, io, subprocess, sys

def launches(path):
    rows = list(csv.reader(open(path)))
    for i, r in enumerate(rows):
        if "Kernel Name" in r:
            h = r; st = i + 1; break
    ki, vi, mi = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Name")
    agg = {}
    for r in rows[st:]:
        if len(r) < len(h) or r[mi] != "gpu__time_duration.sum":
            continue
        k = r[ki].split("(")[0].replace("void ", "")
        agg.setdefault(k, []).append(float(r[vi].replace(",", "")))
    tot = sum(sum(v) for v in agg.values())
    out = ["| kernel | launches | total ms | mean ms | share |", "|---|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
        out.append(f"| {k} | {len(v)} | {sum(v)/1e6:.3f} | {sum(v)/len(v)/1e6:.3f} | {sum(v)*100/tot:.1f}% |")
    return "\n".join(out)

WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "launch__occupancy_limit_shared_mem",
        "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed"]

def full(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u = rows[0], rows[1]
    idx = [h.index(w) for w in WANT if w in h]
    lines = ["| kernel | " + " | ".join(h[i] for i in idx) + " |", "|---" * (len(idx) + 1) + "|"]
    for r in rows[2:]:
        name = r[h.index("Kernel Name")].split("(")[0].replace("void ", "")
        lines.append(f"| {name} | " + " | ".join(f"{r[i]} {u[i]}" for i in idx) + " |")
    return "\n".join(lines)

if __name__ == "__main__":
    print(f"# {sys.argv[3]}\n\n## Launch list (ncu --metrics gpu__time_duration.sum --clock-control none; cold-cache, serialised)\n")
    print(launches(sys.argv[1]))
    if len(sys.argv) > 2 and sys.argv[2] != "-":
        print("\n## ncu --set full (one launch per kernel, M2 N=1)\n")
        print(full(sys.argv[2]))


def traffic_json(path):
    """{kernel: dram_read+dram_write bytes per launch} from a --set full capture."""
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u = rows[0], rows[1]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    res = {}
    for r in rows[2:]:
        name = r[h.index("Kernel Name")].split("(")[0].replace("void ", "").split("<")[0].split("::")[-1]
        tot = 0.0
        for m in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            i = h.index(m)
            tot += float(r[i].replace(",", "")) * scale.get(u[i], 1)
        res[name] = max(res.get(name, 0.0), tot)  # template instances that returned at once move ~0 bytes
    return res
