"""Round-evidence summary for profiles/: the ncu launch list and full-capture
table (tools/ncu_summary.py), the bench line's phases / roofline / baselines,
the reference arm and the GPU test tally, all from one gpurun_out/<TAG>/ run
of tools/gpu_r2_evidence.sh.
usage: python tools/evidence_summary.py gpurun_out/<TAG> "<title>" > profiles/r2/<TAG>_summary.md"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import ncu_summary  # noqa: E402


def main(d, title):
    print(f"# {title}\n")
    print("## Launch list (ncu --metrics gpu__time_duration.sum --clock-control none; cold-cache, serialised)\n")
    print(ncu_summary.launches(os.path.join(d, "launches.csv")))
    rep = os.path.join(d, "full.ncu-rep")
    if os.path.exists(rep):
        print("\n## ncu --set full (one launch per kernel, M2 N=1)\n")
        print(ncu_summary.full(rep))
    b = json.load(open(os.path.join(d, "bench.json")))
    ck = b["clocks"]
    print(f"\n## Bench (`python bench.py`, B200, clocks {ck})\n")
    print(f"{b['ms_per_step']:.3f} ms/step = {b['value'] / 1e9:.1f} G tuples/s; correct = {b['correct']} "
          f"(count {b.get('match_count')}, checksum {b.get('checksum')}, pair digest {b.get('pair_digest')}, from the last timed step); "
          f"{b['gpu_launches']} launches of this repo's kernels in the timed region.\n")
    peak = b["roofline"]["peak"]
    print(f"| phase | ms | algorithmic bytes | of measured HBM ({peak:.0f} GB/s) |\n|---|---|---|---|")
    for k, v in b["phases"].items():
        ab = v.get("alg_bytes")
        print(f"| {k} | {v['ms']:.3f} | {ab if ab else '-'} | {100 * v['frac_hbm']:.1f}% |" if ab else
              f"| {k} | {v['ms']:.3f} | - | - |")
    r = b["roofline"]
    tr = r.get("traffic")
    print(f"\nroofline: {r['kernel']} {r['achieved']:.0f} GB/s of {r['peak']:.0f} = {r['frac']:.3f}; "
          f"ncu traffic {tr / 1e9:.2f} GB per launch (algorithmic {r['alg_bytes_per_launch'] / 1e9:.2f} GB)." if tr else "")
    cb = b["cpu_baseline"]
    print(f"cpu_baseline (oracle): {cb['value'] / 1e6:.1f} M tuples/s, {cb['sample']}.")
    rp = os.path.join(d, "bench_reference.json")
    if os.path.exists(rp):
        try:
            ref = json.load(open(rp))
            print(f"reference arm (oracle): {ref['value'] / 1e6:.1f} M tuples/s ({ref['config']['workload']}).")
        except (ValueError, KeyError):
            pass
    e = b["e2e"]
    print(f"e2e (pinned host columns through mgj_partition): {e['value'] / 1e9:.2f} G tuples/s, "
          f"{e['h2d_bytes_per_step'] / 2**30:.0f} GiB H2D per step.")
    pt = os.path.join(d, "pytest_gpu.txt")
    if os.path.exists(pt):
        tail = [l for l in open(pt).read().splitlines() if l.strip()][-1:]
        print(f"\nGPU tests (`pytest -m gpu`): {tail[0] if tail else '?'}")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
