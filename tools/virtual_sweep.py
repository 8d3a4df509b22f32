"""NEXT-4 on one GPU: the Fig. 13 input-size axis (512M-4096M
tuples in total) run through the 8-rank protocol with N virtual ranks on one
B200 — every rank's own plan, arena, streams and peer stores, the ranks'
kernels sharing the GPU.  Inputs come from the device generator; the result is
checked against the generator's closed form (bench.expected_shard, no join
code).  The time is the whole job on ONE GPU (all N ranks' work), not an N-GPU
time: it shows the protocol at these sizes and its overhead against one rank
doing the same join (`--compare`).

usage: python tools/virtual_sweep.py [--ranks 8] [--log2-total 28 29 30 31] [--steps 3] [--compare]
One JSON line per size."""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def run(mgj, datagen, expected_shard, torch, N, n, steps, **kw):
    """N virtual ranks joining |R| = |S| = n unique tuples; returns (ms, ok, info)."""
    bounds = [datagen.shard_bounds(n, g, N, 0.0) for g in range(N)]
    cols = []
    for g, (lo, hi) in enumerate(bounds):
        c = [torch.empty(hi - lo, dtype=torch.int32, device="cuda") for _ in range(4)]
        mgj.gen_relation("unique", 0, n, n, 0.0, lo, hi - lo, c[0], c[1])
        mgj.gen_relation("unique", 1, n, n, 0.0, lo, hi - lo, c[2], c[3])
        cols.append(c)
    torch.cuda.synchronize()
    cap = max(hi - lo for lo, hi in bounds)
    cfgs = [mgj.make_config(rank=g, world_size=N, r_capacity=cap, s_capacity=cap, **kw) for g in range(N)]
    joins, arenas = [], []
    if N > 1:
        nb = mgj.arena_bytes(cfgs[0])
        arenas = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(N)]
        joins = [mgj.Join(cfgs[g], [a.data_ptr() for a in arenas], nb) for g in range(N)]
    else:
        joins = [mgj.Join(cfgs[0])]
    streams = [torch.cuda.Stream() for _ in range(N)]

    def once():
        for g in range(N):
            joins[g].partition(*cols[g], stream=streams[g])
        for g in range(N):
            joins[g].shuffle(streams[g])
        for g in range(N):
            joins[g].join(streams[g])

    once()  # warm-up
    torch.cuda.synchronize()
    times = []
    for _ in range(steps):
        start = torch.cuda.Event(enable_timing=True)
        start.record(torch.cuda.current_stream())
        for s in streams:
            s.wait_event(start)
        once()
        ends = []
        for s in streams:
            e = torch.cuda.Event(enable_timing=True)
            e.record(s)
            ends.append(e)
        torch.cuda.synchronize()
        times.append(max(start.elapsed_time(e) for e in ends))
    res = [j.result() for j in joins]
    exp = [0, 0, 0]
    for g in range(N):
        for o in range(0, cols[g][2].numel(), 1 << 26):  # slices: the closed form's int64 temporaries
            c, k, d = expected_shard(torch, "unique", 4, n, cols[g][2][o:o + (1 << 26)], cols[g][3][o:o + (1 << 26)])
            exp = [exp[0] + c, exp[1] + k, exp[2] + d]
    m = (1 << 64) - 1
    ok = all(r["status"] == 0 and (r["match_count"], r["checksum"], r["pair_digest"]) ==
             (exp[0], exp[1] & m, exp[2] & m) for r in res)
    info = {"recv_tuples_per_rank_max": max(r["recv_r"] + r["recv_s"] for r in res)}
    for j in joins:
        j.close()
    del arenas, cols
    torch.cuda.empty_cache()
    return sorted(times)[len(times) // 2], ok, info


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ranks", type=int, default=8)
    ap.add_argument("--log2-total", type=int, nargs="+", default=[28, 29, 30, 31],
                    help="log2 of |R| + |S| (Fig. 13: 512M .. 4096M = 2^29 .. 2^32 in the paper's M)")
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--compare", action="store_true", help="also run the same join as one rank")
    ap.add_argument("--radix-bits-global", type=int, default=0, help="B1 (0: the default 10)")
    a = ap.parse_args()
    os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
    import torch
    from paper_conf_sigmod_paullhl21_b200 import datagen, mgj
    sys.path.insert(0, ROOT)
    from bench import expected_shard
    for lt in a.log2_total:
        n = 1 << (lt - 1)  # per relation
        line = {"tuples_total": 2 * n, "ranks": a.ranks, "B1": a.radix_bits_global or 10}
        try:
            ms, ok, info = run(mgj, datagen, expected_shard, torch, a.ranks, n, a.steps,
                               radix_bits_global=a.radix_bits_global)
            line.update({"ms_one_gpu": round(ms, 3), "g_tuples_per_s_one_gpu": round(2 * n / ms / 1e6, 2),
                         "correct": ok, **info})
        except Exception as e:  # ENOMEM at the largest sizes
            line["error"] = str(e)[:200]
            torch.cuda.empty_cache()
        if a.compare:
            try:
                ms1, ok1, _ = run(mgj, datagen, expected_shard, torch, 1, n, a.steps,
                                  radix_bits_global=a.radix_bits_global)
                line.update({"ms_one_rank": round(ms1, 3), "correct_one_rank": ok1})
            except Exception as e:
                line["error_one_rank"] = str(e)[:200]
                torch.cuda.empty_cache()
        print(json.dumps(line), flush=True)
        time.sleep(1)


if __name__ == "__main__":
    main()
