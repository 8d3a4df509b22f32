"""Shuffle traffic and receive balance of the a2 plan at full BASELINE sizes, with and
without selective broadcast (NEXT-2), from the exact per-rank histograms.

Generates every rank's shard of the workload on the GPU (mgj_gen_relation, in
pieces), counts digit1 with torch.bincount, and runs the library's host plan
(mgj_plan_host) for each skew_bcast mode.  Reports per rank: tuples received
(R, S), tuples built/probed (R including the broadcast partitions read from their
roots), and the cross-rank tuples the shuffle moves.  These are exact counts of
the plan, not timings (one GPU here: N > 1 cannot be timed).

usage: python tools/skew_plan.py [--workload zipf|unique] [--z 1.0] [--placement-z 0] [--gpus 8] [--bits 10] > out.json
(--placement-z: rank g holds a 1/(g+1)^z share of the rows, Fig. 9's placement reading;
modes: ranges with/without selective broadcast, and the placement-aware assignment)
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigmod_paullhl21_b200 import mgj  # noqa: E402


def hist_of(kind, rel, n_r, n_s, z, lo, hi, P, piece=1 << 27):
    h = torch.zeros(P, dtype=torch.int64, device="cuda")
    dt = torch.int32
    for a in range(lo, hi, piece):
        cnt = min(piece, hi - a)
        k = torch.empty(cnt, dtype=dt, device="cuda")
        p = torch.empty(cnt, dtype=dt, device="cuda")
        mgj.gen_relation(kind, rel, n_r, n_s, z, a, cnt, k, p)
        h += torch.bincount((k & (P - 1)).long(), minlength=P)
    return h.cpu().numpy()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--z", type=float, default=1.0)
    ap.add_argument("--gpus", type=int, default=8)
    ap.add_argument("--bits", type=int, default=10)
    ap.add_argument("--log2-r-per-gpu", type=int, default=27)
    ap.add_argument("--log2-s-per-gpu", type=int, default=29)
    ap.add_argument("--workload", default="zipf", choices=["zipf", "unique"])
    ap.add_argument("--placement-z", type=float, default=0.0)
    a = ap.parse_args()
    from paper_conf_sigmod_paullhl21_b200 import datagen
    N, P = a.gpus, 1 << a.bits
    n_r, n_s = N << a.log2_r_per_gpu, N << a.log2_s_per_gpu
    H = np.zeros((N, 2, P), np.uint64)
    for g in range(N):
        rlo, rhi = datagen.shard_bounds(n_r, g, N, a.placement_z)
        slo, shi = datagen.shard_bounds(n_s, g, N, a.placement_z)
        H[g, 0] = hist_of(a.workload, 0, n_r, n_s, a.z, rlo, rhi, P)
        H[g, 1] = hist_of(a.workload, 1, n_r, n_s, a.z, slo, shi, P)
    out = {"workload": f"{a.workload} z={a.z}, placement z={a.placement_z}: {n_r} R + {n_s} S tuples over {N} GPUs "
                       f"(8-byte tuples)", "B1": a.bits, "modes": {}}
    tot = H.sum(axis=0)
    for mode, assign, name in ((-1, 0, "hash (single owner per partition, contiguous ranges)"),
                               (0, 0, "selective broadcast (auto)"),
                               (-1, 1, "placement-aware assignment (Track-Join migration)"),
                               (0, 1, "placement-aware + selective broadcast")):
        plans = [mgj.plan_host(N, g, a.bits, H.astype(np.uint32), skew_bcast=mode, with_bcast=True, assign=assign)
                 for g in range(N)]
        owner, _, recv, bc, _skip = plans[0]
        moved = 0  # tuples that leave their rank in the shuffle
        for g in range(N):
            for rel in range(2):
                dest = np.where((bc != 0) & (rel == 1), g, owner)
                moved += int(H[g, rel][dest != g].sum())
        # R read remotely by non-root ranks for broadcast partitions (pull broadcast)
        pulled = int(sum(int(tot[0, p]) * (N - 1) for p in np.nonzero(bc)[0]))
        built = [int(recv[0, d]) + int(sum(int(tot[0, p]) for p in np.nonzero(bc)[0] if owner[p] != d))
                 for d in range(N)]
        work = [built[d] + int(recv[1, d]) for d in range(N)]
        out["modes"][name] = {
            "skew_bcast": mode, "assign": assign, "broadcast_partitions": int(bc.sum()),
            "recv_r": [int(x) for x in recv[0]], "recv_s": [int(x) for x in recv[1]],
            "tuples_joined_per_rank": work,
            "max_over_mean_work": max(work) / (sum(work) / N),
            "shuffle_tuples_moved": moved, "broadcast_r_tuples_pulled": pulled,
            "cross_rank_bytes": 8 * (moved + pulled),
            "max_rank_ingress_bytes": 8 * max(int(recv[0, d] + recv[1, d] - H[d, 0][owner == d].sum()
                                                  - H[d, 1][(owner == d) | (bc != 0)].sum()
                                                  + sum(int(tot[0, p]) for p in np.nonzero(bc)[0] if owner[p] != d))
                                              for d in range(N)),
        }
    json.dump(out, sys.stdout, indent=1)
    print()


if __name__ == "__main__":
    main()
