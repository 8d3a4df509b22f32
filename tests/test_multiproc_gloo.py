"""N>1 host logic on CPU: two (and four) processes over gloo run the paper's
global partitioning with the library's host plan (mgj_plan_host) — histogram
all-gather, owner assignment, exact offsets, all-to-all exchange — then join
their owned co-partitions with the oracle and sum.  Checks that every received
slot is written exactly once, that each rank only receives tuples it owns,
and that the summed result equals the global oracle (placement independence,
PAPER.md P:400-403)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
M64 = (1 << 64) - 1


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, bits, kind, skew, q, assign=0):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_sigmod_paullhl21_b200 import datagen, mgj
        w = datagen.Workload(kind, 1 << 15, 1 << 16, 1.0) if kind == "zipf" else datagen.Workload(kind, 40009, 40009)
        d = w.rank_inputs(rank, world)
        P = 1 << bits
        hist = np.stack([np.bincount((d["r_keys"] & (P - 1)).astype(np.int64), minlength=P),
                         np.bincount((d["s_keys"] & (P - 1)).astype(np.int64), minlength=P)]).astype(np.int64)
        allh = [torch.zeros(2, P, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allh, torch.from_numpy(hist))
        H = np.stack([h.numpy() for h in allh]).astype(np.uint32)
        owner, send_off, recv_size, bc, skip = mgj.plan_host(world, rank, bits, H, skew_bcast=skew, with_bcast=True,
                                                             assign=assign)
        if skew < 0:
            assert not bc.any()
        out = {}
        for rel, (k, p) in enumerate(((d["r_keys"], d["r_pays"]), (d["s_keys"], d["s_pays"]))):
            part = (k & (P - 1)).astype(np.int64)
            # a selectively broadcast partition (NEXT-2) keeps its S on this rank
            dest = np.where(bc[part] != 0, rank, owner[part]) if rel == 1 else owner[part]
            keep = skip[part] == 0  # empty-side partitions are not shuffled
            k, p, part, dest = k[keep], p[keep], part[keep], dest[keep]
            # slot of each tuple inside its owner's receive buffer: send_off[p] + rank inside (rank, p)
            order = np.argsort(part, kind="stable")
            rank_in_p = np.empty(k.size, np.int64)
            starts = np.concatenate([[0], np.cumsum(np.bincount(part, minlength=P))[:-1]])
            rank_in_p[order] = np.arange(k.size) - starts[part[order]]
            slot = send_off[rel][part].astype(np.int64) + rank_in_p
            o2 = np.argsort(dest, kind="stable")
            counts = np.bincount(dest, minlength=world)
            send = np.stack([k.astype(np.int64), p.astype(np.int64), slot]).T[o2].copy()
            rc = torch.zeros(world, dtype=torch.int64)
            dist.all_to_all_single(rc, torch.from_numpy(counts.astype(np.int64)))
            recv = torch.zeros(int(rc.sum()), 3, dtype=torch.int64)
            dist.all_to_all_single(recv, torch.from_numpy(send), rc.tolist(), counts.tolist())
            recv = recv.numpy()
            assert recv.shape[0] == int(recv_size[rel][rank])
            cover = np.bincount(recv[:, 2], minlength=recv.shape[0])
            assert cover.size == recv.shape[0] and np.all(cover == 1), "slots not exactly tiled"
            rp = recv[:, 0] & (P - 1)
            assert np.all((owner[rp] == rank) if rel == 0 else ((owner[rp] == rank) | (bc[rp] != 0)))
            buf = np.empty((recv.shape[0], 2), np.int64)
            buf[recv[:, 2]] = recv[:, :2]
            out[rel] = buf
        # the R side of broadcast partitions is read by every rank from its root (pull broadcast)
        mine_bc = out[0][bc[out[0][:, 0] & (P - 1)] != 0]
        allbc = [None] * world
        dist.all_gather_object(allbc, mine_bc)
        out[0] = np.concatenate([out[0]] + [allbc[g] for g in range(world) if g != rank])
        r = oracle.join(out[0][:, 0].astype(np.uint32), out[0][:, 1].astype(np.uint32),
                        out[1][:, 0].astype(np.uint32), out[1][:, 1].astype(np.uint32))
        t = torch.tensor([r["count"], r["checksum"] & ((1 << 63) - 1), r["checksum"] >> 63], dtype=torch.int64)
        allr = [torch.zeros(3, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allr, t)
        if rank == 0:
            cnt = sum(int(x[0]) for x in allr)
            chk = sum(int(x[1]) + (int(x[2]) << 63) for x in allr) & M64
            full = w.rank_inputs(0, 1)
            g = oracle.join(full["r_keys"], full["r_pays"], full["s_keys"], full["s_pays"])
            q.put((cnt, chk, g["count"], g["checksum"], int(bc.sum())))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,bits,kind,skew,assign", [(2, 8, "unique", 0, 0), (4, 6, "unique", 0, 0),
                                                         (2, 7, "zipf", -1, 0), (2, 7, "zipf", 0, 0), (4, 7, "zipf", 1, 0),
                                                         (3, 6, "unique", 0, 1), (4, 7, "zipf", 1, 1)])
def test_gloo_partitioned_join(world, bits, kind, skew, assign):
    """skew: mgj_config.skew_bcast (selective broadcast of heavy S partitions, NEXT-2)."""
    import __graft_entry__
    __graft_entry__.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, bits, kind, skew, q, assign)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
    assert all(p.exitcode == 0 for p in procs)
    cnt, chk, gc, gk, nbc = q.get(timeout=10)
    assert (cnt, chk) == (gc, gk)
    if kind == "unique" or skew < 0:
        assert nbc == 0
    else:
        assert nbc > 0  # Zipf S with |R|:|S| = 1:2 has partitions worth broadcasting
