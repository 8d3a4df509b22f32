"""Small joins for compute-sanitizer (memcheck / racecheck / synccheck): unique,
duplicate-heavy, wide, and 2 virtual ranks."""
import sys, os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")  # virtual ranks wait for each other inside kernels
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle
from paper_conf_sigmod_paullhl21_b200 import datagen, mgj


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a.view(np.int32 if a.dtype == np.uint32 else np.int64))).cuda()


def one(d, **kw):
    kb = 8 if d["r_keys"].dtype == np.uint64 else 4
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    j = mgj.Join(mgj.make_config(key_bytes=kb, r_capacity=d["r_keys"].size, s_capacity=d["s_keys"].size,
                                 out_capacity=max(ref["count"], 1), **kw))
    r = j.run(*[dev(d[k]) for k in ("r_keys", "r_pays", "s_keys", "s_pays")])
    assert (r["match_count"], r["checksum"], r["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"]), (r, ref)
    j.close()


one(datagen.Workload("unique", 1 << 16, 1 << 16).rank_inputs(), materialize=True)
rng = np.random.default_rng(0)
one({"r_keys": rng.integers(0, 300, 20000, dtype=np.uint64).astype(np.uint32), "r_pays": np.arange(20000, dtype=np.uint32),
     "s_keys": rng.integers(0, 300, 30000, dtype=np.uint64).astype(np.uint32), "s_pays": np.arange(30000, dtype=np.uint32)},
    materialize=False, radix_bits_global=4)
one(datagen.Workload("wide", 1 << 14, 1 << 14).rank_inputs(), materialize=True)
# the bench's probe loop (count only, packed table: B1 + B2 = 16) on duplicate keys
one({"r_keys": rng.integers(0, 1 << 14, 50000, dtype=np.uint64).astype(np.uint32), "r_pays": np.arange(50000, dtype=np.uint32),
     "s_keys": rng.integers(0, 1 << 14, 70000, dtype=np.uint64).astype(np.uint32), "s_pays": np.arange(70000, dtype=np.uint32)},
    materialize=False, radix_bits_global=10, radix_bits_local=6)
# the overlapped shuffle (R's local pass on a second stream beside S's scatter) at one rank
one(datagen.Workload("unique", 1 << 17, 1 << 17).rank_inputs(), materialize=True, shuffle_overlap=1, trace=True)
# chunk streaming (NEXT-3) at one rank, and the compressed shuffle (NEXT-1)
one(datagen.Workload("unique", 1 << 17, 1 << 17).rank_inputs(), materialize=True, shuffle_overlap=2,
    peer_timeout_ms=600000)
one(datagen.Workload("unique", 1 << 17, 1 << 17).rank_inputs(), materialize=True, compress=True)


def virtual(w, N, **kw):
    """N virtual ranks on one GPU (plain device arenas), every phase for all ranks in turn."""
    parts = [w.rank_inputs(g, N) for g in range(N)]
    cfgs = [mgj.make_config(rank=g, world_size=N, r_capacity=max(p["r_keys"].size for p in parts),
                            s_capacity=max(p["s_keys"].size for p in parts), recv_capacity_r=w.n_r,
                            recv_capacity_s=w.n_s, **kw) for g in range(N)]
    nb = mgj.arena_bytes(cfgs[0])
    arenas = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(N)]
    js = [mgj.Join(cfgs[g], [a.data_ptr() for a in arenas], nb) for g in range(N)]
    ts = [[dev(p[k]) for k in ("r_keys", "r_pays", "s_keys", "s_pays")] for p in parts]
    ss = [torch.cuda.Stream() for _ in range(N)]  # one per rank: a6 waits for every peer
    torch.cuda.synchronize()
    for g in range(N): js[g].partition(*ts[g], stream=ss[g])
    for g in range(N): js[g].shuffle(ss[g])
    for g in range(N): js[g].join(ss[g])
    res = [js[g].result() for g in range(N)]
    full = w.rank_inputs()
    ref = oracle.join(full["r_keys"], full["r_pays"], full["s_keys"], full["s_pays"])
    assert (res[0]["match_count"], res[0]["checksum"], res[0]["pair_digest"]) == \
        (ref["count"], ref["checksum"], ref["pair_digest"])
    for j in js: j.close()


# two virtual ranks (with the overlapped shuffle); four with selectively broadcast partitions (NEXT-2),
# also through the first local pass
if os.environ.get("MGJ_SAN_VIRTUAL", "1") == "1":
    virtual(datagen.Workload("unique", 1 << 15, 1 << 15), 2)
    virtual(datagen.Workload("zipf", 1 << 13, 1 << 15, 1.0), 4, skew_bcast=1, radix_bits_global=6)
    virtual(datagen.Workload("zipf", 1 << 13, 1 << 15, 1.0), 4, skew_bcast=1, radix_bits_global=6, local_split_bits=2)
    # round 2: chunk streaming, compressed + streaming, placement-aware assignment
    virtual(datagen.Workload("unique", 1 << 15, 1 << 15), 2, shuffle_overlap=2, peer_timeout_ms=600000)
    virtual(datagen.Workload("unique", 1 << 15, 1 << 15), 2, compress=True, shuffle_overlap=2, peer_timeout_ms=600000)
    virtual(datagen.Workload("unique", 1 << 15, 1 << 15), 3, assign=1, peer_timeout_ms=600000)
print("sanitize workload ok")
