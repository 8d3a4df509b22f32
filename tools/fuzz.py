"""Randomised parity sweep (GPU): random small joins — key width, key domain and
skew, sizes, B1 / B2, forced two-level pass, virtual ranks, shuffle overlap /
chunk streaming, compression, selective broadcast, placement-aware assignment,
materialisation — each checked against the oracle (count, checksum, pair
digest; sorted triples when materialised).  Prints one line per case and a
summary; exits 1 on the first mismatch (with the case's parameters).

usage: python tools/fuzz.py [--cases 200] [--seed 1] [--minutes 15]"""
import argparse
import os
import sys
import time

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")  # virtual ranks wait for each other inside kernels
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
from paper_conf_sigmod_paullhl21_b200 import mgj  # noqa: E402


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a.view(np.int32 if a.dtype == np.uint32 else np.int64))).cuda()


def keys(rng, n, kb, dom, zipf):
    if zipf:
        k = rng.zipf(1.0 + zipf, n).astype(np.uint64) % np.uint64(dom)
    else:
        k = rng.integers(0, dom, n, dtype=np.uint64)
    if kb == 4:
        return k.astype(np.uint32)
    return (k * np.uint64(0x9E3779B97F4A7C15)) if rng.random() < 0.5 else k  # 8-byte: spread or dense


def case(rng):
    kb = 8 if rng.random() < 0.25 else 4
    N = int(rng.choice([1, 1, 2, 3, 4, 8]))
    big = rng.random() < 0.15  # sometimes several chunks and tiles per partition and rank
    nr = int(rng.integers(0, 1 << int(rng.integers(4, 22 if big else 18))))
    ns = int(rng.integers(0, 1 << int(rng.integers(4, 23 if big else 19))))
    dom = int(rng.choice([2, 37, 1000, 1 << 14, 1 << 20, (1 << 32) - 1 if kb == 4 else 1 << 40]))
    zipf = float(rng.choice([0, 0, 0.5, 1.0]))
    kw = dict(radix_bits_global=int(rng.choice([0, 1, 4, 7, 10, 12])),
              radix_bits_local=int(rng.choice([0, 0, 2, 5, 8])),
              materialize=bool(rng.random() < 0.4),
              local_split_bits=int(rng.choice([0, 0, 0, 2, 4])),
              shuffle_overlap=int(rng.choice([0, 1, 2, -1])) if N > 1 else int(rng.choice([0, 1, 2])),
              skew_bcast=int(rng.choice([0, 0, 1, -1])))
    if rng.random() < 0.15:  # EXTERNAL: the caller's all-to-all (emulated with device copies)
        kw["shuffle_mode"] = mgj.SHUFFLE_EXTERNAL
        kw["shuffle_overlap"] = 0
        kw["skew_bcast"] = 0
    elif kb == 4 and kw["radix_bits_global"] <= 10 and rng.random() < 0.25:
        kw["compress"] = True
    if N > 1 and rng.random() < 0.25 and "shuffle_mode" not in kw:
        kw["assign"] = 1
    return dict(kb=kb, N=N, nr=nr, ns=ns, dom=dom, zipf=zipf, kw=kw)


def exchange(joins, N):
    """EXTERNAL mode: the all-to-all NCCL all_to_all_single would do, as device copies."""
    lays = [j.exchange_layout() for j in joins]
    tb = lays[0]["tuple_bytes"]
    for rel in range(2):
        for g in range(N):
            so = 0
            for d in range(N):
                cnt = lays[g]["send_count"][rel][d]
                ro = sum(lays[d]["recv_count"][rel][:g])
                if cnt:
                    mgj.device_bytes(lays[d]["recv"][rel] + ro * tb, cnt * tb).copy_(
                        mgj.device_bytes(lays[g]["send"][rel] + so * tb, cnt * tb))
                so += cnt
    torch.cuda.synchronize()


def dataset(c, rng, nr, ns):
    kb = c["kb"]
    d = {"r_keys": keys(rng, nr, kb, c["dom"], c["zipf"]), "s_keys": keys(rng, ns, kb, c["dom"], c["zipf"])}
    dt = np.uint32 if kb == 4 else np.uint64
    if c["kw"].get("compress"):  # the compressed shuffle needs id payloads (global row ids)
        d["r_pays"] = np.arange(nr, dtype=dt)
        d["s_pays"] = np.arange(ns, dtype=dt)
    else:
        d["r_pays"] = rng.integers(0, 1 << 31, nr, dtype=np.uint64).astype(dt)
        d["s_pays"] = rng.integers(0, 1 << 31, ns, dtype=np.uint64).astype(dt)
    # keep the oracle's work bounded: at most 2e7 matches (a tiny key domain squares the output)
    ur, cr_ = np.unique(d["r_keys"], return_counts=True)
    us, cs_ = np.unique(d["s_keys"], return_counts=True)
    _, ir, is_ = np.intersect1d(ur, us, assume_unique=True, return_indices=True)
    if int((cr_[ir].astype(np.int64) * cs_[is_]).sum()) > 20_000_000:
        return None
    return d


def run(c, rng):
    kb, N = c["kb"], c["N"]
    mat = c["kw"]["materialize"]
    # one plan, one or (30%) two runs: the second with other sizes within the capacities
    sizes = [(c["nr"], c["ns"])]
    if rng.random() < 0.3:
        sizes.append((int(rng.integers(0, c["nr"] + 1)), int(rng.integers(0, c["ns"] + 1))))
    data = [dataset(c, rng, nr, ns) for nr, ns in sizes]
    if any(d is None for d in data):
        return None, "skipped (output too large for the oracle)"
    refs = [oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"], materialize=mat) for d in data]
    cut = lambda n: [n * g // N for g in range(N + 1)]  # contiguous shards (row order), like the generator's
    cap_r = max(1, -(-c["nr"] // N) + 1)
    cap_s = max(1, -(-c["ns"] // N) + 1)
    kw = dict(c["kw"])
    out_cap = max(1, max(r["count"] for r in refs)) if mat else 0
    cfgs = [mgj.make_config(rank=g, world_size=N, key_bytes=kb, r_capacity=cap_r, s_capacity=cap_s,
                            recv_capacity_r=max(1, c["nr"]), recv_capacity_s=max(1, c["ns"]), out_capacity=out_cap,
                            peer_timeout_ms=60000, **kw) for g in range(N)]
    if N > 1:
        nb = mgj.arena_bytes(cfgs[0])
        arenas = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(N)]
        joins = [mgj.Join(cfgs[g], [a.data_ptr() for a in arenas], nb) for g in range(N)]
    else:
        joins = [mgj.Join(cfgs[0])]
    streams = [torch.cuda.Stream() for _ in range(N)]
    ok, st = True, 0
    for d, ref, (nr, ns) in zip(data, refs, sizes):
        cr, cs = cut(nr), cut(ns)
        parts = [{k: d[k][cr[g]:cr[g + 1]] if k[0] == "r" else d[k][cs[g]:cs[g + 1]] for k in d} for g in range(N)]
        tens = [[dev(p[k]) for k in ("r_keys", "r_pays", "s_keys", "s_pays")] for p in parts]
        torch.cuda.synchronize()
        for g in range(N):
            joins[g].partition(*tens[g], stream=streams[g])
        for g in range(N):
            joins[g].shuffle(streams[g])
        if kw.get("shuffle_mode") == mgj.SHUFFLE_EXTERNAL:
            torch.cuda.synchronize()
            exchange(joins, N)
        for g in range(N):
            joins[g].join(streams[g])
        res = [j.result() for j in joins]
        st = res[0]["status"]
        ok = all(r["status"] == 0 and (r["match_count"], r["checksum"], r["pair_digest"]) ==
                 (ref["count"], ref["checksum"], ref["pair_digest"]) for r in res)
        if ok and mat:
            trip = [j.materialized(r) for j, r in zip(joins, res)]
            k = np.concatenate([t[0] for t in trip])
            a = np.concatenate([t[1] for t in trip])
            b = np.concatenate([t[2] for t in trip])
            o = np.lexsort((b, a, k))
            ok = (np.array_equal(k[o], ref["key"]) and np.array_equal(a[o], ref["pay_r"]) and
                  np.array_equal(b[o], ref["pay_s"]))
        if not ok:
            break
    for j in joins:
        j.close()
    return ok, f"{st} runs={len(sizes)}"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cases", type=int, default=200)
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--minutes", type=float, default=15)
    a = ap.parse_args()
    rng = np.random.default_rng(a.seed)
    t0 = time.time()
    n = 0
    for i in range(a.cases):
        if time.time() - t0 > 60 * a.minutes:
            break
        c = case(rng)
        try:
            ok, st = run(c, rng)
        except mgj.MGJError as e:  # a configuration the library rejects (EINVAL) is not a mismatch
            ok, st = ("EINVAL" in str(e) or "MGJ_EINVAL" in str(e)), str(e)
        if ok is None:
            print(i, st, c, flush=True)
            continue
        print(i, "ok" if ok else "MISMATCH", st, c, flush=True)
        n += 1
        if not ok:
            sys.exit(1)
    print(f"fuzz: {n} cases ok in {time.time() - t0:.0f} s (seed {a.seed})")


if __name__ == "__main__":
    main()
