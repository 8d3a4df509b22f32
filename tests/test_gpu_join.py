"""GPU parity tests: the CUDA path through the C ABI vs the CPU oracle.

Bit-exact bar (integer work): match count, 64-bit checksum and the sorted
materialised triples equal the oracle's; per-phase intermediate state is
checked against library routines (np.bincount, sorting) and invariants.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from paper_conf_sigmod_paullhl21_b200 import datagen  # noqa: E402

M64 = (1 << 64) - 1


@pytest.fixture(scope="module")
def mgj():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_sigmod_paullhl21_b200 import mgj as m
    return m


def dev(a: np.ndarray):
    v = a.view(np.int32) if a.dtype == np.uint32 else a.view(np.int64)
    return torch.from_numpy(np.ascontiguousarray(v)).cuda()


def sort_trip(k, a, b):
    o = np.lexsort((b, a, k))
    return k[o], a[o], b[o]


def run_one(mgj, d, materialize=False, **kw):
    kb = 8 if d["r_keys"].dtype == np.uint64 else 4
    cfg = mgj.make_config(key_bytes=kb, r_capacity=max(d["r_keys"].size, 1), s_capacity=max(d["s_keys"].size, 1),
                          materialize=materialize, **kw)
    j = mgj.Join(cfg)
    res = j.run(dev(d["r_keys"]), dev(d["r_pays"]), dev(d["s_keys"]), dev(d["s_pays"]))
    return j, res


def check_vs_oracle(mgj, d, materialize=True, **kw):
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"], materialize=materialize)
    if materialize:
        kw.setdefault("out_capacity", max(ref["count"], 1))
    j, res = run_one(mgj, d, materialize=materialize, **kw)
    assert res["match_count"] == ref["count"]
    assert res["checksum"] == ref["checksum"]
    assert res["pair_digest"] == ref["pair_digest"]
    if materialize:
        assert res["n_materialized"] == ref["count"]
        k, a, b = sort_trip(*j.materialized(res))
        np.testing.assert_array_equal(k, ref["key"])
        np.testing.assert_array_equal(a, ref["pay_r"])
        np.testing.assert_array_equal(b, ref["pay_s"])
    j.close()
    return res


# ----------------------------------------------------------------- generator
@pytest.mark.parametrize("kind,n_r,n_s,z,row0,count", [
    ("unique", 1000003, 1000003, 0.0, 0, 1000003),
    ("unique", 1 << 20, 1 << 20, 0.0, 12345, 99999),
    ("zipf", 1 << 16, 1 << 18, 0.5, 0, 1 << 18),
    ("zipf", 1 << 16, 1 << 18, 1.0, 777, 100000),
    ("zipf", 1 << 16, 1 << 18, 0.0, 0, 1 << 18),
    ("wide", 1 << 16, 1 << 16, 0.0, 5, 60000),
])
def test_gen_matches_numpy(mgj, kind, n_r, n_s, z, row0, count):
    w = datagen.Workload(kind, n_r, n_s, z)
    for rel, name in ((0, "R"), (1, "S")):
        n = n_r if rel == 0 else n_s
        c = min(count, n - row0)
        dt = torch.int64 if kind == "wide" else torch.int32
        k = torch.empty(c, dtype=dt, device="cuda")
        p = torch.empty(c, dtype=dt, device="cuda")
        mgj.gen_relation(kind, rel, n_r, n_s, z, row0, c, k, p)
        torch.cuda.synchronize()
        ek, ep = w.relation(name, row0, row0 + c)
        np.testing.assert_array_equal(k.cpu().numpy().view(ek.dtype), ek)
        np.testing.assert_array_equal(p.cpu().numpy().view(ep.dtype), ep)


# ------------------------------------------------------------ per-phase state
@pytest.mark.parametrize("b1", [10, 4])
def test_phases_m1(mgj, b1):
    """a1 histogram == np.bincount, a2 plan invariants, a3 received multiset,
    a4 sub-partition property, at M1 (2^20 x 2^20, one GPU)."""
    d = datagen.M1().rank_inputs()
    n = d["r_keys"].size
    j, res = run_one(mgj, d, radix_bits_global=b1)
    P = 1 << res["radix_bits_global"]
    B1 = res["radix_bits_global"]
    hist = j.debug("RANK_HIST", np.uint32).reshape(2, P)
    np.testing.assert_array_equal(hist[0], np.bincount(d["r_keys"] & (P - 1), minlength=P))
    np.testing.assert_array_equal(hist[1], np.bincount(d["s_keys"] & (P - 1), minlength=P))
    owner = j.debug("OWNER", np.int32)
    assert (owner == 0).all()
    send_off = j.debug("SEND_OFF", np.uint64).reshape(2, P)
    for rel in range(2):
        exp = np.concatenate([[0], np.cumsum(hist[rel].astype(np.uint64))[:-1]])
        np.testing.assert_array_equal(send_off[rel], exp)
    assert res["recv_r"] == n and res["recv_s"] == n
    for rel, (kk, pp) in enumerate(((d["r_keys"], d["r_pays"]), (d["s_keys"], d["s_pays"]))):
        recv = j.debug("RECV_R" if rel == 0 else "RECV_S", np.uint32).reshape(-1, 2)
        # received layout: partition p occupies [send_off[p], send_off[p] + hist[p])
        digit = recv[:, 0] & (P - 1)
        assert np.all(np.diff(digit.astype(np.int64)) >= 0)
        packed = recv[:, 0].astype(np.uint64) | (recv[:, 1].astype(np.uint64) << np.uint64(32))
        exp = kk.astype(np.uint64) | (pp.astype(np.uint64) << np.uint64(32))
        np.testing.assert_array_equal(np.sort(packed), np.sort(exp))
        # a4: every chunk of every segment is split into q-runs (16-byte padded)
        # whose tuples all have digit2 == q, and the chunk's multiset is kept
        B2 = res["radix_bits_local"]
        Q = 1 << B2
        C = int(j.debug("META", np.int32)[7])  # local-pass chunk size
        seg = j.debug("SEGMENTS", np.uint64).reshape(4, P)
        start, ln = seg[rel], seg[2 + rel]
        E = j.debug("CHUNK_OFF_R" if rel == 0 else "CHUNK_OFF_S", np.uint16).astype(np.int64)
        nch_p = (ln.astype(np.int64) + C - 1) // C
        loc = j.debug("LOCAL_R" if rel == 0 else "LOCAL_S", np.uint32).reshape(-1, 2)
        CR = loc.shape[0] // int(nch_p.sum())
        cb = np.concatenate([[0], np.cumsum(nch_p)])
        for p in range(P):
            for k in range(int(nch_p[p])):
                a = int(start[p]) + k * C
                b = min(int(start[p]) + int(ln[p]), a + C)
                li = cb[p] + k
                row = lambda q: E[(Q + 1) * cb[p] + q * nch_p[p] + k]
                got = []
                for q in range(Q):
                    e0, e1 = row(q), row(q + 1)
                    st, slots = e0 & ~1, (e1 & ~1) - (e0 & ~1)
                    valid = slots - (e0 & 1)
                    run = loc[li * CR + st: li * CR + st + valid]
                    assert np.all(((run[:, 0] >> B1) & (Q - 1)) == q)
                    if valid < slots:  # padding slot: a key of the run with bit 0 (R) / bit 1 (S, P >= 4) flipped
                        flip = 2 if (rel == 1 and P >= 4) else 1
                        assert (loc[li * CR + st + valid, 0] ^ flip) in run[:, 0]
                    got.append(run)
                got = np.concatenate(got)
                src = recv[a:b, 0].astype(np.uint64) | (recv[a:b, 1].astype(np.uint64) << np.uint64(32))
                dst = got[:, 0].astype(np.uint64) | (got[:, 1].astype(np.uint64) << np.uint64(32))
                np.testing.assert_array_equal(np.sort(src), np.sort(dst))
    j.close()


# ------------------------------------------------------------ end-to-end parity
def test_m1_parity_materialized(mgj):
    res = check_vs_oracle(mgj, datagen.M1().rank_inputs(), materialize=True)
    assert res["match_count"] == 1 << 20
    assert res["checksum"] == 0xfff8007ffff80000


# ------------------------------------------------------------ two-level local partitioning
@pytest.mark.parametrize("ba", [1, 3, 6])
def test_two_level_local_phases(mgj, ba):
    """Forced first local pass (BA bits) on M1 with B1 = 4 (16 partitions of
    2^16): every first-pass chunk is stored in place as 2^BA runs; run a holds
    only tuples whose next BA key bits are a (plus, for an odd run, one padding
    tuple: its first tuple with a low key bit flipped, i.e. of another global
    partition), and the runs of all chunks hold exactly the received tuples;
    the join stays exact."""
    d = datagen.M1().rank_inputs()
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"], materialize=False)
    j, res = run_one(mgj, d, radix_bits_global=4, local_split_bits=ba)
    assert (res["match_count"], res["checksum"], res["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    meta = j.debug("META", np.int32)
    B1, P = 4, 16
    BA, QB, L = int(meta[8]), int(meta[9]), int(meta[10])
    assert BA == min(ba, res["radix_bits_local"]) and QB == res["radix_bits_local"] - BA and L == P << BA
    QA = 1 << BA
    for rel, name in ((0, "R"), (1, "S")):
        recv = j.debug("RECV_" + name, np.uint32).reshape(-1, 2)
        mid = j.debug("MID_" + name, np.uint32).reshape(-1, 2)
        E = j.debug("MID_OFF_" + name, np.uint16).reshape(-1, 65).astype(np.int64)
        nch = E.shape[0]
        assert nch == int(meta[4 + rel]) and mid.shape[0] % nch == 0
        region = mid.shape[0] // nch
        real = []
        for k in range(nch):
            for a in range(QA):
                st, en = E[k, a] & ~1, E[k, a + 1] & ~1
                valid = en - st - (E[k, a] & 1)
                run = mid[k * region + st:k * region + en]
                assert np.all(((run[:valid, 0] >> B1) & (QA - 1)) == a)
                if valid < en - st:  # padding: the run's first tuple, a low key bit flipped
                    assert run[valid, 0] == run[0, 0] ^ (2 if (rel == 1 and P >= 4) else 1)
                real.append(run[:valid])
        real = np.concatenate(real)
        pack = lambda x: np.sort(x[:, 0].astype(np.uint64) | (x[:, 1].astype(np.uint64) << np.uint64(32)))
        np.testing.assert_array_equal(pack(real), pack(recv))
    j.close()


@pytest.mark.parametrize("ba", [2, 5])
@pytest.mark.parametrize("kind", ["unique_dup", "zipf", "wide", "edge"])
def test_two_level_local_parity(mgj, ba, kind):
    """Forced two-level local partitioning vs the oracle (materialised)."""
    rng = np.random.default_rng(99)
    if kind == "zipf":
        d = datagen.Workload("zipf", 1 << 16, 1 << 19, 1.0).rank_inputs()
    elif kind == "wide":
        d = datagen.Workload("wide", 1 << 18, 1 << 18).rank_inputs()
    elif kind == "edge":
        ks = np.array([0, 1, 2, 3, 0xFFFFFFFF, 0xFFFFFFFE, 0x80000000, 0x7FFFFFFF], np.uint32)
        d = dict(r_keys=np.repeat(ks, 3), r_pays=np.arange(24, dtype=np.uint32),
                 s_keys=np.tile(ks, 5), s_pays=np.arange(40, dtype=np.uint32) + 100)
    else:
        d = dict(r_keys=rng.integers(0, 1 << 17, 400003, dtype=np.uint32),
                 r_pays=rng.integers(0, 1 << 32, 400003, dtype=np.uint32),
                 s_keys=rng.integers(0, 1 << 17, 500009, dtype=np.uint32),
                 s_pays=rng.integers(0, 1 << 32, 500009, dtype=np.uint32))
    check_vs_oracle(mgj, d, materialize=True, radix_bits_global=3, local_split_bits=ba)


@pytest.mark.parametrize("b1,b2", [(1, 0), (4, 3), (8, 0), (11, 2), (12, 5)])
def test_radix_bit_variants(mgj, b1, b2):
    d = datagen.Workload("unique", 300007, 300007).rank_inputs()
    check_vs_oracle(mgj, d, materialize=True, radix_bits_global=b1, radix_bits_local=b2)


@pytest.mark.parametrize("nr,ns,dom", [(0, 1000, 100), (1000, 0, 100), (0, 0, 1), (1, 1, 1), (3, 5, 2),
                                       (100003, 70001, 1 << 32), (50000, 60000, 4096), (20000, 30000, 37)])
def test_random_duplicates(mgj, nr, ns, dom):
    rng = np.random.default_rng(nr * 7 + ns)
    d = {"r_keys": rng.integers(0, dom, nr, dtype=np.uint64).astype(np.uint32),
         "s_keys": rng.integers(0, dom, ns, dtype=np.uint64).astype(np.uint32),
         "r_pays": rng.integers(0, 1 << 32, nr, dtype=np.uint64).astype(np.uint32),
         "s_pays": rng.integers(0, 1 << 32, ns, dtype=np.uint64).astype(np.uint32)}
    check_vs_oracle(mgj, d, materialize=(nr * ns < 10**8 and dom > 50) or nr * ns < 100)


def test_edge_key_values(mgj):
    edge = np.array([0, 1, 2**31 - 1, 2**31, 2**32 - 2, 2**32 - 1], dtype=np.uint32)
    rng = np.random.default_rng(3)
    d = {"r_keys": rng.choice(edge, 3000), "s_keys": rng.choice(edge, 2000),
         "r_pays": np.arange(3000, dtype=np.uint32) - np.uint32(10), "s_pays": np.arange(2000, dtype=np.uint32)}
    check_vs_oracle(mgj, d, materialize=True)


def test_heavy_single_key(mgj):
    """All R and S tuples share one key: R co-partition 10000 > table capacity
    (chunked builds), S split over several probe items."""
    nr, ns = 10000, 70000
    d = {"r_keys": np.full(nr, 0xDEADBEEF, np.uint32), "s_keys": np.full(ns, 0xDEADBEEF, np.uint32),
         "r_pays": np.arange(nr, dtype=np.uint32), "s_pays": np.arange(ns, dtype=np.uint32) * np.uint32(3)}
    res = check_vs_oracle(mgj, d, materialize=False)
    assert res["match_count"] == nr * ns


@pytest.mark.parametrize("z", [0.5, 1.0])
def test_zipf_small(mgj, z):
    w = datagen.Workload("zipf", 1 << 16, 1 << 18, z)
    d = w.rank_inputs()
    res = check_vs_oracle(mgj, d, materialize=True)
    assert res["match_count"] == 1 << 17


def test_wide_small_materialized(mgj):
    n = 1 << 16
    d = datagen.Workload("wide", n, n).rank_inputs()
    res = check_vs_oracle(mgj, d, materialize=True)
    h = n * (n - 1) // 2
    assert res["checksum"] == (oracle.C_WIDE * (n * (1 << 40) + h) + n * (1 << 41) + h) & M64


def test_wide_high_bits_only(mgj):
    rng = np.random.default_rng(11)
    low = rng.integers(0, 64, 40000, dtype=np.uint64)
    rk = (rng.integers(0, 8, 40000, dtype=np.uint64) << np.uint64(32)) | low
    low2 = rng.integers(0, 64, 30000, dtype=np.uint64)
    sk = (rng.integers(0, 8, 30000, dtype=np.uint64) << np.uint64(32)) | low2
    d = {"r_keys": rk, "s_keys": sk, "r_pays": np.arange(40000, dtype=np.uint64) << np.uint64(33),
         "s_pays": np.arange(30000, dtype=np.uint64) + np.uint64(2**63)}
    check_vs_oracle(mgj, d, materialize=False)


@pytest.mark.parametrize("kind", ["wide", "wide_dup_high", "u32_dup"])
def test_packed_table(mgj, kind):
    """The packed chained table (B1 + B2 >= 16: the R slot's key is replaced by
    khi << 16 | next) at small sizes, forced with B1 = 10, B2 = 6: unique wide
    keys, wide keys that differ only above bit 40 with duplicate R keys (the
    materialisation's re-walk path), and 4-byte duplicate keys."""
    rng = np.random.default_rng(23)
    if kind == "wide":
        d = datagen.Workload("wide", 1 << 17, 1 << 17).rank_inputs()
    elif kind == "wide_dup_high":
        def keys(n):
            return (rng.integers(0, 16, n, dtype=np.uint64) << np.uint64(40)) | rng.integers(0, 256, n, dtype=np.uint64)
        d = {"r_keys": keys(30000), "s_keys": keys(20000),
             "r_pays": np.arange(30000, dtype=np.uint64) << np.uint64(20),
             "s_pays": np.arange(20000, dtype=np.uint64) + np.uint64(2**62)}
    else:
        d = dict(r_keys=rng.integers(0, 1 << 20, 200003, dtype=np.uint32),
                 r_pays=rng.integers(0, 1 << 32, 200003, dtype=np.uint32),
                 s_keys=rng.integers(0, 1 << 20, 300007, dtype=np.uint32),
                 s_pays=rng.integers(0, 1 << 32, 300007, dtype=np.uint32))
    check_vs_oracle(mgj, d, materialize=True, radix_bits_global=10, radix_bits_local=6)


def test_host_pointer_path(mgj):
    """Host (numpy) inputs are staged by the library: same result (end-to-end path)."""
    d = datagen.Workload("unique", 1 << 18, 1 << 18).rank_inputs()
    cfg = mgj.make_config(r_capacity=1 << 18, s_capacity=1 << 18)
    j = mgj.Join(cfg)
    res = j.run(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    assert (res["match_count"], res["checksum"], res["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    j.close()


def test_repeated_runs_same_handle(mgj):
    d = datagen.Workload("unique", 100000, 100000).rank_inputs()
    cfg = mgj.make_config(r_capacity=200000, s_capacity=200000)
    j = mgj.Join(cfg)
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    t = [dev(d[k]) for k in ("r_keys", "r_pays", "s_keys", "s_pays")]
    for _ in range(3):
        res = j.run(*t)
        assert (res["match_count"], res["checksum"], res["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    j.close()


# ------------------------------------------------------------ virtual ranks
def run_virtual(mgj, w: datagen.Workload, N: int, materialize: bool, **kw):
    """N ranks in one process on GPU 0: arenas are plain device buffers, every
    phase is issued for all ranks before the next (mgj.h conventions)."""
    parts = [w.rank_inputs(g, N) for g in range(N)]
    kb = w.key_bytes
    cap_r = max(p["r_keys"].size for p in parts)
    cap_s = max(p["s_keys"].size for p in parts)
    cfgs = [mgj.make_config(rank=g, world_size=N, key_bytes=kb, r_capacity=cap_r, s_capacity=cap_s,
                            materialize=materialize, recv_capacity_r=w.n_r, recv_capacity_s=w.n_s, **kw)
            for g in range(N)]
    nb = mgj.arena_bytes(cfgs[0])
    arenas = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(N)]
    ptrs = [a.data_ptr() for a in arenas]
    joins = [mgj.Join(cfgs[g], ptrs, nb) for g in range(N)]
    tens = [[dev(p[k]) for k in ("r_keys", "r_pays", "s_keys", "s_pays")] for p in parts]
    streams = [torch.cuda.Stream() for _ in range(N)]  # one per rank: a6 waits for every peer (mgj.h)
    torch.cuda.synchronize()
    for g in range(N):
        joins[g].partition(*tens[g], stream=streams[g])
    for g in range(N):
        joins[g].shuffle(streams[g])
    for g in range(N):
        joins[g].join(streams[g])
    res = [joins[g].result() for g in range(N)]
    return joins, res, arenas


@pytest.mark.parametrize("N", [2, 3, 4, 8])
def test_virtual_ranks_m1(mgj, N):
    w = datagen.M1()
    joins, res, _ = run_virtual(mgj, w, N, materialize=True)
    d = w.rank_inputs()
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"], materialize=True)
    for r in res:
        assert (r["match_count"], r["checksum"], r["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    assert sum(r["local_count"] for r in res) == ref["count"]
    assert sum(r["local_pair_digest"] for r in res) % (1 << 64) == ref["pair_digest"]
    trip = [j.materialized(r) for j, r in zip(joins, res)]
    k, a, b = sort_trip(*(np.concatenate([t[i] for t in trip]) for i in range(3)))
    np.testing.assert_array_equal(k, ref["key"])
    np.testing.assert_array_equal(a, ref["pay_r"])
    np.testing.assert_array_equal(b, ref["pay_s"])
    # device plan == host reference plan, and every received tuple belongs to its owner
    P = 1 << res[0]["radix_bits_global"]
    mail = joins[0].debug("MAIL_HIST", np.uint32).reshape(N, 2, P)
    for g, j in enumerate(joins):
        owner, send_off, recv_size = mgj.plan_host(N, g, res[0]["radix_bits_global"], mail)
        np.testing.assert_array_equal(j.debug("OWNER", np.int32), owner)
        np.testing.assert_array_equal(j.debug("SEND_OFF", np.uint64).reshape(2, P), send_off)
        assert res[g]["recv_r"] == recv_size[0, g] and res[g]["recv_s"] == recv_size[1, g]
        recv = j.debug("RECV_R", np.uint32).reshape(-1, 2)
        assert np.all(owner[recv[:, 0] & (P - 1)] == g)
    for j in joins:
        j.close()


@pytest.mark.parametrize("N,ba", [(2, 2), (4, 3), (8, 1)])
def test_virtual_ranks_two_level(mgj, N, ba):
    """N ranks with the first local pass forced on every rank (B1 = 4)."""
    w = datagen.M1()
    joins, res, _ = run_virtual(mgj, w, N, materialize=False, radix_bits_global=4, local_split_bits=ba)
    d = w.rank_inputs()
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    for r in res:
        assert (r["match_count"], r["checksum"], r["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    for j in joins:
        j.close()


def test_virtual_ranks_zipf_skew(mgj):
    w = datagen.Workload("zipf", 1 << 16, 1 << 18, 1.0)
    joins, res, _ = run_virtual(mgj, w, 4, materialize=False)
    d = w.rank_inputs()
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    assert (res[0]["match_count"], res[0]["checksum"], res[0]["pair_digest"]) == \
        (ref["count"], ref["checksum"], ref["pair_digest"])
    for j in joins:
        j.close()


class ArrayWorkload:
    """Fixed arrays split into contiguous rank shards (reading C12), for run_virtual."""

    def __init__(self, rk, ra, sk, sb):
        self.a = dict(r_keys=rk, r_pays=ra, s_keys=sk, s_pays=sb)
        self.n_r, self.n_s = rk.size, sk.size
        self.key_bytes = 8 if rk.dtype == np.uint64 else 4

    def rank_inputs(self, rank=0, world=1):
        out = {}
        for k, v in self.a.items():
            n = v.size
            out[k] = v[n * rank // world: n * (rank + 1) // world].copy()
        return out


def check_bcast_virtual(mgj, w, N, skew, materialize=True, expect_bc=True, **kw):
    """NEXT-2 selective broadcast on N virtual ranks: result == oracle (count, checksum,
    sorted triples), device plan == host plan (owner, offsets, broadcast flags), each
    rank's received S holds its owned partitions and its own share of every broadcast
    partition, and every broadcast partition's R side is built by every rank."""
    joins, res, _ = run_virtual(mgj, w, N, materialize=materialize, skew_bcast=skew, **kw)
    d = w.rank_inputs()
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"], materialize=materialize)
    for r in res:
        assert r["status"] == 0
        assert (r["match_count"], r["checksum"], r["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    assert sum(r["local_count"] for r in res) == ref["count"]
    if materialize:
        trip = [j.materialized(r) for j, r in zip(joins, res)]
        k, a, b = sort_trip(*(np.concatenate([t[i] for t in trip]) for i in range(3)))
        np.testing.assert_array_equal(k, ref["key"])
        np.testing.assert_array_equal(a, ref["pay_r"])
        np.testing.assert_array_equal(b, ref["pay_s"])
    B1 = res[0]["radix_bits_global"]
    P = 1 << B1
    mail = joins[0].debug("MAIL_HIST", np.uint32).reshape(N, 2, P)
    kdt = np.uint32 if w.key_bytes == 4 else np.uint64
    nbc = None
    for g, j in enumerate(joins):
        owner, send_off, recv_size, bc, skip = mgj.plan_host(N, g, B1, mail, skew_bcast=skew, with_bcast=True)
        np.testing.assert_array_equal(j.debug("SKIP", np.uint8), skip)
        np.testing.assert_array_equal(j.debug("OWNER", np.int32), owner)
        np.testing.assert_array_equal(j.debug("BCAST", np.uint8), bc)
        np.testing.assert_array_equal(j.debug("SEND_OFF", np.uint64).reshape(2, P), send_off)
        assert res[g]["recv_r"] == recv_size[0, g] and res[g]["recv_s"] == recv_size[1, g]
        meta = j.debug("META", np.int32)
        nbc = int(bc.sum())
        assert meta[14] == nbc
        plist = j.debug("PLIST", np.int32)
        assert sorted(plist.tolist()) == sorted(set(np.nonzero(owner == g)[0].tolist()) | set(np.nonzero(bc)[0].tolist()))
        recv_s = j.debug("RECV_S", kdt).reshape(-1, 2)
        ps = (recv_s[:, 0] & (P - 1)).astype(np.int64)
        assert np.all((owner[ps] == g) | (bc[ps] != 0))
        # the S of a broadcast partition received by g is exactly g's own shard of it
        mine = w.rank_inputs(g, N)
        for p in np.nonzero(bc)[0][:8]:
            own = np.sort(mine["s_keys"][(mine["s_keys"] & (P - 1)) == p])
            np.testing.assert_array_equal(np.sort(recv_s[ps == p, 0]), own)
    if expect_bc:
        assert nbc > 0
    for j in joins:
        j.close()
    return nbc


@pytest.mark.parametrize("N,skew", [(2, 0), (3, 0), (4, 0), (6, 1), (8, 0), (4, 1), (8, 1), (4, -1)])
def test_virtual_ranks_bcast_zipf(mgj, N, skew):
    """Zipf S (z = 1, |R|:|S| = 1:4, half the S rows match): heavy partitions broadcast."""
    w = datagen.Workload("zipf", 1 << 16, 1 << 18, 1.0)
    check_bcast_virtual(mgj, w, N, skew, materialize=True, expect_bc=skew >= 0, radix_bits_global=8)


@pytest.mark.parametrize("N,ba", [(4, 2), (8, 1)])
def test_virtual_ranks_bcast_two_level(mgj, N, ba):
    """Broadcast partitions' remote R pieces through the first (histogram) local pass."""
    w = datagen.Workload("zipf", 1 << 16, 1 << 18, 1.0)
    check_bcast_virtual(mgj, w, N, 1, materialize=False, radix_bits_global=6, local_split_bits=ba)


def test_virtual_ranks_bcast_duplicates(mgj):
    """Duplicate R keys inside broadcast partitions (bag semantics, C2), 4-byte keys."""
    rng = np.random.default_rng(7)
    rk = rng.integers(0, 3000, 6000, dtype=np.uint64).astype(np.uint32)
    sk = np.concatenate([rng.integers(0, 3000, 20000, dtype=np.uint64),
                         np.full(30000, 7 * 64 + 5, np.uint64)]).astype(np.uint32)
    rng.shuffle(sk)
    w = ArrayWorkload(rk, np.arange(rk.size, dtype=np.uint32), sk, np.arange(sk.size, dtype=np.uint32))
    check_bcast_virtual(mgj, w, 4, 0, materialize=True, radix_bits_global=6)


def test_virtual_ranks_bcast_wide(mgj):
    """8-byte keys and payloads with broadcast partitions (forced)."""
    rng = np.random.default_rng(11)
    dom = rng.integers(0, 1 << 63, 4000, dtype=np.uint64) | np.uint64(1 << 63)
    rk = dom[rng.integers(0, dom.size, 5000)]
    sk = dom[rng.integers(0, dom.size, 60000)]
    w = ArrayWorkload(rk, (np.arange(rk.size) + (1 << 40)).astype(np.uint64), sk,
                      (np.arange(sk.size) + (1 << 41)).astype(np.uint64))
    check_bcast_virtual(mgj, w, 4, 1, materialize=True, radix_bits_global=5)


@pytest.mark.parametrize("N", [1, 4])
def test_bloom_skip_partitions(mgj, N):
    """The histogram as a Bloom filter: partitions with no R or no S tuple
    are not shuffled; the result is unchanged and only the shared partitions arrive."""
    B1, P = 6, 64
    rng = np.random.default_rng(3)
    def keys(n, lo, hi):  # digit1 in [lo, hi)
        return ((rng.integers(0, 1 << 20, n, dtype=np.uint64) << B1) | rng.integers(lo, hi, n, dtype=np.uint64)).astype(np.uint32)
    rk = keys(30000, 0, 48)
    rs = rk[((rk & (P - 1)) >= 16)]  # R keys of the shared partitions [16, 48)
    sk = np.concatenate([keys(20000, 16, 64), rs[rng.integers(0, rs.size, 20000)]])
    w = ArrayWorkload(rk, np.arange(rk.size, dtype=np.uint32), sk, np.arange(sk.size, dtype=np.uint32))
    joins, res, _ = run_virtual(mgj, w, N, materialize=True, radix_bits_global=B1)
    ref = oracle.join(rk, w.a["r_pays"], sk, w.a["s_pays"], materialize=True)
    for r in res:
        assert (r["match_count"], r["checksum"], r["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    trip = [j.materialized(r) for j, r in zip(joins, res)]
    k, a, b = sort_trip(*(np.concatenate([t[i] for t in trip]) for i in range(3)))
    np.testing.assert_array_equal(k, ref["key"])
    np.testing.assert_array_equal(b, ref["pay_s"])
    shared = lambda x: ((x & (P - 1)) >= 16) & ((x & (P - 1)) < 48)
    assert sum(r["recv_r"] for r in res) == int(shared(rk).sum())
    assert sum(r["recv_s"] for r in res) == int(shared(sk).sum())
    skip = joins[0].debug("SKIP", np.uint8)
    np.testing.assert_array_equal(skip != 0, (np.arange(P) < 16) | (np.arange(P) >= 48))
    for j in joins:
        j.close()


def test_virtual_ranks_wide(mgj):
    w = datagen.Workload("wide", 1 << 17, 1 << 17)
    joins, res, _ = run_virtual(mgj, w, 2, materialize=True)
    d = w.rank_inputs()
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    assert (res[1]["match_count"], res[1]["checksum"], res[1]["pair_digest"]) == \
        (ref["count"], ref["checksum"], ref["pair_digest"])
    for j in joins:
        j.close()


# ------------------------------------------------------------ error paths
@pytest.mark.parametrize("sms,kind,mat", [(1, "unique", True), (7, "wide", False), (31, "zipf", False),
                                           (33, "unique", True), (100, "wide", True)])
def test_grid_sizes(mgj, sms, kind, mat):
    """num_sms bounds every persistent grid and the tile count G (= SMs): one CTA,
    fewer tiles than a warp (the tile scan's partial warp), just over a warp, and
    an uneven grid all join bit-exact with the oracle."""
    w = {"unique": datagen.Workload("unique", 200003, 300007), "wide": datagen.Workload("wide", 200003, 300007),
         "zipf": datagen.Workload("zipf", 1 << 16, 1 << 18, 1.0)}[kind]
    d = w.rank_inputs()
    cfg = mgj.make_config(r_capacity=w.n_r, s_capacity=w.n_s, num_sms=sms, materialize=mat,
                          key_bytes=w.key_bytes)
    j = mgj.Join(cfg)
    res = j.run(*[dev(d[x]) for x in ("r_keys", "r_pays", "s_keys", "s_pays")])
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"], materialize=mat)
    assert (res["match_count"], res["checksum"], res["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    if mat:
        k, a, b = sort_trip(*j.materialized(res))
        np.testing.assert_array_equal(k, ref["key"])
        np.testing.assert_array_equal(a, ref["pay_r"])
        np.testing.assert_array_equal(b, ref["pay_s"])
    j.close()


def test_error_paths(mgj):
    n = 4096
    cfg = mgj.make_config(r_capacity=n, s_capacity=n)
    j = mgj.Join(cfg)
    t = torch.zeros(n + 4, dtype=torch.int32, device="cuda")
    with pytest.raises(mgj.MGJError) as e:
        j.shuffle()
    assert e.value.status == -5  # ESTATE
    with pytest.raises(mgj.MGJError) as e:
        j.partition(t[1:n + 1], t[:n], t[:n], t[:n])
    assert e.value.status == -2  # EALIGN
    with pytest.raises(mgj.MGJError) as e:
        j.partition(t, t, t, t)  # n + 4 > capacity
    assert e.value.status == -1
    j.close()
    # receive capacity smaller than the data: sticky ECAPACITY from mgj_result
    d = datagen.Workload("unique", n, n).rank_inputs()
    j = mgj.Join(mgj.make_config(r_capacity=n, s_capacity=n, recv_capacity_r=n // 2, recv_capacity_s=n))
    j.partition(dev(d["r_keys"]), dev(d["r_pays"]), dev(d["s_keys"]), dev(d["s_pays"]))
    j.shuffle()
    j.join()
    with pytest.raises(mgj.MGJError) as e:
        j.result()
    assert e.value.status == -6
    j.close()
    # materialised output larger than out_capacity: sticky ECAPACITY, nothing written past it
    j = mgj.Join(mgj.make_config(r_capacity=n, s_capacity=n, materialize=True, out_capacity=100))
    j.partition(dev(d["r_keys"]), dev(d["r_pays"]), dev(d["s_keys"]), dev(d["s_pays"]))
    j.shuffle()
    j.join()
    with pytest.raises(mgj.MGJError) as e:
        j.result()
    assert e.value.status == -6
    r = j.result(check=False)
    assert r["match_count"] == n  # count and checksum do not depend on the output buffer
    assert r["n_materialized"] <= 100
    j.close()


# ------------------------------------------------------------ full size (bench config)
@pytest.mark.slow
def test_m2_full_size_closed_form(mgj):
    """M2 at N=1 (2^29 R x 2^29 S, the bench workload): closed-form count and
    checksum (tests/golden/appendix_a_closed_forms.json)."""
    n = 1 << 29
    cols = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(4)]
    mgj.gen_relation("unique", 0, n, n, 0.0, 0, n, cols[0], cols[1])
    mgj.gen_relation("unique", 1, n, n, 0.0, 0, n, cols[2], cols[3])
    j = mgj.Join(mgj.make_config(r_capacity=n, s_capacity=n))
    res = j.run(*cols)
    assert res["match_count"] == n
    assert res["checksum"] == 0xf1fffffff0000000
    assert res["pair_digest"] == _device_pair_digest_unique(cols[0], cols[2], cols[3], n)
    # sampled structural check at full size: received R is a permutation of the input
    hist = j.debug("RANK_HIST", np.uint32).reshape(2, -1)
    assert int(hist[0].sum()) == n and int(hist[1].sum()) == n
    j.close()


def _check_materialized_full(mgj, j, res, w: "datagen.Workload", n_sample=1 << 16):
    """Full-size materialised output, unique-key workloads: every R row and
    every S row appears exactly once (payload columns are permutations of the
    row ids, checked on the device), and sampled triples (k, a, b) satisfy
    R.key(row a) == k == S.key(row b) (rows recomputed by the generator)."""
    n = res["n_materialized"]
    kb = w.key_bytes
    dt = torch.int32 if kb == 4 else torch.int64
    col = lambda ptr: mgj.device_bytes(ptr, n * kb).view(dt)
    key, pa, pb = col(res["out_key"]), col(res["out_payload_r"]), col(res["out_payload_s"])
    base_r, base_s = (0, 0) if w.kind == "unique" else (1 << 40, 1 << 41)
    for c, base in ((pa, base_r), (pb, base_s)):
        srt = torch.sort(c - base).values
        assert bool((srt == torch.arange(n, device="cuda", dtype=dt)).all())
        del srt
    g = torch.Generator(device="cuda").manual_seed(5)
    idx = torch.randint(0, n, (n_sample,), device="cuda", generator=g)
    k = key[idx].cpu().numpy().view(np.uint32 if kb == 4 else np.uint64)
    a = (pa[idx] - base_r).cpu().numpy().astype(np.uint64)
    b = (pb[idx] - base_s).cpu().numpy().astype(np.uint64)
    mk = lambda rel, rows, nn: (datagen.perm_n(rows, nn, datagen.SEED_R if rel == "R" else datagen.SEED_S)
                                if w.kind == "unique" else
                                datagen.mix64(datagen.perm_n(rows, nn, datagen.SEED_R if rel == "R" else datagen.SEED_S)))
    np.testing.assert_array_equal(mk("R", a, w.n_r).astype(k.dtype), k)
    np.testing.assert_array_equal(mk("S", b, w.n_s).astype(k.dtype), k)


@pytest.mark.slow
def test_m2_full_size_materialized(mgj):
    """M2 (2^29 x 2^29) with materialisation: closed forms + output properties."""
    n = 1 << 29
    w = datagen.M2()
    cols = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(4)]
    mgj.gen_relation("unique", 0, n, n, 0.0, 0, n, cols[0], cols[1])
    mgj.gen_relation("unique", 1, n, n, 0.0, 0, n, cols[2], cols[3])
    j = mgj.Join(mgj.make_config(r_capacity=n, s_capacity=n, materialize=True, out_capacity=n))
    res = j.run(*cols)
    assert res["match_count"] == n and res["n_materialized"] == n
    assert res["checksum"] == 0xf1fffffff0000000
    del cols
    _check_materialized_full(mgj, j, res, w)
    j.close()


@pytest.mark.slow
def test_m5_full_size_wide_materialized(mgj):
    """M5 per GPU (2^28 x 2^28 wide 8+8-byte tuples, full materialisation):
    closed-form count and checksum (C = 0x9E3779B97F4A7C15) + output properties."""
    n = 1 << 28
    w = datagen.Workload("wide", n, n)
    cols = [torch.empty(n, dtype=torch.int64, device="cuda") for _ in range(4)]
    mgj.gen_relation("wide", 0, n, n, 0.0, 0, n, cols[0], cols[1])
    mgj.gen_relation("wide", 1, n, n, 0.0, 0, n, cols[2], cols[3])
    j = mgj.Join(mgj.make_config(key_bytes=8, r_capacity=n, s_capacity=n, materialize=True, out_capacity=n))
    res = j.run(*cols)
    h = n * (n - 1) // 2
    assert res["match_count"] == n and res["n_materialized"] == n
    assert res["checksum"] == (0x9E3779B97F4A7C15 * (n * (1 << 40) + h) + n * (1 << 41) + h) & M64
    del cols
    _check_materialized_full(mgj, j, res, w)
    j.close()


@pytest.mark.slow
def test_m4_full_size_zipf(mgj):
    """M4 per GPU (|R| = 2^27 unique, |S| = 2^29 Zipf z = 1, 50% selectivity):
    every even S row matches R row r_j exactly once, odd rows never, so
    count = |S|/2 and checksum = sum over even j of (r_j * 2^32 + j).  r_j is
    found with plain torch indexing: R's keys are a permutation of [0, |R|),
    inverted on the device (inv[R.key[r]] = r, r_j = inv[S.key[j]])."""
    n_r, n_s, z = 1 << 27, 1 << 29, 1.0
    cols = [torch.empty(x, dtype=torch.int32, device="cuda") for x in (n_r, n_r, n_s, n_s)]
    mgj.gen_relation("zipf", 0, n_r, n_s, z, 0, n_r, cols[0], cols[1])
    mgj.gen_relation("zipf", 1, n_r, n_s, z, 0, n_s, cols[2], cols[3])
    j = mgj.Join(mgj.make_config(r_capacity=n_r, s_capacity=n_s))
    res = j.run(*cols)
    assert res["match_count"] == n_s // 2
    inv = torch.full((n_r,), -1, dtype=torch.int64, device="cuda")
    inv[cols[0].long()] = torch.arange(n_r, device="cuda")
    assert bool((inv >= 0).all())  # R keys are a permutation of [0, n_r)
    sk = cols[2][0::2].long()
    assert bool((sk < n_r).all()) and bool((cols[2][1::2].long() >= n_r).all())
    rank_sum = int(inv[sk].sum())
    m = n_s // 2
    assert res["checksum"] == ((rank_sum << 32) + m * (m - 1)) & M64
    # pair digest: Σ_{j even} r_j · j (odd rows never match); products < 2^56, int64 sums wrap mod 2^64
    rows = torch.arange(0, n_s, 2, device="cuda", dtype=torch.int64)
    assert res["pair_digest"] == int((inv[sk] * rows).sum()) & M64
    j.close()


# ------------------------------------------------------------ EXTERNAL (NCCL-baseline) shuffle
@pytest.mark.parametrize("N,kind,ba", [(1, "unique", 0), (2, "unique", 0), (4, "unique", 0), (3, "zipf", 0),
                                       (2, "wide", 0), (4, "unique", 3), (3, "zipf", 2)])
def test_external_shuffle_virtual_ranks(mgj, N, kind, ba):
    """shuffle_mode EXTERNAL: the library packs per-destination send buffers, the
    caller's all-to-all (emulated here with device copies, as NCCL
    all_to_all_single would do) fills the receive areas, mgj_join finishes."""
    w = {"unique": datagen.M1(), "zipf": datagen.Workload("zipf", 1 << 16, 1 << 18, 1.0),
         "wide": datagen.Workload("wide", 1 << 17, 1 << 17)}[kind]
    parts = [w.rank_inputs(g, N) for g in range(N)]
    cap_r = max(p["r_keys"].size for p in parts)
    cap_s = max(p["s_keys"].size for p in parts)
    cfgs = [mgj.make_config(rank=g, world_size=N, key_bytes=w.key_bytes, r_capacity=cap_r, s_capacity=cap_s,
                            recv_capacity_r=w.n_r, recv_capacity_s=w.n_s, shuffle_mode=mgj.SHUFFLE_EXTERNAL,
                            local_split_bits=ba, radix_bits_global=4 if ba else 0)
            for g in range(N)]
    nb = mgj.arena_bytes(cfgs[0])
    arenas = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(N)]
    ptrs = [a.data_ptr() for a in arenas]
    joins = [mgj.Join(cfgs[g], ptrs, nb) for g in range(N)]
    tens = [[dev(p[k]) for k in ("r_keys", "r_pays", "s_keys", "s_pays")] for p in parts]
    streams = [torch.cuda.Stream() for _ in range(N)]
    torch.cuda.synchronize()
    for g in range(N):
        joins[g].partition(*tens[g], stream=streams[g])
    for g in range(N):
        joins[g].shuffle(streams[g])
    lays = [j.exchange_layout() for j in joins]
    tb = lays[0]["tuple_bytes"]
    for rel in range(2):
        assert sum(sum(l["send_count"][rel]) for l in lays) == (w.n_r if rel == 0 else w.n_s)
        for g in range(N):
            so = 0
            for d in range(N):
                cnt = lays[g]["send_count"][rel][d]
                assert lays[d]["recv_count"][rel][g] == cnt
                ro = sum(lays[d]["recv_count"][rel][:g])
                mgj.device_bytes(lays[d]["recv"][rel] + ro * tb, cnt * tb).copy_(
                    mgj.device_bytes(lays[g]["send"][rel] + so * tb, cnt * tb))
                so += cnt
    torch.cuda.synchronize()
    for g in range(N):
        joins[g].join(streams[g])
    res = [joins[g].result() for g in range(N)]
    d = w.rank_inputs()
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    for r in res:
        assert (r["match_count"], r["checksum"], r["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    for j in joins:
        j.close()


# ------------------------------------------------------------ torchrun + symmetric memory
@pytest.mark.parametrize("mode", ["p2p", "nccl"])
def test_torchrun_symmetric_memory_path(mgj, mode):
    """bench.py under torchrun with MGJ_SYMM_ARENA=1: the real torch symmetric-memory
    arena (mgj.symmetric_join: symm_mem.empty + rendezvous) and, for mode nccl, the
    EXTERNAL shuffle with NCCL all_to_all_single (mgj.nccl_exchange), at N = 1."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, MGJ_SYMM_ARENA="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "1",
           "--master-addr", "127.0.0.1", "--master-port", str(29600 + (mode == "nccl")), "bench.py", "--gpus", "1",
           "--steps", "2", "--warmup", "3", "--no-cpu-baseline", "--no-e2e", "--log2-per-gpu", "22", "--shuffle", mode]
    out = subprocess.run(cmd, cwd=root, env=env, capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads(out.stdout.strip().splitlines()[-1])
    assert line["correct"] and line["match_count"] == 1 << 22


# ------------------------------------------------------------ the timed count-only probe path
def _set_keys(rng, n, pool):
    """n keys drawn uniformly from a pool of distinct u32 values."""
    return pool[rng.integers(0, pool.size, n)]


def _pool(rng, m):
    return np.unique(rng.integers(0, 1 << 32, 2 * m, dtype=np.uint64).astype(np.uint32))[:m]


@pytest.mark.parametrize("kind", ["pool256", "pool4096", "pool65536", "pool1M", "dense256", "edge",
                                  "zipf1", "zipf05", "stagefill"])
def test_timed_probe_path_parity(mgj, kind):
    """The bench's probe loop — count + checksum only, 4-byte keys, packed
    table (B1 + B2 = 10 + 6 >= 16) — against the oracle on duplicate-heavy,
    edge-key, Zipf and stage-filling inputs, with the pair digest (reading C3b)
    so that a wrong pairing of S with R rows cannot hide behind the linear
    checksum.  (§3.2 Probe.)"""
    rng = np.random.default_rng(abs(hash(kind)) % (1 << 32))
    if kind.startswith("pool"):  # duplicates spread over the whole key space
        m = {"pool256": 256, "pool4096": 4096, "pool65536": 65536, "pool1M": 1 << 20}[kind]
        pool = _pool(rng, m)
        nr, ns = 300007, 500009
        if m == 256:
            nr, ns = 40000, 60000  # ~156 x 234 pairs per key: keep the join small
        d = dict(r_keys=_set_keys(rng, nr, pool), s_keys=_set_keys(rng, ns, pool),
                 r_pays=rng.integers(0, 1 << 32, nr, dtype=np.uint64).astype(np.uint32),
                 s_pays=rng.integers(0, 1 << 32, ns, dtype=np.uint64).astype(np.uint32))
    elif kind == "dense256":  # keys 0..255: every co-partition is one key (khi = 0)
        nr, ns = 20000, 30000
        d = dict(r_keys=rng.integers(0, 256, nr, dtype=np.uint64).astype(np.uint32),
                 s_keys=rng.integers(0, 256, ns, dtype=np.uint64).astype(np.uint32),
                 r_pays=np.arange(nr, dtype=np.uint32), s_pays=np.arange(ns, dtype=np.uint32) * np.uint32(7))
    elif kind == "edge":
        edge = np.array([0, 1, 2, 3, 1023, 1024, 65535, 65536, 2**31 - 1, 2**31, 2**32 - 2, 2**32 - 1],
                        dtype=np.uint32)
        d = dict(r_keys=rng.choice(edge, 5000), s_keys=rng.choice(edge, 7000),
                 r_pays=rng.integers(0, 1 << 32, 5000, dtype=np.uint64).astype(np.uint32),
                 s_pays=rng.integers(0, 1 << 32, 7000, dtype=np.uint64).astype(np.uint32))
    elif kind.startswith("zipf"):
        d = datagen.Workload("zipf", 1 << 18, 1 << 20, 1.0 if kind == "zipf1" else 0.5).rank_inputs()
    else:  # stagefill: 8 co-partitions (low 16 bits fixed) of ~3000-5000 distinct R keys each
        los = rng.choice(1 << 16, 8, replace=False).astype(np.uint32)
        rk, sk = [], []
        for i, lo in enumerate(los):
            hi = rng.choice(1 << 16, 3000 + 300 * i, replace=False).astype(np.uint32)
            r = (hi << np.uint32(16)) | lo
            rk.append(r)
            miss = (rng.integers(0, 1 << 16, 2000, dtype=np.uint64).astype(np.uint32) << np.uint32(16)) | lo
            sk.append(np.concatenate([r[rng.integers(0, r.size, 2500 + 500 * i)], miss]))
        rk, sk = np.concatenate(rk), np.concatenate(sk)
        rng.shuffle(rk)
        rng.shuffle(sk)
        d = dict(r_keys=rk, s_keys=sk, r_pays=np.arange(rk.size, dtype=np.uint32),
                 s_pays=(np.arange(sk.size, dtype=np.uint32) * np.uint32(2654435761)))
    res = check_vs_oracle(mgj, d, materialize=False, radix_bits_global=10, radix_bits_local=6)
    assert res["radix_bits_local"] == 6 and res["status"] == 0


@pytest.mark.parametrize("log2n", [22, 24])
def test_auto_b2_count_only_parity(mgj, log2n):
    """Count-only joins with the automatically chosen B2 (the bench's
    configuration at smaller sizes), unique and duplicate keys, vs the oracle."""
    n = 1 << log2n
    d = datagen.Workload("unique", n, n).rank_inputs()
    check_vs_oracle(mgj, d, materialize=False)
    rng = np.random.default_rng(log2n)
    pool = _pool(rng, n // 8)
    d = dict(r_keys=_set_keys(rng, n // 2, pool), s_keys=_set_keys(rng, n, pool),
             r_pays=rng.integers(0, 1 << 32, n // 2, dtype=np.uint64).astype(np.uint32),
             s_pays=rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32))
    check_vs_oracle(mgj, d, materialize=False)


def _device_pair_digest_unique(r_keys, s_keys, s_pays, n_r):
    """Σ_j a(j)·b_j mod 2^64 for a unique-key R with payload = row id, by plain
    torch indexing (no join code): inv[R.key[i]] = i, a(j) = inv[S.key[j]]."""
    inv = torch.full((n_r,), -1, dtype=torch.int64, device="cuda")
    inv[r_keys.long() & 0xFFFFFFFF] = torch.arange(n_r, device="cuda")
    assert bool((inv >= 0).all())
    a = inv[s_keys.long() & 0xFFFFFFFF]
    b = s_pays.long() & 0xFFFFFFFF
    # products < 2^64 / 2 here (a, b < 2^31); torch int64 sums wrap modulo 2^64
    return int((a * b).sum()) & M64


@pytest.mark.slow
def test_auto_b2_packed_count_only_2p28(mgj):
    """2^28 x 2^28 unique keys, auto B1/B2 (B1 + B2 >= 16 from 2^28 per relation:
    the packed count-only loop the bench times): closed-form count/checksum and
    the pair digest by device inverse permutation."""
    n = 1 << 28
    cols = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(4)]
    mgj.gen_relation("unique", 0, n, n, 0.0, 0, n, cols[0], cols[1])
    mgj.gen_relation("unique", 1, n, n, 0.0, 0, n, cols[2], cols[3])
    j = mgj.Join(mgj.make_config(r_capacity=n, s_capacity=n))
    res = j.run(*cols)
    assert res["radix_bits_global"] + res["radix_bits_local"] >= 16
    assert res["match_count"] == n
    assert res["checksum"] == ((1 << 32) + 1) * n * (n - 1) // 2 & M64
    assert res["pair_digest"] == _device_pair_digest_unique(cols[0], cols[2], cols[3], n)
    j.close()


# ------------------------------------------------------------ error paths (peers, config, items)
def test_peer_timeout_epeer(mgj):
    """A peer that never partitions: every wait of rank 0 is bounded
    (peer_timeout_ms) and the run reports MGJ_EPEER instead of hanging."""
    n, N = 4096, 2
    cfgs = [mgj.make_config(rank=g, world_size=N, r_capacity=n, s_capacity=n, recv_capacity_r=2 * n,
                            recv_capacity_s=2 * n, peer_timeout_ms=200) for g in range(N)]
    nb = mgj.arena_bytes(cfgs[0])
    arenas = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(N)]
    ptrs = [a.data_ptr() for a in arenas]
    joins = [mgj.Join(cfgs[g], ptrs, nb) for g in range(N)]
    d = datagen.Workload("unique", n, n).rank_inputs()
    t = [dev(d[k]) for k in ("r_keys", "r_pays", "s_keys", "s_pays")]
    s0 = torch.cuda.Stream()
    torch.cuda.synchronize()
    joins[0].partition(*t, stream=s0)
    joins[0].shuffle(s0)
    joins[0].join(s0)
    with pytest.raises(mgj.MGJError) as e:
        joins[0].result()
    assert e.value.status == -7  # EPEER
    for j in joins:
        j.close()


def test_config_mismatch_across_ranks(mgj):
    """Receive capacities are job-wide (mgj.h): ranks that planned with
    different ones are detected by k_plan and the run fails with MGJ_EINVAL."""
    n, N = 4096, 2
    cfgs = [mgj.make_config(rank=g, world_size=N, r_capacity=n, s_capacity=n, recv_capacity_r=(g + 2) * n,
                            recv_capacity_s=2 * n) for g in range(N)]
    nb = max(mgj.arena_bytes(c) for c in cfgs)
    arenas = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(N)]
    ptrs = [a.data_ptr() for a in arenas]
    joins = [mgj.Join(cfgs[g], ptrs, nb) for g in range(N)]
    w = datagen.Workload("unique", 2 * n, 2 * n)
    parts = [w.rank_inputs(g, N) for g in range(N)]
    tens = [[dev(p[k]) for k in ("r_keys", "r_pays", "s_keys", "s_pays")] for p in parts]
    streams = [torch.cuda.Stream() for _ in range(N)]
    torch.cuda.synchronize()
    for g in range(N):
        joins[g].partition(*tens[g], stream=streams[g])
    for g in range(N):
        joins[g].shuffle(streams[g])
    for g in range(N):
        joins[g].join(streams[g])
    for g in range(N):
        assert joins[g].result(check=False)["status"] == -1  # EINVAL
    for j in joins:
        j.close()


def test_item_overflow_is_clean_ecapacity(mgj):
    """A single key on both sides (2^20 x 2^20, count-only): the block nested
    loop needs more probe items than the handle holds.  The run must end with
    MGJ_ECAPACITY (the probe never reads reserved-but-unwritten items), and the
    handle must still join correctly afterwards."""
    n = 1 << 20
    cfg = mgj.make_config(r_capacity=n, s_capacity=n)
    j = mgj.Join(cfg)
    k = torch.full((n,), 0x1234567, dtype=torch.int32, device="cuda")
    p = torch.arange(n, dtype=torch.int32, device="cuda")
    j.partition(k, p, k, p)
    j.shuffle()
    j.join()
    r = j.result(check=False)
    assert r["status"] in (0, -6)
    if r["status"] == 0:
        assert r["match_count"] == n * n
    d = datagen.Workload("unique", n, n).rank_inputs()
    res = j.run(*[dev(d[x]) for x in ("r_keys", "r_pays", "s_keys", "s_pays")])
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    assert (res["match_count"], res["checksum"], res["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    j.close()


def test_torchrun_parity_all_gpus(mgj):
    """One process per visible GPU under torchrun (nproc = torch.cuda.device_count(),
    1 on a one-GPU box): M1 split N ways through the symmetric-memory peer path,
    bit-exact against the oracle (count, checksum, pair digest, sorted triples)."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    n = max(1, torch.cuda.device_count())
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(n),
           "--master-addr", "127.0.0.1", "--master-port", "29613", os.path.join(root, "tests", "torchrun_parity_worker.py")]
    out = subprocess.run(cmd, cwd=root, capture_output=True, text=True, timeout=900)
    assert out.returncode == 0, out.stderr[-3000:]
    line = json.loads([l for l in out.stdout.splitlines() if l.startswith("{")][-1])
    assert line["ok"] and line["world"] == n and line["count"] == 1 << 20


# ------------------------------------------------------------ §8(e): shuffle overlapped with the local pass
@pytest.mark.parametrize("N,mat", [(1, True), (2, True), (4, False), (8, True)])
def test_overlap_parity(mgj, N, mat):
    """R's local pass on a second stream beside S's scatter (shuffle_overlap =
    1; auto for N > 1), N virtual ranks: bit-exact vs the oracle."""
    w = datagen.Workload("unique", 300007, 400009)
    joins, res, _ = run_virtual(mgj, w, N, materialize=mat, shuffle_overlap=1, overlap_local_sms=37)
    d = w.rank_inputs()
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"], materialize=mat)
    for r in res:
        assert r["status"] == 0
        assert (r["match_count"], r["checksum"], r["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    if mat:
        trip = [j.materialized(r) for j, r in zip(joins, res)]
        k, a, b = sort_trip(*(np.concatenate([t[i] for t in trip]) for i in range(3)))
        np.testing.assert_array_equal(k, ref["key"])
        np.testing.assert_array_equal(a, ref["pay_r"])
        np.testing.assert_array_equal(b, ref["pay_s"])
    for j in joins:
        j.close()


def test_overlap_timeline(mgj):
    """The kernel timeline (trace=1) of one rank with the overlap on: R's local
    pass runs while S is still being scattered, and S's local pass starts
    only after S's scatter; without the overlap the two never coincide."""
    n = 1 << 24
    cols = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(4)]
    mgj.gen_relation("unique", 0, n, n, 0.0, 0, n, cols[0], cols[1])
    mgj.gen_relation("unique", 1, n, n, 0.0, 0, n, cols[2], cols[3])
    for ov in (1, -1):
        j = mgj.Join(mgj.make_config(r_capacity=n, s_capacity=n, shuffle_overlap=ov, trace=True))
        res = j.run(*cols)
        assert res["match_count"] == n
        t = j.trace()
        if ov == 1:
            assert t["local_R"][0] < t["scatter_S"][1] and t["scatter_S"][0] < t["local_R"][1], t
            assert t["local_S"][0] >= t["scatter_S"][1], t
        else:  # one launch over both relations after both scatters (not stamped)
            assert "local_R" not in t and t["itemize"][0] >= t["scatter_S"][1], t
        j.close()


# ------------------------------------------------------------ NEXT-3: chunk streaming
@pytest.mark.parametrize("N,kind,kw", [(1, "unique", {}), (2, "unique", {"materialize": True}), (4, "unique", {}),
                                       (8, "unique", {"materialize": True}), (3, "zipf", {"skew_bcast": 1}),
                                       (2, "m1", {"compress": True, "materialize": True}), (4, "m1", {"compress": True}),
                                       (2, "wide", {"materialize": True}), (1, "unique", {"radix_bits_global": 4}),
                                       (1, "unique", {"radix_bits_global": 1}), (2, "unique", {"radix_bits_global": 2}),
                                       (2, "unique", {"local_split_bits": 2})])
def test_stream_parity(mgj, N, kind, kw):
    """shuffle_overlap = 2: S's local pass
    runs beside S's scatter and starts every chunk once the scatter rounds that
    fill it are complete at its source rank.  Bit-exact vs the oracle (count,
    checksum, pair digest; sorted triples when materialised) on N virtual
    ranks, with broadcast, compression, 8-byte keys, small P and the
    two-level local pass (which then runs after the shuffle, unstreamed)."""
    w = {"unique": datagen.Workload("unique", 300007, 400009), "m1": datagen.M1(),
         "zipf": datagen.Workload("zipf", 1 << 16, 1 << 18, 1.0),
         "wide": datagen.Workload("wide", 200003, 300007)}[kind]
    kw = dict(kw)
    mat = kw.pop("materialize", False)
    joins, res, _ = run_virtual(mgj, w, N, materialize=mat, shuffle_overlap=2, **kw)
    d = w.rank_inputs()
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"], materialize=mat)
    for r in res:
        assert r["status"] == 0
        assert (r["match_count"], r["checksum"], r["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    if mat:
        trip = [j.materialized(r) for j, r in zip(joins, res)]
        k, a, b = sort_trip(*(np.concatenate([t[i] for t in trip]) for i in range(3)))
        np.testing.assert_array_equal(k, ref["key"])
        np.testing.assert_array_equal(a, ref["pay_r"])
        np.testing.assert_array_equal(b, ref["pay_s"])
    for j in joins:
        j.close()


def test_stream_repeated_runs(mgj):
    """The round counters carry the run's epoch: three runs of one plan with
    different S sizes (so different non-empty tiles per round), 2 virtual ranks."""
    N = 2
    cap = 1 << 18
    cfgs = [mgj.make_config(rank=g, world_size=N, r_capacity=cap, s_capacity=cap, recv_capacity_r=2 * cap,
                            recv_capacity_s=2 * cap, shuffle_overlap=2) for g in range(N)]
    nb = mgj.arena_bytes(cfgs[0])
    arenas = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(N)]
    joins = [mgj.Join(cfgs[g], [a.data_ptr() for a in arenas], nb) for g in range(N)]
    streams = [torch.cuda.Stream() for _ in range(N)]
    for n_s in (cap, 1000, 77777):
        w = datagen.Workload("unique", cap, n_s)
        parts = [w.rank_inputs(g, N) for g in range(N)]
        tens = [[dev(p[k]) for k in ("r_keys", "r_pays", "s_keys", "s_pays")] for p in parts]
        torch.cuda.synchronize()
        for g in range(N):
            joins[g].partition(*tens[g], stream=streams[g])
        for g in range(N):
            joins[g].shuffle(streams[g])
        for g in range(N):
            joins[g].join(streams[g])
        res = [joins[g].result() for g in range(N)]
        d = w.rank_inputs()
        ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
        for r in res:
            assert r["status"] == 0
            assert (r["match_count"], r["checksum"], r["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    for j in joins:
        j.close()


def test_stream_timeline(mgj):
    """With chunk streaming (one rank, trace=1) S's local pass starts while S
    is still being scattered — unlike shuffle_overlap = 1, where it starts
    after S's scatter (test_overlap_timeline) — and the result is exact."""
    n = 1 << 24
    cols = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(4)]
    mgj.gen_relation("unique", 0, n, n, 0.0, 0, n, cols[0], cols[1])
    mgj.gen_relation("unique", 1, n, n, 0.0, 0, n, cols[2], cols[3])
    j = mgj.Join(mgj.make_config(r_capacity=n, s_capacity=n, shuffle_overlap=2, trace=True))
    for _ in range(2):
        res = j.run(*cols)
        assert res["match_count"] == n and res["status"] == 0
    t = j.trace()
    assert t["local_R"][0] < t["scatter_S"][1], t
    assert t["local_S"][0] < t["scatter_S"][1], t
    j.close()


# ------------------------------------------------------------ NEXT-1: the compressed shuffle
@pytest.mark.parametrize("N,kind,kw", [(1, "m1", {}), (2, "m1", {}), (4, "m1", {}), (1, "m1", {"radix_bits_global": 4}),
                                       (3, "zipf", {}), (4, "zipf", {"skew_bcast": 1, "radix_bits_global": 8}),
                                       (2, "m1", {"shuffle_overlap": 1}), (1, "m1", {"radix_bits_global": 10,
                                                                                     "radix_bits_local": 6})])
def test_compress_parity(mgj, N, kind, kw):
    """compress = 1: tuples cross the shuffle as
    (key >> B1, row offset in the source tile) entries, five per 32-byte unit;
    the local pass rebuilds key and id payload.  Bit-exact vs the oracle
    (count, checksum, pair digest, sorted triples) on N virtual ranks."""
    w = datagen.M1() if kind == "m1" else datagen.Workload("zipf", 1 << 16, 1 << 18, 1.0)
    mat = kind == "m1"
    joins, res, _ = run_virtual(mgj, w, N, materialize=mat, compress=True, **kw)
    d = w.rank_inputs()
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"], materialize=mat)
    for r in res:
        assert r["status"] == 0
        assert (r["match_count"], r["checksum"], r["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    if mat:
        trip = [j.materialized(r) for j, r in zip(joins, res)]
        k, a, b = sort_trip(*(np.concatenate([t[i] for t in trip]) for i in range(3)))
        np.testing.assert_array_equal(k, ref["key"])
        np.testing.assert_array_equal(a, ref["pay_r"])
        np.testing.assert_array_equal(b, ref["pay_s"])
    # the receive buffers hold 32-byte units of at most five tuples, at least one each (at this
    # size most (tile, partition) runs are a few tuples, so units are far from full; M2: below)
    tot_units = sum(r["recv_r"] + r["recv_s"] for r in res)
    assert (w.n_r + w.n_s) / 5 <= tot_units <= w.n_r + w.n_s
    for j in joins:
        j.close()


def test_compress_rejects_non_id_payloads(mgj):
    """The compressed shuffle rebuilds payloads from row ids; a payload that is
    not its global row id fails the run with MGJ_EINVAL instead of a wrong join."""
    n = 1 << 16
    d = datagen.Workload("unique", n, n).rank_inputs()
    d["s_pays"] = d["s_pays"].copy()
    d["s_pays"][12345] += np.uint32(1)
    cfg = mgj.make_config(r_capacity=n, s_capacity=n, compress=True)
    j = mgj.Join(cfg)
    j.partition(*[dev(d[k]) for k in ("r_keys", "r_pays", "s_keys", "s_pays")])
    j.shuffle()
    j.join()
    assert j.result(check=False)["status"] == -1
    j.close()


@pytest.mark.slow
def test_compress_full_size_m2(mgj):
    """M2 at one GPU (2^29 x 2^29) through the compressed shuffle: closed-form
    count and checksum, pair digest by device inverse permutation."""
    n = 1 << 29
    cols = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(4)]
    mgj.gen_relation("unique", 0, n, n, 0.0, 0, n, cols[0], cols[1])
    mgj.gen_relation("unique", 1, n, n, 0.0, 0, n, cols[2], cols[3])
    j = mgj.Join(mgj.make_config(r_capacity=n, s_capacity=n, compress=True))
    res = j.run(*cols)
    assert res["match_count"] == n
    assert res["checksum"] == 0xf1fffffff0000000
    assert res["pair_digest"] == _device_pair_digest_unique(cols[0], cols[2], cols[3], n)
    assert (res["recv_r"] + res["recv_s"]) * 32 < 6.5 * 2 * n  # bytes in the receive buffers
    j.close()


# ------------------------------------------------------------ NEXT-2: placement-aware assignment
class PlacedWorkload:
    """Global R and S (unique keys, ids) whose tuples sit on rank key % N with
    probability `alpha`, on a random rank otherwise (placement skew)."""

    def __init__(self, n, N, alpha, seed=5):
        w = datagen.Workload("unique", n, n)
        self.a = w.rank_inputs()
        self.n_r = self.n_s = n
        self.key_bytes = 4
        rng = np.random.default_rng(seed)
        self.where = {}
        for rel in ("r", "s"):
            k = self.a[rel + "_keys"]
            pref = (k % N).astype(np.int64)
            rnd = rng.integers(0, N, k.size)
            self.where[rel] = np.where(rng.random(k.size) < alpha, pref, rnd)

    def rank_inputs(self, rank=0, world=1):
        if world == 1:
            return dict(self.a)
        out = {}
        for rel in ("r", "s"):
            m = self.where[rel] == rank
            out[rel + "_keys"] = self.a[rel + "_keys"][m].copy()
            out[rel + "_pays"] = self.a[rel + "_pays"][m].copy()
        return out


def _moved_tuples(owner, mail):
    """Tuples that leave their rank under owner[] (mail: [N][2][P] histograms)."""
    N = mail.shape[0]
    return int(sum(mail[g, :, owner != g].sum() for g in range(N)))


@pytest.mark.parametrize("N", [2, 4])
def test_placement_aware_assignment(mgj, N):
    """assign = 1 (Track-Join migration): partitions go where most
    of their tuples already are.  Exact vs the oracle either way; the device
    plan equals the host plan; with placement skew (80% of each partition's
    tuples on one rank) far fewer tuples cross ranks than with ranges."""
    w = PlacedWorkload(1 << 18, N, 0.8)
    d = w.rank_inputs()
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"], materialize=True)
    moved = {}
    for assign in (0, 1):
        joins, res, _ = run_virtual(mgj, w, N, materialize=True, assign=assign, radix_bits_global=8)
        for r in res:
            assert r["status"] == 0
            assert (r["match_count"], r["checksum"], r["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
        trip = [j.materialized(r) for j, r in zip(joins, res)]
        k, a, b = sort_trip(*(np.concatenate([t[i] for t in trip]) for i in range(3)))
        np.testing.assert_array_equal(k, ref["key"])
        np.testing.assert_array_equal(b, ref["pay_s"])
        P = 1 << 8
        mail = joins[0].debug("MAIL_HIST", np.uint32).reshape(N, 2, P)
        owner = joins[0].debug("OWNER", np.int32)
        for g, j in enumerate(joins):
            o, send_off, recv_size = mgj.plan_host(N, g, 8, mail, assign=assign)
            np.testing.assert_array_equal(j.debug("OWNER", np.int32), o)
            np.testing.assert_array_equal(j.debug("SEND_OFF", np.uint64).reshape(2, P), send_off)
            assert res[g]["recv_r"] == recv_size[0, g] and res[g]["recv_s"] == recv_size[1, g]
        moved[assign] = _moved_tuples(owner, mail.astype(np.int64))
        if assign:  # the receive load stays within 9/8 of the mean (+ one partition)
            load = np.array([r["recv_r"] + r["recv_s"] for r in res])
            assert load.max() <= load.mean() * 9 / 8 + 2 * (w.n_r + w.n_s) / P
        for j in joins:
            j.close()
    assert moved[1] < 0.5 * moved[0], moved


@pytest.mark.parametrize("N,assign", [(4, 0), (4, 1), (8, 1)])
def test_zipf_placement_parity(mgj, N, assign):
    """Fig. 9's reading of Zipf as placement skew: rank g holds a
    1/(g+1) share of the rows (z = 1).  Exact vs the oracle with range and
    placement-aware assignment; the receive loads stay balanced."""
    w = datagen.Workload("unique", 1 << 19, 1 << 19, placement_z=1.0)
    joins, res, _ = run_virtual(mgj, w, N, materialize=False, assign=assign)
    d = w.rank_inputs()
    ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    for r in res:
        assert r["status"] == 0
        assert (r["match_count"], r["checksum"], r["pair_digest"]) == (ref["count"], ref["checksum"], ref["pair_digest"])
    load = np.array([r["recv_r"] + r["recv_s"] for r in res], dtype=np.float64)
    assert load.max() <= load.mean() * 1.2
    for j in joins:
        j.close()
