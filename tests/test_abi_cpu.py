"""CPU-only checks of the C ABI: the library loads, exports every symbol its
headers declare, rejects bad configs before touching CUDA, and its host plan
(a2) obeys the partitioning invariants."""
import ctypes
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def mgj():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_sigmod_paullhl21_b200 import mgj as m
    return m


def declared_functions():
    names = set()
    for f in os.listdir(os.path.join(ROOT, "include")):
        src = open(os.path.join(ROOT, "include", f)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        for m in re.finditer(r"^\s*(?:const\s+)?[\w\s\*]+?\b(mgj_\w+)\s*\(", src, flags=re.M):
            names.add(m.group(1))
    return names


def test_all_declared_symbols_exported(mgj):
    names = declared_functions()
    assert {"mgj_plan", "mgj_partition", "mgj_shuffle", "mgj_join", "mgj_result", "mgj_destroy",
            "mgj_strerror", "mgj_arena_bytes", "mgj_plan_host", "mgj_gen_relation", "mgj_debug_copy"} <= names
    lib = ctypes.CDLL(mgj.LIB_PATH)
    for n in names:
        assert hasattr(lib, n), n
    assert set(mgj.EXPORTED) == names


def test_strerror(mgj):
    for st in range(-7, 1):
        assert mgj._lib.mgj_strerror(st)


@pytest.mark.parametrize("bad", [dict(key_bytes=3), dict(world_size=0), dict(world_size=9), dict(rank=2, world_size=2),
                                 dict(radix_bits_global=13), dict(radix_bits_local=12), dict(r_capacity=1 << 32),
                                 dict(local_split_bits=7), dict(local_split_bits=-2), dict(skew_bcast=2),
                                 dict(skew_bcast=-2), dict(peer_timeout_ms=-1), dict(shuffle_overlap=3),
                                 dict(shuffle_overlap=2, shuffle_mode=1),
                                 dict(shuffle_overlap=-2), dict(overlap_local_sms=-1),
                                 dict(compress=1, key_bytes=8), dict(compress=1, shuffle_mode=1),
                                 dict(compress=1, radix_bits_global=11), dict(assign=2), dict(assign=1, shuffle_mode=1)])
def test_invalid_config_rejected_without_gpu(mgj, bad):
    kw = dict(r_capacity=1024, s_capacity=1024)
    kw.update(bad)
    cfg = mgj.make_config(**kw)
    assert mgj.arena_bytes(cfg) == 0
    h = ctypes.c_void_p()
    assert mgj._lib.mgj_plan(ctypes.byref(cfg), None, ctypes.byref(h)) == -1
    assert not h.value


def test_reserved_must_be_zero(mgj):
    cfg = mgj.make_config(r_capacity=10, s_capacity=10)
    cfg.reserved[0] = 1
    assert mgj.arena_bytes(cfg) == 0


def test_multi_rank_plan_needs_peers(mgj):
    cfg = mgj.make_config(rank=0, world_size=2, r_capacity=10, s_capacity=10)
    h = ctypes.c_void_p()
    assert mgj._lib.mgj_plan(ctypes.byref(cfg), None, ctypes.byref(h)) == -1


def test_arena_layout_size(mgj):
    cfg = mgj.make_config(r_capacity=1 << 20, s_capacity=1 << 20)
    nb = mgj.arena_bytes(cfg)
    assert 2 * 8 * (1 << 20) <= nb <= 2 * 8 * (1 << 20) + (1 << 20)


def check_plan_invariants(mgj, hist, bits, skew_bcast=0, assign=0):
    """Every rank computes the same plan; for each destination d and relation, the
    (source rank, partition) ranges the plan sends to d tile [0, recv_size[d]) exactly.
    A selectively broadcast partition (NEXT-2) sends R to its owner (the root) and
    keeps each rank's S at that rank."""
    N = hist.shape[0]
    P = 1 << bits
    plans = [mgj.plan_host(N, g, bits, hist, skew_bcast=skew_bcast, with_bcast=True, assign=assign) for g in range(N)]
    owner, recv, bc, skip = plans[0][0], plans[0][2], plans[0][3], plans[0][4]
    for o, _, rs, b, sk in plans:  # every rank computes the same assignment
        assert np.array_equal(o, owner) and np.array_equal(rs, recv) and np.array_equal(b, bc)
        assert np.array_equal(sk, skip)
    tot = hist.astype(np.uint64).sum(axis=0)  # [2][P]
    # the histogram as a Bloom filter: exactly the partitions with one empty side
    np.testing.assert_array_equal(skip != 0, (tot[0] == 0) != (tot[1] == 0))
    assert not (bc.astype(bool) & skip.astype(bool)).any()
    assert owner.min() >= 0 and owner.max() < N
    if not assign:  # contiguous ranges
        assert np.all(np.diff(owner) >= 0)
    if N == 1 or skew_bcast < 0:
        assert not bc.any()
    for rel in range(2):
        assert int(recv[rel].sum()) == int(tot[rel][skip == 0].sum())
        for d in range(N):
            cover = np.zeros(int(recv[rel, d]), np.int32)
            for g in range(N):
                so = plans[g][1][rel]
                for p in range(P):
                    dest = g if (rel == 1 and bc[p]) else owner[p]
                    if dest != d or skip[p]:
                        continue
                    c = int(hist[g, rel, p])
                    cover[int(so[p]):int(so[p]) + c] += 1
            assert np.all(cover == 1)
    return owner, recv, bc, skip


@pytest.mark.parametrize("N", [1, 2, 3, 5, 8])
def test_plan_host_invariants_random(mgj, N):
    rng = np.random.default_rng(N)
    bits = 6
    hist = rng.integers(0, 50, size=(N, 2, 1 << bits)).astype(np.uint32)
    hist[:, :, 5] = 0  # empty partitions
    hist[:, 0, 9] = 0  # no R tuple: partition 9's S is never shuffled
    hist[:, 1, 11] = 0  # no S tuple: partition 11's R neither
    _, _, _, skip = check_plan_invariants(mgj, hist, bits)
    assert skip[9] and skip[11] and not skip[5]
    check_plan_invariants(mgj, hist, bits, skew_bcast=-1)
    hist[:, 1, 7] *= 40  # heavy S partitions: broadcast candidates
    hist[:, 1, 40] = 5000
    _, _, bc, _ = check_plan_invariants(mgj, hist, bits)
    assert bc[40] == (N > 1)
    check_plan_invariants(mgj, hist, bits, skew_bcast=1)


def test_plan_host_uniform_identity_ranges(mgj):
    N, bits = 8, 10
    hist = np.full((N, 2, 1 << bits), 64, np.uint32)
    owner, recv, bc, _ = check_plan_invariants(mgj, hist, bits)
    assert not bc.any()  # uniform data never broadcasts
    assert np.array_equal(owner, np.arange(1 << bits) * N >> bits)
    assert np.all(recv == 64 * N * (1 << bits) // N)


def test_plan_host_skew_balances(mgj):
    """One heavy partition: owner ranges cut on cumulative counts (P:418-444 reduced form)."""
    N, bits = 4, 8
    hist = np.full((N, 2, 1 << bits), 10, np.uint32)
    hist[:, 1, 200] = 5000
    owner, recv, _, _ = check_plan_invariants(mgj, hist, bits, skew_bcast=-1)
    assert owner[200] in (2, 3)
    # partitions below the heavy one spread over the other owners
    assert len(set(owner[:200].tolist())) >= 2


def test_plan_host_selective_broadcast(mgj):
    """NEXT-2 (P:418-444 Track-Join benefit test, P:386-395 heavy hitters): a heavy S
    partition with small R is broadcast: R to its root only (read by every rank), each
    rank keeps its own S; the heavy partition no longer loads one owner."""
    N, bits = 4, 8
    P = 1 << bits
    hist = np.full((N, 2, P), 10, np.uint32)
    hist[:, 1, 200] = 5000
    owner, recv, bc, _ = check_plan_invariants(mgj, hist, bits)
    assert bc.sum() == 1 and bc[200]
    # S receive sizes: every rank holds its own 5000 S tuples of partition 200
    s_range = [sum(10 * N for p in range(P) if owner[p] == d and not bc[p]) for d in range(N)]
    assert [int(x) for x in recv[1]] == [s_range[d] + 5000 for d in range(N)]
    # the owner ranges are balanced on R + S/N for the broadcast partition
    w = hist.astype(np.int64).sum(axis=0)
    load = [int(w[0][owner == d].sum()) + int(w[1][(owner == d) & (bc == 0)].sum()) for d in range(N)]
    assert max(load) - min(load) <= 2 * 20 * N + 5000
    # auto mode leaves the same partition alone when R is not small: (N-1)|R_p| >= |S_p|
    hist[:, 0, 200] = 2000
    _, _, bc2, _ = check_plan_invariants(mgj, hist, bits)
    assert not bc2.any()


def test_plan_host_all_empty(mgj):
    hist = np.zeros((4, 2, 1 << 5), np.uint32)
    owner, recv, _, _ = check_plan_invariants(mgj, hist, 5)
    assert np.array_equal(owner, np.arange(32) * 4 // 32)


@pytest.mark.parametrize("N", [2, 3, 5, 8])
def test_plan_host_placement_aware(mgj, N):
    """assign = 1: the same tiling invariants with non-contiguous owners; a partition
    whose tuples mostly sit on one rank is assigned there while loads allow."""
    rng = np.random.default_rng(10 + N)
    bits = 6
    P = 1 << bits
    hist = rng.integers(0, 20, size=(N, 2, P)).astype(np.uint32)
    for p in range(P):  # partition p lives mostly on rank p % N
        hist[p % N, :, p] += 200
    owner, recv, bc, skip = check_plan_invariants(mgj, hist, bits, assign=1)
    assert np.mean(owner == np.arange(P) % N) > 0.9
    check_plan_invariants(mgj, hist, bits, assign=1, skew_bcast=1)
    load = recv.sum(axis=0)
    assert load.max() <= load.mean() * 9 / 8 + hist.sum(axis=(0, 1)).max()
