"""Pins for the CPU oracle (oracle/oracle.c) against things other than itself.

Each pin would catch a plausible oracle bug: a dropped duplicate (brute force,
multiplicity sums), a swapped a/b or missing 2^32 factor in the checksum
(closed forms, golden), a truncated 8-byte key (high-bits golden case), a bad
sort (brute-force triples), an off-by-one on empty inputs (golden), a pair
digest that sums a+b or a*a instead of a*b, or pairs S rows with the wrong R
row (Σ i(n-1-i) closed form, per-key group-sum products, brute force).
"""
import json
import os

import numpy as np
import pytest

import oracle
from paper_conf_sigmod_paullhl21_b200 import datagen

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
M64 = (1 << 64) - 1


def brute_force(rk, ra, sk, sb, wide=False):
    """Nested-loop definition of the bag equi-join via numpy broadcasting."""
    C = oracle.C_WIDE if wide else 1 << 32
    if rk.size == 0 or sk.size == 0:
        return 0, 0, []
    i, j = np.nonzero(rk[:, None] == sk[None, :])
    trip = [(int(sk[jj]), int(ra[ii]), int(sb[jj])) for ii, jj in zip(i, j)]
    trip.sort()
    checksum = sum(a * C + b for _, a, b in trip) & M64
    return len(trip), checksum, trip


def brute_digest(trip):
    """Pair digest (reading C3b) of brute-force triples: Σ a·b mod 2^64, Python integers."""
    return sum(a * b for _, a, b in trip) & M64


def check_against_brute(rk, ra, sk, sb, wide=False):
    cnt, chk, trip = brute_force(rk, ra, sk, sb, wide)
    got = oracle.join(rk, ra, sk, sb, materialize=True)
    assert got["count"] == cnt
    assert got["checksum"] == chk
    assert got["pair_digest"] == brute_digest(trip)
    gt = list(zip(got["key"].tolist(), got["pay_r"].tolist(), got["pay_s"].tolist()))
    assert gt == trip


@pytest.mark.parametrize("seed", range(6))
def test_oracle_vs_bruteforce_duplicates(seed):
    rng = np.random.default_rng(seed)
    nr, ns = rng.integers(0, 3000, size=2)
    dom = [1, 2, 17, 64, 4096, 1 << 32][seed]
    rk = rng.integers(0, dom, nr, dtype=np.uint64).astype(np.uint32)
    sk = rng.integers(0, dom, ns, dtype=np.uint64).astype(np.uint32)
    ra = rng.integers(0, 1 << 32, nr, dtype=np.uint64).astype(np.uint32)
    sb = rng.integers(0, 1 << 32, ns, dtype=np.uint64).astype(np.uint32)
    if dom <= 2:  # keep the all-equal case's output small
        rk, ra, sk, sb = rk[:200], ra[:200], sk[:300], sb[:300]
    check_against_brute(rk, ra, sk, sb)


def test_oracle_vs_bruteforce_edge_keys():
    edge = np.array([0, 1, 2**31 - 1, 2**31, 2**32 - 2, 2**32 - 1], dtype=np.uint32)
    rng = np.random.default_rng(7)
    rk = rng.choice(edge, 500)
    sk = rng.choice(edge, 700)
    ra = np.arange(500, dtype=np.uint32) + np.uint32(2**32 - 600)  # wrap-around payloads
    sb = np.arange(700, dtype=np.uint32)
    check_against_brute(rk, ra, sk, sb)


def test_oracle_empty_and_disjoint():
    e = np.empty(0, np.uint32)
    a = np.arange(10, dtype=np.uint32)
    for rk, ra, sk, sb in [(e, e, a, a), (a, a, e, e), (e, e, e, e), (a, a, a + 10, a)]:
        check_against_brute(rk, ra, sk, sb)


@pytest.mark.parametrize("seed", range(3))
def test_oracle_wide_vs_bruteforce(seed):
    rng = np.random.default_rng(100 + seed)
    low = rng.integers(0, 8, 1500, dtype=np.uint64)
    rk = (rng.integers(0, 4, 1500, dtype=np.uint64) << np.uint64(32)) | low
    low2 = rng.integers(0, 8, 1200, dtype=np.uint64)
    sk = (rng.integers(0, 4, 1200, dtype=np.uint64) << np.uint64(32)) | low2
    ra = rng.integers(0, 2**63, 1500, dtype=np.uint64) * np.uint64(2)
    sb = rng.integers(0, 2**63, 1200, dtype=np.uint64)
    check_against_brute(rk, ra, sk, sb, wide=True)


def test_oracle_golden_hand_worked():
    cases = json.load(open(os.path.join(GOLDEN, "tiny_bag_join.json")))["cases"]
    for c in cases:
        dt = np.uint64 if c["width"] == 8 else np.uint32
        R = np.array(c["R"], dtype=np.uint64).reshape(-1, 2)
        S = np.array(c["S"], dtype=np.uint64).reshape(-1, 2)
        got = oracle.join(R[:, 0].astype(dt), R[:, 1].astype(dt), S[:, 0].astype(dt),
                          S[:, 1].astype(dt), materialize=True, out_cap=max(c["count"], 1))
        assert got["count"] == c["count"], c["name"]
        assert got["checksum"] == int(c["checksum"], 16), c["name"]
        assert got["pair_digest"] == int(c["pair_digest"], 16), c["name"]
        trip = [list(t) for t in zip(got["key"].tolist(), got["pay_r"].tolist(), got["pay_s"].tolist())]
        assert trip == c["triples"], c["name"]


def closed_form_unique(n):
    return n, ((1 << 32) + 1) * n * (n - 1) // 2 & M64


def closed_form_wide(n):
    C = oracle.C_WIDE
    h = n * (n - 1) // 2
    return n, (C * (n * (1 << 40) + h) + n * (1 << 41) + h) & M64


def test_closed_forms_match_golden_table():
    g = json.load(open(os.path.join(GOLDEN, "appendix_a_closed_forms.json")))
    for row in g["unique_4b"]:
        assert closed_form_unique(row["n"]) == (row["count"], int(row["checksum"], 16))
    for row in g["wide_8b"]:
        assert closed_form_wide(row["n"]) == (row["count"], int(row["checksum"], 16))


@pytest.mark.parametrize("n", [1 << 16, 1 << 20, 1000003])
def test_oracle_closed_form_unique(n):
    w = datagen.Workload("unique", n, n)
    d = w.rank_inputs()
    got = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    assert (got["count"], got["checksum"]) == closed_form_unique(n)


def test_oracle_closed_form_unique_sharded_sum():
    """Sum of the oracle over owner-partitioned pieces equals the global result
    (placement independence)."""
    n, N = 1 << 16, 4
    d = datagen.Workload("unique", n, n).rank_inputs()
    tot_c = tot_s = 0
    for g in range(N):
        mr = (d["r_keys"] % N) == g
        ms = (d["s_keys"] % N) == g
        r = oracle.join(d["r_keys"][mr], d["r_pays"][mr], d["s_keys"][ms], d["s_pays"][ms])
        tot_c += r["count"]
        tot_s = (tot_s + r["checksum"]) & M64
    assert (tot_c, tot_s) == closed_form_unique(n)


def test_oracle_closed_form_wide():
    n = 1 << 16
    d = datagen.Workload("wide", n, n).rank_inputs()
    got = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    assert (got["count"], got["checksum"]) == closed_form_wide(n)


@pytest.mark.parametrize("z", [0.5, 1.0])
def test_oracle_zipf_closed_form(z):
    nr, ns = 1 << 14, 1 << 16
    w = datagen.Workload("zipf", nr, ns, z)
    d = w.rank_inputs()
    got = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    rows = np.arange(ns, dtype=np.uint64)
    r = datagen.zipf_ranks(rows, nr, z)
    even = rows % np.uint64(2) == 0
    # even rows match R row r exactly once (R keys unique); odd rows never match
    exp_sum = (sum(int(x) for x in r[even]) << 32) + sum(int(x) for x in rows[even])
    assert got["count"] == int(even.sum())
    assert got["checksum"] == exp_sum & M64


@pytest.mark.parametrize("seed", range(3))
def test_oracle_vs_multiplicity_sums(seed):
    """Count = Σ m_R(k) m_S(k); checksum = Σ_k 2^32 m_S(k) Σ_{a∈R_k} a + m_R(k) Σ_{b∈S_k} b."""
    rng = np.random.default_rng(50 + seed)
    nr, ns, dom = 1 << 17, 1 << 17, [1 << 10, 1 << 15, 1 << 20][seed]
    rk = rng.integers(0, dom, nr, dtype=np.uint64).astype(np.uint32)
    sk = rng.integers(0, dom, ns, dtype=np.uint64).astype(np.uint32)
    ra = rng.integers(0, 1 << 32, nr, dtype=np.uint64).astype(np.uint32)
    sb = rng.integers(0, 1 << 32, ns, dtype=np.uint64).astype(np.uint32)
    ur, inv_r, cr = np.unique(rk, return_inverse=True, return_counts=True)
    us, inv_s, cs = np.unique(sk, return_inverse=True, return_counts=True)
    sum_a = np.zeros(ur.size, dtype=object)
    np.add.at(sum_a, inv_r, ra.astype(object))
    sum_b = np.zeros(us.size, dtype=object)
    np.add.at(sum_b, inv_s, sb.astype(object))
    _, ir, is_ = np.intersect1d(ur, us, assume_unique=True, return_indices=True)
    count = int(np.sum(cr[ir].astype(object) * cs[is_].astype(object)))
    chk = 0
    for x, y in zip(ir, is_):
        chk += (int(sum_a[x]) * int(cs[y]) << 32) + int(cr[x]) * int(sum_b[y])
    got = oracle.join(rk, ra, sk, sb)
    assert got["count"] == count == oracle.expected_count(rk, sk)
    assert got["checksum"] == chk & M64


def test_oracle_sorted_triples_vs_sortmerge():
    """Materialised triples equal a numpy sort-merge join (lexsort + run expansion)."""
    rng = np.random.default_rng(9)
    nr, ns, dom = 20000, 30000, 5000
    rk = rng.integers(0, dom, nr, dtype=np.uint64).astype(np.uint32)
    sk = rng.integers(0, dom, ns, dtype=np.uint64).astype(np.uint32)
    ra = rng.integers(0, 1 << 32, nr, dtype=np.uint64).astype(np.uint32)
    sb = rng.integers(0, 1 << 32, ns, dtype=np.uint64).astype(np.uint32)
    orr = np.lexsort((ra, rk)); rk2, ra2 = rk[orr], ra[orr]
    oss = np.lexsort((sb, sk)); sk2, sb2 = sk[oss], sb[oss]
    lo = np.searchsorted(sk2, rk2, "left"); hi = np.searchsorted(sk2, rk2, "right")
    cnt = hi - lo
    ks = np.repeat(rk2, cnt)
    as_ = np.repeat(ra2, cnt)
    bs = np.concatenate([sb2[l:h] for l, h in zip(lo, hi)]) if cnt.sum() else np.empty(0, np.uint32)
    o = np.lexsort((bs, as_, ks))
    got = oracle.join(rk, ra, sk, sb, materialize=True)
    np.testing.assert_array_equal(got["key"], ks[o])
    np.testing.assert_array_equal(got["pay_r"], as_[o])
    np.testing.assert_array_equal(got["pay_s"], bs[o])


@pytest.mark.parametrize("n", [1 << 12, 1 << 18, 1000003])
def test_oracle_pair_digest_closed_forms(n):
    """R and S with the SAME key permutation: row i of S matches row i of R only.
    Payloads (i, i) give Σ i² = (n-1)n(2n-1)/6; payloads (i, n-1-i) give
    Σ i(n-1-i) = (n-1)·n(n-1)/2 - (n-1)n(2n-1)/6; a digest of a·a or a+b, or
    any wrong pairing, misses at least one of the two."""
    keys = datagen.perm_n(np.arange(n, dtype=np.uint64), n, datagen.SEED_R).astype(np.uint32)
    ids = np.arange(n, dtype=np.uint32)
    got = oracle.join(keys, ids, keys, ids)
    assert got["count"] == n
    assert got["pair_digest"] == ((n - 1) * n * (2 * n - 1) // 6) & M64
    rev = (np.uint32(n - 1) - ids).astype(np.uint32)
    got = oracle.join(keys, ids, keys, rev)
    # Σ_{i<n} i (n-1-i) = (n-1) Σ i - Σ i²
    exp = (n - 1) * (n * (n - 1) // 2) - (n - 1) * n * (2 * n - 1) // 6
    assert got["pair_digest"] == exp & M64


@pytest.mark.parametrize("wide", [False, True])
@pytest.mark.parametrize("dom", [1 << 6, 1 << 14])
def test_oracle_pair_digest_vs_group_sums(wide, dom):
    """The digest is bilinear: Σ_J a·b = Σ_k (Σ_{R_k} a)(Σ_{S_k} b) mod 2^64 —
    per-key sums by np.unique / np.add.at (library routines), Python integers."""
    rng = np.random.default_rng(dom + wide)
    dt = np.uint64 if wide else np.uint32
    nr, ns = 50000, 70000
    rk = rng.integers(0, dom, nr, dtype=np.uint64).astype(dt)
    sk = rng.integers(0, dom, ns, dtype=np.uint64).astype(dt)
    hi = 1 << 64 if wide else 1 << 32
    ra = rng.integers(0, hi - 1, nr, dtype=np.uint64, endpoint=True).astype(dt)
    sb = rng.integers(0, hi - 1, ns, dtype=np.uint64, endpoint=True).astype(dt)
    ur, inv_r = np.unique(rk, return_inverse=True)
    us, inv_s = np.unique(sk, return_inverse=True)
    sa = np.zeros(ur.size, dtype=object)
    np.add.at(sa, inv_r, ra.astype(object))
    sbb = np.zeros(us.size, dtype=object)
    np.add.at(sbb, inv_s, sb.astype(object))
    _, ir, is_ = np.intersect1d(ur, us, assume_unique=True, return_indices=True)
    exp = sum(int(sa[x]) * int(sbb[y]) for x, y in zip(ir, is_)) & M64
    assert oracle.join(rk, ra, sk, sb)["pair_digest"] == exp
