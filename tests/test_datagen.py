"""Generator properties: bijections, Zipf hit/miss structure."""
import numpy as np
import pytest

from paper_conf_sigmod_paullhl21_b200 import datagen


@pytest.mark.parametrize("k", [1, 2, 5, 16, 20])
def test_perm_k_is_bijection(k):
    x = np.arange(1 << k, dtype=np.uint64)
    y = datagen.perm_k(x, k, datagen.SEED_R)
    assert np.array_equal(np.sort(y), x)


@pytest.mark.parametrize("n", [1, 3, 1000, 65537, 1000003])
def test_perm_n_is_bijection(n):
    x = np.arange(n, dtype=np.uint64)
    y = datagen.perm_n(x, n, datagen.SEED_S)
    assert np.array_equal(np.sort(y), x)


def test_mix64_known_values():
    # splitmix64 finaliser of 0 is 0; of 1 is the published constant below.
    v = datagen.mix64(np.array([0, 1], dtype=np.uint64))
    assert int(v[0]) == 0
    z = 1
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & ((1 << 64) - 1)
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & ((1 << 64) - 1)
    z ^= z >> 31
    assert int(v[1]) == z


def test_unique_workload_shards_cover():
    w = datagen.Workload("unique", 1 << 12, 1 << 12)
    full = w.rank_inputs()
    parts = [w.rank_inputs(g, 4) for g in range(4)]
    assert np.array_equal(np.concatenate([p["r_keys"] for p in parts]), full["r_keys"])
    assert np.array_equal(np.sort(full["s_keys"]), np.arange(1 << 12, dtype=np.uint32))


@pytest.mark.parametrize("z", [0.0, 0.5, 1.0])
def test_zipf_structure(z):
    nr, ns = 1 << 12, 1 << 15
    d = datagen.Workload("zipf", nr, ns, z).rank_inputs()
    rows = np.arange(ns)
    even = rows % 2 == 0
    rset = set(d["r_keys"].tolist())
    assert set(d["s_keys"][even].tolist()) <= rset
    assert not (set(d["s_keys"][~even].tolist()) & rset)
    r = datagen.zipf_ranks(rows.astype(np.uint64), nr, z)
    assert r.min() >= 0 and r.max() < nr
    if z == 1.0:  # heavy head: rank 0 is by far the most frequent
        c = np.bincount(r.astype(np.int64), minlength=nr)
        assert c[0] > 20 * np.median(c)


def test_zipf_exp2_accuracy():
    f = np.linspace(0, 1, 1001, endpoint=False)
    p = datagen._exp2_frac(f)
    assert np.max(np.abs(p - np.exp2(f)) / np.exp2(f)) < 4e-16


@pytest.mark.parametrize("k", [1, 5, 16, 20, 29, 32])
def test_perm_k_inverse(k):
    rng = np.random.default_rng(k)
    x = rng.integers(0, 1 << k, 100000, dtype=np.uint64) if k > 16 else np.arange(1 << k, dtype=np.uint64)
    for seed in (datagen.SEED_R, datagen.SEED_S):
        y = datagen.perm_k(x, k, seed)
        np.testing.assert_array_equal(datagen.perm_k_inverse(y, k, seed), x)


def test_unmix64_inverse():
    rng = np.random.default_rng(1)
    x = rng.integers(0, 2**63, 100000, dtype=np.uint64) * np.uint64(2) + rng.integers(0, 2, 100000, dtype=np.uint64)
    np.testing.assert_array_equal(datagen.unmix64(datagen.mix64(x)), x)


@pytest.mark.parametrize("k", [7, 29, 32])
def test_torch_inverses_match_numpy(k):
    torch = pytest.importorskip("torch")
    rng = np.random.default_rng(k + 1)
    x = rng.integers(0, 1 << k, 50000, dtype=np.uint64)
    y = datagen.perm_k(x, k, datagen.SEED_R)
    got = datagen.perm_k_inverse_t(torch.from_numpy(y.astype(np.int64)), k, datagen.SEED_R).numpy()
    np.testing.assert_array_equal(got.astype(np.uint64), x)
    z = datagen.mix64(x)
    got = datagen.unmix64_t(torch.from_numpy(z.view(np.int64))).numpy().view(np.uint64)
    np.testing.assert_array_equal(got, x)


@pytest.mark.parametrize("world,z", [(1, 1.0), (4, 0.0), (4, 1.0), (8, 0.5)])
def test_placement_shards_tile_rows(world, z):
    """Placement-skewed shards (Fig. 9 reading) still tile [0, n) in rank order, rank 0 largest."""
    n = 1000003
    b = [datagen.shard_bounds(n, g, world, z) for g in range(world)]
    assert b[0][0] == 0 and b[-1][1] == n
    assert all(b[g][1] == b[g + 1][0] for g in range(world - 1))
    sizes = [hi - lo for lo, hi in b]
    assert sizes == sorted(sizes, reverse=True) or z == 0.0
    w = datagen.Workload("unique", n, n, placement_z=z)
    d = w.rank_inputs(world - 1, world)
    assert d["r_keys"].size == sizes[-1] and int(d["r_pays"][0]) == b[-1][0]
