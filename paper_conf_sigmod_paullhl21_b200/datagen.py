"""Seeded synthetic input generator shared by the oracle tests and the CUDA path.

This module holds NO join arithmetic: it only produces the relations R and S
described by the paper's workload (§5.1 "Workload": 8-byte
tuples of a 4-byte key and a 4-byte id, "integer key values generated
sequentially and then shuffled randomly", |R| = |S|, plus a Zipf variant) and
the variants BASELINE.json lists (SURVEY.md §8d generator spec, configs M1-M5).

Everything is counter-based: row i of a relation is a pure function of
(i, seed, config), so any rank can produce any slice of it, and the CUDA
generator in ``csrc/gen.cu`` reproduces it bit for bit (tested in
``tests/test_gen_gpu.py``).  The same spec is stated in DESIGN.md §3.

Bijection on [0, 2^k)  (perm_k):
    x = (x ^ s) & M; x = (x*0x9E3779B1) & M; x ^= x >> h
    x = (x*0x85EBCA6B) & M; x ^= x >> h; x = (x*0xC2B2AE35) & M; x ^= x >> h
with M = 2^k - 1 and h = ceil(k/2).  For n not a power of two, perm_n
cycle-walks perm_k (k = ceil(log2 n)) until the value is < n, which is a
bijection on [0, n).

Zipf ranks (config M4) are drawn from a bounded continuous power law,
r = floor(F^-1(u)) - 1, computed only with IEEE-exact +, -, *, sqrt and a
fixed no-FMA Horner polynomial for 2^f, so numpy and CUDA agree bit for bit.
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

# Seeds; every bench / test JSON records them.
SEED_R = 0x5EED0052
SEED_S = 0x5EED0053
SEED_Z = 0x5EED005A
SEED_X = 0x5EED0058

_U64 = np.uint64
_MASK64 = (1 << 64) - 1

# 1/i! for i = 0..17 as exact double bit patterns (shared with gen.cu).
EXP_COEF_HEX = [
    "0x1.0000000000000p+0", "0x1.0000000000000p+0", "0x1.0000000000000p-1",
    "0x1.5555555555555p-3", "0x1.5555555555555p-5", "0x1.1111111111111p-7",
    "0x1.6c16c16c16c17p-10", "0x1.a01a01a01a01ap-13", "0x1.a01a01a01a01ap-16",
    "0x1.71de3a556c734p-19", "0x1.27e4fb7789f5cp-22", "0x1.ae64567f544e4p-26",
    "0x1.1eed8eff8d898p-29", "0x1.6124613a86d09p-33", "0x1.93974a8c07c9dp-37",
    "0x1.ae7f3e733b81fp-41", "0x1.ae7f3e733b81fp-45", "0x1.952c77030ad4ap-49",
]
LN2_HEX = "0x1.62e42fefa39efp-1"


def ceil_log2(n: int) -> int:
    return max(1, (int(n) - 1).bit_length())


def perm_k(x: np.ndarray, k: int, seed: int) -> np.ndarray:
    """Bijection on [0, 2^k), vectorised over uint64."""
    assert 1 <= k <= 32
    x = np.asarray(x, dtype=_U64)
    M = _U64((1 << k) - 1)
    h = _U64((k + 1) // 2)
    x = (x ^ _U64(seed & _MASK64)) & M
    x = (x * _U64(0x9E3779B1)) & M
    x ^= x >> h
    x = (x * _U64(0x85EBCA6B)) & M
    x ^= x >> h
    x = (x * _U64(0xC2B2AE35)) & M
    x ^= x >> h
    return x


def perm_n(x: np.ndarray, n: int, seed: int) -> np.ndarray:
    """Bijection on [0, n) by cycle-walking perm_k, k = ceil(log2 n)."""
    k = ceil_log2(n)
    y = perm_k(x, k, seed)
    if n == (1 << k):
        return y
    bad = y >= _U64(n)
    while bad.any():
        y[bad] = perm_k(y[bad], k, seed)
        bad = y >= _U64(n)
    return y


def mix64(z: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser, a bijection on u64."""
    z = np.asarray(z, dtype=_U64).copy()
    z = (z ^ (z >> _U64(30))) * _U64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> _U64(27))) * _U64(0x94D049BB133111EB)
    z = z ^ (z >> _U64(31))
    return z


def _exp2_frac(f: np.ndarray) -> np.ndarray:
    """2^f for f in [0,1) by a degree-17 Taylor Horner scheme, no FMA."""
    x = f * float.fromhex(LN2_HEX)
    coef = [float.fromhex(c) for c in EXP_COEF_HEX]
    p = np.full_like(x, coef[-1])
    for c in reversed(coef[:-1]):
        p = p * x
        p = p + c
    return p


def zipf_ranks(rows: np.ndarray, n: int, z: float, seed: int = SEED_Z) -> np.ndarray:
    """Rank r in [0, n) for each S row.

    u = (mix64(j ^ s_Z) >> 11) * 2^-53.
      z = 0   : r = floor(n u)
      z = 0.5 : r = floor(((sqrt(n) - 1) u + 1)^2) - 1
      z = 1   : r = floor(n^u) - 1 = floor(2^(k u)) - 1
    clamped to [0, n-1].  n must be a power of two.
    """
    k = ceil_log2(n)
    assert n == 1 << k
    j = np.asarray(rows, dtype=_U64)
    u = (mix64(j ^ _U64(seed)) >> _U64(11)).astype(np.float64) * (2.0 ** -53)
    if z == 0.0:
        r = np.floor(u * float(n))
    elif z == 0.5:
        a = math.sqrt(float(n))
        t = (a - 1.0) * u
        t = t + 1.0
        r = np.floor(t * t) - 1.0
    elif z == 1.0:
        y = float(k) * u
        e = np.floor(y)
        f = y - e
        p = np.ldexp(_exp2_frac(f), e.astype(np.int32))
        r = np.floor(p) - 1.0
    else:
        raise ValueError("only z in {0, 0.5, 1.0} is specified")
    r = np.clip(r, 0.0, float(n - 1))
    return r.astype(np.uint64)


def shard_bounds(n: int, rank: int, world: int, placement_z: float = 0.0) -> tuple[int, int]:
    """Rows [lo, hi) of `rank` among `world` contiguous slices of n rows; with
    placement_z > 0 slice g holds a share 1/(g+1)^z / sum_h 1/(h+1)^z (exact
    integer boundaries from the cumulative weights)."""
    if placement_z == 0.0:
        return (n * rank) // world, (n * (rank + 1)) // world
    w = [1.0 / (g + 1) ** placement_z for g in range(world)]
    tot = sum(w)
    cum = [0]
    for g in range(world):
        cum.append(n if g == world - 1 else int(n * (sum(w[:g + 1]) / tot)))
    return cum[rank], cum[rank + 1]


@dataclasses.dataclass(frozen=True)
class Workload:
    """A synthetic join input.

    kind:
      "unique" — R.key = perm_n(i; s_R), S.key = perm_n(j; s_S), payload = row id
                 (M1, M2, M3; 100% selectivity when n_r == n_s).
      "zipf"   — R as "unique" over n_r (power of two); S row j draws a Zipf
                 rank r; even j -> key = perm(r; s_R) (matches R row r),
                 odd j -> key = n_r + perm(r; s_X) (never matches). (M4)
      "wide"   — 8-byte keys mix64(perm(i)), payloads 2^40 + i / 2^41 + j. (M5)
    """
    kind: str
    n_r: int
    n_s: int
    z: float = 0.0
    placement_z: float = 0.0  # rank shares of the rows ~ 1/(g+1)^placement_z (0: equal shares)

    @property
    def key_bytes(self) -> int:
        return 8 if self.kind == "wide" else 4

    @property
    def payload_bytes(self) -> int:
        return self.key_bytes

    def shard(self, n: int, rank: int, world: int) -> tuple[int, int]:
        """Rows [lo, hi) held by `rank` (contiguous slices).  With
        placement_z > 0 the slices follow a Zipf law over the ranks (rank g's share
        proportional to 1/(g+1)^z: the placement-skew reading of Fig. 9)."""
        return shard_bounds(n, rank, world, self.placement_z)

    def relation(self, rel: str, lo: int, hi: int) -> tuple[np.ndarray, np.ndarray]:
        rows = np.arange(lo, hi, dtype=_U64)
        if self.kind == "unique":
            n = self.n_r if rel == "R" else self.n_s
            seed = SEED_R if rel == "R" else SEED_S
            keys = perm_n(rows, n, seed).astype(np.uint32)
            return keys, rows.astype(np.uint32)
        if self.kind == "wide":
            n = self.n_r if rel == "R" else self.n_s
            seed = SEED_R if rel == "R" else SEED_S
            keys = mix64(perm_n(rows, n, seed))
            base = _U64(1 << 40) if rel == "R" else _U64(1 << 41)
            return keys, rows + base
        if self.kind == "zipf":
            k = ceil_log2(self.n_r)
            assert self.n_r == 1 << k and self.n_r <= 1 << 31
            if rel == "R":
                return perm_k(rows, k, SEED_R).astype(np.uint32), rows.astype(np.uint32)
            r = zipf_ranks(rows, self.n_r, self.z)
            hit = perm_k(r, k, SEED_R)
            miss = _U64(self.n_r) + perm_k(r, k, SEED_X)
            keys = np.where((rows & _U64(1)) == 0, hit, miss).astype(np.uint32)
            return keys, rows.astype(np.uint32)
        raise ValueError(self.kind)

    def rank_inputs(self, rank: int = 0, world: int = 1) -> dict:
        rlo, rhi = self.shard(self.n_r, rank, world)
        slo, shi = self.shard(self.n_s, rank, world)
        rk, rp = self.relation("R", rlo, rhi)
        sk, sp = self.relation("S", slo, shi)
        return {"r_keys": rk, "r_pays": rp, "s_keys": sk, "s_pays": sp,
                "r_row0": rlo, "s_row0": slo}

    def spec(self) -> dict:
        return {"kind": self.kind, "n_r": self.n_r, "n_s": self.n_s, "z": self.z,
                "seeds": {"R": hex(SEED_R), "S": hex(SEED_S), "Z": hex(SEED_Z), "X": hex(SEED_X)}}


# BASELINE.json configs as generator instances (sizes in tuples; 1M = 2^20).
def M1() -> Workload:
    return Workload("unique", 1 << 20, 1 << 20)


def M2(world: int = 1) -> Workload:
    return Workload("unique", world << 29, world << 29)


def M3() -> Workload:
    return Workload("unique", 1 << 31, 1 << 31)


def M4(z: float, world: int = 8) -> Workload:
    return Workload("zipf", world << 27, world << 29, z)


def M5(world: int = 8) -> Workload:
    return Workload("wide", world << 28, world << 28)


# ---------------------------------------------------------------- inverses
# The generator's bijections inverted, so that a full-size check can find the
# R row an S key was drawn from without any join: R.key[i] = perm_k(i) (or
# mix64(perm_k(i)) for 8-byte keys), hence i = perm_k^-1(key).  Generator
# arithmetic only (no join arithmetic); pinned by tests/test_datagen.py.
_PERM_MUL = (0x9E3779B1, 0x85EBCA6B, 0xC2B2AE35)
_PERM_INV = tuple(pow(c, -1, 1 << 32) for c in _PERM_MUL)  # inverses mod 2^32 (also mod 2^k, k <= 32)
_MIX_MUL = (0xBF58476D1CE4E5B9, 0x94D049BB133111EB)
_MIX_INV = tuple(pow(c, -1, 1 << 64) for c in _MIX_MUL)


def perm_k_inverse(y: np.ndarray, k: int, seed: int) -> np.ndarray:
    """x with perm_k(x, k, seed) == y (y in [0, 2^k)).  x ^= x >> h is an
    involution on [0, 2^k) because 2h >= k."""
    assert 1 <= k <= 32
    x = np.asarray(y, dtype=_U64).copy()
    M = _U64((1 << k) - 1)
    h = _U64((k + 1) // 2)
    x ^= x >> h
    x = (x * _U64(_PERM_INV[2])) & M
    x ^= x >> h
    x = (x * _U64(_PERM_INV[1])) & M
    x ^= x >> h
    x = (x * _U64(_PERM_INV[0])) & M
    return (x ^ _U64(seed & _MASK64)) & M


def unmix64(z: np.ndarray) -> np.ndarray:
    """Inverse of mix64."""
    z = np.asarray(z, dtype=_U64).copy()
    z = z ^ (z >> _U64(31)) ^ (z >> _U64(62))
    z = z * _U64(_MIX_INV[1])
    z = z ^ (z >> _U64(27)) ^ (z >> _U64(54))
    z = z * _U64(_MIX_INV[0])
    return z ^ (z >> _U64(30)) ^ (z >> _U64(60))


def _s64(c: int) -> int:
    """u64 constant as the int64 with the same bits (torch has no uint64 arithmetic)."""
    return c - (1 << 64) if c >= 1 << 63 else c


def _lsr_t(x, s: int):
    """Logical right shift of an int64 torch tensor holding u64 bits."""
    return (x >> s) & ((1 << (64 - s)) - 1)


def perm_k_inverse_t(y, k: int, seed: int):
    """perm_k_inverse on an int64 torch tensor (values in [0, 2^k)), on its device.
    int64 products wrap modulo 2^64, so the low k bits are exact."""
    assert 1 <= k <= 32
    M = (1 << k) - 1
    h = (k + 1) // 2
    x = y & M
    x = x ^ (x >> h)
    x = (x * _PERM_INV[2]) & M
    x = x ^ (x >> h)
    x = (x * _PERM_INV[1]) & M
    x = x ^ (x >> h)
    x = (x * _PERM_INV[0]) & M
    return (x ^ (seed & M)) & M


def unmix64_t(z):
    """unmix64 on an int64 torch tensor holding u64 bits."""
    z = z ^ _lsr_t(z, 31) ^ _lsr_t(z, 62)
    z = z * _s64(_MIX_INV[1])
    z = z ^ _lsr_t(z, 27) ^ _lsr_t(z, 54)
    z = z * _s64(_MIX_INV[0])
    return z ^ _lsr_t(z, 30) ^ _lsr_t(z, 60)
