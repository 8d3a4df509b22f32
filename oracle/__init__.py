"""CPU oracle for the MG-Join hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` leg may import this package.  The
product path (``paper_conf_sigmod_paullhl21_b200``) never imports it and
shares no code with it; see ``oracle.c`` for the definition it follows
 and DESIGN.md §2 for the
readings (C2 bag semantics, C3 checksum, C17 sorted triples).

Parity status: every function here is pinned (tests/test_oracle.py):
brute-force nested loop (tiny), closed forms (generated workloads),
numpy multiplicity sums (sort-merge), per-key group-sum products for the
pair digest (Σ_k (Σ_{R_k} a)(Σ_{S_k} b)), closed forms Σ i² and
Σ i(n-1-i) for identical key permutations, hand-worked golden fixture.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

MASK64 = (1 << 64) - 1
C_WIDE = 0x9E3779B97F4A7C15  # checksum multiplier for 8-byte payloads (reading C3)


class _Res(ctypes.Structure):
    _fields_ = [("count", ctypes.c_uint64), ("checksum", ctypes.c_uint64),
                ("n_out", ctypes.c_uint64), ("pair_digest", ctypes.c_uint64), ("overflow", ctypes.c_int32),
                ("status", ctypes.c_int32)]


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc -O2 (plain C, single thread)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-shared", "-fPIC", "-o", _LIB, _SRC])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        for name in ("oracle_join_k32", "oracle_join_k64"):
            fn = getattr(lib, name)
            fn.restype = ctypes.c_int
            fn.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                           ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                           ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                           ctypes.c_uint64, ctypes.POINTER(_Res)]
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p) if a.size else None


def join(r_keys, r_pays, s_keys, s_pays, materialize: bool = False, out_cap: int | None = None):
    """Return dict(count, checksum, pair_digest[, key, pay_r, pay_s]) for the bag equi-join R ⋈ S.

    pair_digest = Σ_J a·b mod 2^64 (reading C3b): bilinear in the
    matched pair, so a wrong pairing changes it.

    4-byte (uint32) or 8-byte (uint64) keys/payloads; both relations must use
    the same width.  Triples (if requested) are sorted by (k, a, b).
    """
    lib = _load()
    rk = np.ascontiguousarray(r_keys)
    wide = rk.dtype == np.uint64
    dt = np.uint64 if wide else np.uint32
    rk = rk.astype(dt, copy=False)
    ra = np.ascontiguousarray(r_pays).astype(dt, copy=False)
    sk = np.ascontiguousarray(s_keys).astype(dt, copy=False)
    sb = np.ascontiguousarray(s_pays).astype(dt, copy=False)
    assert rk.shape == ra.shape and sk.shape == sb.shape
    res = _Res()
    if materialize:
        if out_cap is None:
            out_cap = expected_count(rk, sk)
        ok = np.empty(max(out_cap, 1), dt)
        oa = np.empty(max(out_cap, 1), dt)
        ob = np.empty(max(out_cap, 1), dt)
        args = (_ptr(ok), _ptr(oa), _ptr(ob), out_cap)
    else:
        args = (None, None, None, 0)
    fn = lib.oracle_join_k64 if wide else lib.oracle_join_k32
    rc = fn(_ptr(rk), _ptr(ra), rk.size, _ptr(sk), _ptr(sb), sk.size, *args, ctypes.byref(res))
    if rc != 0 or res.status != 0:
        raise MemoryError("oracle: allocation failed")
    out = {"count": int(res.count), "checksum": int(res.checksum), "pair_digest": int(res.pair_digest)}
    if materialize:
        n = int(res.n_out)
        out.update(key=ok[:n], pay_r=oa[:n], pay_s=ob[:n], overflow=bool(res.overflow))
    return out


def expected_count(r_keys, s_keys) -> int:
    """Σ_k m_R(k)·m_S(k) via np.unique multiplicities (library routine)."""
    ur, cr = np.unique(r_keys, return_counts=True)
    us, cs = np.unique(s_keys, return_counts=True)
    _, ir, is_ = np.intersect1d(ur, us, assume_unique=True, return_indices=True)
    return int(np.sum(cr[ir].astype(object) * cs[is_].astype(object))) if ir.size else 0
