"""Thin ctypes binding of libmgj.so (include/mgj.h, include/mgj_aux.h).

Argument marshalling only: every step of the join runs in the CUDA kernels of
``csrc/``.  The names follow the C ABI (mgj_plan / mgj_partition /
mgj_shuffle / mgj_join / mgj_result).  Importing this module fails loudly if
the extension has not been built; there is no CPU fallback.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("MGJ_LIB") or os.path.join(_HERE, "libmgj.so")  # MGJ_LIB: A/B experiments only

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libmgj.so not built ({LIB_PATH}); run `python -c 'import __graft_entry__ as g; g.build()'`")

_lib = ctypes.CDLL(LIB_PATH)

STATUS = {0: "MGJ_OK", -1: "MGJ_EINVAL", -2: "MGJ_EALIGN", -3: "MGJ_ENOMEM", -4: "MGJ_ECUDA",
          -5: "MGJ_ESTATE", -6: "MGJ_ECAPACITY", -7: "MGJ_EPEER"}
MAX_RANKS = 8

# mgj_debug_what
DBG = dict(RANK_HIST=1, MAIL_HIST=2, OWNER=3, SEND_OFF=4, RECV_SIZE=5, RECV_R=6, RECV_S=7,
           LOCAL_R=8, LOCAL_S=9, META=10, CHUNK_OFF_R=11, CHUNK_OFF_S=12, CHUNK_BASE=13, SEGMENTS=14,
           OUT_KEY=15, OUT_PAY_R=16, OUT_PAY_S=17, MID_R=18, MID_S=19, MID_OFF_R=20, BCAST=21, PLIST=22, SKIP=23,
           TRACE=24, MID_OFF_S=25)
# trace slots (include/mgj_aux.h MGJ_TR_*), in pipeline order
TRACE_NAMES = ["hist", "plan", "scatter_R", "scatter_S", "local_R", "local_S", "local_RS", "local_split",
               "local_second", "itemize", "probe", "reduce"]
GEN_KIND = {"unique": 0, "zipf": 1, "wide": 2}


class MGJError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        name = STATUS.get(status, str(status))
        msg = _lib.mgj_strerror(status).decode()
        super().__init__(f"{where}: {name} ({msg})")


class Config(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int32), ("world_size", ctypes.c_int32),
                ("key_bytes", ctypes.c_int32), ("payload_bytes", ctypes.c_int32),
                ("r_capacity", ctypes.c_uint64), ("s_capacity", ctypes.c_uint64),
                ("recv_capacity_r", ctypes.c_uint64), ("recv_capacity_s", ctypes.c_uint64),
                ("radix_bits_global", ctypes.c_int32), ("radix_bits_local", ctypes.c_int32),
                ("materialize", ctypes.c_int32), ("num_sms", ctypes.c_int32),
                ("out_capacity", ctypes.c_uint64), ("shuffle_mode", ctypes.c_int32),
                ("local_split_bits", ctypes.c_int32), ("skew_bcast", ctypes.c_int32),
                ("peer_timeout_ms", ctypes.c_int32), ("shuffle_overlap", ctypes.c_int32),
                ("overlap_local_sms", ctypes.c_int32), ("trace", ctypes.c_int32),
                ("compress", ctypes.c_int32), ("assign", ctypes.c_int32), ("reserved", ctypes.c_int32 * 1)]


class Exchange(ctypes.Structure):
    _fields_ = [("send", ctypes.c_void_p * 2), ("recv", ctypes.c_void_p * 2),
                ("send_count", (ctypes.c_uint64 * MAX_RANKS) * 2), ("recv_count", (ctypes.c_uint64 * MAX_RANKS) * 2),
                ("tuple_bytes", ctypes.c_int32), ("world_size", ctypes.c_int32)]


class Peers(ctypes.Structure):
    _fields_ = [("arena_ptrs", ctypes.POINTER(ctypes.c_void_p)), ("arena_bytes", ctypes.c_uint64)]


class Result(ctypes.Structure):
    _fields_ = [("match_count", ctypes.c_uint64), ("checksum", ctypes.c_uint64),
                ("local_count", ctypes.c_uint64), ("local_checksum", ctypes.c_uint64),
                ("n_materialized", ctypes.c_uint64),
                ("out_key", ctypes.c_void_p), ("out_payload_r", ctypes.c_void_p),
                ("out_payload_s", ctypes.c_void_p),
                ("recv_r", ctypes.c_uint64), ("recv_s", ctypes.c_uint64),
                ("phase_ms", ctypes.c_float * 6), ("status", ctypes.c_int32),
                ("radix_bits_global", ctypes.c_int32), ("radix_bits_local", ctypes.c_int32),
                ("n_items", ctypes.c_int32), ("n_launches", ctypes.c_int32),
                ("pair_digest", ctypes.c_uint64), ("local_pair_digest", ctypes.c_uint64)]


_H = ctypes.c_void_p
_P = ctypes.c_void_p
_U64 = ctypes.c_uint64
_lib.mgj_strerror.restype = ctypes.c_char_p
_lib.mgj_strerror.argtypes = [ctypes.c_int]
_lib.mgj_arena_bytes.restype = _U64
_lib.mgj_arena_bytes.argtypes = [ctypes.POINTER(Config)]
_lib.mgj_plan.restype = ctypes.c_int
_lib.mgj_plan.argtypes = [ctypes.POINTER(Config), ctypes.POINTER(Peers), ctypes.POINTER(_H)]
_lib.mgj_partition.restype = ctypes.c_int
_lib.mgj_partition.argtypes = [_H, _P, _P, _U64, _P, _P, _U64, _P]
_lib.mgj_shuffle.restype = ctypes.c_int
_lib.mgj_shuffle.argtypes = [_H, _P]
_lib.mgj_join.restype = ctypes.c_int
_lib.mgj_join.argtypes = [_H, _P]
_lib.mgj_result.restype = ctypes.c_int
_lib.mgj_result.argtypes = [_H, ctypes.POINTER(Result)]
_lib.mgj_destroy.restype = None
_lib.mgj_destroy.argtypes = [_H]
_lib.mgj_plan_host.restype = ctypes.c_int
_lib.mgj_plan_host.argtypes = [ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, _P, _P, _P, _P, ctypes.c_int32, _P, _P,
                               ctypes.c_int32]
_lib.mgj_gen_relation.restype = ctypes.c_int
_lib.mgj_gen_relation.argtypes = [ctypes.c_int32, ctypes.c_int32, _U64, _U64, ctypes.c_double,
                                  _U64, _U64, _P, _P, _P]
_lib.mgj_exchange_layout.restype = ctypes.c_int
_lib.mgj_exchange_layout.argtypes = [_H, ctypes.POINTER(Exchange)]
_lib.mgj_debug_copy.restype = ctypes.c_int
_lib.mgj_debug_copy.argtypes = [_H, ctypes.c_int32, _P, _U64, ctypes.POINTER(_U64)]

EXPORTED = ["mgj_arena_bytes", "mgj_plan", "mgj_partition", "mgj_shuffle", "mgj_join", "mgj_result",
            "mgj_destroy", "mgj_strerror", "mgj_plan_host", "mgj_exchange_layout", "mgj_gen_relation",
            "mgj_debug_copy"]
SHUFFLE_P2P, SHUFFLE_EXTERNAL = 0, 1


def _check(st: int, where: str):
    if st != 0:
        raise MGJError(st, where)


def _ptr(x):
    """Device or host address of a torch tensor / numpy array (None if empty)."""
    if x is None:
        return None
    if isinstance(x, np.ndarray):
        return x.ctypes.data if x.size else None
    return x.data_ptr() if x.numel() else None


def _stream(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return stream if isinstance(stream, int) else stream.cuda_stream


def make_config(rank=0, world_size=1, key_bytes=4, r_capacity=0, s_capacity=0, recv_capacity_r=0,
                recv_capacity_s=0, radix_bits_global=0, radix_bits_local=0, materialize=False,
                num_sms=0, out_capacity=0, shuffle_mode=0, local_split_bits=0, skew_bcast=0,
                peer_timeout_ms=0, shuffle_overlap=0, overlap_local_sms=0, trace=False, compress=False,
                assign=0) -> Config:
    c = Config()
    c.rank, c.world_size = rank, world_size
    c.key_bytes = c.payload_bytes = key_bytes
    c.r_capacity, c.s_capacity = r_capacity, s_capacity
    c.recv_capacity_r, c.recv_capacity_s = recv_capacity_r, recv_capacity_s
    c.radix_bits_global, c.radix_bits_local = radix_bits_global, radix_bits_local
    c.materialize = int(bool(materialize))
    c.num_sms = num_sms
    c.out_capacity = out_capacity
    c.shuffle_mode = shuffle_mode
    c.local_split_bits = local_split_bits
    c.skew_bcast = skew_bcast
    c.peer_timeout_ms = peer_timeout_ms
    c.shuffle_overlap = shuffle_overlap
    c.overlap_local_sms = overlap_local_sms
    c.trace = int(bool(trace))
    c.compress = int(bool(compress))
    c.assign = assign
    return c


def arena_bytes(cfg: Config) -> int:
    return int(_lib.mgj_arena_bytes(ctypes.byref(cfg)))


class Join:
    """One rank's handle (mgj_plan ... mgj_destroy)."""

    def __init__(self, cfg: Config, arena_ptrs=None, arena_nbytes: int = 0):
        self.cfg = cfg
        self._h = _H()
        peers = None
        if arena_ptrs is not None:
            arr = (ctypes.c_void_p * len(arena_ptrs))(*arena_ptrs)
            self._arr = arr
            peers = Peers(ctypes.cast(arr, ctypes.POINTER(ctypes.c_void_p)), arena_nbytes)
        _check(_lib.mgj_plan(ctypes.byref(cfg), ctypes.byref(peers) if peers else None, ctypes.byref(self._h)),
               "mgj_plan")

    def partition(self, r_keys, r_pays, s_keys, s_pays, stream=None):
        n_r = int(r_keys.numel() if hasattr(r_keys, "numel") else r_keys.size)
        n_s = int(s_keys.numel() if hasattr(s_keys, "numel") else s_keys.size)
        self._keep = (r_keys, r_pays, s_keys, s_pays)
        _check(_lib.mgj_partition(self._h, _ptr(r_keys), _ptr(r_pays), n_r, _ptr(s_keys), _ptr(s_pays), n_s,
                                  _stream(stream)), "mgj_partition")

    def shuffle(self, stream=None):
        _check(_lib.mgj_shuffle(self._h, _stream(stream)), "mgj_shuffle")

    def exchange_layout(self) -> dict:
        """EXTERNAL shuffle: buffers and per-rank tuple counts of the exchange (mgj_exchange_layout)."""
        e = Exchange()
        _check(_lib.mgj_exchange_layout(self._h, ctypes.byref(e)), "mgj_exchange_layout")
        W = e.world_size
        return {"send": [e.send[0], e.send[1]], "recv": [e.recv[0], e.recv[1]],
                "send_count": [[int(e.send_count[r][g]) for g in range(W)] for r in range(2)],
                "recv_count": [[int(e.recv_count[r][g]) for g in range(W)] for r in range(2)],
                "tuple_bytes": int(e.tuple_bytes)}

    def join(self, stream=None):
        _check(_lib.mgj_join(self._h, _stream(stream)), "mgj_join")

    def result(self, check: bool = True) -> dict:
        r = Result()
        st = _lib.mgj_result(self._h, ctypes.byref(r))
        if check:
            _check(st, "mgj_result")
        return {"match_count": int(r.match_count), "checksum": int(r.checksum),
                "pair_digest": int(r.pair_digest),
                "local_count": int(r.local_count), "local_checksum": int(r.local_checksum),
                "local_pair_digest": int(r.local_pair_digest),
                "n_materialized": int(r.n_materialized), "out_key": r.out_key,
                "out_payload_r": r.out_payload_r, "out_payload_s": r.out_payload_s,
                "recv_r": int(r.recv_r), "recv_s": int(r.recv_s),
                "phase_ms": [float(x) for x in r.phase_ms], "status": int(r.status),
                "radix_bits_global": int(r.radix_bits_global), "radix_bits_local": int(r.radix_bits_local),
                "n_items": int(r.n_items), "n_launches": int(r.n_launches)}

    def run(self, r_keys, r_pays, s_keys, s_pays, stream=None) -> dict:
        self.partition(r_keys, r_pays, s_keys, s_pays, stream)
        self.shuffle(stream)
        self.join(stream)
        return self.result()

    def debug(self, what: str, dtype=np.uint8) -> np.ndarray:
        size = _U64(0)
        _check(_lib.mgj_debug_copy(self._h, DBG[what], None, 0, ctypes.byref(size)), "mgj_debug_copy")
        buf = np.empty(int(size.value), dtype=np.uint8)
        if buf.size:
            _check(_lib.mgj_debug_copy(self._h, DBG[what], buf.ctypes.data, buf.size, None), "mgj_debug_copy")
        return buf.view(dtype)

    def trace(self) -> dict:
        """Kernel timeline of the last run (needs trace=True): name -> (first start, last end) in ns
        relative to the earliest start; kernels that did not run are left out."""
        t = self.debug("TRACE", np.uint64).reshape(-1, 2)
        live = [(n, int(a), int(b)) for n, (a, b) in zip(TRACE_NAMES, t) if a and b]
        t0 = min(a for _, a, _ in live) if live else 0
        return {n: (a - t0, b - t0) for n, a, b in live}

    def materialized(self, res: dict):
        """Copy this rank's materialised triples to host numpy arrays (key, payR, payS)."""
        dt = np.uint32 if self.cfg.key_bytes == 4 else np.uint64
        n = res["n_materialized"]
        return tuple(self.debug(w, dt)[:n] for w in ("OUT_KEY", "OUT_PAY_R", "OUT_PAY_S"))

    def close(self):
        if self._h:
            _lib.mgj_destroy(self._h)
            self._h = _H()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def symmetric_join(cfg: Config, group=None):
    """One rank's Join over a torch symmetric-memory arena (one process per GPU).

    Allocates this rank's arena with torch.distributed._symmetric_memory (size
    mgj_arena_bytes), zero-fills it, exchanges the peer mappings (rendezvous) and
    barriers, as mgj_peers requires; the process group must be initialised
    (NCCL) and cfg.rank / cfg.world_size must match it.  The arena tensor is kept
    on the returned handle (`.arena`) so it outlives the join.  Memory plumbing
    only: the exchange itself is the library's in-kernel peer stores."""
    import torch
    import torch.distributed as dist
    import torch.distributed._symmetric_memory as symm_mem
    group = group or dist.group.WORLD
    nbytes = arena_bytes(cfg)
    if nbytes == 0:
        raise MGJError(-1, "mgj_arena_bytes")
    arena = symm_mem.empty(nbytes, dtype=torch.uint8, device=torch.device("cuda", torch.cuda.current_device()))
    arena.zero_()
    hdl = symm_mem.rendezvous(arena, group)
    ptrs = [int(p) for p in hdl.buffer_ptrs]
    torch.cuda.synchronize()
    dist.barrier(group)
    j = Join(cfg, ptrs, nbytes)
    j.arena, j._symm = arena, hdl
    return j


def nccl_exchange(join: "Join", stream=None, group=None):
    """MGJ_SHUFFLE_EXTERNAL baseline: all_to_all_single (NCCL) of the per-destination send
    buffers into this rank's receive areas, between join.shuffle() and join.join().
    Synchronises the stream once (the split sizes are computed on the device)."""
    import torch
    import torch.distributed as dist
    lay = join.exchange_layout()
    tb = lay["tuple_bytes"]
    ctx = torch.cuda.stream(stream) if stream is not None else torch.cuda.stream(torch.cuda.current_stream())
    with ctx:
        for rel in range(2):
            sc, rc = lay["send_count"][rel], lay["recv_count"][rel]
            send = device_bytes(lay["send"][rel], sum(sc) * tb)
            recv = device_bytes(lay["recv"][rel], sum(rc) * tb)
            dist.all_to_all_single(recv, send, [x * tb for x in rc], [x * tb for x in sc], group=group)


class _DevBuf:
    """Byte view of a raw device pointer for torch.as_tensor (__cuda_array_interface__)."""

    def __init__(self, ptr: int, nbytes: int):
        self.__cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (ptr, False),
                                         "version": 3}


def device_bytes(ptr: int, nbytes: int):
    """torch uint8 tensor aliasing device memory [ptr, ptr + nbytes)."""
    import torch
    if nbytes == 0:
        return torch.empty(0, dtype=torch.uint8, device="cuda")
    return torch.as_tensor(_DevBuf(ptr, nbytes), device="cuda")


def plan_host(world: int, rank: int, bits: int, hist: np.ndarray, skew_bcast: int = 0, with_bcast: bool = False,
              assign: int = 0):
    """Host reference of the a2 assignment (mgj_plan_host): owner, send offsets, receive sizes
    (and, with with_bcast=True, the selective-broadcast flags and the empty-side skip flags)."""
    P = 1 << bits
    hist = np.ascontiguousarray(hist, dtype=np.uint32).reshape(world, 2, P)
    owner = np.empty(P, np.int32)
    send_off = np.empty((2, P), np.uint64)
    recv_size = np.empty((2, world), np.uint64)
    bcast = np.empty(P, np.uint8)
    skip = np.empty(P, np.uint8)
    _check(_lib.mgj_plan_host(world, rank, bits, hist.ctypes.data, owner.ctypes.data, send_off.ctypes.data,
                              recv_size.ctypes.data, skew_bcast, bcast.ctypes.data, skip.ctypes.data, assign),
           "mgj_plan_host")
    return (owner, send_off, recv_size, bcast, skip) if with_bcast else (owner, send_off, recv_size)


def gen_relation(kind: str, rel: int, n_r: int, n_s: int, z: float, row0: int, count: int, keys, pays,
                 stream=None):
    """Fill device tensors keys/pays with rows [row0, row0+count) of the synthetic workload."""
    _check(_lib.mgj_gen_relation(GEN_KIND[kind], rel, n_r, n_s, float(z), row0, count, _ptr(keys), _ptr(pays),
                                 _stream(stream)), "mgj_gen_relation")
