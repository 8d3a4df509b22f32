#!/usr/bin/env python
"""Benchmark of the MG-Join hot path on B200 (BASELINE.json metric).

One "step" = one pass of the whole hot path (a1 histogram + exchange, a2
plan, a3 scatter/shuffle, a4 local partition, a5 build/probe, a6 reduce) over
the synthetic workload already resident in HBM:
  N=1  : config M2 at one GPU, 2^29 R + 2^29 S tuples (4 B key + 4 B id).
  N>1  : weak scaling, 2^29 R + 2^29 S per GPU (torchrun, one rank per GPU,
         symmetric-memory arenas, in-kernel peer stores over NVSwitch).
Device time per step = CUDA events on the join stream, barrier + synchronize
on both sides, max over ranks.  Inputs (8 GiB per GPU) are larger than L2.

  python bench.py [--gpus N --steps K --warmup W] [--impl reference]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "join input tuples/sec ((|R|+|S|)/T), GPU cycles/tuple; shuffle GB/s vs NVLink"
UNIT = "tuples/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="mgj", choices=["mgj", "reference"])
    ap.add_argument("--log2-per-gpu", type=int, default=29, help="tuples per relation per GPU (M2: 29)")
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="weak: 2^log2-per-gpu per GPU (M2); strong: 2^log2-total per relation over all GPUs (M3)")
    ap.add_argument("--log2-total", type=int, default=31, help="strong scaling: tuples per relation in total (M3: 31)")
    ap.add_argument("--workload", default="unique", choices=["unique", "wide", "zipf"])
    ap.add_argument("--z", type=float, default=1.0)
    ap.add_argument("--materialize", action="store_true")
    ap.add_argument("--radix-bits-global", type=int, default=0)
    ap.add_argument("--radix-bits-local", type=int, default=0)
    ap.add_argument("--local-split-bits", type=int, default=0, help="a4 first pass: 0 auto, -1 never, k forced")
    ap.add_argument("--cpu-sample-log2", type=int, default=28,
                    help="oracle sample: 2^k R + 2^k S unique tuples (cpu_baseline / --impl reference)")
    ap.add_argument("--skew-bcast", type=int, default=0, choices=[-1, 0, 1],
                    help="a2 selective broadcast of heavy S partitions (N>1): 0 auto, -1 never, 1 forced")
    ap.add_argument("--num-sms", type=int, default=0, help="SMs the library's persistent kernels use (0 = all)")
    ap.add_argument("--overlap", default="auto", choices=["auto", "on", "off", "stream"],
                    help="§8(e): R's local pass beside S's scatter (auto: on for N > 1 with the P2P shuffle); stream: S's local pass too, chunk by chunk as scatter rounds complete (NEXT-3)")
    ap.add_argument("--overlap-local-sms", type=int, default=0)
    ap.add_argument("--trace", action="store_true", help="kernel timeline of the last step in the JSON line")
    ap.add_argument("--placement-z", type=float, default=0.0,
                    help="N>1: rank g holds a 1/(g+1)^z share of the rows (Fig. 9's placement-skew reading)")
    ap.add_argument("--assign", type=int, default=0, choices=[0, 1],
                    help="a2 assignment: 0 contiguous ranges, 1 placement-aware (Track-Join migration)")
    ap.add_argument("--compress", action="store_true",
                    help="NEXT-1 compressed shuffle (4-byte keys, id payloads): 32-byte units of five entries")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--profile", action="store_true", help="short run for ncu (no clocks/cpu/e2e)")
    ap.add_argument("--shuffle", default="p2p", choices=["p2p", "nccl"],
                    help="p2p: in-kernel peer stores (product); nccl: NCCL all_to_all_single baseline")
    return ap.parse_args()


def workload_name(a) -> str:
    if a.scaling == "strong":
        return f"M3 ({a.workload}, 2^{a.log2_total} R + 2^{a.log2_total} S in total over all GPUs)"
    if a.workload == "zipf":
        return f"M4-like zipf z={a.z} (2^{a.log2_per_gpu - 2} R + 2^{a.log2_per_gpu} S per GPU)"
    return {"unique": "M2", "wide": "M5"}[a.workload] + \
        f" ({a.workload}, 2^{a.log2_per_gpu} R + 2^{a.log2_per_gpu} S per GPU)"


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clock / throttle sampling during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.1)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, smax, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                smax = float(f[1])
            except ValueError:
                continue
            for nm, v in zip(names, f[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": smax,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------ oracle timing
def cpu_baseline(log2: int) -> dict:
    """The CPU oracle (single thread, plain C) on a bounded sample of the workload."""
    import oracle
    from paper_conf_sigmod_paullhl21_b200 import datagen
    n = 1 << log2
    d = datagen.Workload("unique", n, n).rank_inputs()
    t0 = time.perf_counter()
    r = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    dt = time.perf_counter() - t0
    assert r["count"] == n and r["checksum"] == ((1 << 32) + 1) * n * (n - 1) // 2 % (1 << 64)
    return {"value": 2 * n / dt, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"unique keys, 2^{log2} R + 2^{log2} S tuples (4B key + 4B id), 100% selectivity; "
                      f"{dt:.2f} s single-threaded on 1 of {os.cpu_count()} host cores "
                      f"({_cpu_model()})",
            "seconds": dt}


def _cpu_model() -> str:
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def run_reference(a, out) -> None:
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import oracle
    from paper_conf_sigmod_paullhl21_b200 import datagen
    n = 1 << min(a.cpu_sample_log2, 24)
    d = datagen.Workload("unique", n, n).rank_inputs()
    for _ in range(a.warmup):
        oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
    ts = []
    for _ in range(a.steps):
        t0 = time.perf_counter()
        oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
        ts.append(time.perf_counter() - t0)
    ms = 1000 * sum(ts) / len(ts)
    v = 2 * n / (ms / 1000)
    sample = (f"each step joins a bounded sample: 2^{int(np.log2(n))} R + 2^{int(np.log2(n))} S unique tuples "
              f"of the M2 workload shape, single-threaded, 1 of {os.cpu_count()} cores ({_cpu_model()})")
    emit(out, {
        "impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world, "steps": a.steps,
        "warmup": a.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": f"M2 sample (oracle), 2^{int(np.log2(n))}+2^{int(np.log2(n))} tuples",
                   "tuple_bytes": 8},
        "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample},
        "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    })


# ------------------------------------------------------------------ main bench
def _claim_stdout():
    """Keep the process's stdout for the single JSON line: everything else
    (NCCL banners, library chatter) is redirected to stderr."""
    sys.stdout.flush()
    out = os.fdopen(os.dup(1), "w")
    os.dup2(2, 1)
    return out


def emit(out, obj) -> None:
    out.write(json.dumps(obj) + "\n")
    out.flush()


def self_launch(n: int) -> None:
    """`bench.py --gpus N` (N > 1) started without torchrun: re-execute this
    script under torch.distributed.run, one rank per GPU, on 127.0.0.1."""
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *sys.argv[1:]]
    sys.stdout.flush()
    sys.stderr.flush()
    os.execv(sys.executable, cmd)


def expected_shard(torch, kind: str, kb: int, n_r: int, s_keys, s_pays):
    """(count, checksum, pair digest) of this rank's S shard joined with the
    whole R, from the generator alone (no join code): R.key[i] = perm(i)
    (mix64(perm(i)) for 8-byte keys) with payload i (2^40 + i), so the R row
    an S key matches is i = perm^-1(key); a Zipf miss row has key >= |R|.
    int64 arithmetic wraps modulo 2^64 like the C3 / C3b sums."""
    from paper_conf_sigmod_paullhl21_b200 import datagen
    k = datagen.ceil_log2(n_r)
    assert n_r == 1 << k, "closed-form check needs |R| = 2^k"
    if kb == 4:
        key = s_keys.long() & 0xFFFFFFFF
        b = s_pays.long() & 0xFFFFFFFF
    else:
        key = datagen.unmix64_t(s_keys.long())
        b = s_pays.long()
    hit = key < n_r if kind == "zipf" else torch.ones_like(key, dtype=torch.bool)
    i = datagen.perm_k_inverse_t(key, k, datagen.SEED_R)
    a = i if kb == 4 else i + (1 << 40)
    a = torch.where(hit, a, torch.zeros_like(a))
    b = torch.where(hit, b, torch.zeros_like(b))
    chk = (a << 32) + b if kb == 4 else a * datagen._s64(0x9E3779B97F4A7C15) + b
    return int(hit.sum()), int(chk.sum()), int((a * b).sum())


def main():
    a = parse()
    if a.gpus > 1 and "WORLD_SIZE" not in os.environ:
        self_launch(a.gpus)
    out = _claim_stdout()
    if a.impl == "reference":
        run_reference(a, out)
        return
    import torch
    import torch.distributed as dist

    from paper_conf_sigmod_paullhl21_b200 import mgj

    rank, world, local = dist_env()
    assert world == a.gpus or (world == 1 and a.gpus == 1), "launch N>1 with torchrun --nproc-per-node N"
    torch.cuda.set_device(local)
    # N>1: one rank per GPU over NCCL with symmetric-memory arenas.  MGJ_SYMM_ARENA=1 forces the
    # same symmetric-memory path at N=1 (under torchrun) to exercise it on a single GPU.
    distributed = world > 1 or os.environ.get("MGJ_SYMM_ARENA") == "1"
    assert a.shuffle == "p2p" or distributed, "--shuffle nccl needs torchrun (or MGJ_SYMM_ARENA=1)"
    if distributed:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    stream = torch.cuda.Stream(device=dev)

    wide = a.workload == "wide"
    kb = 8 if wide else 4
    dt = torch.int64 if wide else torch.int32
    per = 1 << a.log2_per_gpu
    if a.scaling == "strong":  # M3: the job size is fixed, each GPU holds 1/N of it
        n_tot = 1 << a.log2_total
        n_r, n_s = (n_tot // 4, n_tot) if a.workload == "zipf" else (n_tot, n_tot)
    elif a.workload == "zipf":
        n_r, n_s = world * per // 4, world * per  # |R|:|S| = 1:4
    else:
        n_r = n_s = world * per
    from paper_conf_sigmod_paullhl21_b200 import datagen as _dg
    r_lo, r_hi = _dg.shard_bounds(n_r, rank, world, a.placement_z)
    s_lo, s_hi = _dg.shard_bounds(n_s, rank, world, a.placement_z)
    nr, ns = r_hi - r_lo, s_hi - s_lo
    cols = [torch.empty(x, dtype=dt, device=dev) for x in (nr, nr, ns, ns)]
    with torch.cuda.stream(stream):
        mgj.gen_relation(a.workload, 0, n_r, n_s, a.z, r_lo, nr, cols[0], cols[1], stream)
        mgj.gen_relation(a.workload, 1, n_r, n_s, a.z, s_lo, ns, cols[2], cols[3], stream)
    stream.synchronize()

    cfg = mgj.make_config(rank=rank, world_size=world, key_bytes=kb, r_capacity=nr, s_capacity=ns,
                          materialize=a.materialize, radix_bits_global=a.radix_bits_global,
                          radix_bits_local=a.radix_bits_local, local_split_bits=a.local_split_bits,
                          # job-wide receive capacities (identical on every rank): skewed keys or
                          # placement can concentrate a relation on one rank
                          recv_capacity_r=(n_r if world > 1 and (a.workload == "zipf" or a.placement_z) else 0),
                          recv_capacity_s=(n_s // 2 if world > 1 and a.workload == "zipf" and not a.placement_z
                                           else (n_s if world > 1 and a.placement_z else 0)),
                          shuffle_mode=(mgj.SHUFFLE_EXTERNAL if a.shuffle == "nccl" else mgj.SHUFFLE_P2P),
                          skew_bcast=a.skew_bcast, num_sms=a.num_sms,
                          shuffle_overlap={"auto": 0, "on": 1, "off": -1, "stream": 2}[a.overlap],
                          overlap_local_sms=a.overlap_local_sms, trace=a.trace, compress=a.compress,
                          assign=a.assign)
    # N>1 (or MGJ_SYMM_ARENA=1): the library's symmetric-memory setup (mgj.symmetric_join)
    join = mgj.symmetric_join(cfg) if distributed else mgj.Join(cfg)

    def nccl_exchange():
        """Baseline shuffle: NCCL all_to_all_single of the per-destination send buffers."""
        mgj.nccl_exchange(join, stream)

    def step(inputs=None):
        join.partition(*(cols if inputs is None else inputs), stream=stream)
        join.shuffle(stream)
        if a.shuffle == "nccl":
            nccl_exchange()
        join.join(stream)

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
            torch.cuda.synchronize()

    for _ in range(max(a.warmup, 1)):
        step()
        res = join.result()

    sampler = ClockSampler(local) if (rank == 0 and not a.profile) else None
    if sampler:
        sampler.start()
        time.sleep(0.3)
    barrier()
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(a.steps + 1)]
    evs[0].record(stream)
    for i in range(a.steps):  # enqueued back to back: no host sync inside the timed region
        step()
        evs[i + 1].record(stream)
    barrier()
    res = join.result()  # the last timed step's result (a6 ran inside it)
    clocks = sampler.stop() if sampler else None
    timeline = {k: [round(v[0] / 1e3, 1), round(v[1] / 1e3, 1)] for k, v in join.trace().items()} if a.trace else None

    # correctness of the timed run: global count, checksum and pair digest
    # against the generator-derived values (every workload; SURVEY.md §8c
    # closed forms, readings C3 / C3b), summed over the ranks' S shards
    M64 = (1 << 64) - 1
    exp = [0, 0, 0] if a.profile else list(expected_shard(torch, a.workload, kb, n_r, cols[2], cols[3]))
    if world > 1:
        t = torch.tensor([x - (1 << 64) if x >= 1 << 63 else x for x in (v & M64 for v in exp)],
                         dtype=torch.int64, device=dev)
        dist.all_reduce(t)  # int64 sums wrap modulo 2^64
        exp = [int(x) for x in t.tolist()]
    exp_count, exp_chk, exp_dig = exp[0] & M64, exp[1] & M64, exp[2] & M64
    expect_ok = (res["status"] == 0 and res["match_count"] == exp_count and res["checksum"] == exp_chk
                 and res["pair_digest"] == exp_dig)
    if a.workload == "unique":  # Appendix A closed forms as well
        n = n_r
        expect_ok = expect_ok and exp_count == n and exp_chk == ((1 << 32) + 1) * n * (n - 1) // 2 & M64
    # per-phase breakdown: the last timed step's phase events (the library records
    # them on the join stream around each phase), plus three untimed steps
    phases = [res["phase_ms"]]
    for _ in range(3):
        step()
        phases.append(join.result()["phase_ms"])
    step_ms = [evs[i].elapsed_time(evs[i + 1]) for i in range(a.steps)]
    total_ms = evs[0].elapsed_time(evs[-1])
    if world > 1:
        t = torch.tensor([total_ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
    ms_per_step = total_ms / a.steps
    tuples_job = n_r + n_s
    value = tuples_job / (ms_per_step / 1000.0)

    # per-phase device times (median over steps) and rooflines
    ph = np.median(np.array(phases), axis=0)
    names = ["hist", "plan", "shuffle", "local_part", "probe", "reduce"]
    tb = 2 * kb
    n_local = nr + ns
    recv = res["recv_r"] + res["recv_s"]
    alg = {"hist": kb * n_local, "shuffle": 2 * tb * n_local, "local_part": 2 * tb * recv,
           "probe": tb * recv + (3 * kb * res["local_count"] if a.materialize else 0)}
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except (OSError, ValueError):
        pass
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0))
    peak_src = "measured (MEASURED_PEAKS.json hbm_gbs)" if "hbm_gbs" in peaks else "fallback (B200_PROFILING.md)"
    phase_report = {}
    for i, nm in enumerate(names):
        d = {"ms": float(ph[i])}
        if nm in alg and ph[i] > 0:
            gbs = alg[nm] / (ph[i] / 1000.0) / 1e9
            d.update(alg_bytes=int(alg[nm]), gbs=gbs, frac_hbm=gbs / hbm_peak)
        phase_report[nm] = d
    kern = {"shuffle": "k_scatter", "local_part": "k_local", "probe": "k_probe", "hist": "k_hist"}
    if a.compress:  # the receive sizes count 32-byte units: the scatter writes, the local pass reads units
        recv_t = n_local  # received tuples, taken as this rank's share (exact at N = 1)
        alg.update(shuffle=tb * n_local + 32 * recv, local_part=32 * recv + tb * recv_t,
                   probe=tb * recv_t + (3 * kb * res["local_count"] if a.materialize else 0))
        for nm in ("shuffle", "local_part", "probe"):
            i = names.index(nm)
            if ph[i] > 0:
                gbs = alg[nm] / (ph[i] / 1000.0) / 1e9
                phase_report[nm].update(alg_bytes=int(alg[nm]), gbs=gbs, frac_hbm=gbs / hbm_peak)
    dom = max(alg, key=lambda k: phase_report[k]["ms"])
    traffic = None
    try:
        tr = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))
        traffic = tr.get(kern[dom])
    except (OSError, ValueError):
        pass
    roof = {"bound": "hbm", "kernel": kern[dom], "achieved": phase_report[dom]["gbs"], "peak": hbm_peak,
            "unit": "GB/s", "frac": phase_report[dom]["gbs"] / hbm_peak, "traffic": traffic,
            "peak_source": peak_src,
            "alg_bytes_per_launch": phase_report[dom]["alg_bytes"]}
    if kern[dom] == "k_scatter":
        # measured (profiles/r2): the scatter keeps the SM's L1 data pipe ~80% busy
        # (shared ranking atomics and random 8-byte stores, the write-out's loads and global stores);
        # its time scales with the SM count, not with HBM
        roof["limiter"] = "per-SM L1 data pipe (~80% busy: ranking atomics, random shared stores, write-out), not DRAM"

    sm_mhz = (clocks or {}).get("sm_mhz") or float(peaks.get("sm_max_mhz", 1965.0))
    nsm = torch.cuda.get_device_properties(dev).multi_processor_count
    cyc = (ms_per_step / 1000.0) * sm_mhz * 1e6 * world / tuples_job
    # shuffle bytes: the wire format (8-byte tuples, or 32-byte units of up to five compressed
    # tuples), from the receive sizes; over NVLink per GPU (egress) the (N-1)/N share
    wire = torch.tensor([float((res["recv_r"] + res["recv_s"]) * (32 if a.compress else tb))], device=dev)
    if world > 1:
        dist.all_reduce(wire)
    wire_per_tuple = float(wire.item()) / tuples_job
    nvl_bytes = wire_per_tuple * n_local * (world - 1) / world
    shuffle_ms = phase_report["shuffle"]["ms"]

    # end-to-end: host (pinned) inputs through the C ABI, H2D inside the timed region
    e2e = None
    if not a.no_e2e and not a.profile:
        host = [torch.empty(c.numel(), dtype=dt, pin_memory=True) for c in cols]
        for h, c in zip(host, cols):
            h.copy_(c)
        hnp = [h.numpy() for h in host]
        barrier()
        step(hnp)
        join.result()
        barrier()
        t0 = time.perf_counter()
        for _ in range(a.e2e_steps):
            step(hnp)
            r2 = join.result()
        t_e2e = time.perf_counter() - t0
        if world > 1:
            t = torch.tensor([t_e2e], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            t_e2e = float(t.item())
        assert (r2["match_count"], r2["checksum"], r2["pair_digest"]) == \
            (res["match_count"], res["checksum"], res["pair_digest"])
        e2e = {"value": tuples_job / (t_e2e / a.e2e_steps), "unit": UNIT,
               "h2d_bytes_per_step": int(sum(h.numel() * h.element_size() for h in host)),
               "d2h_bytes_per_step": 32 + 64, "steps": a.e2e_steps,
               "note": "pinned host columns passed to mgj_partition (library stages H2D on the stream); "
                       "mgj_result reads count/checksum back; host wall clock"}
        del host, hnp

    cpu = None
    if rank == 0 and not a.no_cpu_baseline and not a.profile:
        cpu = cpu_baseline(a.cpu_sample_log2)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": a.scaling,
            "vs_baseline": None, "dtype": "u32" if kb == 4 else "u64", "data": "synthetic",
            "config": {"workload": workload_name(a),
                       "tuples_R": n_r, "tuples_S": n_s, "tuple_bytes": tb, "materialize": a.materialize,
                       "radix_bits_global": res["radix_bits_global"], "radix_bits_local": res["radix_bits_local"],
                       "l2": "inputs (8 GiB/GPU) larger than L2; no flush", "parallelism": f"dp{world}",
                       "shuffle": ("in-kernel peer stores (symmetric memory)" if a.shuffle == "p2p"
                                   else "NCCL all_to_all_single baseline (host sync per step for split sizes)"),
                       "global_batch": tuples_job, "seeds": {"R": "0x5EED0052", "S": "0x5EED0053"},
                       "skew_bcast": a.skew_bcast},
            "correct": None if a.profile else bool(expect_ok),
            "correct_from": "the last timed step's result (count, checksum, pair digest vs generator-derived values)",
            "match_count": res["match_count"], "checksum": hex(res["checksum"]),
            "pair_digest": hex(res["pair_digest"]),
            "gpu_cycles_per_tuple": {"sm_cycles_per_tuple": cyc * nsm, "gpu_cycles_per_tuple": cyc,
                                     "sm_mhz": sm_mhz, "sms": nsm,
                                     "formula": "T*f_SM*SMs*N/(|R|+|S|) and T*f_SM*N/(|R|+|S|)"},
            "phases": phase_report,
            "shuffle": {"wire_bytes_per_tuple": wire_per_tuple, "compress": a.compress,
                        "nvlink_egress_bytes_per_gpu": nvl_bytes,
                        "nvlink_gbs_per_gpu": (nvl_bytes / (shuffle_ms / 1000) / 1e9) if world > 1 else None,
                        "nvlink_peak_gbs": 900.0, "measured_peer_gbs": 770.0},
            "step_ms": {"median": statistics.median(step_ms), "min": min(step_ms), "max": max(step_ms)},
            "roofline": roof,
            "cpu_baseline": None if cpu is None else {k: cpu[k] for k in ("value", "unit", "cores", "kind", "sample")},
            "e2e": e2e,
            "gpu_launches": res["n_launches"] * a.steps,  # counted by the library per run
            "timeline_us": timeline,
            "clocks": clocks,
        }
        emit(out, line)
    join.close()
    if distributed:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
