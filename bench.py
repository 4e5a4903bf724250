#!/usr/bin/env python
"""bench.py — partitioned allreduce bus bandwidth (+ Pready->Parrived latency).

Driver contract (one JSON line on rank 0):
  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl pc|reference]
  N > 1 runs under torchrun, one rank per GPU (real ranks, CUDA IPC over
  NVLink/NVSwitch); `--gpus N` outside torchrun relaunches itself under
  torch.distributed.run.  Beside the allreduce it times NCCL all_reduce on the
  same bytes (default tuning and NCCL_ALGO=Ring, NCCL_DEBUG=INFO on stderr),
  a bare peer-copy floor (the NVLink roofline denominator), the C1/C2 p2p and
  Pready->Parrived latency legs between rank pairs and the C4 Jacobi solver
  over all ranks.  N = 1 runs the same hot path with P virtual ranks
  co-located on the one B200 (--vranks, default 8): every rank's buffers,
  flags and engine live on one GPU, so "NVLink" stores become HBM stores and
  the kernel is HBM-bound.  Beside the headline line N = 1 also reports the
  Pready->Parrived latency pairs, C4 Jacobi, C1 (1 MiB) and C2 at 256 MiB
  (the persistent register-Kernel-Copy producer vs kernel -> copy, with its
  own HBM roofline).

A step = one epoch of the whole hot path for every rank: pc_epoch_all (Start +
ready-to-receive + the user's Pready of every partition, one kernel for all
ranks of the GPU) -> pc_wait_on_stream (the engine: AUTO = the DIRECT
schedule for 3-8 ranks, PULL reduce in registers, the final chunk stored
into every rank's recvbuf).  value = bus bandwidth (nccl-tests convention) =
S/t * 2(P-1)/P with S bytes per rank.
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

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "partitioned allreduce bus GB/s vs msg size at 2/4/8 B200; Pready→Parrived latency (ns)"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="pc", choices=["pc", "reference"])
    ap.add_argument("--bytes", type=int, default=256 << 20, help="bytes per rank (S)")
    ap.add_argument("--partitions", type=int, default=64)
    ap.add_argument("--algo", default="auto", choices=["ring", "rd", "direct", "direct_push", "auto"])
    ap.add_argument("--vranks", type=int, default=8, help="virtual ranks on the one GPU when N = 1")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-latency", action="store_true")
    ap.add_argument("--no-jacobi", action="store_true")
    ap.add_argument("--no-c1", action="store_true",
                    help="skip the C1 leg (its host Progression Engine epochs cannot progress under ncu's serialisation)")
    ap.add_argument("--no-dl", action="store_true", help="N > 1: skip the DL-proxy goodput leg")
    ap.add_argument("--jacobi-n", type=int, default=16384)
    ap.add_argument("--jacobi-iters", type=int, default=50)
    ap.add_argument("--quiet", action="store_true", help="only the JSON line")
    return ap.parse_args()


T0 = time.time()


def log(*a):
    print(f"[bench {time.time() - T0:7.1f}s]", *a, file=sys.stderr, flush=True)


def engine_alg_bytes(algo, P, S):
    """Algorithmic HBM bytes of one grouped engine launch of P co-located ranks
    (DESIGN.md §6).  ring: per rank S/P*(3P-3) reads + S/P*(2P-1) writes;
    direct (PULL): per rank S read (its chunk from all P send buffers) + S
    written (the final chunk into all P recvbufs); rd: per rank log2P steps of
    (read acc + read incoming + write peer staging + write acc) + the final copy."""
    if P == 1:
        return 2 * S
    if algo == "direct":
        return 2 * P * S
    if algo == "direct_push":  # push (P-1)/P*S read + written, then fold S read + S written, per rank
        return int(2 * (P - 1) * S + 2 * P * S)
    if algo == "rd":
        return (4 * (P.bit_length() - 1) + 2) * P * S
    return (5 * P - 4) * S


def busbw(S, sec, P):
    return S / sec * (2.0 * (P - 1) / P) / 1e9 if P > 1 else S / sec / 1e9


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class Clocks:
    """nvidia-smi sampling during the timed region (clocks + throttle reasons)."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index=0):
        self.index = index
        self.p = None
        self.lines = []

    def __enter__(self):
        # NVML (nvidia_ml_py) samples every 2 ms, so even a ~100 ms timed
        # region gets dozens of samples; nvidia-smi -lms 100 is the fallback.
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nvml = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.mx = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.stop = threading.Event()
            self.t = threading.Thread(target=self._nvml_loop, daemon=True)
            self.t.start()
            return self
        except Exception:
            self.nvml = None
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.p = None
        return self

    def _read(self):
        for line in self.p.stdout:
            self.lines.append(line.strip())

    def _nvml_sample(self):
        nv = self.nvml
        bits = [("hw_slowdown", 0x8), ("hw_thermal_slowdown", 0x40), ("sw_thermal_slowdown", 0x20),
                ("sw_power_cap", 0x4)]
        try:
            sm = nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM)
            r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            f = [str(sm), str(self.mx), "0", hex(r)] + ["Active" if r & b else "Not Active" for _, b in bits]
            self.lines.append(", ".join(f))
        except Exception:
            pass

    def _nvml_loop(self):
        while not self.stop.is_set():
            self._nvml_sample()
            time.sleep(0.002)

    def sample_now(self):
        """One synchronous sample (called while the timed work is still queued
        on the GPU), so a short timed region is never left without a sample."""
        if getattr(self, "nvml", None):
            self._nvml_sample()
            return
        try:
            out = subprocess.run(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                  "--format=csv,noheader,nounits"], capture_output=True, text=True, timeout=10)
            self.lines.extend(x.strip() for x in out.stdout.splitlines() if x.strip())
        except Exception:
            pass

    def __exit__(self, *a):
        if getattr(self, "nvml", None):
            self.stop.set()
            self.t.join(timeout=2)
            return
        if self.p:
            self.p.terminate()
            try:
                self.p.wait(timeout=5)
            except Exception:
                self.p.kill()

    def summary(self):
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                mx = max(mx, float(f[1]))
            except ValueError:
                continue
            for n, v in zip(names, f[4:8]):
                if v.lower() == "active":
                    reasons.add(n)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": len(sm)}


# --------------------------------------------------------------------------- CPU oracle legs
def oracle_sample(P=8, S=8 << 20, Np=8, budget_s=12.0):
    """The CPU oracle (literal Alg 1 + Alg 2, P rank threads + P user
    threads) on a bounded sample of the workload; bus GB/s of the sample."""
    import numpy as np

    import oracle
    import synth
    n = S // 4
    x = np.stack([synth.normal_f32(synth.BASE_SEED, r, 0, n) for r in range(P)])
    oalgo, aname = (oracle.DIRECT, "direct") if 3 <= P <= 8 else (oracle.RING, "ring")  # the bench's AUTO choice
    oracle.pallreduce(x[:, : Np * 64], Np, oalgo)  # build + warm
    times = []
    t_end = time.perf_counter() + budget_s
    while time.perf_counter() < t_end or not times:
        t0 = time.perf_counter()
        oracle.pallreduce(x, Np, oalgo)
        times.append(time.perf_counter() - t0)
        if len(times) >= 50:
            break
    sec = statistics.median(times)
    return {"value": busbw(S, sec, P), "unit": "GB/s", "cores": 2 * P, "host_cpus": os.cpu_count(),
            "kind": "oracle",
            "sample": f"{aname} schedule + Alg 2 oracle, P={P} rank threads (+{P} Pready threads), {S >> 20} MiB fp32 "
                      f"per rank, {Np} partitions, median of {len(times)} runs"}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import numpy as np

    import oracle
    import synth
    P = args.vranks if args.gpus == 1 else args.gpus
    S, Np = 8 << 20, 8  # the bounded sample: 8 MiB of each rank's buffer, 8 partitions
    # the schedule the GPU arm's AUTO picks for this workload (DIRECT for 3..8
    # ranks, ring at 2): the oracle runs the same association (O6 / O3)
    oalgo, aname = (oracle.DIRECT, "direct") if 3 <= P <= 8 else (oracle.RING, "ring")
    n = S // 4
    x = np.stack([synth.normal_f32(synth.BASE_SEED, r, 0, n) for r in range(P)])
    for _ in range(args.warmup):
        oracle.pallreduce(x, Np, oalgo)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.pallreduce(x, Np, oalgo)
    sec = (time.perf_counter() - t0) / args.steps
    v = busbw(S, sec, P)
    where = (f"{P} virtual ranks co-located on one B200" if args.gpus == 1 else f"{P} ranks (one per B200)")
    out = {"impl": "reference", "metric": METRIC, "value": v, "unit": "GB/s", "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": sec * 1e3, "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
           "config": {"workload": f"partitioned allreduce (C5/C3 shape) fp32 sum, {where}: the CPU oracle on a "
                                  f"bounded slice of the GPU arm's workload — {S >> 20} MiB per rank in {Np} "
                                  f"partitions per step (GPU arm: {args.bytes >> 20} MiB in {args.partitions}), "
                                  f"{aname} schedule (requested {args.algo})",
                      "ranks": P, "bytes_per_rank": S, "partitions": Np, "algo": aname,
                      "gpu_arm_bytes_per_rank": args.bytes, "gpu_arm_partitions": args.partitions},
           "cpu_baseline": {"value": v, "unit": "GB/s", "cores": 2 * P, "host_cpus": os.cpu_count(), "kind": "oracle",
                            "sample": f"each step: the CPU oracle ({aname} schedule + the Alg 2 loop, {P} rank threads"
                                      f" + {P} Pready threads) on an {S >> 20} MiB-per-rank, {Np}-partition slice of "
                                      f"the workload; bus GB/s of the slice"},
           "e2e": {"value": v, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


# --------------------------------------------------------------------------- GPU legs
def latency_pair(pc, apps, torch, comms, iters=5000, payload=0, copy=None):
    """Pready->Parrived ping-pong between two ranks inside one launch
    (warp-granularity Pready; copy = INLINE flag+fence or LL lines)."""
    copy = pc.COPY_INLINE if copy is None else copy
    cnt = payload // 4
    st = torch.cuda.Stream()
    bufs = [torch.zeros(max(iters * cnt, 4), device="cuda") for _ in range(4)]
    bufs[0].copy_(torch.arange(bufs[0].numel(), dtype=torch.float32))
    a2b = pc.psend_init(bufs[0], iters, cnt, pc.FLOAT32, 1, 101, comms[0])
    b_in = pc.precv_init(bufs[1], iters, cnt, pc.FLOAT32, 0, 101, comms[1])
    b2a = pc.psend_init(bufs[2], iters, cnt, pc.FLOAT32, 0, 102, comms[1])
    a_in = pc.precv_init(bufs[3], iters, cnt, pc.FLOAT32, 1, 102, comms[0])
    for q in (a2b, a_in, b_in, b2a):
        q.start(st)
    pc.run_ranks([lambda: [q.pbuf_prepare(st) for q in (a2b, a_in)], lambda: [q.pbuf_prepare(st) for q in (b_in, b2a)]])
    pa, pai = a2b.prequest_create(pc.GRAN_WARP, 1, copy), a_in.prequest_create(pc.GRAN_WARP, 1, 0)
    pb, pbi = b2a.prequest_create(pc.GRAN_WARP, 1, copy), b_in.prequest_create(pc.GRAN_WARP, 1, 0)
    t = torch.zeros(2, dtype=torch.int64, device="cuda")
    rt = torch.zeros(iters, dtype=torch.int64, device="cuda")
    apps.pingpong_pair(pa, pai, pb, pbi, iters, apps.GRAN_WARP, t, st, rt_ns=rt)
    for q in (a2b, b2a, a_in, b_in):
        q.wait_on_stream(st)
    torch.cuda.synchronize()
    errs = [q.error()[0] for q in (a2b, b2a, a_in, b_in)]
    rts = rt.cpu().numpy()[iters // 10:] / 2.0  # one-way = round trip / 2; drop warm-up
    # the floor: the same ping-pong with two bare flags, no library, at the
    # scope the library uses for these ranks (GPU: relaxed; the release/acquire
    # and system-scope variants are reported beside it)
    floors = {}
    for sc, name in ((0, "relaxed_gpu"), (1, "acq_rel_gpu"), (2, "acq_rel_sys")):
        flags = torch.zeros(64, dtype=torch.int32, device="cuda")
        tb = torch.zeros(2, dtype=torch.int64, device="cuda")
        apps.bare_pingpong_pair(flags[0:], flags[32:], iters, 0, tb, st, scope=sc)
        torch.cuda.synchronize()
        floors[name] = float(tb[0].item()) / iters / 2.0
    bare = floors["relaxed_gpu"]
    for q in (a2b, a_in, b_in, b2a):
        q.free()
    import numpy as np
    ok = bool(torch.equal(bufs[1], bufs[0])) if cnt else True
    return {"p50": float(np.percentile(rts, 50)), "p99": float(np.percentile(rts, 99)),
            "mean": float(rts.mean()), "payload_bytes": payload, "iters": iters, "errors": errs,
            "copy": {0: "inline", 2: "ll"}.get(copy, copy), "payload_ok": ok,
            "bare_flag_floor_mean": bare, "bare_flag_variants_mean": floors,
            "frac_of_floor": bare / float(np.percentile(rts, 50))}


def c2_bench(pc, apps, torch, S=256 << 20, epochs=20):
    """C2 at its largest size (256 MiB): block-granularity Kernel Copy from
    the persistent producer (pc_put_begin + pc_pready_block_put, reading R35;
    Startall/Waitall control) against the traditional model (the same
    persistent vector add with no Pready, then a device copy), device time
    per epoch on one stream.  Parity: the receiver's buffer equals C."""
    n = S // 4
    g, cs = pc.local_comms(2, 0)
    st = torch.cuda.Stream()
    A, B = torch.randn(n, device="cuda"), torch.randn(n, device="cuda")
    Cb, R = torch.empty(n, device="cuda"), torch.empty(n, device="cuda")
    parts = n // 2048
    snd = pc.psend_init(Cb, parts, 2048, pc.FLOAT32, 1, 13, cs[0])
    rcv = pc.precv_init(R, parts, 2048, pc.FLOAT32, 0, 13, cs[1])
    snd.start(st)
    rcv.start(st)
    pc.run_ranks([lambda: snd.pbuf_prepare(st), lambda: rcv.pbuf_prepare(st)])
    sq = snd.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
    apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK_PUT, sq, st, persistent=True)
    pc.waitall_on_stream([snd, rcv], st)

    def epoch():
        pc.epoch_all([snd, rcv], pready=False, stream=st)
        apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK_PUT, sq, st, persistent=True)
        pc.waitall_on_stream([snd, rcv], st)

    def trad():
        apps.vecadd(A, B, Cb, n, apps.GRAN_NONE, None, st, persistent=True)
        with torch.cuda.stream(st):
            R.copy_(Cb)

    out = {}
    for name, fn in (("traditional_us", trad), ("partitioned_us", epoch)):
        for _ in range(3):
            fn()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(st)
        for _ in range(epochs):
            fn()
        e1.record(st)
        torch.cuda.synchronize()
        out[name] = e0.elapsed_time(e1) / epochs * 1e3
    R.zero_()
    epoch()
    torch.cuda.synchronize()
    ok = bool(torch.equal(R, Cb)) and snd.error()[0] == 0 and rcv.error()[0] == 0
    snd.free()
    rcv.free()
    for c in cs:
        c.destroy()
    g.destroy()
    hbm, src = peaks()
    alg = 4 * S  # A and B read, C written, C pushed (the peer is HBM of the same GPU here)
    out["roofline"] = {"bound": "hbm", "algorithmic_bytes_per_epoch": alg,
                       "achieved": alg / (out["partitioned_us"] / 1e6) / 1e9, "peak": hbm, "unit": "GB/s",
                       "frac": alg / (out["partitioned_us"] / 1e6) / 1e9 / hbm, "peak_source": src,
                       "note": "whole epoch (control + producer + both waits), not the producer kernel alone"}
    out.update({"bytes": S, "partitions": parts, "gran": "block_put (R35), persistent producer", "copy": "inline",
                "speedup_vs_traditional": out["traditional_us"] / out["partitioned_us"],
                "goodput_gbs": S / (out["partitioned_us"] / 1e6) / 1e9, "ok": ok,
                "note": "2 virtual ranks on one B200: both models move the same HBM bytes; tools/sweep.py p2p"})
    return out


def c1_bench(pc, apps, torch, epochs=200):
    """C1: 2 ranks, 1 MiB fp32 produced by a vector-add kernel (8 B/thread,
    1024-thread blocks) with block-granularity Pready: 128 user partitions of
    8 KiB aggregated g = 16 -> 8 transport partitions (reading R24), INLINE
    "Kernel Copy".  Goodput = bytes / (kernel + communication) time,
    against the traditional model (kernel -> cudaStreamSynchronize -> copy,
    Listing 1)."""
    import time as _t
    n = 1 << 18
    g, cs = pc.local_comms(2, 0)
    st = torch.cuda.Stream()
    A, B = torch.randn(n, device="cuda"), torch.randn(n, device="cuda")
    Cb, R = torch.empty(n, device="cuda"), torch.empty(n, device="cuda")
    snd = pc.psend_init(Cb, 128, 2048, pc.FLOAT32, 1, 11, cs[0])
    rcv = pc.precv_init(R, 128, 2048, pc.FLOAT32, 0, 11, cs[1])
    snd.start(st)
    rcv.start(st)
    pc.run_ranks([lambda: snd.pbuf_prepare(st), lambda: rcv.pbuf_prepare(st)])
    sq = snd.prequest_create(pc.GRAN_BLOCK, 16, pc.COPY_INLINE)
    apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK, sq, st)
    snd.wait_on_stream(st)
    rcv.wait_on_stream(st)
    torch.cuda.synchronize()

    def epoch():  # Listing 2: Start, Pbuf_prepare, kernel (Pready inside), Wait
        pc.epoch_all([snd, rcv], pready=False, stream=st)  # Startall + Pbuf_prepare of both, one kernel
        apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK, sq, st)
        pc.waitall_on_stream([snd, rcv], st)  # both ranks' waits in one kernel

    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(epochs):
        epoch()
    e1.record(st)
    torch.cuda.synchronize()
    part_us = e0.elapsed_time(e1) / epochs * 1e3
    ok = bool(torch.equal(R, Cb)) and snd.error()[0] == 0 and rcv.error()[0] == 0

    def epoch_put():  # the same epoch from the persistent register-Kernel-Copy producer (R35)
        pc.epoch_all([snd, rcv], pready=False, stream=st)
        apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK_PUT, sq, st, persistent=True)
        pc.waitall_on_stream([snd, rcv], st)

    for _ in range(3):
        epoch_put()
    torch.cuda.synchronize()
    e0.record(st)
    for _ in range(epochs):
        epoch_put()
    e1.record(st)
    torch.cuda.synchronize()
    put_us = e0.elapsed_time(e1) / epochs * 1e3
    ok = ok and bool(torch.equal(R, Cb)) and snd.error()[0] == 0 and rcv.error()[0] == 0
    # traditional: kernel, host synchronisation, then the copy (Listing 1)
    t0 = _t.perf_counter()
    for _ in range(epochs):
        apps.vecadd(A, B, Cb, n, apps.GRAN_NONE, None, st)
        st.synchronize()
        with torch.cuda.stream(st):
            R.copy_(Cb)
        st.synchronize()
    trad_us = (_t.perf_counter() - t0) / epochs * 1e6
    # partitioned, host-observed the same way (Listing 2: ... kernel; MPI_Wait)
    t0 = _t.perf_counter()
    for _ in range(epochs):
        epoch()
        st.synchronize()
    part_host_us = (_t.perf_counter() - t0) / epochs * 1e6
    # the same epoch captured once into a CUDA graph (epochs advance on the device)
    gr = torch.cuda.CUDAGraph()
    with torch.cuda.graph(gr, stream=st):
        epoch()
    t0 = _t.perf_counter()
    for _ in range(epochs):
        with torch.cuda.stream(st):
            gr.replay()
        st.synchronize()
    graph_host_us = (_t.perf_counter() - t0) / epochs * 1e6
    ok = ok and bool(torch.equal(R, Cb)) and snd.error()[0] == 0 and rcv.error()[0] == 0
    # the paper's host Progression Engine (PC_COPY_HOST; NEXT-4):
    # the same epochs with the transfer issued by the library's host thread
    R2 = torch.empty(n, device="cuda")
    snd2 = pc.psend_init(Cb, 128, 2048, pc.FLOAT32, 1, 12, cs[0])
    rcv2 = pc.precv_init(R2, 128, 2048, pc.FLOAT32, 0, 12, cs[1])
    snd2.start(st)
    rcv2.start(st)
    pc.run_ranks([lambda: snd2.pbuf_prepare(st), lambda: rcv2.pbuf_prepare(st)])
    sq2 = snd2.prequest_create(pc.GRAN_BLOCK, 16, pc.COPY_HOST)
    apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK, sq2, st)
    snd2.wait_on_stream(st)
    rcv2.wait_on_stream(st)
    st.synchronize()
    t0 = _t.perf_counter()
    for _ in range(epochs):
        pc.epoch_all([snd2, rcv2], pready=False, stream=st)  # same control path as the Kernel Copy epochs
        apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK, sq2, st)
        pc.waitall_on_stream([snd2, rcv2], st)
        st.synchronize()
    pe_host_us = (_t.perf_counter() - t0) / epochs * 1e6
    ok = ok and bool(torch.equal(R2, Cb)) and snd2.error()[0] == 0 and rcv2.error()[0] == 0
    snd2.free()
    rcv2.free()
    snd.free()
    rcv.free()
    for c in cs:
        c.destroy()
    g.destroy()
    return {"bytes": 4 * n, "partitions": 128, "transport_partitions": 8, "gran": "block", "copy": "inline",
            "partitioned_us_device": part_us, "partitioned_put_persistent_us_device": put_us,
            "partitioned_us_host": part_host_us,
            "partitioned_graph_us_host": graph_host_us, "traditional_us_host": trad_us,
            "goodput_gbs": 4 * n / (part_host_us / 1e6) / 1e9, "speedup_vs_traditional": trad_us / part_host_us,
            "speedup_graph_vs_traditional": trad_us / graph_host_us,
            "progression_engine_us_host": pe_host_us, "speedup_vs_progression_engine": pe_host_us / part_host_us,
            "ok": ok, "note": "2 virtual ranks on one B200; paper: Kernel Copy up to 2.34x vs traditional, PE ~1.0x above 16 MiB (P:L245, GH200)"}


def jacobi_bench(pc, apps, torch, args):
    """C4: Jacobi 16384^2 fp32, 1 rank and 4x2 virtual ranks (intra-kernel
    partitioned halos), GFLOP/s at 4 flops per interior cell update (R17) and
    the HBM fraction at 8 B per cell update."""
    import numpy as np
    N, K = args.jacobi_n, args.jacobi_iters
    hbm_peak, _ = peaks()
    res = {}
    for Py, Px in ((1, 1), (2, 1), (2, 2), (4, 2), (8, 1)):
        P = Py * Px
        g, cs = pc.local_comms(P, 0)
        st = torch.cuda.Stream()
        js = apps.JacobiSolver(cs, list(range(P)), N, Py, Px, K, H=int(os.environ.get("PC_JACOBI_H", "64")))
        res["kernel"] = f"{js.kernel} (W={js.W}, H={js.H})"
        for s in js.local:  # perf init: top edge 1.0, rest 0
            s["grid"][0].zero_()
            if s["py"] == 0:
                s["grid"][0][: js.lx].fill_(1.0)
            s["grid"][1].copy_(s["grid"][0])
        torch.cuda.synchronize()
        fp = lambda lists: pc.run_ranks([(lambda l=l: [q.pbuf_prepare(st) for q in l]) for l in lists])
        js.solve(st, first_prepare=fp)  # warm-up epoch
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 3
        e0.record(st)
        for _ in range(reps):
            js.solve(st)
        e1.record(st)
        torch.cuda.synchronize()
        errs = js.errors()
        ms_iter = e0.elapsed_time(e1) / (reps * K)  # per iteration, the per-epoch init push included
        cells = (N - 2) * (N - 2)
        res[f"{Py}x{Px}"] = {"gflops": 4.0 * cells / (ms_iter / 1e3) / 1e9, "us_per_iter": ms_iter * 1e3,
                             "hbm_frac": (8.0 * N * N / (ms_iter / 1e3) / 1e9) / hbm_peak,
                             "ranks": P, "errors": errs}
        js.free()
        for c in cs:
            c.destroy()
        g.destroy()
    # C4 comparison (i): the same decomposition with kernel -> sync -> copy halos (Listing 1)
    g, cs = pc.local_comms(8, 0)
    st = torch.cuda.Stream()
    js = apps.JacobiSolver(cs, list(range(8)), N, 4, 2, K, H=int(os.environ.get("PC_JACOBI_H", "64")), traditional=True)
    js.solve(st)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(3):
        js.solve(st)
    e1.record(st)
    torch.cuda.synchronize()
    ms_iter = e0.elapsed_time(e1) / (3 * K)
    res["4x2_traditional"] = {"gflops": 4.0 * (N - 2) * (N - 2) / (ms_iter / 1e3) / 1e9, "us_per_iter": ms_iter * 1e3,
                              "hbm_frac": (8.0 * N * N / (ms_iter / 1e3) / 1e9) / hbm_peak, "ranks": 8,
                              "halos": "kernel -> cudaStreamSynchronize -> cudaMemcpyAsync per edge (Listing 1)"}
    res["speedup_partitioned_vs_traditional_4x2"] = res["4x2_traditional"]["us_per_iter"] / res["4x2"]["us_per_iter"]
    js.free()
    for c in cs:
        c.destroy()
    g.destroy()
    res["config"] = f"{N}^2 fp32, {K} iterations per epoch, virtual ranks on one B200, 8 B/cell-update roofline"
    return res


def e2e_pipelined(pc, torch, reqs, send, host_in, recv0, host_out, Np, count, st, steps, chunks=8):
    """End to end through the public API with host buffers: every step copies
    its inputs host -> device and its result device -> host.  The epoch is
    pipelined the partitioned way: pc_epoch_all (Start + ready-to-receive, no
    Pready) forks the engine, then the inputs arrive over PCIe in chunks of
    partitions, each chunk Preadied (pc_pready_range) right after its copy, so
    the engine reduces while the rest is still in flight; the result's D2H of
    step i overlaps the H2D of step i+1 (separate copy streams, PCIe is full
    duplex).  Returns ms per step (CUDA events, all streams joined)."""
    st_in, st_out = torch.cuda.Stream(), torch.cuda.Stream()
    CH = max(1, -(-Np // chunks))
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev_ctl, ev_done, ev_out = torch.cuda.Event(), torch.cuda.Event(), torch.cuda.Event()
    f0.record(st)
    st_in.wait_event(f0)
    st_out.wait_event(f0)
    for i in range(steps):
        if i:
            st_in.wait_event(ev_done)  # step i-1's engine finished reading the send buffers
            st.wait_event(ev_out)      # step i-1's result was read out: recvbuf is free (RTR)
        pc.epoch_all(reqs, pready=False, stream=st)
        ev_ctl.record(st)
        for c0 in range(0, Np, CH):
            c1 = min(c0 + CH, Np)
            with torch.cuda.stream(st_in):
                for r in range(len(reqs)):
                    send[r][c0 * count:c1 * count].copy_(host_in[r][c0 * count:c1 * count], non_blocking=True)
            if c0 == 0:
                st_in.wait_event(ev_ctl)  # the Pready kernels read this epoch's word
            for q in reqs:
                q.pready_range(c0, c1 - 1, st_in)
        for q in reqs:
            q.wait_on_stream(st)
        ev_done.record(st)
        st_out.wait_event(ev_done)
        with torch.cuda.stream(st_out):
            host_out.copy_(recv0, non_blocking=True)
        ev_out.record(st_out)
    st.wait_event(ev_out)
    st.wait_stream(st_in)
    f1.record(st)
    torch.cuda.synchronize()
    return f0.elapsed_time(f1) / steps


def run_virtual(args):
    import numpy as np
    import torch

    import paper_conf_sc_temucinslsga24_b200 as pc
    from paper_conf_sc_temucinslsga24_b200 import apps

    torch.cuda.set_device(0)
    P, S, Np = args.vranks, args.bytes, args.partitions
    count = S // 4 // Np
    S = count * 4 * Np
    algo = {"ring": pc.ALGO_RING, "rd": pc.ALGO_RD, "direct": pc.ALGO_DIRECT, "direct_push": pc.ALGO_DIRECT_PUSH,
            "auto": pc.ALGO_AUTO}[args.algo]
    g, comms = pc.local_comms(P, 0)
    st = torch.cuda.Stream()
    gen = torch.Generator(device="cuda")
    gen.manual_seed(0x5C24)
    send = [torch.randn(Np * count, device="cuda", generator=gen) for _ in range(P)]
    recv = [torch.empty(Np * count, device="cuda") for _ in range(P)]
    reqs = [pc.pallreduce_init(send[r], recv[r], Np, count, pc.FLOAT32, pc.SUM, algo, comms[r]) for r in range(P)]
    torch.cuda.synchronize()

    def step(first=False):
        if first:
            for q in reqs:
                q.start(st)
            pc.run_ranks([(lambda q=q: q.pbuf_prepare(st)) for q in reqs])
            pc.preadyall(reqs, st)  # S_0: the user's Pready of every partition, one kernel
        else:  # pc_epoch_all: Start + ready-to-receive + S_0 Pready of every rank, ONE kernel
            pc.epoch_all(reqs, pready=True, stream=st)
        for q in reqs:
            q.wait_on_stream(st)

    log("init done; first step")
    step(first=True)
    torch.cuda.synchronize()
    log("first step done")
    for _ in range(max(args.warmup - 1, 0)):
        step()
    torch.cuda.synchronize()
    log("warmup done")
    for q in reqs:
        assert q.error()[0] == 0, f"device error {q.error()}"
    info = reqs[0].info()
    reqs[0].set_timing(True)
    reqs[0].engine_times()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n0 = pc.launch_count()
    with Clocks(0) as clk:
        torch.cuda.synchronize()
        e0.record(st)
        for _ in range(args.steps):
            step()
        e1.record(st)
        clk.sample_now()  # the steps are still running: one sample inside the timed region
        torch.cuda.synchronize()
    launches = pc.launch_count() - n0
    ms = e0.elapsed_time(e1) / args.steps
    log(f"timed: {ms:.3f} ms/step")
    eng = reqs[0].engine_times()
    reqs[0].set_timing(False)
    for q in reqs:
        assert q.error()[0] == 0, f"device error {q.error()}"
    # sanity (not parity — tests/ hold parity): every rank holds identical bits
    for r in range(1, P):
        assert torch.equal(recv[r][:4096], recv[0][:4096])

    value = busbw(S, ms / 1e3, P)
    hbm_peak, peak_src = peaks()
    eng_ms = float(np.mean(eng)) if len(eng) else None
    alg_bytes = engine_alg_bytes(info["algo_name"], P, S)
    achieved = alg_bytes / (eng_ms / 1e3) / 1e9 if eng_ms else None
    traffic = None
    tp = os.path.join(ROOT, "profiles", f"engine_traffic_{info['algo_name']}.json")
    if os.path.exists(tp):
        try:
            t = json.load(open(tp))
            if t.get("bytes_per_rank") == S and t.get("ranks") == P and t.get("algo", "ring") == info["algo_name"]:
                traffic = t.get("dram_bytes_per_launch")
        except Exception:
            pass
    roof = {"bound": "hbm", "achieved": achieved, "peak": hbm_peak, "unit": "GB/s",
            "frac": (achieved / hbm_peak) if achieved else None, "traffic": traffic,
            "kernel": f"{info['algo_name']}_engine_group (all co-located ranks' engines in one launch)",
            "engine_ms": eng_ms, "engine_share_of_step": (eng_ms / ms) if eng_ms else None,
            "algorithmic_bytes_per_launch": alg_bytes, "peak_source": peak_src}

    # ---------------- e2e: host buffers, H2D inputs + D2H result inside the timed region
    host_in = [torch.empty(Np * count, dtype=torch.float32, pin_memory=True) for _ in range(P)]
    for r in range(P):
        host_in[r].copy_(send[r].cpu())
    host_out = torch.empty(Np * count, dtype=torch.float32, pin_memory=True)
    torch.cuda.synchronize()
    ke = max(1, args.e2e_steps)
    ref0 = recv[0][: 1 << 16].clone()  # the timed steps' result: the e2e steps reduce the same inputs
    e2e_pipelined(pc, torch, reqs, send, host_in, recv[0], host_out, Np, count, st, 1)  # warm-up
    e2e_ms = e2e_pipelined(pc, torch, reqs, send, host_in, recv[0], host_out, Np, count, st, ke)
    for q in reqs:
        assert q.error()[0] == 0, f"device error {q.error()}"
    assert torch.equal(recv[1][:4096], recv[0][:4096]) and torch.equal(recv[0][: 1 << 16], ref0)
    assert torch.equal(host_out[: 1 << 16], ref0.cpu())
    log(f"e2e: {e2e_ms:.3f} ms/step")
    e2e = {"value": busbw(S, e2e_ms / 1e3, P), "unit": "GB/s", "h2d_bytes_per_step": P * S, "d2h_bytes_per_step": S,
           "ms_per_step": e2e_ms,
           "api": "per step: pc_epoch_all (no Pready) per GPU, then each rank's inputs host->device in 8 chunks of "
                  "partitions, each followed by pc_pready_range (the engine reduces while PCIe delivers the rest), "
                  "pc_wait_on_stream, the result device->host (overlapping the next step's inputs)"}

    for q in reqs:
        q.free()
    for c in comms:
        c.destroy()
    g.destroy()
    lat = None
    if not args.no_latency:
        g2, c2 = pc.local_comms(2, 0)  # the exchange of new requests is collective over the comm
        lat = {"flag_only": latency_pair(pc, apps, torch, c2, payload=0),
               "8B": latency_pair(pc, apps, torch, c2, payload=8),
               "ll_flag_only": latency_pair(pc, apps, torch, c2, payload=0, copy=pc.COPY_LL),
               "ll_8B": latency_pair(pc, apps, torch, c2, payload=8, copy=pc.COPY_LL),
               "ll_256B": latency_pair(pc, apps, torch, c2, payload=256, copy=pc.COPY_LL),
               "note": "2 virtual ranks on one B200 (flags/payload in the same HBM/L2, not NVLink)"}
        for c in c2:
            c.destroy()
        g2.destroy()

    log("latency done")
    jac = None if args.no_jacobi else jacobi_bench(pc, apps, torch, args)
    log("jacobi done")
    c1 = None if args.no_c1 else c1_bench(pc, apps, torch)
    c2p = None if args.no_c1 else c2_bench(pc, apps, torch)
    log("c1 / c2 done")
    cpu = None if args.no_cpu_baseline else oracle_sample(P=P)
    log("cpu baseline done")
    out = {"metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": 1, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "f32", "data": "synthetic",
           "config": {"workload": f"partitioned allreduce (C5/C3 shape) fp32 sum, {P} virtual ranks co-located on one "
                                  f"B200, {S >> 20} MiB per rank in {Np} partitions, {info['algo_name']} schedule"
                                  f" (requested {args.algo})",
                      "ranks": P, "ranks_per_gpu": P, "bytes_per_rank": S, "partitions": Np, "algo": info["algo_name"],
                      "slices_per_chunk": info["slices"], "slice_elems": info["slice_elems"],
                      "engine_warps_per_rank": info["engine_warps"],
                      "l2": f"no flush: working set {3 * P * S >> 20} MiB >> 126 MB L2",
                      "parallelism": f"{P} virtual ranks / 1 GPU"},
           "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches,
           "clocks": clk.summary(), "latency_ns": lat, "jacobi": jac, "c1_p2p": c1, "c2_p2p_256mib": c2p,
           "nccl": None}
    print(json.dumps(out), flush=True)


def _free_port():
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        return so.getsockname()[1]


class MultiCtx:
    """One process per GPU (torchrun): rank / world / device, the process
    group, the max-over-ranks reduction and CUDA-event timing helpers."""

    def __init__(self, torch, dist):
        self.torch, self.dist = torch, dist
        self.rank, self.world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
        ngpu = torch.cuda.device_count()
        local = int(os.environ.get("LOCAL_RANK", self.rank))
        # ranks share GPUs: a correctness run of the N > 1 path on a smaller box
        # (e.g. torchrun --nproc-per-node 2 on the one-GPU box): gloo bootstrap,
        # no NCCL baseline (NCCL needs one GPU per rank), the processes time-slice
        # the GPU, so reduced sizes and no meaningful times
        self.shared = ngpu < int(os.environ.get("LOCAL_WORLD_SIZE", self.world))
        self.dev = local % ngpu
        torch.cuda.set_device(self.dev)
        if self.shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", self.dev))
        self.tdev = "cpu" if self.shared else "cuda"

    def max(self, v):
        t = self.torch.tensor([float(v)], dtype=self.torch.float64, device=self.tdev)
        self.dist.all_reduce(t, op=self.dist.ReduceOp.MAX)
        return float(t.item())

    def barrier(self):
        self.dist.barrier()

    def time_ms(self, fn, iters, stream, warm=2):
        """CUDA events on `stream` around `iters` calls, barrier + sync on both
        sides, max over ranks (ms per call)."""
        torch = self.torch
        for _ in range(warm):
            fn()
        torch.cuda.synchronize()
        self.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(iters):
            fn()
        e1.record(stream)
        torch.cuda.synchronize()
        self.barrier()
        return self.max(e0.elapsed_time(e1) / iters)


def multi_nvlink_floor(ctx, pc, apps, torch, chunk):
    """Bare peer-copy floor (no library): every
    rank writes (push) / reads (pull) `chunk` bytes to / from each of its P-1
    peers at once — the all-to-all pattern of the DIRECT schedule over
    NVSwitch.  Peer addresses come from a pc_pallgather_init request (its
    recvbuf holds one chunk slot per rank).  GB/s per GPU per direction."""
    P, r = ctx.world, ctx.rank
    n = chunk // 4
    st = torch.cuda.Stream()
    comm = pc.Comm.from_process_group(ctx.dev)
    send = torch.ones(n, device="cuda")
    recv = torch.zeros(P * n, device="cuda")
    q = pc.pallgather_init(send, recv, 1, n, pc.FLOAT32, comm)
    q.start(st)
    q.pbuf_prepare(st)
    q.pready_range(0, 0, st)
    q.wait_on_stream(st)
    torch.cuda.synchronize()
    peers = [q.peer_buffer(j) for j in range(P - 1)]  # (allgather: DIRECT peer mapping)
    # push: my chunk -> slot r of every peer's recvbuf; pull: slot (peer) of every peer -> my slot (peer)
    push_dst = [p + r * chunk for p in peers]
    pull_src = [peers[j] + ((r + 1 + j) % P) * chunk for j in range(P - 1)]
    pull_dst = [recv.data_ptr() + ((r + 1 + j) % P) * chunk for j in range(P - 1)]
    iters = 3 if ctx.shared else 20
    ms_push = ctx.time_ms(lambda: apps.peer_copy([send] * (P - 1), push_dst, chunk, stream=st), iters, st)
    ms_pull = ctx.time_ms(lambda: apps.peer_copy(pull_src, pull_dst, chunk, stream=st), iters, st)
    out_bytes = (P - 1) * chunk
    res = {"push_gbs_per_gpu": out_bytes / (ms_push / 1e3) / 1e9, "pull_gbs_per_gpu": out_bytes / (ms_pull / 1e3) / 1e9,
           "bytes_per_peer": chunk, "peers": P - 1, "kernel": "peer_copy_kernel (16-B vectors, no flags)"}
    q.free()
    comm.destroy()
    return res


def multi_nccl(ctx, torch, dist, send, steps):
    """NCCL all_reduce on the same bytes: default tuning and NCCL_ALGO=Ring (a
    second communicator created with the variable set; NCCL_DEBUG=INFO logs
    each communicator's nranks and the chosen algorithm / protocol)."""
    out = {}
    x = send.clone()
    st = torch.cuda.current_stream()
    out["default"] = ctx.time_ms(lambda: dist.all_reduce(x), steps, st, warm=3)
    old = os.environ.get("NCCL_ALGO")
    os.environ["NCCL_ALGO"] = "Ring"
    try:
        g_ring = dist.new_group(list(range(ctx.world)), backend="nccl")
        out["ring"] = ctx.time_ms(lambda: dist.all_reduce(x, group=g_ring), steps, st, warm=3)
    finally:
        if old is None:
            os.environ.pop("NCCL_ALGO", None)
        else:
            os.environ["NCCL_ALGO"] = old
    return out


def multi_p2p(ctx, pc, apps, torch, dist):
    """C1 / C2 / latency between rank pairs (2k, 2k+1), all pairs at once (one
    pc comm per pair: the first pbuf_prepare is collective over its comm).
    Even ranks produce (vector add, 8 B/thread, 1024-thread blocks, Pready
    inside) and send; odd ranks receive.  Reported for pair (0, 1); times are
    max over the pair."""
    import numpy as np
    P, r = ctx.world, ctx.rank
    pairs = [dist.new_group([2 * k, 2 * k + 1]) for k in range(P // 2)]
    if r >= 2 * (P // 2):  # odd world: the last rank sits this leg out
        return None
    grp = pairs[r // 2]
    side = r % 2
    comm = pc.Comm.from_process_group(ctx.dev, group=grp)
    st = torch.cuda.Stream()

    def pmax(v):
        t = torch.tensor([float(v)], dtype=torch.float64, device=ctx.tdev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=grp)
        return float(t.item())

    def ptime(fn, iters, warm=2):
        for _ in range(warm):
            fn()
        torch.cuda.synchronize()
        dist.barrier(group=grp)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(iters):
            fn()
        e1.record(st)
        torch.cuda.synchronize()
        dist.barrier(group=grp)
        return pmax(e0.elapsed_time(e1) / iters)

    res = {"pair": [0, 1], "note": "ranks 2k -> 2k+1, all pairs concurrently"}
    sizes = [1 << 24] if ctx.shared else [1 << 20, 1 << 24, 1 << 28]
    elems = {apps.GRAN_BLOCK: 2048, apps.GRAN_WARP: 64, apps.GRAN_THREAD: 2}
    tag = 200
    for S in sizes:
        n = S // 4
        A = torch.randn(n, device="cuda")
        B = torch.randn(n, device="cuda")
        Cb = torch.empty(n, device="cuda")
        Rb = torch.zeros(n, device="cuda")
        wts = (torch.arange(n, device="cuda", dtype=torch.int64) % 1021) + 1
        row = {}
        # traditional (Listing 1): kernel -> cudaStreamSynchronize -> copy into
        # the peer's buffer (cudaMemcpyAsync, peer-mapped) -> synchronize
        snd0 = pc.psend_init(Cb, 1, n, pc.FLOAT32, 1, tag, comm) if side == 0 else None
        rcv0 = pc.precv_init(Rb, 1, n, pc.FLOAT32, 0, tag, comm) if side == 1 else None
        tag += 1
        q0 = snd0 or rcv0
        q0.start(st)
        q0.pbuf_prepare(st)
        if side == 0:
            q0.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
            q0.pready_range(0, 0, st)
        q0.wait_on_stream(st)
        torch.cuda.synchronize()
        if side == 0:
            peer = q0.peer_buffer(0)

            def trad():
                apps.vecadd(A, B, Cb, n, apps.GRAN_NONE, None, st)
                st.synchronize()
                apps.memcpy_async(peer, Cb, S, st)
                st.synchronize()
        else:
            def trad():
                pass
        it = 5 if ctx.shared else (50 if S <= (1 << 24) else 10)
        for _ in range(2):
            trad()
        dist.barrier(group=grp)
        t0 = time.perf_counter()
        for _ in range(it):
            trad()
        torch.cuda.synchronize()
        row["traditional_us_host"] = pmax((time.perf_counter() - t0) / it * 1e6)
        if not ctx.shared:  # the same with NCCL point-to-point (kernel -> sync -> ncclSend / ncclRecv)
            def trad_nccl():
                if side == 0:
                    apps.vecadd(A, B, Cb, n, apps.GRAN_NONE, None, st)
                    st.synchronize()
                    with torch.cuda.stream(st):
                        dist.send(Cb, dst=r + 1, group=grp)
                else:
                    with torch.cuda.stream(st):
                        dist.recv(Rb, src=r - 1, group=grp)
                st.synchronize()
            for _ in range(2):
                trad_nccl()
            dist.barrier(group=grp)
            t0 = time.perf_counter()
            for _ in range(it):
                trad_nccl()
            row["traditional_nccl_us_host"] = pmax((time.perf_counter() - t0) / it * 1e6)
        q0.free()
        if side == 0:  # the same traditional model, device-timed, with the persistent producer (C2 leg of N = 1)
            def trad_dev():
                apps.vecadd(A, B, Cb, n, apps.GRAN_NONE, None, st, persistent=True)
                apps.memcpy_async(peer, Cb, S, st)
        else:
            def trad_dev():
                pass
        row["traditional_persistent_us_device"] = ptime(trad_dev, it) * 1e3
        configs = [("block", apps.GRAN_BLOCK, 1, pc.COPY_INLINE, False),
                   ("block", apps.GRAN_BLOCK, 1, pc.COPY_ENGINE, False),
                   ("block->1MiB", apps.GRAN_BLOCK, 128, pc.COPY_INLINE, False),
                   ("block_put persistent", apps.GRAN_BLOCK_PUT, 1, pc.COPY_INLINE, True),
                   ("warp->all", apps.GRAN_WARP, None, pc.COPY_INLINE, False),
                   ("thread->all", apps.GRAN_THREAD, None, pc.COPY_INLINE, False)]
        if S == (1 << 20):  # C1: 128 block partitions aggregated into 8 transport partitions (R24)
            configs = [("C1 block->128KiB", apps.GRAN_BLOCK, 16, pc.COPY_INLINE, False)] + configs
        elems[apps.GRAN_BLOCK_PUT] = 2048
        for name, gran, agg, copy, pers in configs:
            cnt = elems[gran]
            parts = n // cnt
            g = parts if agg is None else min(agg, parts)
            if side == 0:
                q = pc.psend_init(Cb, parts, cnt, pc.FLOAT32, 1, tag, comm)
            else:
                Rb.zero_()
                q = pc.precv_init(Rb, parts, cnt, pc.FLOAT32, 0, tag, comm)
            tag += 1
            q.start(st)
            q.pbuf_prepare(st)
            sq = q.prequest_create(min(gran, apps.GRAN_BLOCK), g, copy) if side == 0 else None

            def epoch(first=False):
                if not first:
                    q.start(st)
                    q.pbuf_prepare(st)
                if side == 0:
                    apps.vecadd(A, B, Cb, n, gran, sq, st, persistent=pers)
                q.wait_on_stream(st)

            epoch(first=True)
            torch.cuda.synchronize()
            us = ptime(epoch, it) * 1e3
            err = q.error()
            # parity gate of the point: the receiver's bytes equal the sender's C
            # (exact: sums of the 32-bit patterns with position weights, exchanged)
            buf = Cb if side == 0 else Rb
            h = torch.tensor([int((buf.view(torch.int32).long() * wts).sum().item()) if side == 0 else 0,
                              int((buf.view(torch.int32).long() * wts).sum().item()) if side == 1 else 0],
                             dtype=torch.int64, device=ctx.tdev)
            dist.all_reduce(h, group=grp)
            q.free()
            row[f"{name} {['inline', 'engine', 'll', 'host'][copy]}"] = {
                "us": us, "gbs": S / (us / 1e6) / 1e9, "error": list(err), "parity": bool(h[0].item() == h[1].item())}
        res[f"{S >> 20}MiB"] = row
    # Pready -> Parrived latency: one persistent ping-pong kernel per side
    iters = 50 if ctx.shared else 10000
    lat = {}
    for name, payload, copy in (("flag_only", 0, pc.COPY_INLINE), ("8B", 8, pc.COPY_INLINE),
                                ("ll_8B", 8, pc.COPY_LL), ("ll_256B", 256, pc.COPY_LL)):
        cnt = payload // 4
        sbuf = torch.arange(max(iters * cnt, 4), dtype=torch.float32, device="cuda")
        rbuf = torch.zeros(max(iters * cnt, 4), device="cuda")
        snd = pc.psend_init(sbuf, iters, cnt, pc.FLOAT32, 1 - side, 300 + side, comm)
        rcv = pc.precv_init(rbuf, iters, cnt, pc.FLOAT32, 1 - side, 300 + (1 - side), comm)
        for q in (snd, rcv):
            q.start(st)
        for q in (snd, rcv):
            q.pbuf_prepare(st)
        sq = snd.prequest_create(pc.GRAN_WARP, 1, copy)
        rq = rcv.prequest_create(pc.GRAN_WARP, 1, pc.COPY_INLINE)
        t = torch.zeros(1, dtype=torch.int64, device="cuda")
        torch.cuda.synchronize()
        dist.barrier(group=grp)
        apps.pingpong(sq, rq, side, iters, apps.GRAN_WARP, t, st)
        snd.wait_on_stream(st)
        rcv.wait_on_stream(st)
        torch.cuda.synchronize()
        one_way = pmax(float(t.item()) / iters / 2.0)
        lat[name] = {"mean_ns": one_way, "payload_bytes": payload, "iters": iters,
                     "copy": ["inline", "engine", "ll"][copy], "errors": [snd.error()[0], rcv.error()[0]]}
        snd.free()
        rcv.free()
    # the floor: bare release/acquire system-scope flag ping-pong, no library
    fl = torch.zeros(64, dtype=torch.int32, device="cuda")
    q = pc.psend_init(fl, 1, 64, pc.INT32, 1 - side, 400 + side, comm)
    q2 = pc.precv_init(fl, 1, 64, pc.INT32, 1 - side, 400 + (1 - side), comm)
    for x in (q, q2):
        x.start(st)
    for x in (q, q2):
        x.pbuf_prepare(st)
    q.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
    q.pready_range(0, 0, st)
    q.wait_on_stream(st)
    q2.wait_on_stream(st)
    torch.cuda.synchronize()
    peer_flag = q.peer_buffer(0)
    fl.zero_()
    torch.cuda.synchronize()
    dist.barrier(group=grp)
    t = torch.zeros(1, dtype=torch.int64, device="cuda")
    apps.bare_pingpong(fl, peer_flag, side, iters, 0, t, st)
    torch.cuda.synchronize()
    lat["bare_sys_flag_floor_ns"] = pmax(float(t.item()) / iters / 2.0)
    q.free()
    q2.free()
    res["latency_ns"] = lat
    comm.destroy()
    return res


def multi_dl(ctx, pc, apps, torch, dist, args):
    """NEXT-2 / Figs 10-11 analogue across GPUs (§VI-D2): every
    rank computes the BCE gradient of a ResNet-50-sized flat buffer (25.56 M
    fp32, 64 KiB partitions) and the ranks allreduce it, three ways:
      traditional: producer kernel -> NCCL all_reduce (Listing 1);
      serial:      producer kernel -> pc_epoch_all(pready) -> engine;
      partitioned: pc_epoch_all -> producer that Preadies each partition ->
                   engine forked at the epoch's control call (overlap, a6).
    ms per step (max over ranks) and the gradient goodput."""
    NPARAM, L = 25_557_032, 16384
    Np = -(-NPARAM // L)
    if ctx.shared:
        Np, L = 64, 16384
    n = Np * L
    gen = torch.Generator(device="cuda")
    gen.manual_seed(0x5C24 + ctx.rank)
    p = 0.02 + 0.96 * torch.rand(n, device="cuda", generator=gen)
    y = torch.randint(0, 2, (n,), device="cuda", generator=gen).float()
    g = torch.empty(n, device="cuda")
    out = torch.empty(n, device="cuda")
    comm = pc.Comm.from_process_group(ctx.dev)
    st = torch.cuda.Stream()
    q = pc.pallreduce_init(g, out, Np, L, pc.FLOAT32, pc.SUM, pc.ALGO_AUTO, comm)
    q.start(st)
    q.pbuf_prepare(st)
    pq = q.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_ENGINE)
    apps.bce_grad(p, y, g, Np, L, float(n), None, stream=st)
    q.pready_range(0, Np - 1, st)
    q.wait_on_stream(st)
    torch.cuda.synchronize()
    it = 3 if ctx.shared else 20

    def serial():
        apps.bce_grad(p, y, g, Np, L, float(n), None, stream=st)
        pc.epoch_all([q], pready=True, stream=st)
        q.wait_on_stream(st)

    def partitioned():
        pc.epoch_all([q], pready=False, stream=st)
        apps.bce_grad(p, y, g, Np, L, float(n), pq, stream=st)
        q.wait_on_stream(st)

    res = {"partitions": Np, "partition_bytes": 4 * L, "bytes_per_rank": 4 * n, "algo": q.info()["algo_name"]}
    res["serial_ms"] = ctx.time_ms(serial, it, st)
    res["partitioned_ms"] = ctx.time_ms(partitioned, it, st)
    assert q.error()[0] == 0
    if not ctx.shared:
        def traditional():
            apps.bce_grad(p, y, g, Np, L, float(n), None, stream=st)
            with torch.cuda.stream(st):
                dist.all_reduce(g)
        res["traditional_nccl_ms"] = ctx.time_ms(traditional, it, st)
    for k in ("serial", "partitioned", "traditional_nccl"):
        if f"{k}_ms" in res:
            res[f"{k}_goodput_gbs"] = 4 * n * ctx.world / (res[f"{k}_ms"] / 1e3) / 1e9
    q.free()
    comm.destroy()
    return res


def multi_jacobi(ctx, pc, apps, torch, args):
    """C4 at N GPUs: 16384^2 fp32, 1D (P x 1) and 2D decompositions, halos by
    intra-kernel partitioned sends (pc_pready_warp into the neighbour's halo
    over NVLink); GFLOP/s over all ranks (4 flops per interior cell)."""
    P = ctx.world
    N = 4096 if ctx.shared else args.jacobi_n
    K = 5 if ctx.shared else args.jacobi_iters
    decomps = [(P, 1)] + ([{2: (2, 1), 4: (2, 2), 8: (4, 2)}[P]] if P in (4, 8) else [])
    comm = pc.Comm.from_process_group(ctx.dev)
    res = {}
    for Py, Px in decomps:
        st = torch.cuda.Stream()
        js = apps.JacobiSolver([comm], [ctx.rank], N, Py, Px, K, H=int(os.environ.get("PC_JACOBI_H", "64")),
                               device=ctx.dev)
        for s_ in js.local:
            s_["grid"][0].zero_()
            if s_["py"] == 0:
                s_["grid"][0][: js.lx].fill_(1.0)
            s_["grid"][1].copy_(s_["grid"][0])
        torch.cuda.synchronize()
        js.solve(st)  # first epoch: exchange + mapping
        torch.cuda.synchronize()
        reps = 1 if ctx.shared else 3
        ms = ctx.time_ms(lambda: js.solve(st), reps, st, warm=1)
        ms_iter = ms / K
        errs = js.errors()
        nerr = ctx.max(len(errs))
        cells = (N - 2) * (N - 2)
        res[f"{Py}x{Px}"] = {"gflops": 4.0 * cells / (ms_iter / 1e3) / 1e9, "us_per_iter": ms_iter * 1e3,
                             "errors": int(nerr)}
        js.free()
    comm.destroy()
    res["config"] = f"{N}^2 fp32, {K} iterations per epoch, one rank per GPU"
    return res


def run_multi(args):
    import numpy as np
    # NCCL logs every communicator's rank / nranks and the tuning decision
    # (algorithm, protocol) — to stderr, so stdout keeps the one JSON line
    os.environ.setdefault("NCCL_DEBUG", "INFO")
    os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT,TUNING,ENV")
    os.environ.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
    import torch
    import torch.distributed as dist

    import paper_conf_sc_temucinslsga24_b200 as pc
    from paper_conf_sc_temucinslsga24_b200 import apps

    ctx = MultiCtx(torch, dist)
    rank, world, local = ctx.rank, ctx.world, ctx.dev
    shared = ctx.shared
    P, S, Np = world, args.bytes, args.partitions
    if shared:
        S = min(S, 16 << 20)
    count = S // 4 // Np
    S = count * 4 * Np
    algo = {"ring": pc.ALGO_RING, "rd": pc.ALGO_RD, "direct": pc.ALGO_DIRECT, "direct_push": pc.ALGO_DIRECT_PUSH,
            "auto": pc.ALGO_AUTO}[args.algo]
    comm = pc.Comm.from_process_group(local)
    st = torch.cuda.Stream()
    gen = torch.Generator(device="cuda")
    gen.manual_seed(0x5C24 + rank)
    send = torch.randn(Np * count, device="cuda", generator=gen)
    recv = torch.empty_like(send)
    q = pc.pallreduce_init(send, recv, Np, count, pc.FLOAT32, pc.SUM, algo, comm)
    steps = min(args.steps, 5) if shared else args.steps

    def first_step():  # the first Pbuf_prepare exchanges and maps (blocking)
        q.start(st)
        q.pbuf_prepare(st)
        q.pready_range(0, Np - 1, st)
        q.wait_on_stream(st)

    def step():  # Start + RTR + Pready of every partition in one kernel, then the engine
        pc.epoch_all([q], pready=True, stream=st)
        q.wait_on_stream(st)

    first_step()
    info = q.info()
    for _ in range(max(args.warmup, 1)):
        step()
    torch.cuda.synchronize()
    assert q.error()[0] == 0
    # parity gate (sampled): the allreduce of the rank-seeded inputs equals the
    # fp64 sum within the north_star bound (R16); bit-identical on every rank
    xs = [torch.empty_like(send) for _ in range(P)]
    if shared:
        dist.all_gather(xs_cpu := [torch.empty(send.numel()) for _ in range(P)], send.cpu())
        xs = [x.cuda() for x in xs_cpu]
    else:
        dist.all_gather(xs, send)
    gidx = torch.Generator(device="cuda")
    gidx.manual_seed(0x5C24)  # the same sample on every rank
    idx = torch.randint(0, send.numel(), (4096,), device="cuda", generator=gidx)
    ref = torch.stack([x[idx].double() for x in xs]).sum(0)
    bound = 1e-5 * torch.stack([x[idx].double().abs() for x in xs]).sum(0)
    parity_ok = bool(((recv[idx].double() - ref).abs() <= bound).all().item())
    h = torch.tensor([float(recv[idx].double().sum().item())], dtype=torch.float64, device=ctx.tdev)
    hs = [torch.empty_like(h) for _ in range(P)]
    dist.all_gather(hs, h)
    parity_ok = parity_ok and all(float(x.item()) == float(h.item()) for x in hs)
    parity_ok = ctx.max(0.0 if parity_ok else 1.0) == 0.0
    del xs

    q.set_timing(True)
    q.engine_times()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n0 = pc.launch_count()
    with Clocks(local) as clk:
        dist.barrier()
        torch.cuda.synchronize()
        e0.record(st)
        for _ in range(steps):
            step()
        e1.record(st)
        clk.sample_now()  # the steps are still running: one sample inside the timed region
        torch.cuda.synchronize()
        dist.barrier()
    launches = pc.launch_count() - n0
    ms = ctx.max(e0.elapsed_time(e1) / steps)
    eng = q.engine_times()
    eng_ms = ctx.max(float(np.mean(eng)) if len(eng) else 0.0)
    assert q.error()[0] == 0

    # the DIRECT schedule's other variant on the same bytes (PULL <-> PUSH):
    # whichever direction of NVLink traffic the fabric serves better
    other = None
    if info["algo_name"] in ("direct", "direct_push"):
        oalgo = pc.ALGO_DIRECT_PUSH if info["algo_name"] == "direct" else pc.ALGO_DIRECT
        q2 = pc.pallreduce_init(send, recv, Np, count, pc.FLOAT32, pc.SUM, oalgo, comm)
        q2.start(st)
        q2.pbuf_prepare(st)
        q2.pready_range(0, Np - 1, st)
        q2.wait_on_stream(st)

        def step2():
            pc.epoch_all([q2], pready=True, stream=st)
            q2.wait_on_stream(st)

        ms2 = ctx.time_ms(step2, steps, st, warm=max(args.warmup, 1))
        ok2 = bool(((recv[idx].double() - ref).abs() <= bound).all().item()) and q2.error()[0] == 0
        ok2 = ctx.max(0.0 if ok2 else 1.0) == 0.0
        other = {"algo": q2.info()["algo_name"], "value": busbw(S, ms2 / 1e3, P), "ms_per_step": ms2, "unit": "GB/s",
                 "parity": ok2}
        q2.free()
    log("direct variant done")

    nccl = {"skipped": "ranks share a GPU (debug run): NCCL needs one GPU per rank"}
    if not shared:
        t = multi_nccl(ctx, torch, dist, send, steps)
        nccl = {k: {"value": busbw(S, v / 1e3, P), "ms_per_step": v, "unit": "GB/s"} for k, v in t.items()}
        nccl["call"] = "torch.distributed.all_reduce (NCCL 2.28.9); 'ring' = a communicator created with NCCL_ALGO=Ring"
        nccl["debug_log"] = "NCCL_DEBUG=INFO, NCCL_DEBUG_SUBSYS=INIT,TUNING,ENV on stderr"
    log("allreduce + nccl done")

    # e2e: H2D input in chunks each Preadied, allreduce, D2H result (pipelined, e2e_pipelined)
    host_in = send.cpu().pin_memory()
    host_out = torch.empty_like(host_in).pin_memory()
    torch.cuda.synchronize()
    ke = max(1, args.e2e_steps)
    e2e_pipelined(pc, torch, [q], [send], [host_in], recv, host_out, Np, count, st, 1)
    dist.barrier()
    ems = ctx.max(e2e_pipelined(pc, torch, [q], [send], [host_in], recv, host_out, Np, count, st, ke))
    q.free()
    comm.destroy()

    floor = multi_nvlink_floor(ctx, pc, apps, torch, min(S, 64 << 20))
    log("nvlink floor done")
    p2p = None if args.no_c1 else multi_p2p(ctx, pc, apps, torch, dist)
    log("p2p legs done")
    jac = None if args.no_jacobi else multi_jacobi(ctx, pc, apps, torch, args)
    log("jacobi done")
    dl = None if args.no_dl else multi_dl(ctx, pc, apps, torch, dist, args)
    log("dl proxy done")
    cpu = None
    if rank == 0 and not args.no_cpu_baseline:
        cpu = oracle_sample(P=min(P, 8))
    dist.barrier()
    if rank == 0:
        eng_ms_v = eng_ms or None
        # NVLink bytes per rank per direction: ring and DIRECT 2(P-1)/P*S, RD log2(P)*S
        nvl_bytes = (P.bit_length() - 1) * S if info["algo_name"] == "rd" else 2 * (P - 1) / P * S
        achieved = nvl_bytes / (eng_ms_v / 1e3) / 1e9 if eng_ms_v else None
        # the roofline denominator: the measured bare peer-copy floor of this box
        # (DIRECT: half its bytes are peer-load responses, half peer stores)
        peak = 0.5 * (floor["push_gbs_per_gpu"] + floor["pull_gbs_per_gpu"]) if info["algo_name"] == "direct" \
            else floor["push_gbs_per_gpu"]
        where = "ranks sharing GPUs (debug run: time-sliced, not a measurement)" if shared else "one per B200"
        out = {"metric": METRIC, "value": busbw(S, ms / 1e3, P), "unit": "GB/s", "n_gpus": world,
               "steps": steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
               "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
               "config": {"workload": f"partitioned allreduce fp32 sum, {P} ranks ({where}), {S >> 20} MiB "
                                      f"per rank in {Np} partitions, {info['algo_name']} schedule "
                                      f"(requested {args.algo})", "ranks": P,
                          "bytes_per_rank": S, "partitions": Np, "algo": info["algo_name"],
                          "algo_requested": args.algo,
                          "l2": "no flush: per-rank working set > 126 MB L2" if S >= (64 << 20) else
                                "working set within L2 (debug size)",
                          "parallelism": f"dp{P}"},
               "parity": {"ok": parity_ok, "check": "4096 sampled elements vs the fp64 sum within 1e-5*sum|x| "
                                                   "(R16), bit-identical on every rank"},
               "roofline": {"bound": "nvlink", "achieved": achieved, "peak": peak, "unit": "GB/s",
                            "frac": achieved / peak if achieved and peak else None, "traffic": None,
                            "kernel": f"{info['algo_name']}_engine", "engine_ms": eng_ms_v,
                            "nvlink_bytes_per_rank_per_launch": nvl_bytes,
                            "peak_source": "measured on this box: bare peer-copy floor (nvlink_floor)"},
               "nvlink_floor": floor, "cpu_baseline": cpu,
               "e2e": {"value": busbw(S, ems / 1e3, P), "unit": "GB/s", "h2d_bytes_per_step": S,
                       "d2h_bytes_per_step": S, "ms_per_step": ems,
                       "api": "pc_epoch_all + chunked H2D each followed by pc_pready_range + pc_wait_on_stream + "
                              "D2H (pipelined, e2e_pipelined)"},
               "gpu_launches": launches, "clocks": clk.summary(), "nccl": nccl, "direct_other_variant": other,
               "p2p": p2p, "jacobi": jac, "dl_proxy": dl}
        print(json.dumps(out), flush=True)
    dist.destroy_process_group()


def main():
    args = parse()
    if args.quiet:
        sys.stderr = open(os.devnull, "w")
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        # --gpus N outside torchrun: relaunch as N processes, one per GPU
        # (never fall back to virtual ranks reporting n_gpus 1)
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr=127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
        log("relaunching under torchrun:", " ".join(cmd))
        sys.exit(subprocess.call(cmd))
    if args.impl == "reference":
        run_reference(args)
        return
    if world > 1:
        run_multi(args)
    else:
        run_virtual(args)


if __name__ == "__main__":
    main()
