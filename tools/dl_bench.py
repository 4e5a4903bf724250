"""DL proxy (§VI-D2, Figs 10/11 analogue) on one B200 with co-located virtual
ranks: per step each rank computes the BCE gradient of a ResNet-50-sized flat
buffer (25.56 M fp32) and the ranks allreduce it; pc_startall +
pc_pbuf_prepare_all are inside the step.  Modes: pready (the producer
Preadies each partition from the kernel; the engine overlaps the producers),
pready_nooverlap (the same with the engine forked at the wait), serial
(producers, then host Pready of all partitions), and the two halves alone.
Each rank's producer runs on its own stream.
JSON lines to stdout; CUDA-event timing on the control stream."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

import torch  # noqa: E402

import paper_conf_sc_temucinslsga24_b200 as pc  # noqa: E402
from paper_conf_sc_temucinslsga24_b200 import apps  # noqa: E402

NPARAM = 25_557_032  # ResNet-50


def timeit(fn, st, reps=20, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(reps):
        fn()
    e1.record(st)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def run(P, L, algo, modes):
    Np = -(-NPARAM // L)
    n = Np * L
    g, cs = pc.local_comms(P, 0)
    gen = torch.Generator(device="cuda")
    gen.manual_seed(0x5C24)
    p = [(0.02 + 0.96 * torch.rand(n, device="cuda", generator=gen)) for _ in range(P)]
    y = [torch.randint(0, 2, (n,), device="cuda", generator=gen).float() for _ in range(P)]
    dl = apps.DLProxy(cs, Np, L, algo, p, y)
    dl.step("serial")  # the first epoch exchanges and maps (every mode below starts from there)
    torch.cuda.synchronize()
    dl_no = None
    dl_in = None
    multi = {}
    out = []
    for mode in modes:
        if mode in ("pready", "serial"):
            ms = timeit(lambda: dl.step(mode), dl.ctl)
        elif mode in ("timeline", "timeline_serial"):  # where the time of one overlapped step goes
            import statistics
            sm = "pready" if mode == "timeline" else "serial"
            dl.step(sm)
            torch.cuda.synchronize()
            dl.reqs[0].set_timing(True)
            dl.reqs[0].engine_times()
            prod, tot = [], []
            for _ in range(10):
                t0 = torch.cuda.Event(enable_timing=True)
                te = [torch.cuda.Event(enable_timing=True) for _ in range(P)]
                t1 = torch.cuda.Event(enable_timing=True)
                dl.ev_p = te  # the step records the producers' ends into these
                t0.record(dl.ctl)
                dl.step(sm)
                t1.record(dl.ctl)
                torch.cuda.synchronize()
                prod.append(max(t0.elapsed_time(e) for e in te))
                tot.append(t0.elapsed_time(t1))
            eng = dl.reqs[0].engine_times()
            dl.reqs[0].set_timing(False)
            dl.ev_p = [torch.cuda.Event() for _ in range(P)]
            ms = statistics.median(tot)
            extra = {"producers_end_ms": statistics.median(prod), "engine_ms": float(statistics.median(list(eng))) if len(eng) else None}
            out.append({"P": P, "partition_bytes": 4 * L, "partitions": Np, "algo": algo, "mode": mode,
                        "ms_per_step": ms, **extra})
            print(json.dumps(out[-1]), flush=True)
            continue
        elif mode == "pready_inline":  # R33: the completing producer block folds (no engine)
            if dl_in is None:
                dl_in = apps.DLProxy(cs, Np, L, pc.ALGO_DIRECT, p, y, copy=pc.COPY_INLINE)
                dl_in.step("pready")
                torch.cuda.synchronize()
            ms = timeit(lambda: dl_in.step("pready"), dl_in.ctl)
            assert dl_in.errors() == [], dl_in.errors()
        elif mode in ("serial_multi", "pready_multi", "pready_inline_multi", "pready_coop_multi"):
            # every rank's producer in ONE launch, partition u of all ranks side by side (bce_grad_multi)
            key = {"pready_inline_multi": "inline", "pready_coop_multi": "coop"}.get(mode, "engine")
            if key not in multi:
                multi[key] = apps.DLProxy(cs, Np, L, pc.ALGO_DIRECT if key != "engine" else algo, p, y,
                                          copy=pc.COPY_INLINE if key != "engine" else None, multi=True,
                                          coop=key == "coop")
                multi[key].step("serial" if mode == "serial_multi" else "pready")
                torch.cuda.synchronize()
            dm = multi[key]
            sm = "serial" if mode == "serial_multi" else "pready"
            ms = timeit(lambda: dm.step(sm), dm.ctl)
            assert dm.errors() == [], dm.errors()
            if key != "engine":  # parity of the fused step against the serial one (same bits: R25 rank order)
                ref = multi.get("engine")
                if ref is not None:
                    ref.step("serial")
                    dm.step("pready")
                    torch.cuda.synchronize()
                    assert all(torch.equal(ref.out[r], dm.out[r]) for r in range(P)), "fused != serial"
        elif mode == "pready_nooverlap":  # engine forked at the wait (no producer/engine concurrency)
            if dl_no is None:
                dl_no = apps.DLProxy(cs, Np, L, algo, p, y, overlap=False)
            ms = timeit(lambda: dl_no.step("pready"), dl_no.ctl)
        elif mode == "bce_only":  # the producers alone, concurrently on their per-rank streams
            def f():
                dl.ev_ctl.record(dl.ctl)
                for r in range(P):
                    dl.pst[r].wait_event(dl.ev_ctl)
                    apps.bce_grad(p[r], y[r], dl.g[r], Np, L, float(n), None, stream=dl.pst[r])
                    dl.ev_p[r].record(dl.pst[r])
                for r in range(P):
                    dl.ctl.wait_event(dl.ev_p[r])
            ms = timeit(f, dl.ctl)
        elif mode == "allreduce_bounded":  # the engine alone at its overlap width (thin CTAs)
            def f():
                pc.startall(dl.reqs, dl.ctl)
                pc.pbuf_prepare_all(dl.reqs, dl.ctl)
                for q in dl.reqs:  # two ranges: not "every partition by one host op" -> overlap width
                    q.pready_range(0, Np - 2, dl.ctl)
                    q.pready_range(Np - 1, Np - 1, dl.ctl)
                for q in dl.reqs:
                    q.wait_on_stream(dl.ctl)
            ms = timeit(f, dl.ctl)
        else:  # allreduce only (host Pready of every partition)
            def f():
                pc.startall(dl.reqs, dl.ctl)
                pc.pbuf_prepare_all(dl.reqs, dl.ctl)
                pc.preadyall(dl.reqs, dl.ctl)
                for q in dl.reqs:
                    q.wait_on_stream(dl.ctl)
            ms = timeit(f, dl.ctl)
        errs = dl.errors()
        assert errs == [], (mode, errs)
        out.append({"P": P, "partition_bytes": 4 * L, "partitions": Np, "algo": algo, "mode": mode,
                    "ms_per_step": ms, "grad_GB_per_s_all_ranks": P * 4 * n / (ms / 1e3) / 1e9})
        print(json.dumps(out[-1]), flush=True)
    dl.free()
    if dl_no is not None:
        dl_no.free()
    if dl_in is not None:
        dl_in.free()
    for dm in multi.values():
        dm.free()
    for c in cs:
        c.destroy()
    g.destroy()
    return out


if __name__ == "__main__":
    torch.cuda.set_device(0)
    modes = sys.argv[1].split(",") if len(sys.argv) > 1 else ["pready", "serial", "bce_only", "allreduce_only"]
    Ps = [int(v) for v in sys.argv[2].split(",")] if len(sys.argv) > 2 else [8, 4, 2]
    Ls = [int(v) for v in sys.argv[3].split(",")] if len(sys.argv) > 3 else [16384, 65536, 262144]
    algos = [int(v) for v in sys.argv[4].split(",")] if len(sys.argv) > 4 else [pc.ALGO_RING, pc.ALGO_DIRECT]
    for P in Ps:
        for L in Ls:
            for algo in algos:
                try:
                    run(P, L, algo, modes)
                except AssertionError as ex:
                    print(json.dumps({"P": P, "L": L, "algo": algo, "error": str(ex)}), flush=True)
