"""C5 / C3 / C2 sweeps on one B200 (virtual ranks), JSONL to stdout.

  python tools/sweep.py allreduce [--ranks 2,4,8] [--algos ring,rd]
  python tools/sweep.py dl                      # ResNet-50 / BERT-large gradient buffers
  python tools/sweep.py p2p                     # C2: Pready granularity x aggregation x copy mode

Each point: busBW (allreduce) or GB/s (p2p) from CUDA events over many
back-to-back epochs on one stream (the bench step), median of 3 blocks."""
import argparse
import collections
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

import torch  # noqa: E402

import paper_conf_sc_temucinslsga24_b200 as pc  # noqa: E402
import synth  # noqa: E402
from paper_conf_sc_temucinslsga24_b200 import apps  # noqa: E402


def busbw(S, sec, P):
    return S / sec * 2.0 * (P - 1) / P / 1e9 if P > 1 else S / sec / 1e9


# ------------------------------------------------------------ parity gate (§8(d).2)
# Before a point is reported: (1) the timed fp32 run's result is bit-identical
# on every rank and within the north_star bound |y - y64| <= 1e-5 * sum|x|
# (reading R16) on sampled elements against the fp64 sum of the inputs; (2)
# for S <= 64 MiB an int32 run of the same shape (partitions, count, schedule)
# equals the plain definition, the wrapping sum mod 2^32, on every element.
# Plain definitions only (no oracle import: tools/ is product-side).
def fp32_gate(send, recv, nsample=65536):
    n = send[0].numel()
    ok = all(torch.equal(recv[0][:n], r[:n]) for r in recv[1:])
    g = torch.Generator(device="cuda")
    g.manual_seed(0x5C24)
    idx = torch.randint(0, n, (min(nsample, n),), device="cuda", generator=g)
    x = torch.stack([t[idx].double() for t in send])
    y64, sabs = x.sum(0), x.abs().sum(0)
    return ok and bool(((recv[0][idx].double() - y64).abs() <= 1e-5 * sabs).all().item())


def int32_gate(cs, Np, count, algo, st):
    P = len(cs)
    send = [torch.randint(-2**31, 2**31 - 1, (Np * count,), dtype=torch.int32, device="cuda") for _ in range(P)]
    recv = [torch.empty_like(send[0]) for _ in range(P)]
    reqs = [pc.pallreduce_init(send[r], recv[r], Np, count, pc.INT32, pc.SUM, algo, cs[r]) for r in range(P)]
    for q in reqs:
        q.start(st)
    pc.run_ranks([(lambda q=q: q.pbuf_prepare(st)) for q in reqs])
    pc.preadyall(reqs, st)
    for q in reqs:
        q.wait_on_stream(st)
    pc.epoch_all(reqs, pready=True, stream=st)  # and a second epoch through the bench's control path
    for q in reqs:
        q.wait_on_stream(st)
    torch.cuda.synchronize()
    tot = torch.zeros(Np * count, dtype=torch.int64, device="cuda")
    for t in send:
        tot += t.long()
    want = ((tot + 2**31) % 2**32 - 2**31).int()
    ok = all(torch.equal(r, want) for r in recv) and all(q.error()[0] == 0 for q in reqs)
    for q in reqs:
        q.free()
    return ok


def time_allreduce(cs, S, Np, algo, min_ms=30.0, graph=False):
    P = len(cs)
    count = max(S // 4 // Np, 1)
    n = count * Np
    st = torch.cuda.Stream()
    send = [torch.randn(n, device="cuda") for _ in range(P)]
    recv = [torch.empty(n, device="cuda") for _ in range(P)]
    reqs = [pc.pallreduce_init(send[r], recv[r], Np, count, pc.FLOAT32, pc.SUM, algo, cs[r]) for r in range(P)]

    def step(first=False):
        if first:
            for q in reqs:
                q.start(st)
            pc.run_ranks([(lambda q=q: q.pbuf_prepare(st)) for q in reqs])
            pc.preadyall(reqs, st)  # S_0: the user's Pready of every partition, one kernel
        elif os.environ.get("PC_SWEEP_SEPARATE_CTL"):
            pc.startall(reqs, st)  # one kernel for every rank's epoch
            pc.pbuf_prepare_all(reqs, st)  # one kernel for every RTR
            pc.preadyall(reqs, st)
        else:  # Start + RTR + S_0 Pready of every rank in ONE kernel
            pc.epoch_all(reqs, pready=True, stream=st)
        for q in reqs:
            q.wait_on_stream(st)

    step(True)
    torch.cuda.synchronize()
    run = step
    if graph:  # capture one epoch of every rank; each replay is a new epoch
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            step()

        def run():
            with torch.cuda.stream(st):  # replay on the timed stream
                g.replay()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    run()
    e1.record(st)
    torch.cuda.synchronize()
    one = max(e0.elapsed_time(e1), 1e-3)
    iters = int(max(5, min(2000, min_ms / one)))
    blocks = []
    for _ in range(3):
        e0.record(st)
        for _ in range(iters):
            run()
        e1.record(st)
        torch.cuda.synchronize()
        blocks.append(e0.elapsed_time(e1) / iters)
    errs = [q.error() for q in reqs if q.error()[0] != 0]
    info = reqs[0].info()
    parity = fp32_gate(send, recv)
    for q in reqs:
        q.free()
    if n * 4 <= (64 << 20):
        parity = parity and int32_gate(cs, Np, count, algo, st)
    ms = statistics.median(blocks)
    return {"bytes_per_rank": n * 4, "partitions": Np, "ranks": P,
            "algo": ["auto", "ring", "rd", "direct", "direct_push", "ll"][algo],
            "us_per_step": ms * 1e3, "busbw_gbs": busbw(n * 4, ms / 1e3, P), "slices": info["slices"],
            "graph": graph, "errors": errs, "parity": parity}


def sweep_allreduce(args):
    for P in [int(x) for x in args.ranks.split(",")]:
        g, cs = pc.local_comms(P, 0)
        for algo in args.algos.split(","):
            a = {"ring": pc.ALGO_RING, "rd": pc.ALGO_RD, "direct": pc.ALGO_DIRECT, "direct_push": pc.ALGO_DIRECT_PUSH,
                 "ll": pc.ALGO_LL,
                 "auto": pc.ALGO_AUTO}[algo]
            if a == pc.ALGO_RD and P & (P - 1):
                continue
            S = 1 << 10
            while S <= args.max_bytes:
                for Np in [int(x) for x in args.partitions.split(",")]:
                    if S // 4 // Np < P:
                        continue
                    r = time_allreduce(cs, S, Np, a, graph=args.graph)
                    print(json.dumps(r), flush=True)
                S <<= 2
        for c in cs:
            c.destroy()
        g.destroy()


def time_coll(cs, kind, S, Np, min_ms=30.0):
    """NEXT-3 collectives, nccl-tests conventions: S = the full buffer (reduce-
    scatter input, allgather output, broadcast buffer) per rank; busBW =
    S/t * (P-1)/P for reduce-scatter / allgather, S/t for broadcast."""
    P = len(cs)
    st = torch.cuda.Stream()
    if kind == "rs":
        count = max(S // 4 // (Np * P), 1)
        send = [torch.randn(Np * P * count, device="cuda") for _ in range(P)]
        recv = [torch.empty(Np * count, device="cuda") for _ in range(P)]
        reqs = [pc.preduce_scatter_init(send[r], recv[r], Np, count, pc.FLOAT32, pc.SUM, cs[r]) for r in range(P)]
        full = Np * P * count * 4
    elif kind == "ag":
        count = max(S // 4 // (Np * P), 1)
        send = [torch.randn(Np * count, device="cuda") for _ in range(P)]
        recv = [torch.empty(P * Np * count, device="cuda") for _ in range(P)]
        reqs = [pc.pallgather_init(send[r], recv[r], Np, count, pc.FLOAT32, cs[r]) for r in range(P)]
        full = P * Np * count * 4
    else:
        count = max(S // 4 // Np, 1)
        buf = [torch.randn(Np * count, device="cuda") for _ in range(P)]
        reqs = [pc.pbcast_init(buf[r], Np, count, pc.FLOAT32, 0, cs[r]) for r in range(P)]
        full = Np * count * 4
    producers = reqs if kind != "bc" else reqs[:1]

    def step(first=False):
        if first:
            for q in reqs:
                q.start(st)
            pc.run_ranks([(lambda q=q: q.pbuf_prepare(st)) for q in reqs])
        else:
            pc.startall(reqs, st)
            pc.pbuf_prepare_all(reqs, st)
        pc.preadyall(producers, st)
        for q in reqs:
            q.wait_on_stream(st)

    step(True)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    step()
    e1.record(st)
    torch.cuda.synchronize()
    iters = int(max(5, min(2000, min_ms / max(e0.elapsed_time(e1), 1e-3))))
    blocks = []
    for _ in range(3):
        e0.record(st)
        for _ in range(iters):
            step()
        e1.record(st)
        torch.cuda.synchronize()
        blocks.append(e0.elapsed_time(e1) / iters)
    errs = [q.error() for q in reqs if q.error()[0] != 0]
    # parity gate: the plain definition of the collective on every element
    # (reduce-scatter: the rank-order fp32 fold (R25) of block r of every
    # partition; allgather: rank-major concatenation; broadcast: the root's)
    if kind == "rs":
        parity = True
        for r in range(P):
            blk = [send[k].view(Np, P, count)[:, r, :] for k in range(P)]
            acc = blk[0].clone()
            for k in range(1, P):
                acc = acc + blk[k]  # fp32 adds in rank order, round to nearest
            parity = parity and torch.equal(recv[r].view(Np, count), acc)
    elif kind == "ag":
        want = torch.cat([send[k] for k in range(P)])
        parity = all(torch.equal(recv[r], want) for r in range(P))
    else:
        parity = all(torch.equal(buf[r], buf[0]) for r in range(P))
    for q in reqs:
        q.free()
    ms = statistics.median(blocks)
    fac = 1.0 if kind == "bc" else (P - 1) / P
    return {"coll": kind, "ranks": P, "bytes": full, "partitions": Np, "us_per_step": ms * 1e3,
            "busbw_gbs": full / (ms / 1e3) * fac / 1e9, "errors": errs, "parity": bool(parity)}


def sweep_coll(args):
    for P in [int(x) for x in args.ranks.split(",")]:
        g, cs = pc.local_comms(P, 0)
        for kind in ("rs", "ag", "bc"):
            for S in [1 << 20, 16 << 20, 256 << 20, 1 << 30]:
                if S > args.max_bytes:
                    continue
                print(json.dumps(time_coll(cs, kind, S, 64)), flush=True)
        for c in cs:
            c.destroy()
        g.destroy()


def sweep_dl(args):
    for P in [int(x) for x in args.ranks.split(",")]:
        g, cs = pc.local_comms(P, 0)
        for name, sizes, part_bytes in (("resnet50", synth.RESNET50_SIZES, 1 << 20),
                                        ("bert_large", synth.BERT_LARGE_SIZES, 4 << 20)):
            total = sum(sizes) * 4
            Np = max(1, total // part_bytes)
            for an in args.algos.split(","):
                algo = {"ring": pc.ALGO_RING, "rd": pc.ALGO_RD, "direct": pc.ALGO_DIRECT, "auto": pc.ALGO_AUTO}[an]
                if algo == pc.ALGO_RD and P & (P - 1):
                    continue
                r = time_allreduce(cs, total, Np, algo)
                r["model"] = name
                r["tensors"] = len(sizes)
                print(json.dumps(r), flush=True)
        for c in cs:
            c.destroy()
        g.destroy()


def sweep_dl_per_tensor(args):
    """C3 workload (ii): one partitioned-allreduce request per gradient tensor
    (AUTO schedule per size), one epoch of all of them captured in a CUDA graph."""
    for P in [int(x) for x in args.ranks.split(",")]:
        g, cs = pc.local_comms(P, 0)
        for name, sizes in (("resnet50", synth.RESNET50_SIZES),):
            st = torch.cuda.Stream()
            bufs = [[torch.randn(n, device="cuda") for n in sizes] for _ in range(P)]
            outs = [[torch.empty(n, device="cuda") for n in sizes] for _ in range(P)]
            reqs = [[pc.pallreduce_init(bufs[r][t], outs[r][t], 1, n, pc.FLOAT32, pc.SUM, pc.ALGO_AUTO, cs[r])
                     for t, n in enumerate(sizes)] for r in range(P)]
            flat = [q for r in range(P) for q in reqs[r]]
            for q in flat:
                q.start(st)
            pc.run_ranks([(lambda r=r: [q.pbuf_prepare(st) for q in reqs[r]]) for r in range(P)])

            def epoch_rest():
                pc.preadyall(flat, st) if len(flat) <= 16 else [pc.preadyall(flat[i:i + 16], st)
                                                                  for i in range(0, len(flat), 16)]
                for t in range(len(sizes)):
                    for r in range(P):
                        reqs[r][t].wait_on_stream(st)

            epoch_rest()
            torch.cuda.synchronize()

            if args.batched:  # one pc_epoch_all (table kernel) + one batched engine launch
                def epoch():
                    pc.epoch_all(flat, pready=True, stream=st)
                    pc.waitall_on_stream(flat, st)

                epoch()  # eager first: the batch tables are built outside the capture
                torch.cuda.synchronize()
            else:
                def epoch():
                    pc.startall(flat, st)
                    pc.pbuf_prepare_all(flat, st)
                    epoch_rest()

            gr = torch.cuda.CUDAGraph()
            with torch.cuda.graph(gr, stream=st):
                epoch()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            it = 10
            e0.record(st)
            for _ in range(it):
                with torch.cuda.stream(st):
                    gr.replay()
            e1.record(st)
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / it
            total = sum(sizes) * 4
            errs = [q.error() for q in flat if q.error()[0] != 0]
            parity = all(fp32_gate([bufs[r][t] for r in range(P)], [outs[r][t] for r in range(P)], 4096)
                         for t in range(len(sizes)))
            algos = collections.Counter(["auto", "ring", "rd", "direct"][q.info()["algo"]] for q in reqs[0])
            print(json.dumps({"model": name, "mode": "per-tensor (graph%s)" % (", batched" if args.batched else ""),
                              "ranks": P, "tensors": len(sizes),
                              "bytes_per_rank": total, "us_per_step": ms * 1e3,
                              "busbw_gbs": busbw(total, ms / 1e3, P), "algos": dict(algos), "errors": errs,
                              "parity": parity}),
                  flush=True)
            for q in flat:
                q.free()
        for c in cs:
            c.destroy()
        g.destroy()


def sweep_p2p(args):
    """C2: vector-add producer + Pready at thread/warp/block granularity with
    aggregation g, INLINE vs ENGINE; goodput = bytes / (kernel + comm) time."""
    g2, cs = pc.local_comms(2, 0)
    st = torch.cuda.Stream()
    elems = {apps.GRAN_THREAD: 2, apps.GRAN_WARP: 64, apps.GRAN_BLOCK: 2048, apps.GRAN_BLOCK_PUT: 2048}
    sizes = [int(x) for x in args.sizes.split(",")] if args.sizes else [64 << 10, 1 << 20, 16 << 20, 256 << 20]
    grans = {"thread": apps.GRAN_THREAD, "warp": apps.GRAN_WARP, "block": apps.GRAN_BLOCK,
             "block_put": apps.GRAN_BLOCK_PUT}
    gsel = [grans[g] for g in args.grans.split(",")] if args.grans else [apps.GRAN_BLOCK, apps.GRAN_WARP,
                                                                           apps.GRAN_THREAD]
    aggsel = args.aggs.split(",") if args.aggs else None
    pers = args.persistent
    producer = "persistent" if pers else "block-per-partition"
    for S in sizes:
        n = S // 4
        A = torch.randn(n, device="cuda")
        B = torch.randn(n, device="cuda")
        Cb = torch.empty(n, device="cuda")
        R = torch.empty(n, device="cuda")
        # traditional baseline: kernel, then a device copy (no library)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        it = 20

        def trad():
            apps.vecadd(A, B, Cb, n, apps.GRAN_NONE, None, st, persistent=pers)
            with torch.cuda.stream(st):
                R.copy_(Cb)

        for _ in range(3):  # warm-up (module load, first-touch)
            trad()
        if args.graph:  # both arms replay a captured CUDA graph of their epoch
            gt = torch.cuda.CUDAGraph()
            with torch.cuda.graph(gt, stream=st):
                trad()
            trad = gt.replay  # noqa: F811
        torch.cuda.synchronize()
        e0.record(st)
        for _ in range(it):
            with torch.cuda.stream(st):
                trad()
        e1.record(st)
        torch.cuda.synchronize()
        print(json.dumps({"bytes": S, "mode": "kernel+copy (traditional, same GPU)", "producer": producer, "graph": bool(args.graph),
                          "us": e0.elapsed_time(e1) / it * 1e3,
                          "gbs": S / (e0.elapsed_time(e1) / it / 1e3) / 1e9}), flush=True)
        for gran in gsel:
            cnt = elems[gran]
            parts = n // cnt
            for agg_name, agg in (("none", 1), ("block", max(1, 2048 // cnt)), ("1MiB", max(1, (1 << 18) // cnt)),
                                  ("all", parts)):
                if aggsel and agg_name not in aggsel:
                    continue
                agg = min(agg, parts)
                for copy in (pc.COPY_INLINE, pc.COPY_ENGINE):
                    if gran == apps.GRAN_THREAD and agg == 1 and S > (16 << 20):
                        continue  # 33 M flags: covered up to 16 MiB
                    snd = pc.psend_init(Cb, parts, cnt, pc.FLOAT32, 1, 5, cs[0])
                    rcv = pc.precv_init(R, parts, cnt, pc.FLOAT32, 0, 5, cs[1])

                    def epoch(first=False):
                        if args.batched:  # MPI_Startall + Pbuf_prepare in one kernel, MPI_Waitall in one kernel
                            pc.epoch_all([snd, rcv], False, st)
                            apps.vecadd(A, B, Cb, n, gran, sq[0], st, persistent=pers)
                            pc.waitall_on_stream([snd, rcv], st)
                            return
                        snd.start(st)
                        rcv.start(st)
                        if first:
                            pc.run_ranks([lambda: snd.pbuf_prepare(st), lambda: rcv.pbuf_prepare(st)])
                        else:
                            rcv.pbuf_prepare(st)
                            snd.pbuf_prepare(st)
                        apps.vecadd(A, B, Cb, n, gran, sq[0], st, persistent=pers)
                        snd.wait_on_stream(st)
                        rcv.wait_on_stream(st)

                    snd.start(st)
                    rcv.start(st)
                    pc.run_ranks([lambda: snd.pbuf_prepare(st), lambda: rcv.pbuf_prepare(st)])
                    sq = [snd.prequest_create(min(gran, apps.GRAN_BLOCK), agg, copy)]
                    apps.vecadd(A, B, Cb, n, gran, sq[0], st, persistent=pers)
                    snd.wait_on_stream(st)
                    rcv.wait_on_stream(st)
                    run = epoch
                    if args.graph:
                        for _ in range(2):
                            epoch()
                        torch.cuda.synchronize()
                        ge = torch.cuda.CUDAGraph()
                        with torch.cuda.graph(ge, stream=st):
                            epoch()
                        run = ge.replay
                    torch.cuda.synchronize()
                    e0.record(st)
                    for _ in range(it):
                        with torch.cuda.stream(st):
                            run()
                    e1.record(st)
                    torch.cuda.synchronize()
                    us = e0.elapsed_time(e1) / it * 1e3
                    errs = [q.error() for q in (snd, rcv) if q.error()[0] != 0]
                    ok = torch.equal(R, Cb)
                    print(json.dumps({"bytes": S, "gran": ["thread", "warp", "block", "block_put"][gran], "agg": agg_name,
                                      "g": agg, "copy": ["inline", "engine"][copy], "producer": producer,
                                      "control": "epoch_all+waitall" if args.batched else "per-request",
                                      "graph": bool(args.graph), "us": us,
                                      "goodput_gbs": S / (us / 1e6) / 1e9, "ok": ok, "parity": ok and not errs,
                                      "errors": errs}), flush=True)
                    snd.free()
                    rcv.free()
    for c in cs:
        c.destroy()
    g2.destroy()


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("what", choices=["allreduce", "dl", "dl_tensor", "p2p", "coll"])
    ap.add_argument("--ranks", default="8")
    ap.add_argument("--algos", default="ring,rd")
    ap.add_argument("--partitions", default="1,16,64")
    ap.add_argument("--max-bytes", type=int, default=1 << 30)
    ap.add_argument("--graph", action="store_true", help="replay a captured CUDA graph of the epoch")
    ap.add_argument("--sizes", default="", help="p2p: buffer bytes, comma separated")
    ap.add_argument("--batched", action="store_true",
                    help="dl_tensor / p2p: pc_epoch_all + pc_waitall_on_stream batch (one control and one wait kernel)")
    ap.add_argument("--grans", default="", help="p2p: thread,warp,block")
    ap.add_argument("--aggs", default="", help="p2p: none,block,1MiB,all")
    ap.add_argument("--persistent", action="store_true",
                    help="p2p: persistent vecadd producer (both arms) instead of one CTA per logical block")
    a = ap.parse_args()
    {"allreduce": sweep_allreduce, "dl": sweep_dl, "dl_tensor": sweep_dl_per_tensor, "p2p": sweep_p2p,
     "coll": sweep_coll}[a.what](a)
