"""NEXT-4 context measurements on one B200 (paper Table I and Fig 2 analogues).

Table I: host cost of the non-blocking inits, of
pc_prequest_create (blocking) and of pc_pbuf_prepare (first call = exchange +
mapping, later = ready-to-receive only); mean +- sd over repetitions.
Fig 2: cost of cudaStreamSynchronize after a vector-add kernel
of G 1024-thread blocks (8 B per thread), and the kernel + sync total.
Two virtual ranks (one process); JSON lines to stdout."""
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

import torch  # noqa: E402

import paper_conf_sc_temucinslsga24_b200 as pc  # noqa: E402
from paper_conf_sc_temucinslsga24_b200 import apps  # noqa: E402


def us(ts):
    return {"mean_us": statistics.mean(ts) * 1e6, "sd_us": statistics.pstdev(ts) * 1e6, "n": len(ts)}


def table1(reps=10):
    g, cs = pc.local_comms(2, 0)
    st = torch.cuda.Stream()
    n = 2048 * 64
    buf = [torch.zeros(n, device="cuda") for _ in range(4)]
    t_init, t_ar, t_preq, t_first, t_later = [], [], [], [], []
    for _ in range(reps):
        t0 = time.perf_counter()
        s = pc.psend_init(buf[0], 64, 2048, pc.FLOAT32, 1, 3, cs[0])
        t_init.append(time.perf_counter() - t0)
        r = pc.precv_init(buf[1], 64, 2048, pc.FLOAT32, 0, 3, cs[1])
        t0 = time.perf_counter()
        a = pc.pallreduce_init(buf[2], buf[3], 64, 2048, pc.FLOAT32, pc.SUM, pc.ALGO_RING, cs[0])
        t_ar.append(time.perf_counter() - t0)
        a.free()
        s.start(st)
        r.start(st)
        times = [0.0, 0.0]

        def prep(q, k):
            t0 = time.perf_counter()
            q.pbuf_prepare(st)
            times[k] = time.perf_counter() - t0

        pc.run_ranks([lambda: prep(s, 0), lambda: prep(r, 1)])
        t_first.append(max(times))
        t0 = time.perf_counter()
        pq = s.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
        t_preq.append(time.perf_counter() - t0)
        apps.vecadd(buf[0], buf[0], buf[0], n, apps.GRAN_BLOCK, pq, st)
        s.wait_on_stream(st)
        r.wait_on_stream(st)
        for _ in range(100):  # later pbuf_prepare calls: ready-to-receive only
            s.start(st)
            r.start(st)
            t0 = time.perf_counter()
            r.pbuf_prepare(st)
            t_later.append(time.perf_counter() - t0)
            s.pbuf_prepare(st)
            apps.vecadd(buf[0], buf[0], buf[0], n, apps.GRAN_BLOCK, pq, st)
            s.wait_on_stream(st)
            r.wait_on_stream(st)
        torch.cuda.synchronize()
        s.free()
        r.free()
    for c in cs:
        c.destroy()
    g.destroy()
    return {"pc_psend_init/pc_precv_init": us(t_init), "pc_pallreduce_init": us(t_ar),
            "pc_prequest_create": us(t_preq), "pc_pbuf_prepare first": us(t_first),
            "pc_pbuf_prepare later": us(t_later),
            "paper (GH200, Table I)": {"init": "17.2 +- 10.2", "pallreduce_init": "62.3 +- 6.2",
                                       "prequest_create": "110.7 +- 37.8", "pbuf_prepare": "193.4 first, 3.4 +- 1.4"}}


def fig2():
    st = torch.cuda.Stream()
    out = []
    for G in [1, 16, 256, 2048, 16384, 131072]:
        n = G * 2048
        A = torch.randn(n, device="cuda")
        Cb = torch.empty(n, device="cuda")
        for _ in range(5):
            apps.vecadd(A, A, Cb, n, apps.GRAN_NONE, None, st)
        st.synchronize()
        ks, ss = [], []
        for _ in range(50):
            t0 = time.perf_counter()
            apps.vecadd(A, A, Cb, n, apps.GRAN_NONE, None, st)
            t1 = time.perf_counter()
            st.synchronize()
            t2 = time.perf_counter()
            ks.append(t2 - t0)
            ss.append(t2 - t1)
        out.append({"grid_blocks": G, "bytes": 8 * 1024 * G, "kernel_plus_sync_us": statistics.median(ks) * 1e6,
                    "sync_us": statistics.median(ss) * 1e6})
    return out


if __name__ == "__main__":
    print(json.dumps({"table1_overheads": table1()}))
    print(json.dumps({"fig2_sync_cost": fig2(), "paper": "cudaStreamSynchronize 7.8 +- 0.1 us on GH200 (P:L105)"}))
