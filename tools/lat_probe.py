"""Latency decomposition: the 2-rank Pready->Parrived ping-pong with the
library wait / Pready swapped for raw flag operations (apps.cu
lat_probe_pair_kernel).  One-way ns = total / iters / 2."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_sc_temucinslsga24_b200 as pc
from paper_conf_sc_temucinslsga24_b200 import _lib

MODES = ["lib wait + lib pready_warp", "raw wait + lib pready_warp", "lib wait + raw pready",
         "raw wait + raw pready", "lib wait + lib pready(thread)", "raw wait + lib pready(thread)",
         "lib wait + lane0 epoch_rtr+publish", "lib wait + lane0 epoch_rtr+shfl+publish", "lib wait + lane0 relaxed epoch+publish", "warp wait + lib pready_warp", "lane0 ld.acquire.gpu+publish", "lane0 ld.acquire.sys+publish", "lane0 ld.relaxed.gpu+publish", "lane0 ld.acquire.sys.v2+publish", "lane0 ld.acquire.gpu.v2+publish"]


def run(payload, iters=20000, copy=0):
    g, comms = pc.local_comms(2, 0)
    st = torch.cuda.Stream()
    cnt = payload // 4
    bufs = [torch.zeros(max(iters * cnt, 4), device="cuda") for _ in range(4)]
    a2b = pc.psend_init(bufs[0], iters, cnt, pc.FLOAT32, 1, 101, comms[0])
    b_in = pc.precv_init(bufs[1], iters, cnt, pc.FLOAT32, 0, 101, comms[1])
    b2a = pc.psend_init(bufs[2], iters, cnt, pc.FLOAT32, 0, 102, comms[1])
    a_in = pc.precv_init(bufs[3], iters, cnt, pc.FLOAT32, 1, 102, comms[0])
    t = torch.zeros(8, dtype=torch.int64, device="cuda")
    res = {}
    first = True
    pq = None
    for mode in (range(len(MODES)) if copy == pc.COPY_INLINE else (0, 4, 9)):
        for rep in range(2):
            for q in (a2b, a_in, b_in, b2a):
                q.start(st)
            if first:
                pc.run_ranks([lambda: [q.pbuf_prepare(st) for q in (a2b, a_in)],
                              lambda: [q.pbuf_prepare(st) for q in (b_in, b2a)]])
                pq = [q.prequest_create(pc.GRAN_WARP, 1, c) for q, c in zip((a2b, a_in, b2a, b_in), (copy, 0, copy, 0))]
                first = False
            else:
                for q in (a2b, a_in, b_in, b2a):
                    q.pbuf_prepare(st)
            _lib.apps().pcapp_lat_probe_pair(pq[0].ptr, pq[1].ptr, pq[2].ptr, pq[3].ptr, mode, iters,
                                             t.data_ptr(), st.cuda_stream)
            for q in (a2b, b2a, a_in, b_in):
                q.wait_on_stream(st)
            torch.cuda.synchronize()
        res[MODES[mode]] = t[0].item() / iters / 2
        tt = t.cpu().tolist()
        print(f"copy {copy} payload {payload:4d} B  {MODES[mode]:40s} one-way {res[MODES[mode]]:8.1f} ns  "
              f"pready A {tt[2] / iters:7.0f} B {tt[4] / iters:7.0f} cyc  wait B {tt[5] / iters:7.0f} cyc", flush=True)
    for q in (a2b, a_in, b_in, b2a):
        q.free()
    for c in comms:
        c.destroy()
    g.destroy()
    return res


if __name__ == "__main__":
    torch.cuda.set_device(0)
    for copy in (pc.COPY_INLINE, pc.COPY_LL):
        for payload in (0, 8, 256):
            run(payload, copy=copy)
