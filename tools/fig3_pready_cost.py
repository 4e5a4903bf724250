"""Fig 3 analogue: the cost of marking ONE block's
data ready at thread, warp and block granularity, for block sizes t = 1 ...
1024 threads (8 B per thread, INLINE "Kernel Copy" to a second virtual rank),
plus thread granularity with library aggregation to one transport partition
(g = t, the paper's recommendation).  Cost = %globaltimer around the
block's Pready calls (block barrier on both sides), median over epochs.
Every epoch's received bytes are checked.  JSONL to stdout."""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import torch  # noqa: E402

import paper_conf_sc_temucinslsga24_b200 as pc  # noqa: E402
from gpu_util import comms, first_prepare  # noqa: E402
from paper_conf_sc_temucinslsga24_b200 import apps  # noqa: E402

EPOCHS = int(os.environ.get("EPOCHS", "200"))
torch.cuda.set_device(0)
modes = [("thread", apps.GRAN_THREAD, False), ("warp", apps.GRAN_WARP, False), ("block", apps.GRAN_BLOCK, False),
         ("thread_agg_block", apps.GRAN_THREAD, True)]
for t in [1, 2, 4, 8, 16, 32, 64, 128, 256, 512, 1024]:
    for name, gran, agg_all in modes:
        if gran == apps.GRAN_WARP and t % 32:
            continue
        n = 2 * t  # floats: 8 B per thread
        parts = {apps.GRAN_THREAD: t, apps.GRAN_WARP: t // 32, apps.GRAN_BLOCK: 1}[gran]
        count = n // parts
        agg = parts if agg_all else 1
        with comms(2) as cs:
            s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
            A, B = torch.randn(n, device="cuda"), torch.randn(n, device="cuda")
            Cb, R = torch.empty(n, device="cuda"), torch.zeros(n, device="cuda")
            ns = torch.zeros(1, dtype=torch.int64, device="cuda")
            snd = pc.psend_init(Cb, parts, count, pc.FLOAT32, 1, 2, cs[0])
            rcv = pc.precv_init(R, parts, count, pc.FLOAT32, 0, 2, cs[1])
            samples, ok = [], True
            for e in range(EPOCHS + 5):
                snd.start(s0)
                rcv.start(s1)
                if e == 0:
                    first_prepare([[snd], [rcv]], [s0, s1])
                    sq = snd.prequest_create(gran, agg, pc.COPY_INLINE)
                else:
                    rcv.pbuf_prepare(s1)
                    snd.pbuf_prepare(s0)
                apps.pready_cost(A, B, Cb, t, gran, sq, ns, stream=s0)
                snd.wait_on_stream(s0)
                rcv.wait_on_stream(s1)
                torch.cuda.synchronize()
                if e >= 5:
                    samples.append(int(ns.item()))
                ok = ok and bool(torch.equal(R, A + B))
            ok = ok and snd.error()[0] == 0 and rcv.error()[0] == 0
            snd.free()
            rcv.free()
        print(json.dumps({"threads": t, "mode": name, "partitions": parts, "aggregation": agg,
                          "ns_p50": statistics.median(samples), "ns_min": min(samples), "ok": ok}), flush=True)
