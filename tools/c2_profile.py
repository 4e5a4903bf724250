"""C2 profiling driver: vecadd (8 B/thread, 1024-thread blocks) at 256 MiB
[S copies gran persistent]
alone (GRAN_NONE) and with block-granularity Pready (INLINE / ENGINE, g=1)
into a 2-rank partitioned send on one B200.  Run under ncu -k regex:vecadd."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_sc_temucinslsga24_b200 as pc  # noqa: E402
from paper_conf_sc_temucinslsga24_b200 import apps  # noqa: E402

S = int(sys.argv[1]) if len(sys.argv) > 1 else 256 << 20
copies = [int(c) for c in sys.argv[2].split(",")] if len(sys.argv) > 2 else [pc.COPY_INLINE]
gran = int(sys.argv[3]) if len(sys.argv) > 3 else apps.GRAN_BLOCK  # 3 = block_put (R35)
pers = len(sys.argv) > 4 and sys.argv[4] == "persistent"
n = S // 4
g2, cs = pc.local_comms(2, 0)
st = torch.cuda.Stream()
A, B = torch.randn(n, device="cuda"), torch.randn(n, device="cuda")
Cb, R = torch.empty(n, device="cuda"), torch.empty(n, device="cuda")
for _ in range(2):
    apps.vecadd(A, B, Cb, n, apps.GRAN_NONE, None, st, persistent=pers)
torch.cuda.synchronize()
for copy in copies:
    snd = pc.psend_init(Cb, n // 2048, 2048, pc.FLOAT32, 1, 5 + copy, cs[0])
    rcv = pc.precv_init(R, n // 2048, 2048, pc.FLOAT32, 0, 5 + copy, cs[1])
    for e in range(3):
        snd.start(st)
        rcv.start(st)
        if e == 0:
            pc.run_ranks([lambda: snd.pbuf_prepare(st), lambda: rcv.pbuf_prepare(st)])
            sq = snd.prequest_create(pc.GRAN_BLOCK, 1, copy)
        else:
            rcv.pbuf_prepare(st)
            snd.pbuf_prepare(st)
        apps.vecadd(A, B, Cb, n, gran, sq, st, persistent=pers)
        snd.wait_on_stream(st)
        rcv.wait_on_stream(st)
    torch.cuda.synchronize()
    assert torch.equal(R, Cb)
    snd.free()
    rcv.free()
for c in cs:
    c.destroy()
g2.destroy()
print("ok")
