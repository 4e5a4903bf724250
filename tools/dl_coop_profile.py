"""ncu driver: one DL-proxy step with all ranks' producers in one launch and the
cooperative INLINE fold (R36), P ranks, partition L floats.  argv: P L [mode]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_sc_temucinslsga24_b200 as pc  # noqa: E402
from paper_conf_sc_temucinslsga24_b200 import apps  # noqa: E402

P = int(sys.argv[1]) if len(sys.argv) > 1 else 8
L = int(sys.argv[2]) if len(sys.argv) > 2 else 16384
mode = sys.argv[3] if len(sys.argv) > 3 else "coop"
Np = -(-25_557_032 // L)
n = Np * L
g, cs = pc.local_comms(P, 0)
p = [(0.02 + 0.96 * torch.rand(n, device="cuda")) for _ in range(P)]
y = [torch.randint(0, 2, (n,), device="cuda").float() for _ in range(P)]
dl = apps.DLProxy(cs, Np, L, pc.ALGO_DIRECT, p, y, copy=pc.COPY_INLINE if mode != "serial" else None,
                  multi=True, coop=mode == "coop")
for _ in range(3):
    dl.step("serial" if mode == "serial" else "pready")
torch.cuda.synchronize()
assert dl.errors() == []
dl.free()
for c in cs:
    c.destroy()
g.destroy()
print("ok")
