"""Flag ping-pong latency by memory-order variant (same GPU, two blocks)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_temucinslsga24_b200 import _lib
names = ["release/acquire.sys", "relaxed.sys", "release/acquire.gpu", "relaxed.gpu", "fence.sys+relaxed/acquire.sys", "volatile"]
flags = torch.zeros(1024, dtype=torch.int32, device="cuda")
t = torch.zeros(2, dtype=torch.int64, device="cuda")
iters = 20000
base = 0
for v in range(6):
    for rep in range(2):
        _lib.apps().pcapp_flag_variant(flags[0:].data_ptr(), flags[512:].data_ptr(), v, iters, base, t.data_ptr(), 0)
        torch.cuda.synchronize()
        base += iters
    print(f"{names[v]:32s} one-way {t[0].item() / iters / 2:8.1f} ns")
