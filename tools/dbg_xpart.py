"""Debug: MPI-4 different partition counts (R30) — receiver words after one epoch."""
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sc_temucinslsga24_b200 as pc  # noqa: E402
import synth  # noqa: E402
from gpu_util import comms, first_prepare  # noqa: E402
from paper_conf_sc_temucinslsga24_b200 import apps  # noqa: E402

Ns, Nr, total = int(sys.argv[1]), int(sys.argv[2]), 13440
sb, rb = total // Ns, total // Nr
with comms(2) as cs:
    s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
    payload = synth.bytes_tagged(1, 1, 0, total)
    src = torch.from_numpy(payload).cuda()
    sbuf, rbuf = torch.empty_like(src), torch.zeros_like(src)
    snd = pc.psend_init(sbuf, Ns, sb, pc.BYTE, 1, 9, cs[0])
    rcv = pc.precv_init(rbuf, Nr, rb, pc.BYTE, 0, 9, cs[1])
    torch.cuda.synchronize()
    snd.start(s0)
    rcv.start(s1)
    first_prepare([[snd], [rcv]], [s0, s1])
    sq = snd.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
    print("layout", [hex(v) for v in rcv.words("layout", 0, 1)], "epoch", rcv.words("epoch", 0, 1))
    apps.produce(sbuf, src, Ns, sb, apps.GRAN_BLOCK, sq, stream=s0)
    torch.cuda.synchronize()
    print("recv flags", rcv.words("flags", 0, Nr), "sent", snd.words("sent", 0, Ns), "errs", snd.error(), rcv.error())
    print("bytes ok", bool((rbuf.cpu().numpy() == payload).all()))
    print("parrived", [rcv.parrived(p) for p in range(Nr)])
