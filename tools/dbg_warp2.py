import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
os.environ["CUDA_DEVICE_MAX_CONNECTIONS"] = "32"
import numpy as np, torch
import paper_conf_sc_temucinslsga24_b200 as pc, synth
from paper_conf_sc_temucinslsga24_b200 import apps
from gpu_util import comms, first_prepare
n = 30720
for gran, count in ((1, 64), (0, 2), (2, 2048)):
  partitions = n // count
  with comms(2, timeout_ms=1000) as cs:
    s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
    A = torch.from_numpy(synth.uniform_f32(1, 0, 0, n)).cuda(); B = torch.from_numpy(synth.uniform_f32(1, 0, 1, n)).cuda()
    Cb = torch.empty(n, device="cuda"); R = torch.full((n,), -1.0, device="cuda")
    out = torch.zeros(n, device="cuda"); status = torch.zeros(1, dtype=torch.int32, device="cuda")
    snd = pc.psend_init(Cb, partitions, count, pc.FLOAT32, 1, 7, cs[0])
    rcv = pc.precv_init(R, partitions, count, pc.FLOAT32, 0, 7, cs[1])
    snd.start(s0); rcv.start(s1)
    first_prepare([[snd], [rcv]], [s0, s1])
    sq = snd.prequest_create(gran, 1, 0); rq = rcv.prequest_create(gran, 1, 0)
    torch.cuda.synchronize()
    print("gran", gran, "before: layout", rcv.words("layout", 0, 1), "err", rcv.words("err", 0, 2), "epoch", rcv.words("epoch", 0, 1))
    apps.vecadd(A, B, Cb, n, gran, sq, s0)
    torch.cuda.synchronize()
    print("  after vecadd: flags min", rcv.words("flags", 0, partitions).min(), "err", rcv.words("err", 0, 2), snd.words("err", 0, 2))
    apps.check_recv(rq, R, out, partitions, count * 4, status, blocks=64, stream=s1)
    torch.cuda.synchronize()
    print("  after check: status", status.item(), "err", rcv.words("err", 0, 2), "out ok", (out == R).float().mean().item(), "R ok", (R == A + B).float().mean().item())
    snd.wait_on_stream(s0); rcv.wait_on_stream(s1); torch.cuda.synchronize()
    print("  after wait: err", rcv.words("err", 0, 2))
