"""Small-message allreduce (C5 latency end): 8 virtual ranks, DIRECT, one
epoch = pc_epoch_all(pready) + the grouped engine, replayed from a CUDA graph;
prints us per epoch.  Run under ncu to split the epoch into its kernels."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_sc_temucinslsga24_b200 as pc  # noqa: E402

P = int(sys.argv[1]) if len(sys.argv) > 1 else 8
S = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
algo = {"direct": pc.ALGO_DIRECT, "rd": pc.ALGO_RD, "ring": pc.ALGO_RING, "ll": pc.ALGO_LL}[sys.argv[3] if len(sys.argv) > 3 else "direct"]
n = S // 4
g, cs = pc.local_comms(P, 0)
st = torch.cuda.Stream()
send = [torch.randn(n, device="cuda") for _ in range(P)]
recv = [torch.empty(n, device="cuda") for _ in range(P)]
reqs = [pc.pallreduce_init(send[r], recv[r], 1, n, pc.FLOAT32, pc.SUM, algo, cs[r]) for r in range(P)]
for q in reqs:
    q.start(st)
pc.run_ranks([(lambda q=q: q.pbuf_prepare(st)) for q in reqs])
pc.preadyall(reqs, st)
for q in reqs:
    q.wait_on_stream(st)
torch.cuda.synchronize()


def epoch():
    pc.epoch_all(reqs, pready=True, stream=st)
    for q in reqs:
        q.wait_on_stream(st)


gr = torch.cuda.CUDAGraph()
with torch.cuda.graph(gr, stream=st):
    epoch()
for _ in range(20):
    with torch.cuda.stream(st):
        gr.replay()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
it = 200
e0.record(st)
for _ in range(it):
    with torch.cuda.stream(st):
        gr.replay()
e1.record(st)
torch.cuda.synchronize()
print(f"P={P} S={S} algo={sys.argv[3] if len(sys.argv) > 3 else 'direct'}: {e0.elapsed_time(e1) / it * 1e3:.2f} us/epoch")
assert all(q.error()[0] == 0 for q in reqs)
