"""Worker for test_gpu_multiproc: one process per rank, every rank on cuda:0
(the box has one GPU), bootstrap over a gloo process group, peers mapped with
CUDA IPC — the N > 1 code path of bench.py except that ranks share a GPU."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import paper_conf_sc_temucinslsga24_b200 as pc  # noqa: E402
import synth  # noqa: E402
from paper_conf_sc_temucinslsga24_b200 import apps  # noqa: E402

out_dir = sys.argv[1]
dist.init_process_group("gloo")
r, P = dist.get_rank(), dist.get_world_size()
torch.cuda.set_device(0)
comm = pc.Comm.from_process_group(0)
st = torch.cuda.Stream()
res = {}
for name, algo in (("ring", pc.ALGO_RING), ("rd", pc.ALGO_RD), ("direct", pc.ALGO_DIRECT),
                   ("direct_push", pc.ALGO_DIRECT_PUSH), ("ll", pc.ALGO_LL)):
    Np, L = 3, 1000
    x = synth.normal_f32(synth.BASE_SEED, r, 0, Np * L)
    send = torch.from_numpy(x).cuda()
    recv = torch.zeros_like(send)
    q = pc.pallreduce_init(send, recv, Np, L, pc.FLOAT32, pc.SUM, algo, comm)
    for e in range(2):
        q.start(st)
        q.pbuf_prepare(st)
        q.pready_range(0, Np - 1, st)
        q.wait_on_stream(st)
    st.synchronize()
    assert q.error() == (0, 0), q.error()
    res[name] = recv.cpu().numpy()
    # later epochs as bench.py's N > 1 step runs them: Start + RTR + Pready in
    # one pc_epoch_all kernel (RTR words of the other PROCESS, via CUDA IPC)
    for e in range(3):
        recv.zero_()
        st.wait_stream(torch.cuda.current_stream())
        pc.epoch_all([q], pready=True, stream=st)
        q.wait_on_stream(st)
        st.synchronize()
        assert q.error() == (0, 0), q.error()
        res[name + "_epoch_all%d" % e] = recv.cpu().numpy()
    q.free()
# INLINE allreduce across the processes (reading R33): the producer's block
# Pready that completes a partition on the last rank folds it for both ranks
# (system-scope arrival counter in rank 0's control block, peer stores).
Np, L = 5, 777
x = synth.normal_f32(synth.BASE_SEED + 3, r, 0, Np * L)
srcb = torch.from_numpy(x).cuda()
send = torch.zeros_like(srcb)
recv = torch.zeros_like(srcb)
q = pc.pallreduce_init(send, recv, Np, L, pc.FLOAT32, pc.SUM, pc.ALGO_DIRECT, comm)
for e in range(3):
    recv.zero_()
    st.wait_stream(torch.cuda.current_stream())
    q.start(st)
    q.pbuf_prepare(st)
    if e == 0:
        pq = q.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
    apps.produce(send, srcb, Np, L * 4, apps.GRAN_BLOCK, pq, order_stride=3, stream=st)
    q.wait_on_stream(st)
    st.synchronize()
    assert q.error() == (0, 0), q.error()
    res["inline%d" % e] = recv.cpu().numpy()
q.free()
# engine/producer overlap across the processes: each rank's producer waits on
# the device pc_parrived(0) of the collective before it Preadies the rest
Np, L = 4, 4099
x = synth.normal_f32(synth.BASE_SEED + 4, r, 0, Np * L)
send = torch.from_numpy(x).cuda()
recv = torch.zeros_like(send)
q = pc.pallreduce_init(send, recv, Np, L, pc.FLOAT32, pc.SUM, pc.ALGO_DIRECT, comm)
q.start(st)
q.pbuf_prepare(st)
pq = q.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_ENGINE)
stamps = torch.zeros((1, 4), dtype=torch.int64, device="cuda")
apps.overlap_probe([pq], Np, 20000, stamps, st)
q.wait_on_stream(st)
st.synchronize()
assert q.error() == (0, 0), q.error()
res["overlap"] = recv.cpu().numpy()
res["overlap_stamps"] = stamps.cpu().numpy()
q.free()
# p2p 0 -> 1 with block-granularity Pready from the producer kernel
n = 2048 * 8
if r == 0:
    a = torch.from_numpy(synth.uniform_f32(synth.BASE_SEED, 0, 0, n)).cuda()
    b = torch.from_numpy(synth.uniform_f32(synth.BASE_SEED, 0, 1, n)).cuda()
    c = torch.empty(n, device="cuda")
    q = pc.psend_init(c, 8, 2048, pc.FLOAT32, 1, 9, comm)
else:
    rb = torch.zeros(n, device="cuda")
    q = pc.precv_init(rb, 8, 2048, pc.FLOAT32, 0, 9, comm)
q.start(st)
q.pbuf_prepare(st)
pq = q.prequest_create(pc.GRAN_BLOCK, 2, pc.COPY_INLINE)
if r == 0:
    apps.vecadd(a, b, c, n, apps.GRAN_BLOCK, pq, st)
q.wait()
assert q.error() == (0, 0), q.error()
if r == 1:
    res["p2p"] = rb.cpu().numpy()
q.free()
# ENGINE-mode p2p 1 -> 0 (library warps push), warp-granularity Pready
if r == 1:
    a2 = torch.from_numpy(synth.uniform_f32(synth.BASE_SEED, 1, 0, n)).cuda()
    c2 = torch.empty(n, device="cuda")
    q = pc.psend_init(c2, n // 64, 64, pc.FLOAT32, 0, 12, comm)
else:
    rb2 = torch.zeros(n, device="cuda")
    q = pc.precv_init(rb2, n // 64, 64, pc.FLOAT32, 1, 12, comm)
for e in range(2):
    q.start(st)
    q.pbuf_prepare(st)
    if e == 0:
        pq = q.prequest_create(pc.GRAN_WARP, 4, pc.COPY_ENGINE)
    if r == 1:
        apps.vecadd(a2, a2, c2, n, apps.GRAN_WARP, pq, st)
    q.wait()
    assert q.error() == (0, 0), q.error()
if r == 0:
    res["p2p_engine"] = rb2.cpu().numpy()
q.free()
# LL p2p 0 -> 1 (16-B lines over CUDA IPC), warp-granularity Pready, 3 epochs
# (both line-area parities, the sender's completion acquires the receiver's RTR)
nl = 2048 * 2  # whole 1024-thread blocks (vecadd launches ceil(n/2048) blocks)
if r == 0:
    a3 = torch.from_numpy(synth.uniform_f32(synth.BASE_SEED, 0, 7, nl)).cuda()
    c3 = torch.empty(nl, device="cuda")
    q = pc.psend_init(c3, nl // 64, 64, pc.FLOAT32, 1, 13, comm)
else:
    rb3 = torch.zeros(nl, device="cuda")
    q = pc.precv_init(rb3, nl // 64, 64, pc.FLOAT32, 0, 13, comm)
for e in range(3):
    q.start(st)
    q.pbuf_prepare(st)
    if e == 0:
        pq = q.prequest_create(pc.GRAN_WARP, 1, pc.COPY_LL if r == 0 else pc.COPY_INLINE)
    if r == 0:
        apps.vecadd(a3, a3, c3, nl, apps.GRAN_WARP, pq, st)
    q.wait()
    assert q.error() == (0, 0), q.error()
if r == 1:
    res["p2p_ll"] = rb3.cpu().numpy()
q.free()
# Jacobi 2 x 1 across the two processes (one rank each), halos over CUDA IPC
js = apps.JacobiSolver([comm], [r], 256, 2, 1, 30, H=32)
js.set_initial(synth.jacobi_init(256, 256, "random"))
torch.cuda.synchronize()
js.solve(st)
torch.cuda.synchronize()
assert js.errors() == [], js.errors()
res["jacobi"] = js.result()
js.free()
np.savez(os.path.join(out_dir, f"rank{r}.npz"), **res)
comm.destroy()
dist.destroy_process_group()
print("worker OK", r)
