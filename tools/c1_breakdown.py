"""Where the C1 epoch's device time goes (2 virtual ranks, 1 MiB, block Pready g=16)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
import torch
import paper_conf_sc_temucinslsga24_b200 as pc
from paper_conf_sc_temucinslsga24_b200 import apps

n = 1 << 18
g, cs = pc.local_comms(2, 0)
st = torch.cuda.Stream()
A, B = torch.randn(n, device="cuda"), torch.randn(n, device="cuda")
Cb, R = torch.empty(n, device="cuda"), torch.empty(n, device="cuda")
snd = pc.psend_init(Cb, 128, 2048, pc.FLOAT32, 1, 11, cs[0])
rcv = pc.precv_init(R, 128, 2048, pc.FLOAT32, 0, 11, cs[1])
snd.start(st); rcv.start(st)
pc.run_ranks([lambda: snd.pbuf_prepare(st), lambda: rcv.pbuf_prepare(st)])
sq = snd.prequest_create(pc.GRAN_BLOCK, 16, pc.COPY_INLINE)
apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK, sq, st)
snd.wait_on_stream(st); rcv.wait_on_stream(st)
torch.cuda.synchronize()

def timeit(f, it=300):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for _ in range(10): f()
    torch.cuda.synchronize()
    e0.record(st)
    for _ in range(it): f()
    e1.record(st)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / it * 1e3

def full_batched():
    pc.startall([snd, rcv], st); pc.pbuf_prepare_all([snd, rcv], st)
    apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK, sq, st)
    snd.wait_on_stream(st); rcv.wait_on_stream(st)

def full_memops():
    snd.start(st); rcv.start(st); rcv.pbuf_prepare(st); snd.pbuf_prepare(st)
    apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK, sq, st)
    snd.wait_on_stream(st); rcv.wait_on_stream(st)

def vec_only():
    apps.vecadd(A, B, Cb, n, apps.GRAN_NONE, None, st)

def trad_dev():
    apps.vecadd(A, B, Cb, n, apps.GRAN_NONE, None, st)
    with torch.cuda.stream(st):
        R.copy_(Cb)

def ctl_only():
    pc.startall([snd, rcv], st); pc.pbuf_prepare_all([snd, rcv], st)
    pc.preadyall([snd], st)
    snd.wait_on_stream(st); rcv.wait_on_stream(st)

st2 = torch.cuda.Stream()
ev_a, ev_b = torch.cuda.Event(), torch.cuda.Event()

def epoch_all_serial():  # bench.py c1 epoch: one stream, both waits serialised
    pc.epoch_all([snd, rcv], pready=False, stream=st)
    apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK, sq, st)
    snd.wait_on_stream(st); rcv.wait_on_stream(st)

def epoch_all_waitall():  # bench.py c1 epoch: both waits in one pc_waitall_on_stream kernel
    pc.epoch_all([snd, rcv], pready=False, stream=st)
    apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK, sq, st)
    pc.waitall_on_stream([snd, rcv], st)

def epoch_all_2stream():  # the receiver's wait on its own stream, as on its own GPU
    pc.epoch_all([snd, rcv], pready=False, stream=st)
    ev_a.record(st)
    st2.wait_event(ev_a)
    rcv.wait_on_stream(st2)
    ev_b.record(st2)
    apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK, sq, st)
    snd.wait_on_stream(st)
    st.wait_event(ev_b)

for name, f in [("epoch_all + vecadd + 2 waits", epoch_all_serial),
                ("epoch_all + vecadd + waitall (bench c1)", epoch_all_waitall),
                ("epoch_all; recv wait on 2nd stream", epoch_all_2stream),
                ("full epoch (startall/prepare_all)", full_batched), ("full epoch (start/pbuf_prepare memops)", full_memops),
                ("vecadd only", vec_only), ("vecadd + copy (device only)", trad_dev),
                ("control only (startall, prepare_all, preadyall, waits)", ctl_only)]:
    print(f"{name:55s} {timeit(f):8.2f} us")
print("errors", snd.error(), rcv.error())
