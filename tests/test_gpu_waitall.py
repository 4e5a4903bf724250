"""GPU parity: pc_waitall_on_stream (MPI_Waitall, stream-ordered; Listing 2's
MPI_Wait per request) — the p2p waits of several requests fused into one
kernel — against the CPU oracle O1 (byte-exact), 2 virtual ranks on one B200,
every epoch's control, producer and waits on ONE stream as bench.py's C1 leg
runs them."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_temucinslsga24_b200 as pc
import synth
from paper_conf_sc_temucinslsga24_b200 import apps

from gpu_util import comms, first_prepare

pytestmark = pytest.mark.gpu
SEED = synth.BASE_SEED
GRAN_ELEMS = {apps.GRAN_THREAD: 2, apps.GRAN_WARP: 64, apps.GRAN_BLOCK: 2048}  # 8 B / 256 B / 8 KiB


def _inputs(e, n, A, B):
    a = synth.uniform_f32(SEED, 0, 2 * e, n)
    b = synth.uniform_f32(SEED, 0, 2 * e + 1, n)
    A.copy_(torch.from_numpy(a))
    B.copy_(torch.from_numpy(b))
    return (a + b).astype(np.float32)


def _check(sent, got, partitions, agg):
    E = len(sent)
    send = np.stack(sent).view(np.uint8).reshape(E, -1)
    orders = np.stack([synth.permutation(SEED, 0, e, partitions) for e in range(E)])
    consumed, arrivals = oracle.p2p(send, partitions, agg, orders)
    assert (arrivals == 1).all()
    np.testing.assert_array_equal(np.stack(got).view(np.uint8).reshape(E, -1), consumed)


@pytest.mark.parametrize("n,gran,agg,copy", [
    (1 << 18, apps.GRAN_BLOCK, 16, pc.COPY_INLINE),    # C1
    (3 * 2048 * 5, apps.GRAN_BLOCK, 1, pc.COPY_INLINE),
    (1 << 15, apps.GRAN_WARP, 4, pc.COPY_INLINE),
    (1 << 14, apps.GRAN_WARP, 1, pc.COPY_LL),          # receive wait unpacks lines (multi-block range)
    (1 << 14, apps.GRAN_THREAD, 32, pc.COPY_LL),
    (3 * 2048 * 5, apps.GRAN_BLOCK, 2, pc.COPY_ENGINE),  # engine-moved send: pc_wait_on_stream's path
    (3 * 2048 * 5, apps.GRAN_BLOCK, 3, pc.COPY_HOST),
])
def test_waitall_p2p_epochs(n, gran, agg, copy):
    count = GRAN_ELEMS[gran]
    partitions = n // count
    E = 4
    with comms(2) as cs:
        st = torch.cuda.Stream()
        A, B = torch.empty(n, device="cuda"), torch.empty(n, device="cuda")
        Cb = torch.empty(n, device="cuda")
        R = torch.full((n,), -1.0, device="cuda")
        snd = pc.psend_init(Cb, partitions, count, pc.FLOAT32, 1, 21, cs[0])
        rcv = pc.precv_init(R, partitions, count, pc.FLOAT32, 0, 21, cs[1])
        sent, got = [], []
        for e in range(E):
            sent.append(_inputs(e, n, A, B))
            torch.cuda.synchronize()
            if e == 0:
                snd.start(st)
                rcv.start(st)
                first_prepare([[snd], [rcv]], [st, st])
                sq = snd.prequest_create(gran, agg, copy)
            else:
                pc.epoch_all([snd, rcv], pready=False, stream=st)
            apps.vecadd(A, B, Cb, n, gran, sq, st)
            pc.waitall_on_stream([snd, rcv], st)
            st.synchronize()
            assert snd.error() == (0, 0) and rcv.error() == (0, 0), (snd.error(), rcv.error())
            got.append(R.cpu().numpy().copy())
        snd.free()
        rcv.free()
    _check(sent, got, partitions, agg)


def test_waitall_graph_replayed_c1():
    """The C1 epoch (pc_epoch_all, producer with block Pready, waitall) captured
    once into a CUDA graph and replayed with new inputs: epochs advance on the
    device, every replay's bytes arrive intact."""
    n, gran, agg = 1 << 18, apps.GRAN_BLOCK, 16
    count = GRAN_ELEMS[gran]
    partitions = n // count
    with comms(2) as cs:
        st = torch.cuda.Stream()
        A, B = torch.empty(n, device="cuda"), torch.empty(n, device="cuda")
        Cb = torch.empty(n, device="cuda")
        R = torch.full((n,), -1.0, device="cuda")
        snd = pc.psend_init(Cb, partitions, count, pc.FLOAT32, 1, 22, cs[0])
        rcv = pc.precv_init(R, partitions, count, pc.FLOAT32, 0, 22, cs[1])
        sent, got = [_inputs(0, n, A, B)], []
        torch.cuda.synchronize()
        snd.start(st)
        rcv.start(st)
        first_prepare([[snd], [rcv]], [st, st])
        sq = snd.prequest_create(gran, agg, pc.COPY_INLINE)
        apps.vecadd(A, B, Cb, n, gran, sq, st)
        pc.waitall_on_stream([snd, rcv], st)
        st.synchronize()
        got.append(R.cpu().numpy().copy())
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            pc.epoch_all([snd, rcv], pready=False, stream=st)
            apps.vecadd(A, B, Cb, n, gran, sq, st)
            pc.waitall_on_stream([snd, rcv], st)
        for e in range(1, 5):
            sent.append(_inputs(e, n, A, B))
            R.fill_(-1.0)
            torch.cuda.synchronize()
            with torch.cuda.stream(st):
                g.replay()
            st.synchronize()
            assert snd.error() == (0, 0) and rcv.error() == (0, 0)
            got.append(R.cpu().numpy().copy())
        snd.free()
        rcv.free()
    _check(sent, got, partitions, agg)


def test_waitall_many_requests_grouped():
    """Three send/receive pairs (6 requests: two fused launches of <= 4) plus an
    inactive request in the list (skipped) — every pair's bytes arrive."""
    n, gran, agg = 3 * 2048 * 4, apps.GRAN_BLOCK, 2
    count = GRAN_ELEMS[gran]
    partitions = n // count
    with comms(2) as cs:
        st = torch.cuda.Stream()
        A, B = torch.empty(n, device="cuda"), torch.empty(n, device="cuda")
        idle_buf = torch.empty(n, device="cuda")
        idle = pc.psend_init(idle_buf, partitions, count, pc.FLOAT32, 1, 99, cs[0])  # never started
        Cs = [torch.empty(n, device="cuda") for _ in range(3)]
        Rs = [torch.full((n,), -1.0, device="cuda") for _ in range(3)]
        snds = [pc.psend_init(Cs[k], partitions, count, pc.FLOAT32, 1, 30 + k, cs[0]) for k in range(3)]
        rcvs = [pc.precv_init(Rs[k], partitions, count, pc.FLOAT32, 0, 30 + k, cs[1]) for k in range(3)]
        reqs = [x for k in range(3) for x in (snds[k], rcvs[k])]
        sent, got = [[] for _ in range(3)], [[] for _ in range(3)]
        for e in range(3):
            ab = _inputs(e, n, A, B)
            torch.cuda.synchronize()
            if e == 0:
                for q in reqs:
                    q.start(st)
                first_prepare([snds, rcvs], [st, st])
                sqs = [s.prequest_create(gran, agg, pc.COPY_INLINE) for s in snds]
            else:
                pc.epoch_all(reqs, pready=False, stream=st)
            for k in range(3):
                apps.vecadd(A, B, Cs[k], n, gran, sqs[k], st)
            pc.waitall_on_stream(reqs + [idle], st)
            st.synchronize()
            for k in range(3):
                assert snds[k].error() == (0, 0) and rcvs[k].error() == (0, 0)
                sent[k].append(ab)
                got[k].append(Rs[k].cpu().numpy().copy())
        for q in reqs + [idle]:
            q.free()
    for k in range(3):
        _check(sent[k], got[k], partitions, agg)
