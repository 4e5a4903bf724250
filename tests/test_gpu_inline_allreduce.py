"""GPU parity: the INLINE partitioned allreduce (reading R33 — P:L277 §VI-B,
"the Pready could trigger computation"; the paper's Kernel Copy applied to
the collective).  No engine: the Pready that completes partition u on the
last of the P ranks folds u over every rank's send buffer in rank order
(R25) and stores it into every rank's recvbuf.  The bits are the DIRECT
schedule's, so the pin is oracle O6 (oracle.pallreduce(..., DIRECT)) for
floating point and the plain definition for int32 — bit-exact, on every rank,
over several epochs, for block / warp / thread Pready from a producer kernel,
for the host Pready bindings, in place, with ragged (unaligned) partitions."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_temucinslsga24_b200 as pc
import synth
from paper_conf_sc_temucinslsga24_b200 import apps

from gpu_util import comms, first_prepare
from test_gpu_allreduce import _bits, _inputs, run_allreduce, wrap_sum

pytestmark = pytest.mark.gpu

SEED = synth.BASE_SEED + 900


def _fp_ref(x, Np):
    ref, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT)
    return ref


@pytest.mark.parametrize("P", [1, 2, 3, 5, 8])
@pytest.mark.parametrize("Np,L", [(1, 1), (3, 17), (7, 64), (4, 1001), (2, 30001)])
@pytest.mark.parametrize("gran", [apps.GRAN_BLOCK, apps.GRAN_WARP, apps.GRAN_THREAD])
def test_inline_fp32_producer(P, Np, L, gran):
    if gran == apps.GRAN_THREAD and L > 2000:
        pytest.skip("thread-granularity fold of a 30k partition by one thread: covered at small L")
    xs = [np.stack([synth.normal_f32(SEED, r, e, Np * L) for r in range(P)]) for e in range(3)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_DIRECT, producer=3 if Np % 3 else 1, gran=gran, copy=pc.COPY_INLINE)
    for x, y in zip(xs, ys):
        ref = _fp_ref(x, Np)
        for r in range(P):
            np.testing.assert_array_equal(y[r].view(np.uint32), ref[r].view(np.uint32))


@pytest.mark.parametrize("op", [pc.SUM, pc.MAX, pc.MIN])
@pytest.mark.parametrize("P", [2, 4, 8])
def test_inline_int32(op, P):
    Np, L = 5, 777
    xs = [np.stack([synth.int32_full(SEED + 1, r, e, Np * L) for r in range(P)]) for e in range(2)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_DIRECT, op=op, producer=1, copy=pc.COPY_INLINE)
    for x, y in zip(xs, ys):
        ref = wrap_sum(x) if op == pc.SUM else oracle.allreduce_def_i32(x, op)
        for r in range(P):
            np.testing.assert_array_equal(y[r], ref)


@pytest.mark.parametrize("kind", ["f64", "bf16"])
@pytest.mark.parametrize("Np,L", [(3, 17), (2, 4099)])
def test_inline_fp64_bf16(kind, Np, L):
    P = 4
    xs = [_inputs(kind, SEED + 2, P, Np * L, e) for e in range(2)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_DIRECT, producer=1, copy=pc.COPY_INLINE)
    for x, y in zip(xs, ys):
        ref = _fp_ref(x, Np)
        for r in range(P):
            np.testing.assert_array_equal(_bits(y[r]), _bits(ref[r]))


@pytest.mark.parametrize("P", [3, 8])
def test_inline_inplace_and_host_pready(P):
    """In place (sendbuf == recvbuf) from the producer, then the host Pready
    bindings (pc_pready_range: the library's warp kernel folds)."""
    Np, L = 6, 515
    xs = [np.stack([synth.normal_f32(SEED + 4, r, e, Np * L) for r in range(P)]) for e in range(3)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_DIRECT, inplace=True, producer=5, copy=pc.COPY_INLINE)
    for x, y in zip(xs, ys):
        ref = _fp_ref(x, Np)
        for r in range(P):
            np.testing.assert_array_equal(y[r].view(np.uint32), ref[r].view(np.uint32))


def test_inline_host_pready_range():
    P, Np, L = 4, 5, 2049
    with comms(P) as cs:
        st = [torch.cuda.Stream() for _ in range(P)]
        x = np.stack([synth.normal_f32(SEED + 5, r, 0, Np * L) for r in range(P)])
        send = [torch.from_numpy(x[r]).cuda() for r in range(P)]
        recv = [torch.zeros(Np * L, device="cuda") for _ in range(P)]
        reqs = [pc.pallreduce_init(send[r], recv[r], Np, L, pc.FLOAT32, pc.SUM, pc.ALGO_DIRECT, cs[r])
                for r in range(P)]
        for e in range(2):
            for r in range(P):
                reqs[r].start(st[r])
            if e == 0:
                first_prepare([[q] for q in reqs], st)
                for q in reqs:
                    q.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
            else:
                for r in range(P):
                    reqs[r].pbuf_prepare(st[r])
            for r in range(P):
                reqs[r].pready_range(0, 1, st[r])
                reqs[r].pready_range(2, Np - 1, st[r])
            for r in range(P):
                reqs[r].wait_on_stream(st[r])
            torch.cuda.synchronize()
            ref = _fp_ref(x, Np)
            for r in range(P):
                assert reqs[r].error() == (0, 0)
                np.testing.assert_array_equal(recv[r].cpu().numpy().view(np.uint32), ref[r].view(np.uint32))
                f = reqs[r].parrived(Np - 1)
                assert f == 1
        with pytest.raises(pc.PcError) as ex:  # pc_epoch_all's Pready only marks ready: it cannot fold
            pc.epoch_all(reqs, pready=True, stream=st[0])
        assert ex.value.code == pc.ERR_ARG
        for q in reqs:
            q.free()


def test_inline_needs_direct():
    with comms(2) as cs:
        st = torch.cuda.Stream()
        a = [torch.zeros(64, device="cuda") for _ in range(2)]
        reqs = [pc.pallreduce_init(a[r], a[r], 1, 64, pc.FLOAT32, pc.SUM, pc.ALGO_RING, cs[r]) for r in range(2)]
        for q in reqs:
            q.start(st)
        first_prepare([[q] for q in reqs], [st, st])
        for q in reqs:
            with pytest.raises(pc.PcError) as ex:
                q.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
            assert ex.value.code == pc.ERR_UNSUPPORTED
            q.pready_range(0, 0, st)
        for q in reqs:
            q.wait_on_stream(st)
        torch.cuda.synchronize()
        for q in reqs:
            q.free()


@pytest.mark.parametrize("P", [2, 4, 8])
def test_inline_parrived_inside_the_producer(P):
    """The a6 probe with the INLINE allreduce: partition 0 completes (folded by
    the last rank's Pready) while every rank's producer waits for it inside
    the kernel — there is no engine at all."""
    from test_gpu_overlap import _run
    for stamps in _run(P, pc.ALGO_DIRECT, overlap=True, copy=pc.COPY_INLINE):
        assert (stamps[:, 2] > 0).all() and (stamps[:, 2] < stamps[:, 3]).all()
