"""GPU parity: the DIRECT schedule's PUSH variant (PC_ALGO_DIRECT_PUSH): every
rank stores its copy of chunk o of partition u into owner o's staging with
peer stores, the owner folds from local memory in rank order (reading R25)
and stores the final chunk into every rank's recvbuf.  Same bits as the PULL
variant, so the pin is oracle O6 (fp) and the plain definition (int32):
bit-exact on every rank, several epochs, ragged partitions (the staging slots
are 16-B aligned while the send buffer offsets need not be), in place,
producer-kernel Pready and host Pready, and the bench's control path."""
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
SEED = synth.BASE_SEED + 1500


@pytest.mark.parametrize("P", [2, 3, 5, 8])
@pytest.mark.parametrize("Np,L", [(1, 1), (3, 17), (7, 64), (2, 4099), (4, 30000)])
def test_push_fp32_bitexact(P, Np, L):
    xs = [np.stack([synth.normal_f32(SEED, r, e, Np * L) for r in range(P)]) for e in range(3)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_DIRECT_PUSH)
    for x, y in zip(xs, ys):
        ref, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT)
        for r in range(P):
            np.testing.assert_array_equal(y[r].view(np.uint32), ref[r].view(np.uint32))


@pytest.mark.parametrize("op", [pc.SUM, pc.MAX, pc.MIN])
def test_push_int32(op):
    P, Np, L = 8, 5, 1001
    xs = [np.stack([synth.int32_full(SEED + 1, r, e, Np * L) for r in range(P)]) for e in range(2)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_DIRECT_PUSH, op=op, producer=3, gran=apps.GRAN_WARP)
    for x, y in zip(xs, ys):
        ref = wrap_sum(x) if op == pc.SUM else oracle.allreduce_def_i32(x, op)
        for r in range(P):
            np.testing.assert_array_equal(y[r], ref)


@pytest.mark.parametrize("kind", ["f64", "bf16"])
def test_push_wide_narrow(kind):
    P, Np, L = 4, 3, 4099
    x = _inputs(kind, SEED + 2, P, Np * L)
    (y,) = run_allreduce(P, Np, L, [x], pc.ALGO_DIRECT_PUSH)
    ref, _, _ = oracle.pallreduce(x, Np, pc.ALGO_DIRECT)
    for r in range(P):
        np.testing.assert_array_equal(_bits(y[r]), _bits(ref[r]))


def test_push_inplace_producer():
    P, Np, L = 8, 6, 2050
    xs = [np.stack([synth.normal_f32(SEED + 3, r, e, Np * L) for r in range(P)]) for e in range(3)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_DIRECT_PUSH, inplace=True, producer=5)
    for x, y in zip(xs, ys):
        ref, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT)
        for r in range(P):
            np.testing.assert_array_equal(y[r].view(np.uint32), ref[r].view(np.uint32))


def test_push_epoch_all_bench_path():
    """pc_epoch_all(pready) epochs on one stream, the bench's step."""
    P, Np, L = 8, 16, 65536
    with comms(P) as cs:
        st = torch.cuda.Stream()
        x = np.stack([synth.normal_f32(SEED + 4, r, 0, Np * L) for r in range(P)])
        send = [torch.from_numpy(x[r]).cuda() for r in range(P)]
        recv = [torch.empty(Np * L, device="cuda") for _ in range(P)]
        reqs = [pc.pallreduce_init(send[r], recv[r], Np, L, pc.FLOAT32, pc.SUM, pc.ALGO_DIRECT_PUSH, cs[r])
                for r in range(P)]
        for q in reqs:
            q.start(st)
        first_prepare([[q] for q in reqs], [st] * P)
        assert reqs[0].info()["algo_name"] == "direct_push"
        for q in reqs:
            q.pready_range(0, Np - 1, st)
        for q in reqs:
            q.wait_on_stream(st)
        for _ in range(3):
            pc.epoch_all(reqs, pready=True, stream=st)
            for q in reqs:
                q.wait_on_stream(st)
        torch.cuda.synchronize()
        ref, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT)
        for r in range(P):
            assert reqs[r].error() == (0, 0)
            np.testing.assert_array_equal(recv[r].cpu().numpy().view(np.uint32), ref[r].view(np.uint32))
        for q in reqs:
            q.free()


def test_push_and_pull_do_not_match():
    """Every rank must choose the same variant: a PULL request and a PUSH
    request do not match (PC_ERR_MATCH at the first pbuf_prepare)."""
    with comms(2) as cs:
        st = torch.cuda.Stream()
        a = [torch.zeros(64, device="cuda") for _ in range(2)]
        reqs = [pc.pallreduce_init(a[0], a[0], 1, 64, pc.FLOAT32, pc.SUM, pc.ALGO_DIRECT, cs[0]),
                pc.pallreduce_init(a[1], a[1], 1, 64, pc.FLOAT32, pc.SUM, pc.ALGO_DIRECT_PUSH, cs[1])]
        for q in reqs:
            q.start(st)
        with pytest.raises(pc.PcError) as ex:
            pc.run_ranks([(lambda q=q: q.pbuf_prepare(st)) for q in reqs])
        assert ex.value.code == pc.ERR_MATCH
        for q in reqs:
            q.free()
