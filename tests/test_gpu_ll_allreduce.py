"""GPU parity: the one-shot LL allreduce (PC_ALGO_LL, small messages): every
rank stores each ready partition as 16-B LL lines into every peer's line
area (no fence, no flag) and folds all P contributions itself in rank order
(reading R25) — oracle O6's bits for floating point, the plain definition for
int32; bit-exact on every rank over 6 epochs (both line parities, three times
each), ragged partitions (a partial last 8-B word), in place, producer-kernel
and host Pready, the pc_epoch_all path and CUDA-graph replay."""
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
SEED = synth.BASE_SEED + 1700


@pytest.mark.parametrize("P", [2, 3, 5, 8])
@pytest.mark.parametrize("Np,L", [(1, 1), (3, 17), (7, 64), (2, 999), (16, 256)])
def test_ll_fp32_bitexact(P, Np, L):
    xs = [np.stack([synth.normal_f32(SEED, r, e, Np * L) for r in range(P)]) for e in range(6)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_LL, producer=3 if Np % 3 else 1)
    for x, y in zip(xs, ys):
        ref, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT)
        for r in range(P):
            np.testing.assert_array_equal(y[r].view(np.uint32), ref[r].view(np.uint32))


@pytest.mark.parametrize("op", [pc.SUM, pc.MAX, pc.MIN])
def test_ll_int32(op):
    P, Np, L = 8, 4, 333
    xs = [np.stack([synth.int32_full(SEED + 1, r, e, Np * L) for r in range(P)]) for e in range(4)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_LL, op=op)
    for x, y in zip(xs, ys):
        ref = wrap_sum(x) if op == pc.SUM else oracle.allreduce_def_i32(x, op)
        for r in range(P):
            np.testing.assert_array_equal(y[r], ref)


@pytest.mark.parametrize("kind", ["f64", "bf16"])
@pytest.mark.parametrize("Np,L", [(3, 17), (2, 1001)])
def test_ll_fp64_bf16(kind, Np, L):
    P = 4
    xs = [_inputs(kind, SEED + 2, P, Np * L, e) for e in range(4)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_LL)
    for x, y in zip(xs, ys):
        ref, _, _ = oracle.pallreduce(x, Np, pc.ALGO_DIRECT)
        for r in range(P):
            np.testing.assert_array_equal(_bits(y[r]), _bits(ref[r]))


def test_ll_inplace_warp_producer():
    P, Np, L = 8, 6, 515
    xs = [np.stack([synth.normal_f32(SEED + 3, r, e, Np * L) for r in range(P)]) for e in range(5)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_LL, inplace=True, producer=5, gran=apps.GRAN_WARP)
    for x, y in zip(xs, ys):
        ref, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT)
        for r in range(P):
            np.testing.assert_array_equal(y[r].view(np.uint32), ref[r].view(np.uint32))


@pytest.mark.parametrize("graph", [False, True])
def test_ll_epoch_all_and_graph_replay(graph):
    """The bench's control path (pc_epoch_all with Pready) for 7 epochs, eager
    or replayed from one captured epoch; AUTO picks LL at this size (64 KiB)."""
    P, Np, L = 8, 4, 4096  # 64 KiB per rank: AUTO picks LL on one GPU
    with comms(P) as cs:
        st = torch.cuda.Stream()
        x = np.stack([synth.normal_f32(SEED + 4, r, 0, Np * L) for r in range(P)])
        send = [torch.from_numpy(x[r]).cuda() for r in range(P)]
        recv = [torch.zeros(Np * L, device="cuda") for _ in range(P)]
        reqs = [pc.pallreduce_init(send[r], recv[r], Np, L, pc.FLOAT32, pc.SUM, pc.ALGO_AUTO, cs[r])
                for r in range(P)]
        for q in reqs:
            q.start(st)
        first_prepare([[q] for q in reqs], [st] * P)
        assert reqs[0].info()["algo_name"] == "ll"
        pc.preadyall(reqs, st)
        for q in reqs:
            q.wait_on_stream(st)

        def epoch():
            pc.epoch_all(reqs, pready=True, stream=st)
            for q in reqs:
                q.wait_on_stream(st)

        ref, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT)
        gr = None
        if graph:
            torch.cuda.synchronize()
            gr = torch.cuda.CUDAGraph()
            with torch.cuda.graph(gr, stream=st):
                epoch()
        for _ in range(7):
            for r in range(P):
                recv[r].zero_()
            torch.cuda.synchronize()
            if graph:
                with torch.cuda.stream(st):
                    gr.replay()
            else:
                epoch()
            torch.cuda.synchronize()
            for r in range(P):
                assert reqs[r].error() == (0, 0)
                np.testing.assert_array_equal(recv[r].cpu().numpy().view(np.uint32), ref[r].view(np.uint32))
        for q in reqs:
            q.free()
