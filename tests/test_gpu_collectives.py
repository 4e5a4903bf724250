"""GPU parity: partitioned reduce-scatter / allgather / broadcast (SURVEY
NEXT-3) through the C ABI vs the CPU oracle's plain definitions O8 / O9 / O10,
with P virtual ranks on one B200.  Bar: bit-exact for every dtype (the
reduce-scatter fold is the rank-order association of reading R25, which O8
writes out), over several epochs, with host Pready and with Pready from a
producer kernel, and device Parrived (pc_wait_arrived) on every receive
partition."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_temucinslsga24_b200 as pc
import synth
from paper_conf_sc_temucinslsga24_b200 import apps

from gpu_util import comms, first_prepare
from test_gpu_allreduce import DTYPES, _to_numpy, _to_torch

pytestmark = pytest.mark.gpu
SEED = synth.BASE_SEED


def run_coll(kind, P, Np, count, xs_epochs, op=pc.SUM, root=0, producer=None):
    """xs_epochs: list over epochs of (P, send elements) host arrays.
    Returns a list over epochs of (P, recv elements) results."""
    dt, tdtype = DTYPES[xs_epochs[0].dtype.type]
    es = pc.ESIZE[dt]
    ns = {"rs": Np * P * count, "ag": Np * count, "bc": Np * count}[kind]
    nr = {"rs": Np * count, "ag": P * Np * count, "bc": Np * count}[kind]
    part_send = ns // Np  # elements per send partition
    outs = []
    with comms(P) as cs:
        streams = [torch.cuda.Stream() for _ in range(P)]
        send = [torch.zeros(max(ns, 8), dtype=tdtype, device="cuda") for _ in range(P)]
        recv = send if kind == "bc" else [torch.full((max(nr, 8),), 0, dtype=tdtype, device="cuda") for _ in range(P)]
        src = [torch.zeros(max(ns, 8), dtype=tdtype, device="cuda") for _ in range(P)]
        out = [torch.zeros(max(nr, 8) * es, dtype=torch.uint8, device="cuda") for _ in range(P)]
        status = torch.zeros(1, dtype=torch.int32, device="cuda")
        if kind == "rs":
            reqs = [pc.preduce_scatter_init(send[r], recv[r], Np, count, dt, op, cs[r]) for r in range(P)]
        elif kind == "ag":
            reqs = [pc.pallgather_init(send[r], recv[r], Np, count, dt, cs[r]) for r in range(P)]
        else:
            reqs = [pc.pbcast_init(send[r], Np, count, dt, root, cs[r]) for r in range(P)]
        preqs = None
        for e, xs in enumerate(xs_epochs):
            for r in range(P):
                (src if producer else send)[r][:ns].copy_(_to_torch(xs[r]).to("cuda"))
            torch.cuda.synchronize()
            for r in range(P):
                reqs[r].start(streams[r])
            if e == 0:
                first_prepare([[reqs[r]] for r in range(P)], streams)
                preqs = [reqs[r].prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_ENGINE) for r in range(P)]
            else:
                for r in range(P):
                    reqs[r].pbuf_prepare(streams[r])
            for r in range(P):
                if kind == "bc" and r != root:
                    continue
                if producer:
                    apps.produce(send[r], src[r], Np, part_send * es, apps.GRAN_BLOCK, preqs[r],
                                 order_stride=producer, stream=streams[r])
                else:
                    reqs[r].pready_range(0, Np - 1, streams[r])
            for r in range(P):
                reqs[r].wait_on_stream(streams[r])
            # device Parrived of every receive partition, after completion
            nparts = P * Np if kind == "ag" else Np
            for r in range(P):
                apps.check_recv(preqs[r], recv[r], out[r], nparts, count * es, status, blocks=16, stream=streams[r])
            torch.cuda.synchronize()
            assert int(status.item()) == 0
            for r in range(P):
                code, part = reqs[r].error()
                assert code == 0, f"rank {r} device error {code} at {part}"
            res = np.stack([_to_numpy(recv[r][:nr]) for r in range(P)])
            for r in range(P):
                np.testing.assert_array_equal(out[r][:nr * es].cpu().numpy(), res[r].view(np.uint8))
            outs.append(res)
        for q in reqs:
            q.free()
    return outs


def gen(dtype, P, n, epoch, seed_off=0):
    if dtype == np.int32:
        return np.stack([synth.int32_full(SEED + seed_off, r, epoch, n) for r in range(P)])
    x = np.stack([synth.normal_f32(SEED + seed_off, r, epoch, n) for r in range(P)])
    if dtype == np.uint16:
        return np.stack([oracle.bf16_round(v.astype(np.float64)) for v in x])
    return x.astype(dtype)


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("Np,count", [(1, 1), (3, 17), (7, 64), (2, 1000)])
@pytest.mark.parametrize("dtype", [np.int32, np.float32])
def test_reduce_scatter_sum(P, Np, count, dtype):
    xs = [gen(dtype, P, Np * P * count, e) for e in range(2)]
    ys = run_coll("rs", P, Np, count, xs)
    for x, y in zip(xs, ys):
        np.testing.assert_array_equal(y.view(np.uint8), oracle.reduce_scatter_def(x, Np).view(np.uint8))


@pytest.mark.parametrize("dtype", [np.float64, np.uint16, np.int32])
@pytest.mark.parametrize("op", [pc.SUM, pc.MAX, pc.MIN])
def test_reduce_scatter_dtypes_ops(dtype, op):
    P, Np, count = 4, 3, 40
    xs = [gen(dtype, P, Np * P * count, 0, 5)]
    (y,) = run_coll("rs", P, Np, count, xs, op=op)
    np.testing.assert_array_equal(y.view(np.uint8), oracle.reduce_scatter_def(xs[0], Np, op).view(np.uint8))


def test_reduce_scatter_producer_large():
    """Pready from a producer kernel (permuted order), slices of 8 KiB, 8 ranks."""
    P, Np, count = 8, 5, 9000
    xs = [gen(np.float32, P, Np * P * count, e, 9) for e in range(2)]
    ys = run_coll("rs", P, Np, count, xs, producer=3)
    for x, y in zip(xs, ys):
        np.testing.assert_array_equal(y, oracle.reduce_scatter_def(x, Np))


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("Np,count", [(1, 1), (3, 17), (7, 64), (2, 3000)])
def test_allgather(P, Np, count):
    xs = [gen(np.float32, P, Np * count, e, 2) for e in range(3)]
    ys = run_coll("ag", P, Np, count, xs)
    for x, y in zip(xs, ys):
        np.testing.assert_array_equal(y, oracle.allgather_def(x))


def test_allgather_producer_bf16():
    P, Np, count = 8, 6, 5000
    xs = [gen(np.uint16, P, Np * count, e, 4) for e in range(2)]
    ys = run_coll("ag", P, Np, count, xs, producer=5)
    for x, y in zip(xs, ys):
        np.testing.assert_array_equal(y, oracle.allgather_def(x))


@pytest.mark.parametrize("P,root", [(1, 0), (2, 1), (3, 0), (4, 2), (8, 7)])
@pytest.mark.parametrize("Np,count", [(1, 1), (5, 33), (2, 4000)])
def test_bcast(P, root, Np, count):
    xs = [gen(np.int32, P, Np * count, e, 3) for e in range(3)]
    ys = run_coll("bc", P, Np, count, xs, root=root)
    for x, y in zip(xs, ys):
        np.testing.assert_array_equal(y, oracle.bcast_def(x, root))
