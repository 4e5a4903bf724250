"""GPU parity: partitioned allreduce (ring = Alg 1, RD) through the C ABI vs
the CPU oracle, with P virtual ranks on one B200 (tests/gpu_util.py).

Bar: int32 bit-exact against the oracle's plain
definition; fp32 bit-exact against the schedule-faithful oracle (O3 ring fold /
O4 RD tree) AND |y - y64| <= 1e-5 * sum|x| against fp64 (reading R16).
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_temucinslsga24_b200 as pc
import synth
from paper_conf_sc_temucinslsga24_b200 import apps

from gpu_util import comms, first_prepare, to_dev

pytestmark = pytest.mark.gpu

SEED = synth.BASE_SEED


# host arrays: bf16 travels as uint16 bit patterns (oracle reading R27)
DTYPES = {np.int32: (pc.INT32, torch.int32), np.float32: (pc.FLOAT32, torch.float32),
          np.float64: (pc.FLOAT64, torch.float64), np.uint16: (pc.BF16, torch.bfloat16)}


def _to_torch(a):
    if a.dtype == np.uint16:
        return torch.from_numpy(a.view(np.int16).copy()).view(torch.bfloat16)
    return torch.from_numpy(np.ascontiguousarray(a))


def _to_numpy(t):
    if t.dtype == torch.bfloat16:
        return t.view(torch.int16).cpu().numpy().view(np.uint16)
    return t.cpu().numpy()


def run_allreduce(P, Np, L, xs_epochs, algo, op=pc.SUM, inplace=False, producer=None, gran=apps.GRAN_BLOCK,
                  copy=pc.COPY_ENGINE):
    """xs_epochs: list over epochs of (P, Np*L) host arrays.  Returns a list over
    epochs of (P, Np*L) results (each rank's recvbuf after its wait).  copy:
    the prequest's mode (COPY_INLINE on DIRECT: the completing Pready folds,
    reading R33)."""
    dt, tdtype = DTYPES[xs_epochs[0].dtype.type]
    es = pc.ESIZE[dt]
    n = Np * L
    outs = []
    with comms(P) as cs:
        streams = [torch.cuda.Stream() for _ in range(P)]
        nd = max(n, 4)
        send = [torch.zeros(nd, dtype=tdtype, device="cuda") for _ in range(P)]
        recv = send if inplace else [torch.zeros(nd, dtype=tdtype, device="cuda") for _ in range(P)]
        src = [torch.zeros(nd, dtype=tdtype, device="cuda") for _ in range(P)]
        reqs = [pc.pallreduce_init(send[r], recv[r], Np, L, dt, op, algo, cs[r]) for r in range(P)]
        preqs = None
        for e, xs in enumerate(xs_epochs):
            for r in range(P):
                with torch.cuda.stream(streams[r]):
                    (src if producer else send)[r][:n].copy_(_to_torch(xs[r]).to("cuda", non_blocking=False))
            torch.cuda.synchronize()
            for r in range(P):
                reqs[r].start(streams[r])
            if e == 0:
                first_prepare([[reqs[r]] for r in range(P)], streams)
                preqs = [reqs[r].prequest_create(pc.GRAN_BLOCK, 1, copy) for r in range(P)]
            else:
                for r in range(P):
                    reqs[r].pbuf_prepare(streams[r])
            for r in range(P):
                if producer:
                    apps.produce(send[r], src[r], Np, L * es, gran, preqs[r], order_stride=producer,
                                 stream=streams[r])
                else:
                    reqs[r].pready_range(0, Np - 1, streams[r])
            for r in range(P):
                reqs[r].wait_on_stream(streams[r])
            torch.cuda.synchronize()
            for r in range(P):
                code, part = reqs[r].error()
                assert code == 0, f"rank {r} device error {code} at {part}"
            outs.append(np.stack([_to_numpy(recv[r][:n]) for r in range(P)]))
        for q in reqs:
            q.free()
    return outs


def wrap_sum(x):
    s = x.astype(np.int64).sum(axis=0)
    return ((s + 2**31) % 2**32 - 2**31).astype(np.int32)


@pytest.mark.parametrize("P", [1, 2, 3, 4, 5, 8])
@pytest.mark.parametrize("Np,L", [(1, 1), (3, 17), (7, 64), (8, 5), (2, 1000), (1, 4)])
def test_ring_int32_sum(P, Np, L):
    x = np.stack([synth.int32_full(SEED, r, 0, Np * L) for r in range(P)])
    (y,) = run_allreduce(P, Np, L, [x], pc.ALGO_RING)
    ref = oracle.allreduce_def_i32(x)
    for r in range(P):
        np.testing.assert_array_equal(y[r], ref)


@pytest.mark.parametrize("P", [1, 2, 4, 8])
@pytest.mark.parametrize("Np,L", [(1, 1), (3, 17), (8, 5), (2, 1000)])
def test_rd_int32_sum(P, Np, L):
    x = np.stack([synth.int32_full(SEED + 1, r, 0, Np * L) for r in range(P)])
    (y,) = run_allreduce(P, Np, L, [x], pc.ALGO_RD)
    ref = oracle.allreduce_def_i32(x)
    for r in range(P):
        np.testing.assert_array_equal(y[r], ref)


@pytest.mark.parametrize("op", [pc.MAX, pc.MIN])
@pytest.mark.parametrize("algo,P", [(pc.ALGO_RING, 3), (pc.ALGO_RING, 8), (pc.ALGO_RD, 4)])
def test_int32_maxmin(op, algo, P):
    Np, L = 4, 333
    x = np.stack([synth.int32_full(SEED + 2, r, 0, Np * L) for r in range(P)])
    (y,) = run_allreduce(P, Np, L, [x], algo, op=op)
    ref = oracle.allreduce_def_i32(x, op)
    for r in range(P):
        np.testing.assert_array_equal(y[r], ref)


def check_fp32(x, y, algo, Np, L):
    P = x.shape[0]
    y64, sabs = oracle.allreduce_def_f64(x)
    if algo == pc.ALGO_RING:
        lit, _, _ = oracle.pallreduce(x, Np, oracle.RING) if x.size <= 4_000_000 else (None, 0, 0)
        cf = oracle.ring_fold_f32(x, oracle.chunk_ids(L, P, Np))
    elif algo == pc.ALGO_DIRECT:  # R25: left fold over ranks 0..P-1
        lit, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT) if x.size <= 4_000_000 else (None, 0, 0)
        cf = oracle.ring_fold_f32(x, np.zeros(x.shape[1], np.int32))
    else:
        lit, _, _ = oracle.pallreduce(x, Np, oracle.RD) if x.size <= 4_000_000 else (None, 0, 0)
        cf = oracle.rd_tree_f32(x)
    for r in range(P):
        np.testing.assert_array_equal(y[r].view(np.uint32), cf.view(np.uint32))
        if lit is not None:
            np.testing.assert_array_equal(y[r].view(np.uint32), lit[r].view(np.uint32))
    assert (np.abs(y[0].astype(np.float64) - y64) <= 1e-5 * sabs).all()


@pytest.mark.parametrize("P", [2, 3, 5, 8])
@pytest.mark.parametrize("Np,L", [(1, 1), (3, 17), (7, 64), (2, 4099)])
def test_ring_fp32_bitexact(P, Np, L):
    x = np.stack([synth.normal_f32(SEED + 3, r, 0, Np * L) for r in range(P)])
    (y,) = run_allreduce(P, Np, L, [x], pc.ALGO_RING)
    check_fp32(x, y, pc.ALGO_RING, Np, L)


@pytest.mark.parametrize("P", [2, 4, 8])
@pytest.mark.parametrize("Np,L", [(1, 1), (3, 17), (2, 4099)])
def test_rd_fp32_bitexact(P, Np, L):
    x = np.stack([synth.normal_f32(SEED + 4, r, 0, Np * L) for r in range(P)])
    (y,) = run_allreduce(P, Np, L, [x], pc.ALGO_RD)
    check_fp32(x, y, pc.ALGO_RD, Np, L)


@pytest.mark.parametrize("algo,P", [(pc.ALGO_RING, 4), (pc.ALGO_RING, 8), (pc.ALGO_RD, 8)])
def test_multi_slice_ragged_epochs_inplace(algo, P):
    """Sizes spanning many slices per chunk with a ragged tail (L % 4 != 0 so
    partitions are not 16-B aligned), 3 epochs with epoch-tagged inputs,
    in place (sendbuf == recvbuf, reading R22), device producer with a
    permuted Pready order."""
    Np, L = 3, 300_001
    xs = [np.stack([synth.normal_f32(SEED + 5, r, e, Np * L) for r in range(P)]) for e in range(3)]
    ys = run_allreduce(P, Np, L, xs, algo, inplace=True, producer=2)
    for x, y in zip(xs, ys):
        check_fp32(x, y, algo, Np, L)


@pytest.mark.parametrize("gran", [apps.GRAN_THREAD, apps.GRAN_WARP, apps.GRAN_BLOCK])
def test_device_producer_granularities(gran):
    P, Np, L = 4, 16, 4096
    x = np.stack([synth.int32_full(SEED + 6, r, 0, Np * L) for r in range(P)])
    (y,) = run_allreduce(P, Np, L, [x], pc.ALGO_RING, producer=5, gran=gran)
    for r in range(P):
        np.testing.assert_array_equal(y[r], wrap_sum(x))


def test_many_epochs_int():
    """50 back-to-back epochs with epoch-tagged inputs: no stale or early reads."""
    P, Np, L = 4, 5, 777
    xs = [np.stack([synth.int32_full(SEED + 7, r, e, Np * L) for r in range(P)]) for e in range(50)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_RING)
    for x, y in zip(xs, ys):
        for r in range(P):
            np.testing.assert_array_equal(y[r], wrap_sum(x))


def test_1000_epochs_direct_tagged():
    """>= 1000 back-to-back epochs with epoch-tagged inputs on
    the bench's schedule (DIRECT, 8 ranks): no stale or early reads."""
    P, Np, L = 8, 3, 1000
    xs = [np.stack([synth.int32_full(SEED + 8, r, e, Np * L) for r in range(P)]) for e in range(1000)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_DIRECT)
    for x, y in zip(xs, ys):
        for r in range(P):
            np.testing.assert_array_equal(y[r], wrap_sum(x))


def test_nan_propagates():
    P, Np, L = 4, 2, 64
    x = np.stack([synth.normal_f32(SEED + 8, r, 0, Np * L) for r in range(P)])
    x[1, 7] = np.nan
    for algo in (pc.ALGO_RING, pc.ALGO_RD):
        (y,) = run_allreduce(P, Np, L, [x], algo)
        assert np.isnan(y[:, 7]).all() and not np.isnan(np.delete(y, 7, axis=1)).any()


def test_integer_valued_fp32_exact():
    P, Np, L = 8, 4, 10_000
    x = np.stack([synth.int_valued_f32(SEED + 9, r, 0, Np * L, (1 << 24) // P) for r in range(P)])
    for algo in (pc.ALGO_RING, pc.ALGO_RD):
        (y,) = run_allreduce(P, Np, L, [x], algo)
        ref = x.astype(np.int64).sum(0).astype(np.float32)
        for r in range(P):
            np.testing.assert_array_equal(y[r], ref)


def test_cuda_graph_replay_of_epochs():
    """Start -> Pbuf_prepare -> Pready -> Wait of every rank captured once into
    a CUDA graph and replayed: the epoch lives on the device (pc_start bumps it
    there), so each replay is a new, correct epoch."""
    P, Np, L = 4, 3, 5000
    with comms(P) as cs:
        st = torch.cuda.Stream()
        send = [torch.zeros(Np * L, device="cuda") for _ in range(P)]
        recv = [torch.zeros(Np * L, device="cuda") for _ in range(P)]
        reqs = [pc.pallreduce_init(send[r], recv[r], Np, L, pc.FLOAT32, pc.SUM, pc.ALGO_RING, cs[r]) for r in range(P)]

        def step(first=False):
            if first:
                for q in reqs:
                    q.start(st)
                first_prepare([[q] for q in reqs], [st] * P)
            else:  # MPI_Startall analogue + batched ready-to-receive
                pc.startall(reqs, st)
                pc.pbuf_prepare_all(reqs, st)
            if first:
                for q in reqs:
                    q.pready_range(0, Np - 1, st)
            else:
                pc.preadyall(reqs, st)
            for q in reqs:
                q.wait_on_stream(st)

        step(first=True)  # eager first epoch: exchange, mapping
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            step()
        for e in range(6):
            x = np.stack([synth.normal_f32(SEED + 20, r, e, Np * L) for r in range(P)])
            for r in range(P):
                send[r].copy_(torch.from_numpy(x[r]))
            torch.cuda.synchronize()
            g.replay()
            torch.cuda.synchronize()
            ref = oracle.ring_fold_f32(x, oracle.chunk_ids(L, P, Np))
            for r in range(P):
                np.testing.assert_array_equal(recv[r].cpu().numpy().view(np.uint32), ref.view(np.uint32))
        # 1 eager + 1 captured (not executed at capture) + 6 replays
        assert int(reqs[0].words("epoch", 0, 1)[0]) == 7
        for q in reqs:
            assert q.error() == (0, 0)
            q.free()


# ------------------------------------------------------------------ DIRECT
@pytest.mark.parametrize("P", [1, 2, 3, 5, 8])
@pytest.mark.parametrize("Np,L", [(1, 1), (3, 17), (7, 64), (2, 1000)])
def test_direct_int32_sum(P, Np, L):
    x = np.stack([synth.int32_full(SEED + 30, r, 0, Np * L) for r in range(P)])
    (y,) = run_allreduce(P, Np, L, [x], pc.ALGO_DIRECT)
    for r in range(P):
        np.testing.assert_array_equal(y[r], wrap_sum(x))


@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("Np,L", [(1, 1), (3, 17), (2, 4099)])
def test_direct_fp32_bitexact(P, Np, L):
    x = np.stack([synth.normal_f32(SEED + 31, r, 0, Np * L) for r in range(P)])
    (y,) = run_allreduce(P, Np, L, [x], pc.ALGO_DIRECT)
    check_fp32(x, y, pc.ALGO_DIRECT, Np, L)


def test_direct_ragged_inplace_epochs_producer():
    P, Np, L = 8, 3, 300_001
    xs = [np.stack([synth.normal_f32(SEED + 32, r, e, Np * L) for r in range(P)]) for e in range(3)]
    ys = run_allreduce(P, Np, L, xs, pc.ALGO_DIRECT, inplace=True, producer=2)
    for x, y in zip(xs, ys):
        check_fp32(x, y, pc.ALGO_DIRECT, Np, L)


@pytest.mark.parametrize("op", [pc.MAX, pc.MIN])
def test_direct_maxmin(op):
    P, Np, L = 5, 4, 333
    x = np.stack([synth.int32_full(SEED + 33, r, 0, Np * L) for r in range(P)])
    (y,) = run_allreduce(P, Np, L, [x], pc.ALGO_DIRECT, op=op)
    for r in range(P):
        np.testing.assert_array_equal(y[r], oracle.allreduce_def_i32(x, op))


# ------------------------------------------------------------ fp64 and bf16 (R27)
def _inputs(kind, seed, P, n, e=0):
    gen = synth.normal_f64 if kind == "f64" else synth.bf16_bits
    return np.stack([gen(seed, r, e, n) for r in range(P)])


def _bits(a):
    return a.view(np.uint64) if a.dtype == np.float64 else a


@pytest.mark.parametrize("kind", ["f64", "bf16"])
@pytest.mark.parametrize("algo,Ps", [(pc.ALGO_RING, [2, 3, 8]), (pc.ALGO_RD, [2, 4, 8]),
                                     (pc.ALGO_DIRECT, [3, 8])])
@pytest.mark.parametrize("Np,L", [(1, 1), (3, 17), (7, 64), (2, 4099)])
def test_wide_and_narrow_dtypes_bitexact(kind, algo, Ps, Np, L):
    """fp64 / bf16 allreduce bit-exact against the schedule-faithful oracle,
    including ragged L (partitions not 16-B aligned)."""
    for P in Ps:
        x = _inputs(kind, SEED + 41, P, Np * L)
        (y,) = run_allreduce(P, Np, L, [x], algo)
        ref, _, _ = oracle.pallreduce(x, Np, algo)
        for r in range(P):
            np.testing.assert_array_equal(_bits(y[r]), _bits(ref[r]))


@pytest.mark.parametrize("kind", ["f64", "bf16"])
@pytest.mark.parametrize("algo,P", [(pc.ALGO_RING, 8), (pc.ALGO_RD, 4), (pc.ALGO_DIRECT, 8)])
def test_dtypes_multi_slice_ragged_epochs_inplace(kind, algo, P):
    """Many slices per chunk, ragged tail, in place, device producer with a
    permuted Pready order, 2 epochs; plus the fp64 error bound of the sum."""
    Np, L = 3, 100_003
    xs = [_inputs(kind, SEED + 42, P, Np * L, e) for e in range(2)]
    ys = run_allreduce(P, Np, L, xs, algo, inplace=True, producer=2)
    for x, y in zip(xs, ys):
        ref, _, _ = oracle.pallreduce(x, Np, algo)
        for r in range(P):
            np.testing.assert_array_equal(_bits(y[r]), _bits(ref[r]))
        xf = x if kind == "f64" else oracle.bf16_to_f64(x)
        yf = y[0] if kind == "f64" else oracle.bf16_to_f64(y[0])
        u = 2.0**-53 if kind == "f64" else 2.0**-8   # unit roundoff
        bound = (P - 1) * u * np.abs(xf).sum(0) * 1.01 + (0 if kind == "f64" else 2.0**-133)
        assert (np.abs(yf - xf.sum(0)) <= bound).all()


@pytest.mark.parametrize("kind", ["f64", "bf16"])
@pytest.mark.parametrize("op", [pc.MAX, pc.MIN])
def test_dtypes_maxmin(kind, op):
    P, Np, L = 5, 4, 333
    x = _inputs(kind, SEED + 43, P, Np * L)
    for algo in (pc.ALGO_RING, pc.ALGO_DIRECT):
        (y,) = run_allreduce(P, Np, L, [x], algo, op=op)
        xf = x if kind == "f64" else oracle.bf16_to_f64(x)
        want = xf.max(0) if op == pc.MAX else xf.min(0)
        for r in range(P):
            got = y[r] if kind == "f64" else oracle.bf16_to_f64(y[r])
            np.testing.assert_array_equal(got, want)


# ------------------------------------------------------------------ c.5 matrix corners
@pytest.mark.parametrize("algo,Ps", [(pc.ALGO_RING, [2, 3, 8]), (pc.ALGO_RD, [2, 4, 8]),
                                     (pc.ALGO_DIRECT, [2, 3, 5, 8])])
@pytest.mark.parametrize("Np,L", [(8, 0), (2, 3), (7, 4), (3, 16), (8, 17)])
def test_c5_matrix_empty_and_short_chunks(algo, Ps, Np, L):
    """SURVEY §8(c).5 corners: L = 0 (every partition empty: flags still move,
    the wait still completes), L < P (empty trailing chunks under reading R4)
    and non-16-B lengths; int32 wrap sum against the brute-force definition and
    fp32 bit-exact against the schedule's fold (O3 / O4 / O6), 2 epochs."""
    oalgo = {pc.ALGO_RING: oracle.RING, pc.ALGO_RD: oracle.RD, pc.ALGO_DIRECT: oracle.DIRECT}[algo]
    for P in Ps:
        xi = [np.stack([synth.int32_full(SEED + 70 + e, r, 0, Np * L) for r in range(P)]) for e in range(2)]
        for x, y in zip(xi, run_allreduce(P, Np, L, xi, algo)):
            for r in range(P):
                np.testing.assert_array_equal(y[r], wrap_sum(x))
        xf = [np.stack([synth.normal_f32(SEED + 80 + e, r, 0, Np * L) for r in range(P)]) for e in range(2)]
        for x, y in zip(xf, run_allreduce(P, Np, L, xf, algo)):
            ref, _, _ = oracle.pallreduce(x, Np, oalgo)
            for r in range(P):
                assert (y[r].view(np.uint32) == ref[r].view(np.uint32)).all(), (P, r)


@pytest.mark.parametrize("algo,P", [(pc.ALGO_RING, 4), (pc.ALGO_RD, 8), (pc.ALGO_DIRECT, 8), (pc.ALGO_DIRECT, 3)])
@pytest.mark.parametrize("graph", [False, True])
def test_epoch_all_single_control_kernel(algo, P, graph):
    """pc_epoch_all (Start + Pbuf_prepare + Pready of every partition in one
    kernel) drives correct epochs, eagerly and replayed from a CUDA graph:
    fp32 bit-exact vs the schedule's oracle fold every epoch."""
    Np, L = 5, 999
    oalgo = {pc.ALGO_RING: oracle.RING, pc.ALGO_RD: oracle.RD, pc.ALGO_DIRECT: oracle.DIRECT}[algo]
    with comms(P) as cs:
        st = torch.cuda.Stream()
        send = [torch.zeros(Np * L, device="cuda") for _ in range(P)]
        recv = [torch.zeros(Np * L, device="cuda") for _ in range(P)]
        reqs = [pc.pallreduce_init(send[r], recv[r], Np, L, pc.FLOAT32, pc.SUM, algo, cs[r]) for r in range(P)]
        for q in reqs:
            q.start(st)
        first_prepare([[q] for q in reqs], [st] * P)
        for q in reqs:
            q.pready_range(0, Np - 1, st)
        for q in reqs:
            q.wait_on_stream(st)
        torch.cuda.synchronize()

        def step():
            pc.epoch_all(reqs, pready=True, stream=st)
            for q in reqs:
                q.wait_on_stream(st)

        g = None
        if graph:
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=st):
                step()
        for e in range(4):
            x = np.stack([synth.normal_f32(SEED + 90, r, e, Np * L) for r in range(P)])
            for r in range(P):
                send[r].copy_(torch.from_numpy(x[r]))
            torch.cuda.synchronize()
            if graph:
                g.replay()
            else:
                step()
            torch.cuda.synchronize()
            ref, _, _ = oracle.pallreduce(x, Np, oalgo)
            for r in range(P):
                assert (recv[r].cpu().numpy().view(np.uint32) == ref[r].view(np.uint32)).all(), (e, r)
        for q in reqs:
            assert q.error() == (0, 0)
            q.free()
