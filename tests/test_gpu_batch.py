"""GPU parity: batched control and completion over MANY partitioned
allreduces of one GPU (one request per gradient tensor;
MPI_Startall / MPI_Waitall).  pc_epoch_all with more requests / RTR words than
one kernel's parameters hold runs one table-driven kernel; pc_waitall_on_stream
over DIRECT allreduces runs ONE batched engine launch (units ordered
[request][unit][local rank]).  Results bit-exact against the schedule-faithful
oracle (O6: rank-order fold, reading R25) for every tensor, every rank, several
epochs — eager and replayed from a captured CUDA graph."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_temucinslsga24_b200 as pc
import synth

from gpu_util import comms, first_prepare

pytestmark = pytest.mark.gpu
SEED = synth.BASE_SEED + 1200


def _run(P, sizes, Np_of, epochs=3, graph=False, control="epoch_all", dtype=np.float32, algo=pc.ALGO_DIRECT):
    T = len(sizes)
    dt = pc.FLOAT32 if dtype == np.float32 else pc.INT32
    tdt = torch.float32 if dtype == np.float32 else torch.int32
    with comms(P, timeout_ms=20000) as cs:
        st = torch.cuda.Stream()
        send = [[torch.zeros(n, dtype=tdt, device="cuda") for n in sizes] for _ in range(P)]
        recv = [[torch.zeros(n, dtype=tdt, device="cuda") for n in sizes] for _ in range(P)]
        reqs = [[pc.pallreduce_init(send[r][t], recv[r][t], Np_of(n), n // Np_of(n), dt, pc.SUM, algo, cs[r])
                 for t, n in enumerate(sizes)] for r in range(P)]
        flat = [reqs[r][t] for t in range(T) for r in range(P)]
        for q in flat:
            q.start(st)
        first_prepare(reqs, [st] * P)
        pc.preadyall(flat[:16], st) if len(flat) <= 16 else [pc.preadyall(flat[i:i + 16], st)
                                                            for i in range(0, len(flat), 16)]
        pc.waitall_on_stream(flat, st)
        torch.cuda.synchronize()

        def epoch():
            if control == "epoch_all":
                pc.epoch_all(flat, pready=True, stream=st)
            else:
                pc.startall(flat, st)
                pc.pbuf_prepare_all(flat, st)
                for i in range(0, len(flat), 16):
                    pc.preadyall(flat[i:i + 16], st)
            pc.waitall_on_stream(flat, st)

        gr = None
        results = []
        for e in range(epochs):
            xs = []
            for t, n in enumerate(sizes):
                gen = synth.normal_f32 if dtype == np.float32 else synth.int32_full
                x = np.stack([gen(SEED + t, r, e, n) for r in range(P)])
                xs.append(x)
                for r in range(P):
                    send[r][t].copy_(torch.from_numpy(x[r]))
            torch.cuda.synchronize()
            if graph:
                if gr is None:
                    epoch()  # eager first: the batch tables are built outside the capture
                    torch.cuda.synchronize()
                    gr = torch.cuda.CUDAGraph()
                    with torch.cuda.graph(gr, stream=st):
                        epoch()
                with torch.cuda.stream(st):
                    gr.replay()
            else:
                epoch()
            torch.cuda.synchronize()
            for q in flat:
                assert q.error() == (0, 0)
            results.append((xs, [[recv[r][t].cpu().numpy() for t in range(T)] for r in range(P)]))
        for q in flat:
            q.free()
    return results


SIZES = [64, 1000, 4096, 9408, 36864, 65536, 147456, 3, 16384]


@pytest.mark.parametrize("P", [2, 4, 8])
@pytest.mark.parametrize("control", ["epoch_all", "startall"])
def test_batched_per_tensor_fp32(P, control):
    for xs, got in _run(P, SIZES, lambda n: 1 if n < 4096 else 4, control=control):
        for t, x in enumerate(xs):
            ref, _, _ = oracle.pallreduce(x, 1 if x.shape[1] < 4096 else 4, oracle.DIRECT)
            for r in range(P):
                np.testing.assert_array_equal(got[r][t].view(np.uint32), ref[r].view(np.uint32))


def test_batched_int32_graph_replay():
    P = 8
    sizes = SIZES * 3  # 27 tensors x 8 ranks = 216 requests (RTR words: 1512)
    for xs, got in _run(P, sizes, lambda n: 1, graph=True, dtype=np.int32, epochs=3):
        for t, x in enumerate(xs):
            ref = oracle.allreduce_def_i32(x)
            for r in range(P):
                np.testing.assert_array_equal(got[r][t], ref)


def test_batched_falls_back_for_ring():
    """Ring requests are not batched (different engine): pc_waitall_on_stream
    takes each request's own path; results stay exact."""
    P = 4
    for xs, got in _run(P, [1000, 4096, 17], lambda n: 1, algo=pc.ALGO_RING, epochs=2):
        for t, x in enumerate(xs):
            ref, _, _ = oracle.pallreduce(x, 1, oracle.RING)
            for r in range(P):
                np.testing.assert_array_equal(got[r][t].view(np.uint32), ref[r].view(np.uint32))
