"""GPU parity at BASELINE sizes, in the launch configuration bench.py times
(8 virtual ranks on one B200, 256 MiB fp32 per rank, 64 partitions, ring /
DIRECT / RD, default slicing, one shared stream, pc_epoch_all after the first
epoch): sampled outputs are checked bit-exactly
against the oracle's closed-form ring fold computed element by element from
regenerated inputs, plus the R16 fp64 bound; RD at 64 MiB likewise; int32 at
64 MiB on every element against numpy's exact sum."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_temucinslsga24_b200 as pc
import synth

from gpu_util import comms, first_prepare

pytestmark = pytest.mark.gpu
SEED = synth.BASE_SEED + 100


def run_bench_shape(P, S, Np, algo, gen_rank, dtype=torch.float32, steps=2):
    count = S // 4 // Np
    n = count * Np
    with comms(P, timeout_ms=20000) as cs:
        st = torch.cuda.Stream()
        send = [torch.from_numpy(gen_rank(r, n)).to("cuda") for r in range(P)]
        recv = [torch.empty(n, dtype=dtype, device="cuda") for _ in range(P)]
        dt = pc.FLOAT32 if dtype == torch.float32 else pc.INT32
        reqs = [pc.pallreduce_init(send[r], recv[r], Np, count, dt, pc.SUM, algo, cs[r]) for r in range(P)]
        torch.cuda.synchronize()
        for e in range(steps):  # several epochs, exactly as bench.py's step()
            if e == 0:
                for q in reqs:
                    q.start(st)
                first_prepare([[q] for q in reqs], [st] * P)
                for q in reqs:
                    q.pready_range(0, Np - 1, st)
            else:  # bench.py: Start + RTR + Pready of every rank in one kernel
                pc.epoch_all(reqs, pready=True, stream=st)
            for q in reqs:
                q.wait_on_stream(st)
        torch.cuda.synchronize()
        for q in reqs:
            assert q.error() == (0, 0)
        info = reqs[0].info()
        for q in reqs:
            q.free()
        return recv, count, info


@pytest.mark.parametrize("algo,S", [(pc.ALGO_RING, 256 << 20), (pc.ALGO_RD, 64 << 20), (pc.ALGO_DIRECT, 256 << 20)])
def test_fullsize_sampled_fp32(algo, S):
    P, Np = 8, 64
    recv, L, info = run_bench_shape(P, S, Np, algo, lambda r, n: synth.uniform_f32(SEED, r, 0, n))
    rng = np.random.default_rng(7)
    n = L * Np
    idx = np.unique(np.concatenate([rng.integers(0, n, 20000), [0, n - 1, L - 1, L, n // 2]]))
    xs = np.stack([synth.uniform_f32_at(SEED, r, 0, idx) for r in range(P)])
    if algo == pc.ALGO_RING:
        chunk = oracle.chunk_ids(L, P, 1)[idx % L]
        ref = oracle.ring_fold_f32(xs, chunk)
    elif algo == pc.ALGO_DIRECT:
        ref = oracle.ring_fold_f32(xs, np.zeros(len(idx), np.int32))
    else:
        ref = oracle.rd_tree_f32(xs)
    y64, sabs = oracle.allreduce_def_f64(xs)
    for r in range(P):
        got = recv[r][torch.from_numpy(idx).cuda()].cpu().numpy()
        np.testing.assert_array_equal(got.view(np.uint32), ref.view(np.uint32))
    assert (np.abs(ref.astype(np.float64) - y64) <= 1e-5 * sabs).all()
    # every rank holds identical bits everywhere (AG copies / commutativity)
    for r in range(1, P):
        assert torch.equal(recv[r], recv[0])


@pytest.mark.parametrize("algo", [pc.ALGO_RING, pc.ALGO_DIRECT])
def test_fullsize_int32_every_element(algo):
    P, Np, S = 8, 64, 64 << 20
    recv, L, _ = run_bench_shape(P, S, Np, algo, lambda r, n: synth.int32_full(SEED, r, 1, n),
                                 dtype=torch.int32)
    n = L * Np
    acc = np.zeros(n, dtype=np.int64)
    for r in range(P):
        acc += synth.int32_full(SEED, r, 1, n)
    ref = ((acc + 2**31) % 2**32 - 2**31).astype(np.int32)
    for r in range(P):
        np.testing.assert_array_equal(recv[r].cpu().numpy(), ref)
