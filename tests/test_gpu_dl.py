"""GPU parity: the DL proxy (§VI-D2; reading R28) — the BCE
gradient producer alone bit-exact against oracle O7, and producer →
partitioned allreduce (the producer Preadies each partition from the kernel,
or the host Preadies all after it) bit-exact against oracle.pallreduce of the
oracle's gradients, over several epochs."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_temucinslsga24_b200 as pc
import synth
from paper_conf_sc_temucinslsga24_b200 import apps

from gpu_util import comms

pytestmark = pytest.mark.gpu

SEED = synth.BASE_SEED + 90


@pytest.mark.parametrize("Np,L", [(1, 1), (5, 1001), (3, 4096), (7, 65539)])
def test_bce_grad_bitexact(Np, L):
    n = Np * L
    p, y = synth.bce_inputs(SEED, 0, 0, n)
    pt, yt = torch.from_numpy(p).cuda(), torch.from_numpy(y).cuda()
    g = torch.zeros(n, device="cuda")
    apps.bce_grad(pt, yt, g, Np, L, float(n), None, order_stride=3 if Np % 3 else 1)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(g.cpu().numpy().view(np.uint32), oracle.bce_grad(p, y, float(n)).view(np.uint32))


def _oracle_step(ps, ys, Np, L, algo):
    n = Np * L
    grads = np.stack([oracle.bce_grad(ps[r], ys[r], float(n)) for r in range(len(ps))])
    ref, _, _ = oracle.pallreduce(grads, Np, {pc.ALGO_RING: oracle.RING, pc.ALGO_RD: oracle.RD,
                                              pc.ALGO_DIRECT: oracle.DIRECT}[algo])
    return ref


@pytest.mark.parametrize("mode", ["pready", "serial"])
@pytest.mark.parametrize("algo,P", [(pc.ALGO_RING, 4), (pc.ALGO_RING, 8), (pc.ALGO_RD, 8), (pc.ALGO_DIRECT, 8)])
@pytest.mark.parametrize("Np,L", [(6, 3000), (4, 30001)])
def test_dl_proxy_epochs(mode, algo, P, Np, L):
    n = Np * L
    with comms(P) as cs:
        inputs = [[synth.bce_inputs(SEED + 1, r, e, n) for r in range(P)] for e in range(3)]
        p = [torch.empty(n, device="cuda") for _ in range(P)]
        y = [torch.empty(n, device="cuda") for _ in range(P)]
        dl = apps.DLProxy(cs, Np, L, algo, p, y)
        for e in range(3):
            torch.cuda.synchronize()
            for r in range(P):
                p[r].copy_(torch.from_numpy(inputs[e][r][0]))
                y[r].copy_(torch.from_numpy(inputs[e][r][1]))
            torch.cuda.synchronize()
            dl.step(mode, order_stride=5)
            torch.cuda.synchronize()
            assert dl.errors() == []
            ref = _oracle_step([inputs[e][r][0] for r in range(P)], [inputs[e][r][1] for r in range(P)], Np, L, algo)
            for r in range(P):
                np.testing.assert_array_equal(dl.out[r][:n].cpu().numpy().view(np.uint32), ref[r].view(np.uint32))
        dl.free()


def test_dl_proxy_mode_switch_and_many_epochs():
    """Alternate device-Pready / host-Pready epochs on the same persistent
    requests; 20 epochs, constant inputs."""
    P, Np, L = 8, 16, 8192
    n = Np * L
    with comms(P) as cs:
        pin = [synth.bce_inputs(SEED + 2, r, 0, n) for r in range(P)]
        p = [torch.from_numpy(a).cuda() for a, _ in pin]
        y = [torch.from_numpy(b).cuda() for _, b in pin]
        dl = apps.DLProxy(cs, Np, L, pc.ALGO_RING, p, y)
        ref = _oracle_step([a for a, _ in pin], [b for _, b in pin], Np, L, pc.ALGO_RING)
        for e in range(20):
            dl.step("pready" if e % 3 else "serial", order_stride=7)
            if e % 5 == 4:
                torch.cuda.synchronize()
                assert dl.errors() == []
                for r in (0, P - 1):
                    np.testing.assert_array_equal(dl.out[r][:n].cpu().numpy(), ref[r])
        dl.free()


@pytest.mark.parametrize("mode,copy,algo,coop", [("pready", pc.COPY_INLINE, pc.ALGO_DIRECT, False),
                                                 ("pready", pc.COPY_INLINE, pc.ALGO_DIRECT, True),
                                                 ("mixed", pc.COPY_INLINE, pc.ALGO_DIRECT, True),
                                                 ("pready", None, pc.ALGO_DIRECT, False),
                                                 ("serial", None, pc.ALGO_RING, False),
                                                 ("pready", None, pc.ALGO_RING, False)])
@pytest.mark.parametrize("P,Np,L", [(8, 6, 3000), (4, 13, 4099), (2, 3, 65536), (8, 700, 1024)])
def test_dl_proxy_multi_launch(mode, copy, algo, coop, P, Np, L):
    """All ranks' producers in one launch (bce_grad_multi, partition u of
    every rank side by side), with the INLINE fold (R33), the cooperative
    INLINE fold (R36: the P blocks of u fold one slice each; "mixed"
    alternates it with host-Pready epochs on the same request) or the engine,
    over 3 epochs: bit-exact against the oracle's gradients + pallreduce."""
    n = Np * L
    with comms(P) as cs:
        inputs = [[synth.bce_inputs(SEED + 3, r, e, n) for r in range(P)] for e in range(3)]
        p = [torch.empty(n, device="cuda") for _ in range(P)]
        y = [torch.empty(n, device="cuda") for _ in range(P)]
        dl = apps.DLProxy(cs, Np, L, algo, p, y, copy=copy, multi=True, coop=coop)
        for e in range(3):
            torch.cuda.synchronize()
            for r in range(P):
                p[r].copy_(torch.from_numpy(inputs[e][r][0]))
                y[r].copy_(torch.from_numpy(inputs[e][r][1]))
            torch.cuda.synchronize()
            dl.step(("serial" if e == 1 else "pready") if mode == "mixed" else mode)
            torch.cuda.synchronize()
            assert dl.errors() == []
            ref = _oracle_step([inputs[e][r][0] for r in range(P)], [inputs[e][r][1] for r in range(P)], Np, L, algo)
            for r in range(P):
                np.testing.assert_array_equal(dl.out[r][:n].cpu().numpy().view(np.uint32), ref[r].view(np.uint32))
        dl.free()
