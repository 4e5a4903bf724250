"""GPU: producer/engine overlap (§8(a) a6 — "each partition forwarded and
reduced as soon as it is ready", §IV-B1; the paper's own remedy of
moving the collective's progress beside the user kernel, §VI-B).

The probe producer (apps.overlap_probe: one launch, block r = rank r's
producer, so the P spinning producers are co-resident by construction)
Preadies partition 0, then spins on the DEVICE pc_parrived(0) of
the partitioned collective before it Preadies the remaining partitions.
Partition 0 can only complete while the producer is still running if the
engine runs concurrently with it: with the default fork point (the epoch's
pbuf_prepare) every rank sees Parrived(0) inside its kernel, stamped by
%globaltimer before the kernel's exit; with pc_request_set_overlap(0) (engine
forked at the wait, after the producer — the round-1 order) the spin times out.
Results stay bit-exact against the schedule-faithful oracle in both cases."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_temucinslsga24_b200 as pc
import synth
from paper_conf_sc_temucinslsga24_b200 import apps

from gpu_util import comms, first_prepare

pytestmark = pytest.mark.gpu

SEED = synth.BASE_SEED + 700
OALGO = {pc.ALGO_RING: oracle.RING, pc.ALGO_RD: oracle.RD, pc.ALGO_DIRECT: oracle.DIRECT}


def _run(P, algo, overlap, Np=4, L=4099, epochs=3, spin_ms=3000, copy=pc.COPY_ENGINE):
    n = Np * L
    with comms(P, timeout_ms=20000) as cs:
        streams = [torch.cuda.Stream() for _ in range(P)]
        send = [torch.empty(n, device="cuda") for _ in range(P)]
        recv = [torch.zeros(n, device="cuda") for _ in range(P)]
        reqs = [pc.pallreduce_init(send[r], recv[r], Np, L, pc.FLOAT32, pc.SUM, algo, cs[r]) for r in range(P)]
        for q in reqs:
            q.set_overlap(overlap)
        stamps = []
        for e in range(epochs):
            x = np.stack([synth.normal_f32(SEED, r, e, n) for r in range(P)])
            torch.cuda.synchronize()
            for r in range(P):
                send[r].copy_(torch.from_numpy(x[r]))
            torch.cuda.synchronize()
            for r in range(P):
                reqs[r].start(streams[r])
            if e == 0:
                first_prepare([[q] for q in reqs], streams)
                preqs = [q.prequest_create(pc.GRAN_BLOCK, 1, copy) for q in reqs]
            else:
                for r in range(P):
                    reqs[r].pbuf_prepare(streams[r])
            out = torch.zeros((P, 4), dtype=torch.int64, device="cuda")
            # every rank's producer (one launch, block r = rank r, on rank 0's
            # stream after every rank's control calls), then every rank's wait
            # (Listing 2 order)
            ev = [torch.cuda.Event() for _ in range(P)]
            for r in range(P):
                ev[r].record(streams[r])
                streams[0].wait_event(ev[r])
            apps.overlap_probe(preqs, Np, spin_ms, out, streams[0])
            for r in range(P):
                reqs[r].wait_on_stream(streams[r])
            torch.cuda.synchronize()
            for q in reqs:
                assert q.error() == (0, 0)
            ref, _, _ = oracle.pallreduce(x, Np, OALGO[algo])
            for r in range(P):
                got = recv[r].cpu().numpy()
                np.testing.assert_array_equal(got.view(np.uint32), ref[r].view(np.uint32))
            stamps.append(out.cpu().numpy())
        return stamps


CASES = [(pc.ALGO_DIRECT, 2), (pc.ALGO_DIRECT, 4), (pc.ALGO_DIRECT, 8), (pc.ALGO_RING, 3), (pc.ALGO_RING, 8),
         (pc.ALGO_RD, 4)]


@pytest.mark.parametrize("algo,P", CASES)
def test_engine_runs_while_producer_runs(algo, P):
    for st in _run(P, algo, overlap=True):
        t_entry, t_ready0, t_arr0, t_exit = st[:, 0], st[:, 1], st[:, 2], st[:, 3]
        assert (t_arr0 > 0).all(), f"partition 0 never completed inside the producer: {st.tolist()}"
        # on every rank the collective's partition 0 completed while that
        # rank's producer kernel was still running (it waited for it inside)
        assert (t_arr0 >= t_ready0).all() and (t_arr0 < t_exit).all()


@pytest.mark.parametrize("algo,P", [(pc.ALGO_DIRECT, 4), (pc.ALGO_RING, 3)])
def test_no_overlap_mode_times_out_the_probe(algo, P):
    """Control: with the engine forked at the wait (after the producer) the
    probe's in-kernel Parrived(0) cannot succeed; it gives up after spin_ms and
    the collective then completes correctly."""
    for st in _run(P, algo, overlap=False, epochs=2, spin_ms=50):
        assert (st[:, 2] == 0).all(), st.tolist()


def test_overlap_width_bound():
    """The engine width while a producer may run beside it: whole CTAs on at
    most PC_OVERLAP_FRAC (0.5) of the SMs per GPU in total."""
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    for P in (1, 2, 8):
        with comms(P) as cs:
            assert cs[0].overlap_warps * P <= sms * 8 // 2
            assert cs[0].overlap_warps % 8 == 0 and cs[0].overlap_warps >= 8


@pytest.mark.parametrize("algo,P", [(pc.ALGO_DIRECT, 8), (pc.ALGO_RING, 4), (pc.ALGO_DIRECT_PUSH, 4)])
def test_back_to_back_epochs_without_host_sync(algo, P):
    """The early fork must keep every epoch ordered after the previous epoch's
    consumer: 24 epochs back to back on per-rank streams with NO host
    synchronisation — each epoch a producer kernel writes new (epoch-tagged)
    inputs and Preadies them, the engine (forked at pbuf_prepare) reduces, and
    a consumer copies recvbuf into that epoch's slot on the same stream before
    the next pc_start.  Every epoch's slot must equal the oracle's fold of that
    epoch's inputs."""
    Np, L, E = 6, 3001, 24
    n = Np * L
    with comms(P, timeout_ms=20000) as cs:
        streams = [torch.cuda.Stream() for _ in range(P)]
        xs = [np.stack([synth.normal_f32(SEED + 9, r, e, n) for r in range(P)]) for e in range(E)]
        src = [torch.from_numpy(np.stack([xs[e][r] for e in range(E)])).cuda() for r in range(P)]  # [E, n]
        send = [torch.zeros(n, device="cuda") for _ in range(P)]
        recv = [torch.zeros(n, device="cuda") for _ in range(P)]
        slots = [torch.zeros(E, n, device="cuda") for _ in range(P)]
        reqs = [pc.pallreduce_init(send[r], recv[r], Np, L, pc.FLOAT32, pc.SUM, algo, cs[r]) for r in range(P)]
        torch.cuda.synchronize()
        for e in range(E):
            for r in range(P):
                reqs[r].start(streams[r])
            if e == 0:
                first_prepare([[q] for q in reqs], streams)
                preqs = [q.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_ENGINE) for q in reqs]
            else:
                for r in range(P):
                    reqs[r].pbuf_prepare(streams[r])
            for r in range(P):
                apps.produce(send[r], src[r][e], Np, L * 4, apps.GRAN_BLOCK, preqs[r],
                             order_stride=(1, 5, 7)[e % 3], stream=streams[r])  # coprime with Np = 6
            for r in range(P):
                reqs[r].wait_on_stream(streams[r])
            for r in range(P):
                with torch.cuda.stream(streams[r]):
                    slots[r][e].copy_(recv[r])  # the consumer of this epoch's result
        torch.cuda.synchronize()
        for q in reqs:
            assert q.error() == (0, 0)
        oalgo = oracle.RING if algo == pc.ALGO_RING else oracle.DIRECT
        for e in range(E):
            ref, _, _ = oracle.pallreduce(xs[e], Np, oalgo)
            for r in range(P):
                np.testing.assert_array_equal(slots[r][e].cpu().numpy().view(np.uint32), ref[r].view(np.uint32))
        for q in reqs:
            q.free()
