"""GPU parity: partitioned send/recv (Pready at thread / warp / block
granularity, aggregation, INLINE "Kernel Copy" and ENGINE copy) through the C
ABI vs the CPU oracle O1 (byte-exact), with 2 virtual ranks on one B200."""
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

GRAN_ELEMS = {apps.GRAN_THREAD: 2, apps.GRAN_WARP: 64, apps.GRAN_BLOCK: 2048,
              apps.GRAN_BLOCK_PUT: 2048}  # 8 B / 256 B / 8 KiB / 8 KiB


def run_vecadd(n, gran, agg, copy, epochs=3, check_in_kernel=True, persistent=False):
    """C1/C2 shape: sender computes C = A + B and Preadies from the kernel
    (persistent: the same partitions from one CTA per resident slot)."""
    count = GRAN_ELEMS[gran]
    partitions = n // count
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        A = torch.empty(n, device="cuda")
        B = torch.empty(n, device="cuda")
        Cb = torch.empty(n, device="cuda")
        R = torch.full((n,), -1.0, device="cuda")
        out = torch.zeros(n, device="cuda")
        status = torch.zeros(1, dtype=torch.int32, device="cuda")
        snd = pc.psend_init(Cb, partitions, count, pc.FLOAT32, 1, 7, cs[0])
        rcv = pc.precv_init(R, partitions, count, pc.FLOAT32, 0, 7, cs[1])
        sent_all, got_all, got_kernel = [], [], []
        for e in range(epochs):
            a = synth.uniform_f32(SEED, 0, 2 * e, n)
            b = synth.uniform_f32(SEED, 0, 2 * e + 1, n)
            A.copy_(torch.from_numpy(a))
            B.copy_(torch.from_numpy(b))
            torch.cuda.synchronize()
            snd.start(s0)
            rcv.start(s1)
            if e == 0:
                first_prepare([[snd], [rcv]], [s0, s1])
                sq = snd.prequest_create(min(gran, apps.GRAN_BLOCK), agg, copy)
                rq = rcv.prequest_create(min(gran, apps.GRAN_BLOCK), 1, pc.COPY_INLINE)
            else:
                rcv.pbuf_prepare(s1)
                snd.pbuf_prepare(s0)
            # Producers first, consumers second: virtual ranks share hardware
            # queues, so a spinning consumer must never be enqueued before the
            # work it waits for.  The sender's wait launches its ENGINE (lazy
            # launch), so it precedes the in-kernel Parrived consumer.
            apps.vecadd(A, B, Cb, n, gran, sq, s0, persistent=persistent)
            snd.wait_on_stream(s0)
            if check_in_kernel:
                apps.check_recv(rq, R, out, partitions, count * 4, status, blocks=64, stream=s1)
            rcv.wait_on_stream(s1)
            torch.cuda.synchronize()
            if snd.error()[0] != 0 or rcv.error()[0] != 0:
                f = rcv.words("flags", 0, -(-partitions // agg))
                st = snd.words("sent", 0, -(-partitions // agg))
                raise AssertionError(
                    f"epoch {e}: snd err {snd.error()} rcv err {rcv.error()} status {int(status.item())} "
                    f"flags<e+1 at {np.nonzero(f < e + 1)[0][:8]} vals {f[np.nonzero(f < e + 1)[0][:4]]} "
                    f"sent<e+1 at {np.nonzero(st < e + 1)[0][:8]} layout/epoch {rcv.words('epoch', 0, 1)} "
                    f"rtr {snd.words('rtr', 0, 2)} raw flags {[hex(v) for v in f[:12]]} max {hex(f.max())} "
                    f"R[:4] {R[:4].tolist()} out[:4] {out[:4].tolist()}")
            sent_all.append((a + b).astype(np.float32))
            got_all.append(R.cpu().numpy().copy())
            got_kernel.append(out.cpu().numpy().copy())
        assert int(status.item()) == 0
        snd.free()
        rcv.free()
    send = np.stack(sent_all).view(np.uint8).reshape(epochs, -1)
    orders = np.stack([synth.permutation(SEED, 0, e, partitions) for e in range(epochs)])
    consumed, arrivals = oracle.p2p(send, partitions, agg, orders)
    assert (arrivals == 1).all()
    got = np.stack(got_all).view(np.uint8).reshape(epochs, -1)
    np.testing.assert_array_equal(got, consumed)
    if check_in_kernel:
        np.testing.assert_array_equal(np.stack(got_kernel).view(np.uint8).reshape(epochs, -1), consumed)


@pytest.mark.parametrize("copy", [pc.COPY_INLINE, pc.COPY_ENGINE])
@pytest.mark.parametrize("agg", [1, 128])
def test_c2_block_256mib(copy, agg):
    """C2 at its largest size (256 MiB, 32768 block partitions of 8 KiB; agg
    128 = 1 MiB transport partitions): byte-exact vs O1 over 2 epochs with
    seeded inputs, in-kernel Parrived consumer included."""
    run_vecadd(1 << 26, apps.GRAN_BLOCK, agg, copy, epochs=2)


@pytest.mark.parametrize("gran", [apps.GRAN_BLOCK, apps.GRAN_BLOCK_PUT])
@pytest.mark.parametrize("copy", [pc.COPY_INLINE, pc.COPY_ENGINE])
def test_c2_persistent_256mib(gran, copy):
    """C2 at 256 MiB from the persistent producer (296 CTAs walking 32768
    logical blocks), block Pready with read-back and from registers
    (pc_pready_block_put, R35): byte-exact vs O1 over 2 epochs."""
    run_vecadd(1 << 26, gran, 1, copy, epochs=2, persistent=True)


@pytest.mark.parametrize("gran", [apps.GRAN_BLOCK_PUT, apps.GRAN_BLOCK])
@pytest.mark.parametrize("batch", ["1", "3", "32"])
@pytest.mark.parametrize("agg", [1, 5])
def test_put_batched_release(gran, batch, agg, monkeypatch):
    """Persistent producers releasing `batch` logical blocks at a time
    (pc_put_begin batch, pc_put_end flushing the tail; 1000 logical blocks
    over 296 CTAs leave partial batches) — the register Kernel Copy and the
    MPI-shaped pc_pready_block checked once — with and without aggregation:
    byte-exact vs O1, in-kernel Parrived consumer included."""
    monkeypatch.setenv("PCAPP_PUT_BATCH", batch)
    run_vecadd(2048 * 1000, gran, agg, pc.COPY_INLINE, epochs=3, persistent=True)


@pytest.mark.parametrize("persistent", [False, True])
@pytest.mark.parametrize("gran", [apps.GRAN_THREAD, apps.GRAN_WARP, apps.GRAN_BLOCK, apps.GRAN_BLOCK_PUT])
@pytest.mark.parametrize("agg_kind", ["none", "odd", "all"])
@pytest.mark.parametrize("copy", [pc.COPY_INLINE, pc.COPY_ENGINE, pc.COPY_LL])
def test_producer_shapes(persistent, gran, agg_kind, copy):
    """Every granularity from both producer shapes, over more logical blocks
    (1000) than resident CTAs so persistent CTAs loop; block_put falls back to
    pc_pready_block for ENGINE / LL."""
    n = 2048 * 1000
    partitions = n // GRAN_ELEMS[gran]
    agg = {"none": 1, "odd": max(1, partitions // 3 - 1), "all": partitions}[agg_kind]
    if copy == pc.COPY_LL and agg * GRAN_ELEMS[gran] * 4 > 1024:
        pytest.skip("LL: transport partitions of at most 1 KiB")
    run_vecadd(n, gran, agg, copy, epochs=2, persistent=persistent)


def test_c1_block_agg16_inline():
    """C1: 1 MiB fp32, block Pready (128 x 8 KiB user partitions) aggregated
    16 per transport partition -> 8 transport partitions (reading R24)."""
    run_vecadd(1 << 18, apps.GRAN_BLOCK, 16, pc.COPY_INLINE, epochs=5)


@pytest.mark.parametrize("gran", [apps.GRAN_THREAD, apps.GRAN_WARP, apps.GRAN_BLOCK])
@pytest.mark.parametrize("agg_kind", ["none", "odd", "all"])
@pytest.mark.parametrize("copy", [pc.COPY_INLINE, pc.COPY_ENGINE, pc.COPY_HOST])
def test_granularity_aggregation_copy(gran, agg_kind, copy):
    n = 3 * 2048 * 5 + 0  # 15 blocks of 1024 threads
    partitions = n // GRAN_ELEMS[gran]
    agg = {"none": 1, "odd": max(1, partitions // 3 - 1), "all": partitions}[agg_kind]
    run_vecadd(n, gran, agg, copy, epochs=2)


def test_thread_granularity_warp_aggregation_large():
    """Thread granularity with g = 1024 (one transport partition per block):
    the library's warp aggregation of thread Preadies."""
    run_vecadd(1 << 20, apps.GRAN_THREAD, 1024, pc.COPY_INLINE, epochs=2)


def test_many_epochs_tagged_bytes():
    """1000 back-to-back epochs of epoch-tagged bytes with a permuted Pready
    order: every epoch's bytes arrive intact and exactly once."""
    partitions, pbytes, E = 16, 4096, 1000
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        src = torch.empty(partitions * pbytes, dtype=torch.uint8, device="cuda")
        sbuf = torch.empty_like(src)
        rbuf = torch.empty_like(src)
        snd = pc.psend_init(sbuf, partitions, pbytes, pc.BYTE, 1, 1, cs[0])
        rcv = pc.precv_init(rbuf, partitions, pbytes, pc.BYTE, 0, 1, cs[1])
        for e in range(E):
            payload = synth.bytes_tagged(SEED, 0, e, partitions * pbytes)
            src.copy_(torch.from_numpy(payload))
            torch.cuda.synchronize()
            snd.start(s0)
            rcv.start(s1)
            if e == 0:
                first_prepare([[snd], [rcv]], [s0, s1])
                sq = snd.prequest_create(pc.GRAN_BLOCK, 4, pc.COPY_INLINE)
            else:
                rcv.pbuf_prepare(s1)
                snd.pbuf_prepare(s0)
            apps.produce(sbuf, src, partitions, pbytes, apps.GRAN_BLOCK, sq, order_stride=5, stream=s0)
            snd.wait_on_stream(s0)
            rcv.wait_on_stream(s1)
            s1.synchronize()
            np.testing.assert_array_equal(rbuf.cpu().numpy(), payload)
        snd.wait()
        assert snd.error()[0] == 0 and rcv.error()[0] == 0
        snd.free()
        rcv.free()


def test_host_wait_and_test():
    n = 2048 * 4
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        A = torch.ones(n, device="cuda")
        Cb = torch.empty(n, device="cuda")
        R = torch.zeros(n, device="cuda")
        snd = pc.psend_init(Cb, 4, 2048, pc.FLOAT32, 1, 0, cs[0])
        rcv = pc.precv_init(R, 4, 2048, pc.FLOAT32, 0, 0, cs[1])
        snd.start(s0)
        rcv.start(s1)
        first_prepare([[snd], [rcv]], [s0, s1])
        sq = snd.prequest_create(pc.GRAN_BLOCK, 2, pc.COPY_ENGINE)
        assert not rcv.parrived(0)
        apps.vecadd(A, A, Cb, n, apps.GRAN_BLOCK, sq, s0)
        snd.wait()
        rcv.wait()
        assert rcv.parrived(3)
        assert (R.cpu().numpy() == 2.0).all()
        assert rcv.test()  # inactive request: complete
        snd.free()
        rcv.free()


def test_duplicate_pready_is_reported():
    n = 2048 * 2
    with comms(2, timeout_ms=2000) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        Cb = torch.zeros(n, device="cuda")
        R = torch.zeros(n, device="cuda")
        snd = pc.psend_init(Cb, 2, 2048, pc.FLOAT32, 1, 0, cs[0])
        rcv = pc.precv_init(R, 2, 2048, pc.FLOAT32, 0, 0, cs[1])
        snd.start(s0)
        rcv.start(s1)
        first_prepare([[snd], [rcv]], [s0, s1])
        # g = 2: both partitions feed one transport partition, so a duplicate
        # Pready overshoots the aggregation counter (g = 1 has no counter)
        snd.prequest_create(pc.GRAN_BLOCK, 2, pc.COPY_INLINE)
        snd.pready(0, s0)
        snd.pready(0, s0)  # duplicate in the same epoch
        snd.pready(1, s0)
        rcv.wait()
        with pytest.raises(pc.PcError) as ei:
            snd.wait()
        assert ei.value.code == pc.ERR_DEVICE
        snd.free()
        rcv.free()


def test_missing_pready_times_out():
    n = 2048 * 2
    with comms(2, timeout_ms=300) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        Cb = torch.zeros(n, device="cuda")
        R = torch.zeros(n, device="cuda")
        snd = pc.psend_init(Cb, 2, 2048, pc.FLOAT32, 1, 0, cs[0])
        rcv = pc.precv_init(R, 2, 2048, pc.FLOAT32, 0, 0, cs[1])
        snd.start(s0)
        rcv.start(s1)
        first_prepare([[snd], [rcv]], [s0, s1])
        snd.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
        snd.pready(0, s0)  # partition 1 never readied
        with pytest.raises(pc.PcError) as ei:
            rcv.wait()
        assert ei.value.code == pc.ERR_TIMEOUT
        with pytest.raises(pc.PcError):
            snd.wait()
        snd.free()
        rcv.free()


@pytest.mark.parametrize("payload", [0, 8, 256, 8192])
def test_pingpong_latency_roundtrip(payload):
    """Pready->Parrived ping-pong inside persistent kernels (one per side)."""
    iters = 2000
    cnt = payload // 4
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        bufs = [torch.zeros(max(iters * cnt, 4), device="cuda") for _ in range(4)]
        a2b = pc.psend_init(bufs[0], iters, cnt, pc.FLOAT32, 1, 1, cs[0])
        b_in = pc.precv_init(bufs[1], iters, cnt, pc.FLOAT32, 0, 1, cs[1])
        b2a = pc.psend_init(bufs[2], iters, cnt, pc.FLOAT32, 0, 2, cs[1])
        a_in = pc.precv_init(bufs[3], iters, cnt, pc.FLOAT32, 1, 2, cs[0])
        bufs[0].copy_(torch.arange(bufs[0].numel(), dtype=torch.float32))
        # the pair kernel runs on s0: every epoch word it reads is written on s0
        for q in (a2b, a_in, b_in, b2a):
            q.start(s0)
        first_prepare([[a2b, a_in], [b_in, b2a]], [s0, s0])
        pa = a2b.prequest_create(pc.GRAN_WARP, 1, pc.COPY_INLINE)
        pai = a_in.prequest_create(pc.GRAN_WARP, 1, pc.COPY_INLINE)
        pb = b2a.prequest_create(pc.GRAN_WARP, 1, pc.COPY_INLINE)
        pbi = b_in.prequest_create(pc.GRAN_WARP, 1, pc.COPY_INLINE)
        t = torch.zeros(2, dtype=torch.int64, device="cuda")
        apps.pingpong_pair(pa, pai, pb, pbi, iters, apps.GRAN_WARP, t, s0)
        for q in (a2b, b2a, a_in, b_in):
            q.wait_on_stream(s0)
        torch.cuda.synchronize()
        ns = int(t[0].item()) / iters / 2
        print(f"payload {payload} B: one-way {ns:.0f} ns (same-GPU virtual ranks)")
        assert ns > 0
        if cnt:
            np.testing.assert_array_equal(bufs[1].cpu().numpy(), bufs[0].cpu().numpy())
        for q in (a2b, a_in, b_in, b2a):
            assert q.error()[0] == 0
            q.free()


# ---------------------------------------------------------------- PC_COPY_LL
@pytest.mark.parametrize("gran", [apps.GRAN_THREAD, apps.GRAN_WARP])
@pytest.mark.parametrize("agg_kind", ["none", "odd", "all"])
def test_ll_granularity_aggregation(gran, agg_kind):
    """LL lines (8 payload bytes + the epoch per 16-B line) at thread (8 B) and
    warp (256 B) granularity: byte-exact vs O1, in-kernel pc_wait_arrived and
    the stream wait both unpack the lines into recvbuf."""
    n = 3 * 2048 * 5
    partitions = n // GRAN_ELEMS[gran]
    agg = {"none": 1, "odd": max(1, partitions // 3 - 1), "all": partitions}[agg_kind]
    run_vecadd(n, gran, agg, pc.COPY_LL, epochs=3)


@pytest.mark.parametrize("pbytes", [1, 3, 8, 12, 100, 256, 1000, 1024])
@pytest.mark.parametrize("gran", [apps.GRAN_THREAD, apps.GRAN_WARP, apps.GRAN_BLOCK])
def test_ll_epochs_tagged_bytes(pbytes, gran):
    """LL over many back-to-back epochs of epoch-tagged bytes (both line-area
    parities reused many times), ragged partition sizes (partial last line,
    unaligned partitions), permuted Pready order; recvbuf checked every epoch."""
    partitions, E = 37, 60
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        src = torch.empty(partitions * pbytes, dtype=torch.uint8, device="cuda")
        sbuf = torch.empty_like(src)
        rbuf = torch.empty_like(src)
        out = torch.zeros_like(src)
        status = torch.zeros(1, dtype=torch.int32, device="cuda")
        snd = pc.psend_init(sbuf, partitions, pbytes, pc.BYTE, 1, 1, cs[0])
        rcv = pc.precv_init(rbuf, partitions, pbytes, pc.BYTE, 0, 1, cs[1])
        for e in range(E):
            payload = synth.bytes_tagged(SEED, 0, e, partitions * pbytes)
            src.copy_(torch.from_numpy(payload))
            torch.cuda.synchronize()
            snd.start(s0)
            rcv.start(s1)
            if e == 0:
                first_prepare([[snd], [rcv]], [s0, s1])
                sq = snd.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_LL)
                rq = rcv.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
            else:
                rcv.pbuf_prepare(s1)
                snd.pbuf_prepare(s0)
            apps.produce(sbuf, src, partitions, pbytes, gran, sq, order_stride=5, stream=s0)
            snd.wait_on_stream(s0)
            if e % 2:
                apps.check_recv(rq, rbuf, out, partitions, pbytes, status, blocks=8, stream=s1)
            rcv.wait_on_stream(s1)
            s1.synchronize()
            np.testing.assert_array_equal(rbuf.cpu().numpy(), payload)
            if e % 2:
                np.testing.assert_array_equal(out.cpu().numpy(), payload)
        snd.wait()
        assert int(status.item()) == 0
        assert snd.error()[0] == 0 and rcv.error()[0] == 0
        snd.free()
        rcv.free()


def test_ll_host_parrived_and_test():
    """Host pc_parrived / pc_test on an LL receive request check (and unpack)
    the lines on the device."""
    partitions, count = 8, 16  # 64 B partitions
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        sbuf = torch.arange(partitions * count, dtype=torch.float32, device="cuda")
        rbuf = torch.zeros_like(sbuf)
        snd = pc.psend_init(sbuf, partitions, count, pc.FLOAT32, 1, 0, cs[0])
        rcv = pc.precv_init(rbuf, partitions, count, pc.FLOAT32, 0, 0, cs[1])
        snd.start(s0)
        rcv.start(s1)
        first_prepare([[snd], [rcv]], [s0, s1])
        snd.prequest_create(pc.GRAN_WARP, 1, pc.COPY_LL)
        assert not rcv.parrived(0)
        assert not rcv.test()
        snd.pready_range(0, 2, s0)
        s0.synchronize()
        assert rcv.parrived(1)
        assert not rcv.parrived(5)
        assert torch.equal(rbuf[count:2 * count], sbuf[count:2 * count])
        assert not rcv.test()
        snd.pready_range(3, partitions - 1, s0)
        s0.synchronize()
        while not rcv.test():
            pass
        assert torch.equal(rbuf, sbuf)
        snd.wait()
        snd.free()
        rcv.free()


def test_ll_unsupported_large_partitions():
    """LL is for small partitions (<= PC_LL_MAX_PART_BYTES): larger ones are
    refused at pc_prequest_create."""
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        sbuf = torch.zeros(4 * 2048, device="cuda")
        rbuf = torch.zeros_like(sbuf)
        snd = pc.psend_init(sbuf, 4, 2048, pc.FLOAT32, 1, 0, cs[0])
        rcv = pc.precv_init(rbuf, 4, 2048, pc.FLOAT32, 0, 0, cs[1])
        snd.start(s0)
        rcv.start(s1)
        first_prepare([[snd], [rcv]], [s0, s1])
        with pytest.raises(pc.PcError) as ei:
            snd.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_LL)
        assert ei.value.code == pc.ERR_UNSUPPORTED
        snd.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
        snd.pready_range(0, 3, s0)
        rcv.wait()
        snd.wait()
        snd.free()
        rcv.free()


@pytest.mark.parametrize("payload", [0, 8, 256, 1024])
def test_ll_pingpong_latency_roundtrip(payload):
    """Pready->Parrived ping-pong with LL lines: data intact at every size."""
    iters = 2000
    cnt = payload // 4
    with comms(2) as cs:
        s0 = torch.cuda.Stream()
        bufs = [torch.zeros(max(iters * cnt, 4), device="cuda") for _ in range(4)]
        a2b = pc.psend_init(bufs[0], iters, cnt, pc.FLOAT32, 1, 1, cs[0])
        b_in = pc.precv_init(bufs[1], iters, cnt, pc.FLOAT32, 0, 1, cs[1])
        b2a = pc.psend_init(bufs[2], iters, cnt, pc.FLOAT32, 0, 2, cs[1])
        a_in = pc.precv_init(bufs[3], iters, cnt, pc.FLOAT32, 1, 2, cs[0])
        bufs[0].copy_(torch.arange(bufs[0].numel(), dtype=torch.float32))
        bufs[2].copy_(-torch.arange(bufs[2].numel(), dtype=torch.float32))
        for q in (a2b, a_in, b_in, b2a):
            q.start(s0)
        first_prepare([[a2b, a_in], [b_in, b2a]], [s0, s0])
        pa = a2b.prequest_create(pc.GRAN_WARP, 1, pc.COPY_LL)
        pai = a_in.prequest_create(pc.GRAN_WARP, 1, pc.COPY_INLINE)
        pb = b2a.prequest_create(pc.GRAN_WARP, 1, pc.COPY_LL)
        pbi = b_in.prequest_create(pc.GRAN_WARP, 1, pc.COPY_INLINE)
        t = torch.zeros(2, dtype=torch.int64, device="cuda")
        apps.pingpong_pair(pa, pai, pb, pbi, iters, apps.GRAN_WARP, t, s0)
        for q in (a2b, b2a, a_in, b_in):
            q.wait_on_stream(s0)
        torch.cuda.synchronize()
        ns = int(t[0].item()) / iters / 2
        print(f"LL payload {payload} B: one-way {ns:.0f} ns (same-GPU virtual ranks)")
        if cnt:
            np.testing.assert_array_equal(bufs[1].cpu().numpy(), bufs[0].cpu().numpy())
            np.testing.assert_array_equal(bufs[3].cpu().numpy(), bufs[2].cpu().numpy())
        for q in (a2b, a_in, b_in, b2a):
            assert q.error()[0] == 0
            q.free()


# ---------------------------------------------------------------- MPI-4: different partition counts (R30)
XP_TOTAL = 840 * 16  # bytes: divisible by every partition count 1..8


@pytest.mark.parametrize("Ns,Nr", [(8, 3), (3, 8), (6, 4), (1, 5), (5, 1)])
@pytest.mark.parametrize("agg", [1, 2])
@pytest.mark.parametrize("copy", [pc.COPY_INLINE, pc.COPY_ENGINE])
def test_xpart_different_partition_counts(Ns, Nr, agg, copy):
    """Sender and receiver partition the same bytes differently (MPI-4, P:L46;
    reading R30): byte-exact delivery over 3 epochs of epoch-tagged payloads,
    device pc_wait_arrived on every RECEIVE partition (check_recv kernel),
    stream wait, and host pc_parrived afterwards."""
    agg = min(agg, Ns)
    sb, rb = XP_TOTAL // Ns, XP_TOTAL // Nr
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        src = torch.empty(XP_TOTAL, dtype=torch.uint8, device="cuda")
        sbuf, rbuf, out = torch.empty_like(src), torch.zeros_like(src), torch.zeros_like(src)
        status = torch.zeros(1, dtype=torch.int32, device="cuda")
        snd = pc.psend_init(sbuf, Ns, sb, pc.BYTE, 1, 9, cs[0])
        rcv = pc.precv_init(rbuf, Nr, rb, pc.BYTE, 0, 9, cs[1])
        for e in range(3):
            payload = synth.bytes_tagged(SEED, 1, e, XP_TOTAL)
            src.copy_(torch.from_numpy(payload))
            torch.cuda.synchronize()
            snd.start(s0)
            rcv.start(s1)
            if e == 0:
                first_prepare([[snd], [rcv]], [s0, s1])
                sq = snd.prequest_create(pc.GRAN_BLOCK, agg, copy)
                rq = rcv.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
            else:
                rcv.pbuf_prepare(s1)
                snd.pbuf_prepare(s0)
            apps.produce(sbuf, src, Ns, sb, apps.GRAN_BLOCK, sq, stream=s0)
            snd.wait_on_stream(s0)
            apps.check_recv(rq, rbuf, out, Nr, rb, status, blocks=8, stream=s1)
            rcv.wait_on_stream(s1)
            torch.cuda.synchronize()
            assert snd.error()[0] == 0 and rcv.error()[0] == 0, (snd.error(), rcv.error())
            assert int(status.item()) == 0
            np.testing.assert_array_equal(rbuf.cpu().numpy(), payload)
            np.testing.assert_array_equal(out.cpu().numpy(), payload)
            assert all(rcv.parrived(p) for p in range(Nr))
        snd.free()
        rcv.free()


@pytest.mark.parametrize("Ns,Nr,agg", [(2, 3, 1), (6, 4, 2), (4, 6, 1), (5, 3, 2), (3, 5, 3)])
def test_xpart_partial_arrival_matches_oracle(Ns, Nr, agg):
    """Pready the send partitions one at a time (host binding, INLINE copy) in a
    seeded order; after each, the set of receive partitions the library reports
    arrived (host pc_parrived, pc_test) equals O11's byte-coverage definition,
    and every arrived partition already holds its bytes."""
    total = 960
    sb, rb = total // Ns, total // Nr
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        payload = synth.bytes_tagged(SEED, 2, Ns * 10 + Nr, total)
        sbuf = torch.from_numpy(payload).cuda()
        rbuf = torch.zeros_like(sbuf)
        snd = pc.psend_init(sbuf, Ns, sb, pc.BYTE, 1, 4, cs[0])
        rcv = pc.precv_init(rbuf, Nr, rb, pc.BYTE, 0, 4, cs[1])
        torch.cuda.synchronize()
        snd.start(s0)
        rcv.start(s1)
        first_prepare([[snd], [rcv]], [s0, s1])
        sq = snd.prequest_create(pc.GRAN_THREAD, agg, pc.COPY_INLINE)  # noqa: F841 (publishes the layout)
        readied = np.zeros(Ns, dtype=bool)
        for u in synth.permutation(SEED, 3, Ns * 10 + Nr, Ns):
            snd.pready(int(u), s0)
            s0.synchronize()
            readied[u] = True
            want = oracle.xpart_arrived(Ns, sb, agg, Nr, rb, readied)
            got = np.array([rcv.parrived(p) for p in range(Nr)])
            np.testing.assert_array_equal(got, want, err_msg=f"after readying {np.nonzero(readied)[0]}")
            host = rbuf.cpu().numpy()
            for p in np.nonzero(want)[0]:
                np.testing.assert_array_equal(host[p * rb:(p + 1) * rb], payload[p * rb:(p + 1) * rb])
            assert rcv.test() == bool(want.all())
        snd.wait()
        assert snd.error()[0] == 0 and rcv.error()[0] == 0
        snd.free()
        rcv.free()


def test_xpart_ll_unsupported_and_size_mismatch():
    """LL lines are laid out per receive partition, so a different partitioning
    cannot use them (PC_ERR_UNSUPPORTED); different TOTAL sizes do not match."""
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        sbuf = torch.zeros(960, dtype=torch.uint8, device="cuda")
        rbuf = torch.zeros_like(sbuf)
        snd = pc.psend_init(sbuf, 2, 480, pc.BYTE, 1, 5, cs[0])
        rcv = pc.precv_init(rbuf, 3, 320, pc.BYTE, 0, 5, cs[1])
        snd.start(s0)
        rcv.start(s1)
        first_prepare([[snd], [rcv]], [s0, s1])
        with pytest.raises(pc.PcError) as ei:
            snd.prequest_create(pc.GRAN_THREAD, 1, pc.COPY_LL)
        assert ei.value.code == pc.ERR_UNSUPPORTED
        snd.prequest_create(pc.GRAN_THREAD, 1, pc.COPY_INLINE)
        snd.pready(0, s0)
        snd.pready(1, s0)
        snd.wait()
        rcv.wait()
        snd.free()
        rcv.free()


# ---------------------------------------------------------------- host progression engine (NEXT-4)
@pytest.mark.parametrize("agg", [1, 4])
def test_host_progression_engine_tagged_epochs(agg):
    """PC_COPY_HOST (the paper's Progression Engine): device
    Pready marks pinned host flags, the library's host thread copies and
    signals.  50 back-to-back epochs of epoch-tagged bytes with a permuted
    Pready order, device Parrived on every partition, host wait/test."""
    partitions, pbytes, E = 16, 4096, 50
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        src = torch.empty(partitions * pbytes, dtype=torch.uint8, device="cuda")
        sbuf, rbuf, out = torch.empty_like(src), torch.empty_like(src), torch.zeros_like(src)
        status = torch.zeros(1, dtype=torch.int32, device="cuda")
        snd = pc.psend_init(sbuf, partitions, pbytes, pc.BYTE, 1, 1, cs[0])
        rcv = pc.precv_init(rbuf, partitions, pbytes, pc.BYTE, 0, 1, cs[1])
        for e in range(E):
            payload = synth.bytes_tagged(SEED, 5, e, partitions * pbytes)
            src.copy_(torch.from_numpy(payload))
            torch.cuda.synchronize()
            snd.start(s0)
            rcv.start(s1)
            if e == 0:
                first_prepare([[snd], [rcv]], [s0, s1])
                sq = snd.prequest_create(pc.GRAN_BLOCK, agg, pc.COPY_HOST)
                rq = rcv.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
            else:
                rcv.pbuf_prepare(s1)
                snd.pbuf_prepare(s0)
            apps.produce(sbuf, src, partitions, pbytes, apps.GRAN_BLOCK, sq, order_stride=5, stream=s0)
            apps.check_recv(rq, rbuf, out, partitions, pbytes, status, blocks=16, stream=s1)
            if e % 2:
                snd.wait()
                rcv.wait()
            else:
                snd.wait_on_stream(s0)
                rcv.wait_on_stream(s1)
                torch.cuda.synchronize()
            assert int(status.item()) == 0
            np.testing.assert_array_equal(rbuf.cpu().numpy(), payload)
            np.testing.assert_array_equal(out.cpu().numpy(), payload)
        assert snd.error()[0] == 0 and rcv.error()[0] == 0
        snd.free()
        rcv.free()


def test_host_progression_engine_unsupported_cases():
    """PE mode moves p2p bytes only: no allreduce requests, no different
    partitionings (its signals are stores, R30 needs counters)."""
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        sbuf = torch.zeros(960, dtype=torch.uint8, device="cuda")
        rbuf = torch.zeros_like(sbuf)
        snd = pc.psend_init(sbuf, 2, 480, pc.BYTE, 1, 6, cs[0])
        rcv = pc.precv_init(rbuf, 3, 320, pc.BYTE, 0, 6, cs[1])
        snd.start(s0)
        rcv.start(s1)
        first_prepare([[snd], [rcv]], [s0, s1])
        with pytest.raises(pc.PcError) as ei:
            snd.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_HOST)
        assert ei.value.code == pc.ERR_UNSUPPORTED
        snd.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
        snd.pready(0, s0)
        snd.pready(1, s0)
        snd.wait()
        rcv.wait()
        snd.free()
        rcv.free()


@pytest.mark.parametrize("t", [1, 7, 64, 1024])
@pytest.mark.parametrize("mode", ["thread", "warp", "block", "thread_agg_block"])
def test_fig3_single_block_pready(t, mode):
    """Fig 3 analogue's kernel (one block of t threads, 8 B each, Pready at
    thread / warp / block granularity or thread with aggregation to one
    transport partition): bytes delivered every epoch, cost recorded."""
    gran = {"thread": apps.GRAN_THREAD, "warp": apps.GRAN_WARP, "block": apps.GRAN_BLOCK,
            "thread_agg_block": apps.GRAN_THREAD}[mode]
    if gran == apps.GRAN_WARP and t % 32:
        pytest.skip("warp granularity needs whole warps (reading R11)")
    n = 2 * t
    parts = {apps.GRAN_THREAD: t, apps.GRAN_WARP: t // 32, apps.GRAN_BLOCK: 1}[gran]
    agg = parts if mode == "thread_agg_block" else 1
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        A = torch.from_numpy(synth.uniform_f32(SEED, 0, t, n)).cuda()
        B = torch.from_numpy(synth.uniform_f32(SEED, 1, t, n)).cuda()
        Cb, R = torch.empty(n, device="cuda"), torch.zeros(n, device="cuda")
        ns = torch.zeros(1, dtype=torch.int64, device="cuda")
        snd = pc.psend_init(Cb, parts, n // parts, pc.FLOAT32, 1, 2, cs[0])
        rcv = pc.precv_init(R, parts, n // parts, pc.FLOAT32, 0, 2, cs[1])
        for e in range(3):
            R.zero_()
            torch.cuda.synchronize()
            snd.start(s0)
            rcv.start(s1)
            if e == 0:
                first_prepare([[snd], [rcv]], [s0, s1])
                sq = snd.prequest_create(gran, agg, pc.COPY_INLINE)
            else:
                rcv.pbuf_prepare(s1)
                snd.pbuf_prepare(s0)
            apps.pready_cost(A, B, Cb, t, gran, sq, ns, stream=s0)
            snd.wait_on_stream(s0)
            rcv.wait_on_stream(s1)
            torch.cuda.synchronize()
            want = (A.cpu().numpy() + B.cpu().numpy()).astype(np.float32)
            np.testing.assert_array_equal(R.cpu().numpy(), want)
            assert 0 < int(ns.item()) < 10**8
        assert snd.error()[0] == 0 and rcv.error()[0] == 0
        snd.free()
        rcv.free()


@pytest.mark.parametrize("gran", [apps.GRAN_THREAD, apps.GRAN_WARP])
@pytest.mark.parametrize("agg", [1024, 5000, "all"])
@pytest.mark.parametrize("copy", [pc.COPY_INLINE, pc.COPY_ENGINE, pc.COPY_LL, pc.COPY_HOST])
def test_two_level_aggregation_counters(gran, agg, copy):
    """g >= 1024: two-level counting (reading R32) — sub-counters of 256
    partitions, ragged last sub-group (g = 5000) and last transport partition;
    byte-exact vs O1 over several epochs.  Every copy mode goes through the
    counters: INLINE / ENGINE (publish / mark_ready), LL (ll_account, 4 MiB
    within the LL cap) and HOST (mark_ready into pinned host memory)."""
    n = 1 << 20
    partitions = n // GRAN_ELEMS[gran]
    run_vecadd(n, gran, partitions if agg == "all" else min(agg, partitions), copy, epochs=3)


_SCOPE_PROBE = r"""
import ctypes, os, sys
sys.path.insert(0, os.environ["PC_ROOT"]); sys.path.insert(0, os.path.join(os.environ["PC_ROOT"], "tests"))
import torch
import paper_conf_sc_temucinslsga24_b200 as pc
from gpu_util import comms, first_prepare
with comms(2) as cs:
    st = torch.cuda.Stream()
    a, b = torch.zeros(1024, device="cuda"), torch.zeros(1024, device="cuda")
    snd = pc.psend_init(a, 4, 256, pc.FLOAT32, 1, 3, cs[0])
    rcv = pc.precv_init(b, 4, 256, pc.FLOAT32, 0, 3, cs[1])
    snd.start(st); rcv.start(st)
    first_prepare([[snd], [rcv]], [st, st])
    pq = snd.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
    # pc_prequest_t.sys_scope: after 6 x 4-B fields, part_bytes and 11 pointers (include/pc_prequest.h)
    print(int.from_bytes(pq.buf.raw[128:132], "little"))
    snd.pready_range(0, 3, st)
    snd.wait(); rcv.wait()
    assert snd.error() == (0, 0) and rcv.error() == (0, 0)
    snd.free(); rcv.free()
"""


@pytest.mark.parametrize("force", ["0", "1"])
def test_force_sys_scope_env(force):
    """PC_FORCE_SYS_SCOPE=1 (tools/gpu_sys_scope_check.sh runs the whole GPU
    suite with it) really gives ranks of one GPU system-scope ordering."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, PC_ROOT=root, PC_FORCE_SYS_SCOPE=force)
    p = subprocess.run([sys.executable, "-c", _SCOPE_PROBE], capture_output=True, text=True, env=env, timeout=240)
    assert p.returncode == 0, p.stderr[-2000:]
    assert p.stdout.strip().splitlines()[-1] == force


# ------------------------------------------------ stream waits over many flag words (session 2)
@pytest.mark.parametrize("Ns,Nr", [(100003, 100003), (3000, 5000), (5000, 3000)])
def test_stream_wait_many_partitions(Ns, Nr):
    """MPI_Wait on the stream over ~10^5 flag words (the bulk wait: relaxed
    16-B loads over up to one block per SM, head / tail words at odd
    offsets) and over per-receive-partition counters of different
    partitionings (R30, grid-stride over several blocks): every byte
    delivered over 3 epochs, MPI_Test false before the sender's Pready
    (the pending-count path) and true after."""
    total = Ns * 16 if Ns == Nr else 240000
    sb, rb = total // Ns, total // Nr
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        sbuf = torch.empty(total, dtype=torch.uint8, device="cuda")
        rbuf = torch.zeros_like(sbuf)
        snd = pc.psend_init(sbuf, Ns, sb, pc.BYTE, 1, 21, cs[0])
        rcv = pc.precv_init(rbuf, Nr, rb, pc.BYTE, 0, 21, cs[1])
        for e in range(3):
            payload = synth.bytes_tagged(SEED, 4, e, total)
            sbuf.copy_(torch.from_numpy(payload))
            torch.cuda.synchronize()
            snd.start(s0)
            rcv.start(s1)
            if e == 0:
                first_prepare([[snd], [rcv]], [s0, s1])
                snd.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
                rcv.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
            else:
                rcv.pbuf_prepare(s1)
                snd.pbuf_prepare(s0)
            torch.cuda.synchronize()
            assert not rcv.test()  # nothing readied yet in this epoch
            snd.pready_range(0, Ns - 1, s0)
            snd.wait_on_stream(s0)
            rcv.wait_on_stream(s1)
            torch.cuda.synchronize()
            assert snd.error()[0] == 0 and rcv.error()[0] == 0, (snd.error(), rcv.error())
            np.testing.assert_array_equal(rbuf.cpu().numpy(), payload)
            assert rcv.test()
        snd.free()
        rcv.free()


@pytest.mark.parametrize("elem,pbytes,agg", [(16, 4096, 1), (4, 1024, 1), (8, 2048, 3), (16, 1000, 1), (4, 1022, 2),
                                             (16, 16, 1)])
@pytest.mark.parametrize("copy", [pc.COPY_INLINE, pc.COPY_ENGINE])
def test_pready_block_put_element_types(elem, pbytes, agg, copy):
    """pc_pready_block_put with 4-, 8- and 16-byte elements from a 256-thread
    producer over 37 partitions (more than one per CTA), and the fallback to
    pc_pready_block when the partition size does not suit the element type or
    the copy mode is not INLINE: byte-exact delivery over 2 epochs."""
    parts = 37
    total = parts * pbytes
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        src = torch.empty(total, dtype=torch.uint8, device="cuda")
        sbuf, rbuf = torch.zeros_like(src), torch.zeros_like(src)
        snd = pc.psend_init(sbuf, parts, pbytes, pc.BYTE, 1, 23, cs[0])
        rcv = pc.precv_init(rbuf, parts, pbytes, pc.BYTE, 0, 23, cs[1])
        for e in range(2):
            payload = synth.bytes_tagged(SEED, 5, e, total)
            src.copy_(torch.from_numpy(payload))
            torch.cuda.synchronize()
            snd.start(s0)
            rcv.start(s1)
            if e == 0:
                first_prepare([[snd], [rcv]], [s0, s1])
                sq = snd.prequest_create(pc.GRAN_BLOCK, agg, copy)
                rcv.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
            else:
                rcv.pbuf_prepare(s1)
                snd.pbuf_prepare(s0)
            apps.produce_put(sbuf, src, parts, pbytes, elem, sq, threads=256, blocks=8, stream=s0)
            snd.wait_on_stream(s0)
            rcv.wait_on_stream(s1)
            torch.cuda.synchronize()
            assert snd.error()[0] == 0 and rcv.error()[0] == 0, (snd.error(), rcv.error())
            np.testing.assert_array_equal(rbuf.cpu().numpy(), payload)
        snd.free()
        rcv.free()


def test_persistent_put_many_epochs():
    """200 back-to-back epochs of the persistent register Kernel Copy with
    batched releases (epoch-tagged inputs, no host sync between epochs except
    every 50th): every epoch's bytes arrive intact (the last epoch checked
    byte-exact, every 50th epoch's too), no device error."""
    n = 2048 * 600  # 600 logical blocks over 296 CTAs: partial batches every epoch
    with comms(2) as cs:
        st = torch.cuda.Stream()
        A = torch.empty(n, device="cuda")
        B = torch.zeros(n, device="cuda")
        Cb = torch.empty(n, device="cuda")
        R = torch.zeros(n, device="cuda")
        parts = n // 2048
        snd = pc.psend_init(Cb, parts, 2048, pc.FLOAT32, 1, 31, cs[0])
        rcv = pc.precv_init(R, parts, 2048, pc.FLOAT32, 0, 31, cs[1])
        base = torch.arange(n, device="cuda", dtype=torch.float32)
        torch.cuda.synchronize()
        for e in range(200):
            with torch.cuda.stream(st):
                A.copy_(base + float(e))  # epoch tag in every element
            if e == 0:
                snd.start(st)
                rcv.start(st)
                first_prepare([[snd], [rcv]], [st, st])
                sq = snd.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
                rcv.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
            else:
                pc.epoch_all([snd, rcv], False, st)
            apps.vecadd(A, B, Cb, n, apps.GRAN_BLOCK_PUT, sq, st, persistent=True)
            pc.waitall_on_stream([snd, rcv], st)
            if e % 50 == 49:
                torch.cuda.synchronize()
                assert snd.error()[0] == 0 and rcv.error()[0] == 0
                assert torch.equal(R, base + float(e)), f"epoch {e}"
        snd.free()
        rcv.free()


@pytest.mark.parametrize("pbytes,parts,agg", [(8, 37, 2), (16, 101, 1), (48, 33, 8), (8, 1001, 64), (8, 77, 1),
                                              (24, 41, 3), (12, 50, 1)])
def test_engine_small_units(pbytes, parts, agg):
    """ENGINE copy of small transport partitions (<= 512 B: the engine gives
    each lane a unit), including a ragged last transport partition whose
    bytes are not a multiple of 16: byte-exact over 3 epochs."""
    total = parts * pbytes
    with comms(2) as cs:
        s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
        src = torch.empty(total, dtype=torch.uint8, device="cuda")
        sbuf, rbuf = torch.zeros_like(src), torch.zeros_like(src)
        snd = pc.psend_init(sbuf, parts, pbytes, pc.BYTE, 1, 25, cs[0])
        rcv = pc.precv_init(rbuf, parts, pbytes, pc.BYTE, 0, 25, cs[1])
        for e in range(3):
            payload = synth.bytes_tagged(SEED, 6, e, total)
            src.copy_(torch.from_numpy(payload))
            torch.cuda.synchronize()
            snd.start(s0)
            rcv.start(s1)
            if e == 0:
                first_prepare([[snd], [rcv]], [s0, s1])
                sq = snd.prequest_create(pc.GRAN_BLOCK, agg, pc.COPY_ENGINE)
                rcv.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
            else:
                rcv.pbuf_prepare(s1)
                snd.pbuf_prepare(s0)
            apps.produce(sbuf, src, parts, pbytes, apps.GRAN_BLOCK, sq, stream=s0)
            snd.wait_on_stream(s0)
            rcv.wait_on_stream(s1)
            torch.cuda.synchronize()
            assert snd.error()[0] == 0 and rcv.error()[0] == 0, (snd.error(), rcv.error())
            np.testing.assert_array_equal(rbuf.cpu().numpy(), payload)
        snd.free()
        rcv.free()
