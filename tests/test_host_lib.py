"""CPU tests of the C-ABI library: it loads, exports every symbol include/*.h
declares, and its pure host logic (schedules, chunking, matching, request
state machine) is right.  No compute calls — there is no GPU here.  Host-only
("dry", device = -1) comms run the real bootstrap / exchange / matching code."""
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
import paper_conf_sc_temucinslsga24_b200 as pc
from paper_conf_sc_temucinslsga24_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_header_symbol():
    lib = _lib.pc()
    syms = _lib.header_symbols("pc.h")
    assert len(syms) >= 30
    for s in syms:
        assert hasattr(lib, s), f"libpc.so does not export {s}"
    assert lib.pc_prequest_size() == _lib.apps().pcapp_prequest_size()


def test_app_launchers_reject_bad_arguments_before_the_gpu():
    """The producer launchers of libpcapps (session 2: the persistent vector
    add, the one-launch multi-rank BCE producer) validate their arguments on
    the host and return -1 without touching the GPU."""
    import ctypes as C
    lib = _lib.apps()
    for name in ("pcapp_vecadd", "pcapp_vecadd_persistent", "pcapp_bce_grad_multi"):
        assert hasattr(lib, name)
    a16 = C.c_void_p(0x10000)
    a8 = C.c_void_p(0x10008)
    assert lib.pcapp_vecadd(a16, a16, a16, 3, -1, None, None) == -1  # odd element count
    assert lib.pcapp_vecadd(a16, a16, a16, 4, 4, None, None) == -1  # unknown granularity
    assert lib.pcapp_vecadd(a16, a16, a16, 4, 2, None, None) == -1  # Pready without a prequest
    assert lib.pcapp_vecadd_persistent(a8, a16, a16, 4, -1, None, None) == -1  # TMA needs 16-B sources
    assert lib.pcapp_vecadd_persistent(a16, a16, a16, 1 << 33, -1, None, None) == -1  # 32-bit indices
    assert lib.pcapp_vecadd_persistent(a16, a16, a16, 4, 3, None, None) == -1  # block_put needs a prequest
    arr = (C.c_void_p * 9)(*([0x10000] * 9))
    assert lib.pcapp_bce_grad_multi(0, arr, arr, arr, 4, 16, 1.0, 0, None, 0, None) == -1  # no ranks
    assert lib.pcapp_bce_grad_multi(9, arr, arr, arr, 4, 16, 1.0, 0, None, 0, None) == -1  # > 8 ranks
    assert lib.pcapp_bce_grad_multi(2, arr, arr, arr, 0, 16, 1.0, 0, None, 0, None) == -1  # no partitions
    q = C.create_string_buffer(4096)  # (a request image: never read before the argument checks fail)
    assert lib.pcapp_produce_put(a16, a16, 4, 4097, 16, 256, 0, q, None) == -1  # > one element per thread
    assert lib.pcapp_produce_put(a16, a16, 4, 64, 16, 16, 0, q, None) == -1  # < one warp
    assert lib.pcapp_produce_put(a16, a16, 4, 64, 16, 256, 0, None, None) == -1  # no prequest


def test_no_oracle_in_product():
    """The product never links or imports the oracle."""
    out = subprocess.run(["nm", "-D", "--defined-only", _lib.LIBPC], capture_output=True, text=True).stdout
    assert "orc_" not in out
    for f in os.listdir(os.path.join(ROOT, "paper_conf_sc_temucinslsga24_b200")):
        if f.endswith(".py"):
            src = open(os.path.join(ROOT, "paper_conf_sc_temucinslsga24_b200", f)).read()
            assert "import oracle" not in src and "from oracle" not in src


@pytest.mark.parametrize("P", range(1, 9))
def test_ring_schedule_matches_oracle_alg1(P):
    """Two independent implementations of Alg 1 agree."""
    for r in range(P):
        np.testing.assert_array_equal(pc.schedule_ring(P, r), oracle.alg1_table(P, r))


@pytest.mark.parametrize("P", [1, 2, 4, 8, 16])
def test_rd_schedule(P):
    k = int(np.log2(P))
    for r in range(P):
        t = pc.schedule_rd(P, r)
        assert len(t) == k
        partners = sorted(int(row[0]) for row in t)
        assert partners == sorted(r ^ (1 << j) for j in range(k))
        # symmetric: my partner at step j has me as its partner at step j
        for j, row in enumerate(t):
            assert pc.schedule_rd(P, int(row[0]))[j][0] == r


def test_rd_schedule_rejects_non_power_of_two():
    with pytest.raises(pc.PcError):
        pc.schedule_rd(6, 0)


@pytest.mark.parametrize("L", [0, 1, 3, 4, 5, 16, 17, 64, 1000, 300001])
@pytest.mark.parametrize("P", [1, 2, 3, 5, 8])
def test_chunk_bounds_match_oracle(L, P):
    b = pc.chunk_bounds(L, P)
    assert b[0] == 0 and b[-1] == L and (np.diff(b) >= 0).all()
    ids = oracle.chunk_ids(L, P, 1)
    for c in range(P):
        assert (ids[b[c]:b[c + 1]] == c).all()
    for c in range(1, P):
        if b[c] < L:
            assert b[c] % 4 == 0, "chunk starts are 16-byte aligned (reading R4)"


def _dry(P):
    return pc.local_comms(P, -1)


def test_dry_p2p_matching_by_tag_and_order():
    g, cs = _dry(2)
    # rank 0 posts two sends with tag 5 and one with tag 9; rank 1 posts the
    # receives in a different order: matching is by (peer, tag, posting order)
    s = [pc.psend_init(0x1000, 4, 8, pc.FLOAT32, 1, 5, cs[0]), pc.psend_init(0x2000, 4, 8, pc.FLOAT32, 1, 9, cs[0]),
         pc.psend_init(0x3000, 4, 8, pc.FLOAT32, 1, 5, cs[0])]
    r = [pc.precv_init(0x4000, 4, 8, pc.FLOAT32, 0, 9, cs[1]), pc.precv_init(0x5000, 4, 8, pc.FLOAT32, 0, 5, cs[1]),
         pc.precv_init(0x6000, 4, 8, pc.FLOAT32, 0, 5, cs[1])]
    for q in s + r:
        q.start()
    pc.run_ranks([lambda: [q.pbuf_prepare() for q in s], lambda: [q.pbuf_prepare() for q in r]])
    # request indices on the peer: s[0] <-> r[1], s[1] <-> r[0], s[2] <-> r[2]
    assert s[0].match() == (1, 1) and s[1].match() == (1, 0) and s[2].match() == (1, 2)
    assert r[1].match() == (0, 0) and r[0].match() == (0, 1) and r[2].match() == (0, 2)
    for q in s + r:
        q.wait()
        q.free()
    for c in cs:
        c.destroy()
    g.destroy()


@pytest.mark.parametrize("recv,want", [
    ((8, 4, "FLOAT32"), 0),                 # same bytes, different partitions: MPI-4 allows it (R30)
    ((3, 8, "FLOAT32"), pc.ERR_MATCH),      # different total size
    ((4, 8, "INT32"), pc.ERR_MATCH),        # different type signature
    ((8, 0, "FLOAT32"), pc.ERR_MATCH),      # empty vs non-empty
])
def test_dry_p2p_matching_rules(recv, want):
    g, cs = _dry(2)
    a = pc.psend_init(0x1000, 4, 8, pc.FLOAT32, 1, 1, cs[0])
    b = pc.precv_init(0x2000, recv[0], recv[1], getattr(pc, recv[2]), 0, 1, cs[1])
    a.start()
    b.start()
    res = pc.run_ranks([lambda: _try(a.pbuf_prepare), lambda: _try(b.pbuf_prepare)])
    assert res == [want, want]
    if want == 0:
        a.wait()
        b.wait()
    for c in cs:
        c.destroy()
    g.destroy()


def _try(f):
    try:
        f()
        return 0
    except pc.PcError as e:
        return e.code


def test_dry_allreduce_agreement_and_algo_choice():
    g, cs = _dry(4)
    reqs = [pc.pallreduce_init(0, 0, 2, 1 << 20, pc.FLOAT32, pc.SUM, pc.ALGO_AUTO, c) for c in cs]
    small = [pc.pallreduce_init(0, 0, 1, 256, pc.FLOAT32, pc.SUM, pc.ALGO_AUTO, c) for c in cs]
    for q in reqs + small:
        q.start()
    pc.run_ranks([(lambda r=r: (reqs[r].pbuf_prepare(), small[r].pbuf_prepare())) for r in range(4)])
    # AUTO (profiles/r01_sweep_allreduce_pull.jsonl): DIRECT (pull) for 3 <= P <= 8
    # (the one-shot LL variant only from 32 KiB per rank on one GPU)
    assert all(q.info()["algo"] == pc.ALGO_DIRECT for q in reqs)
    assert all(q.info()["algo"] == pc.ALGO_DIRECT for q in small)
    infos = {tuple(sorted(q.info().items())) for q in reqs}
    assert len(infos) == 1, "every rank must derive the same slicing"
    # disagreeing allreduce (different count on rank 3) -> PC_ERR_MATCH everywhere it is checked
    bad = [pc.pallreduce_init(0, 0, 1, 100 if r < 3 else 101, pc.INT32, pc.SUM, pc.ALGO_RING, cs[r]) for r in range(4)]
    for q in bad:
        q.start()
    res = pc.run_ranks([(lambda r=r: _try(bad[r].pbuf_prepare)) for r in range(4)])
    assert all(x == pc.ERR_MATCH for x in res)
    for q in reqs + small:
        q.wait()
    for c in cs:
        c.destroy()
    g.destroy()


def test_dry_state_errors():
    g, cs = _dry(1)
    q = pc.pallreduce_init(0, 0, 1, 16, pc.FLOAT32, pc.SUM, pc.ALGO_RING, cs[0])
    with pytest.raises(pc.PcError) as e:
        q.pbuf_prepare()  # not started
    assert e.value.code == pc.ERR_STATE
    q.start()
    with pytest.raises(pc.PcError) as e:
        q.start()  # start on an active request
    assert e.value.code == pc.ERR_STATE
    q.pbuf_prepare()
    with pytest.raises(pc.PcError) as e:
        q.free()  # free of an active (matched) request
    assert e.value.code == pc.ERR_STATE
    q.wait()
    q.wait()  # wait on an inactive request: success
    q.free()
    cs[0].destroy()
    g.destroy()


def test_bad_arguments():
    g, cs = _dry(2)
    for f in (lambda: pc.psend_init(0, 0, 8, pc.FLOAT32, 1, 0, cs[0]),      # no partitions
              lambda: pc.psend_init(0, 4, 8, pc.FLOAT32, 5, 0, cs[0]),      # bad peer
              lambda: pc.pallreduce_init(0, 0, 1, 8, pc.BYTE, pc.SUM, 0, cs[0]),  # bad dtype
              lambda: pc.pallreduce_init(0, 0, 1, 8, pc.FLOAT32, 7, 0, cs[0])):   # bad op
        with pytest.raises(pc.PcError) as e:
            f()
        assert e.value.code == pc.ERR_ARG
    for c in cs:
        c.destroy()
    g.destroy()


_GLOO_WORKER = r"""
import os, sys
sys.path.insert(0, {root!r})
import torch.distributed as dist
import paper_conf_sc_temucinslsga24_b200 as pc
dist.init_process_group("gloo", rank=int(os.environ["RANK"]), world_size=2)
r = dist.get_rank()
comm = pc.Comm.from_process_group(-1)
assert comm.rank == r and comm.size == 2
if r == 0:
    a = pc.psend_init(0x1000, 4, 8, pc.FLOAT32, 1, 3, comm)
    b = pc.precv_init(0x2000, 4, 8, pc.FLOAT32, 1, 4, comm)
else:
    b = pc.psend_init(0x1000, 4, 8, pc.FLOAT32, 0, 4, comm)
    a = pc.precv_init(0x2000, 4, 8, pc.FLOAT32, 0, 3, comm)
ar = pc.pallreduce_init(0, 0, 3, 1000, pc.FLOAT32, pc.SUM, pc.ALGO_RING, comm)
for q in (a, b, ar):
    q.start()
for q in (a, b, ar):
    q.pbuf_prepare()
# request indices on the peer: rank 0 created (a, b), rank 1 created (b, a)
exp = ((1, 1), (1, 0)) if r == 0 else ((0, 0), (0, 1))
assert (a.match(), b.match()) == exp, (a.match(), b.match())
info = ar.info()
for q in (a, b, ar):
    q.wait()
    q.free()
comm.destroy()
print("OK", r, info["slices"])
dist.destroy_process_group()
"""


def test_gloo_two_process_bootstrap_and_matching(tmp_path):
    """The N>1 host path: two processes, torch.distributed gloo all-gather as
    the bootstrap, request exchange + matching across processes."""
    script = tmp_path / "w.py"
    script.write_text(_GLOO_WORKER.format(root=ROOT))
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", MASTER_PORT=str(29500 + os.getpid() % 1000), WORLD_SIZE="2")
    procs = [subprocess.Popen([sys.executable, str(script)], env=dict(env, RANK=str(r)), stdout=subprocess.PIPE,
                              stderr=subprocess.STDOUT, text=True) for r in range(2)]
    outs = [p.communicate(timeout=120)[0] for p in procs]
    for r, (p, o) in enumerate(zip(procs, outs)):
        assert p.returncode == 0, o
        assert f"OK {r}" in o


@pytest.mark.parametrize("P,nbytes,want", [(2, 1024, "RD"), (2, 32 << 10, "LL"), (2, 64 << 10, "LL"),
                                          (2, 256 << 10, "LL"), (2, 512 << 10, "RD"), (2, 4 << 20, "RD"),
                                          (2, 8 << 20, "DIRECT"), (8, 128 << 10, "DIRECT"),
                                          (3, 1024, "DIRECT"), (8, 1024, "DIRECT"), (8, 64 << 10, "LL"),
                                          (8, 1 << 20, "DIRECT"), (8, 64 << 20, "DIRECT")])
def test_dry_auto_schedule_policy(P, nbytes, want):
    """AUTO on one GPU (dry ranks count as one): the one-shot LL variant from
    32 KiB to 64 KiB per rank (256 KiB for P <= 4), RD for P = 2 up to 4 MiB, DIRECT for P <= 8
    otherwise (beyond DIRECT's peer limit — more ranks than one process can
    host dry — RD for small messages, ring above)."""
    g, cs = _dry(P)
    reqs = [pc.pallreduce_init(0, 0, 1, nbytes // 4, pc.FLOAT32, pc.SUM, pc.ALGO_AUTO, c) for c in cs]
    for q in reqs:
        q.start()
    pc.run_ranks([(lambda r=r: reqs[r].pbuf_prepare()) for r in range(P)])
    assert all(q.info()["algo"] == getattr(pc, "ALGO_" + want) for q in reqs)
    for q in reqs:
        q.wait()
    for c in cs:
        c.destroy()
    g.destroy()


def test_dry_epoch_all_state_rules():
    """pc_epoch_all bookkeeping (no device): needs exchanged, inactive
    requests; Pready of every partition only for allreduce-kind requests;
    at most 16 requests."""
    g, cs = _dry(2)
    ar = [pc.pallreduce_init(0, 0, 2, 64, pc.FLOAT32, pc.SUM, pc.ALGO_RING, c) for c in cs]
    assert _try(lambda: pc.epoch_all(ar, pready=True)) == pc.ERR_STATE  # not exchanged yet
    for q in ar:
        q.start()
    pc.run_ranks([lambda q=q: q.pbuf_prepare() for q in ar])
    assert _try(lambda: pc.epoch_all(ar, pready=True)) == pc.ERR_STATE  # still active
    for q in ar:
        q.wait()
    for _ in range(3):
        pc.epoch_all(ar, pready=True)
        for q in ar:
            q.wait()
    snd = pc.psend_init(0x1000, 4, 8, pc.FLOAT32, 1, 1, cs[0])
    rcv = pc.precv_init(0x2000, 4, 8, pc.FLOAT32, 0, 1, cs[1])
    snd.start()
    rcv.start()
    pc.run_ranks([lambda: snd.pbuf_prepare(), lambda: rcv.pbuf_prepare()])
    snd.wait()
    rcv.wait()
    assert _try(lambda: pc.epoch_all([snd, rcv], pready=True)) == pc.ERR_ARG  # p2p: no library-side Pready
    pc.epoch_all([snd, rcv], pready=False)
    snd.wait()
    rcv.wait()
    for q in ar + [snd, rcv]:
        q.free()
    for c in cs:
        c.destroy()
    g.destroy()


def test_dry_waitall_state_rules():
    """pc_waitall_on_stream bookkeeping (no device): completes every active
    request of the list (a later pc_epoch_all, which needs inactive requests,
    succeeds), skips inactive ones, accepts an empty list."""
    g, cs = _dry(2)
    snd = pc.psend_init(0x1000, 4, 8, pc.FLOAT32, 1, 1, cs[0])
    rcv = pc.precv_init(0x2000, 4, 8, pc.FLOAT32, 0, 1, cs[1])
    ar = [pc.pallreduce_init(0, 0, 2, 64, pc.FLOAT32, pc.SUM, pc.ALGO_RING, c) for c in cs]
    pc.waitall_on_stream([])
    pc.waitall_on_stream([snd, rcv] + ar)  # nothing started: all inactive
    for q in [snd, rcv] + ar:
        q.start()
    pc.run_ranks([lambda: (snd.pbuf_prepare(), ar[0].pbuf_prepare()),
                  lambda: (rcv.pbuf_prepare(), ar[1].pbuf_prepare())])
    assert _try(lambda: pc.epoch_all([snd, rcv] + ar)) == pc.ERR_STATE  # still active
    pc.waitall_on_stream([snd, rcv] + ar)
    for _ in range(3):
        pc.epoch_all([snd, rcv] + ar)
        pc.waitall_on_stream([rcv, snd] + ar)
    for q in [snd, rcv] + ar:
        q.free()
    for c in cs:
        c.destroy()
    g.destroy()


def test_dry_direct_push_variant(monkeypatch):
    """PC_ALGO_DIRECT_PUSH is the DIRECT schedule's PUSH variant: reported as
    such, matched only against itself (every rank must pick the same variant),
    and AUTO picks it with PC_DIRECT_MODE=push."""
    g, cs = _dry(4)
    push = [pc.pallreduce_init(0, 0, 2, 4096, pc.FLOAT32, pc.SUM, pc.ALGO_DIRECT_PUSH, c) for c in cs]
    for q in push:
        q.start()
    pc.run_ranks([(lambda q=q: q.pbuf_prepare()) for q in push])
    assert all(q.info()["algo_name"] == "direct_push" for q in push)
    mixed = [pc.pallreduce_init(0, 0, 1, 64, pc.FLOAT32, pc.SUM, pc.ALGO_DIRECT if r else pc.ALGO_DIRECT_PUSH, cs[r])
             for r in range(4)]
    for q in mixed:
        q.start()
    res = pc.run_ranks([(lambda q=q: _try(q.pbuf_prepare)) for q in mixed])
    assert all(x == pc.ERR_MATCH for x in res)
    monkeypatch.setenv("PC_DIRECT_MODE", "push")
    auto = [pc.pallreduce_init(0, 0, 1, 1 << 22, pc.FLOAT32, pc.SUM, pc.ALGO_AUTO, c) for c in cs]
    for q in auto:
        q.start()
    pc.run_ranks([(lambda q=q: q.pbuf_prepare()) for q in auto])
    assert all(q.info()["algo_name"] == "direct_push" for q in auto)
    for q in push + auto:
        q.wait()
    for q in push + auto + mixed:
        q.free()
    for c in cs:
        c.destroy()
    g.destroy()


def test_dry_epoch_all_beyond_one_kernel():
    """pc_epoch_all takes any number of requests (more than one kernel's
    parameters hold: the device path uses a table-driven kernel); the same
    request twice in one call is refused before any request is touched."""
    g, cs = _dry(2)
    ar = [[pc.pallreduce_init(0, 0, 1, 64, pc.FLOAT32, pc.SUM, pc.ALGO_DIRECT, c) for _ in range(20)] for c in cs]
    flat = ar[0] + ar[1]
    for q in flat:
        q.start()
    pc.run_ranks([(lambda r=r: [q.pbuf_prepare() for q in ar[r]]) for r in range(2)])
    pc.waitall_on_stream(flat)
    for _ in range(3):
        pc.epoch_all(flat, pready=True)
        pc.waitall_on_stream(flat)
    assert _try(lambda: pc.epoch_all(flat + flat[:1], pready=True)) == pc.ERR_ARG
    pc.epoch_all(flat, pready=True)  # nothing was started by the refused call
    pc.waitall_on_stream(flat)
    for q in flat:
        q.free()
    for c in cs:
        c.destroy()
    g.destroy()


def test_dry_overlap_and_inline_rules():
    """pc_request_set_overlap only on inactive requests; an INLINE prequest
    (reading R33) only on DIRECT (PULL) allreduces; pc_epoch_all cannot Pready
    an INLINE allreduce (its Pready folds)."""
    g, cs = _dry(2)
    d = [pc.pallreduce_init(0, 0, 2, 64, pc.FLOAT32, pc.SUM, pc.ALGO_DIRECT, c) for c in cs]
    ring = [pc.pallreduce_init(0, 0, 2, 64, pc.FLOAT32, pc.SUM, pc.ALGO_RING, c) for c in cs]
    for q in d + ring:
        q.set_overlap(False)
        q.set_overlap(True)
        q.start()
    assert _try(lambda: d[0].set_overlap(False)) == pc.ERR_STATE
    pc.run_ranks([(lambda r=r: (d[r].pbuf_prepare(), ring[r].pbuf_prepare())) for r in range(2)])
    for q in ring:
        assert _try(lambda q=q: q.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)) == pc.ERR_UNSUPPORTED
    for q in d:
        q.prequest_create(pc.GRAN_BLOCK, 1, pc.COPY_INLINE)
    for q in d + ring:
        q.wait()
    assert _try(lambda: pc.epoch_all(d, pready=True)) == pc.ERR_ARG
    pc.epoch_all(d, pready=False)
    for q in d:
        q.wait()
    for q in d + ring:
        q.free()
    for c in cs:
        c.destroy()
    g.destroy()


def test_device_header_compiles_in_a_user_kernel(tmp_path):
    """include/pc_device.cuh is the user's device API: a stand-alone user
    translation unit calling every binding (Pready at thread / warp / block
    granularity, the register Kernel Copy with its persistent begin / end,
    the check-once warp Pready, the cooperative INLINE fold, Parrived) builds
    for sm_100a with nvcc alone (no GPU needed)."""
    import shutil
    nvcc = shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc"
    if not os.path.exists(nvcc):
        pytest.skip("nvcc not available")
    src = tmp_path / "user.cu"
    src.write_text(r'''
#include "pc_device.cuh"
__global__ void user_producer(float2 *out, pc_prequest_t sendq, pc_prequest_t recvq, pc_prequest_t arq, int n) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const float2 v = make_float2((float)i, 1.f);
  if (i < n) out[i] = v;
  pc_pready(i, sendq);
  pc_pready_warp(i >> 5, sendq);
  pc_pready_block(blockIdx.x, sendq);
  pc_pready_block_put(blockIdx.x, sendq, (uint64_t)threadIdx.x, v);
  pc_put_state st;
  if (pc_put_begin<float2>(sendq, &st, 4) == 0) {
    pc_pready_block_put(blockIdx.x, sendq, (uint64_t)threadIdx.x, v, st);
    pc_put_end(sendq, st);
  }
  pc_put_state bs;
  if (pc_put_begin<uint8_t>(sendq, &bs, 2) == 0) {
    pc_pready_block(blockIdx.x, sendq, bs);
    pc_put_end(sendq, bs);
  }
  pc_warp_state ws;
  pc_warp_begin(sendq, &ws);
  pc_pready_warp(i >> 5, sendq, ws);
  pc_pready_block_coop(blockIdx.x, arq);
  if (threadIdx.x == 0 && pc_parrived(recvq, blockIdx.x)) out[0].x += 1.f;
  pc_wait_arrived_warp(recvq, blockIdx.x);
}
''')
    inc = os.path.join(ROOT, "include")
    r = subprocess.run([nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-std=c++17", "-DPC_INLINE_ALLREDUCE",
                        "-I", inc, "-c", "-o", str(tmp_path / "user.o"), str(src)], capture_output=True, text=True)
    assert r.returncode == 0, r.stderr[-2000:]
