"""Thin Python binding over libpc's C ABI (include/pc.h).  Argument
marshalling only: every step of the hot path runs in the CUDA kernels of
libpc.so; PyTorch supplies device memory, streams and (optionally) the
process group used for the bootstrap all-gather.

Names follow the C ABI / the paper (MPI-4 partitioned + MPIX extensions):
``psend_init``, ``precv_init``, ``pallreduce_init``, ``Request.start``,
``Request.pbuf_prepare``, ``Request.prequest_create``, ``Request.wait`` …
"""
from __future__ import annotations

import ctypes as C
import threading
from typing import Callable, Sequence

from . import _lib

INT32, FLOAT32, BYTE, FLOAT64, BF16 = 0, 1, 2, 3, 4
ESIZE = {INT32: 4, FLOAT32: 4, BYTE: 1, FLOAT64: 8, BF16: 2}
SUM, MAX, MIN = 0, 1, 2
GRAN_THREAD, GRAN_WARP, GRAN_BLOCK = 0, 1, 2
COPY_INLINE, COPY_ENGINE, COPY_LL, COPY_HOST = 0, 1, 2, 3
ALGO_AUTO, ALGO_RING, ALGO_RD, ALGO_DIRECT, ALGO_DIRECT_PUSH, ALGO_LL = 0, 1, 2, 3, 4, 5
KIND_PSEND, KIND_PRECV, KIND_PALLREDUCE = 1, 2, 3

SUCCESS, ERR_ARG, ERR_CUDA, ERR_STATE, ERR_MATCH, ERR_TIMEOUT, ERR_DEVICE, ERR_NOMEM, ERR_UNSUPPORTED = (
    0, -1, -2, -3, -4, -5, -6, -7, -8)


class PcError(RuntimeError):
    def __init__(self, code: int, what: str):
        msg = _lib.pc().pc_strerror(code).decode()
        super().__init__(f"{what}: {msg} ({code})")
        self.code = code


def check(rc: int, what: str) -> int:
    if rc < 0:
        raise PcError(rc, what)
    return rc


def _ptr(x) -> int:
    """Device pointer of a torch tensor, or an int address, or None."""
    if x is None:
        return 0
    if isinstance(x, int):
        return x
    return x.data_ptr()


def _stream(s) -> int:
    if s is None:
        return 0
    if isinstance(s, int):
        return s
    return s.cuda_stream


def _dtype_code(t) -> int:
    import torch
    if t.dtype == torch.float32:
        return FLOAT32
    if t.dtype == torch.int32:
        return INT32
    if t.dtype == torch.uint8:
        return BYTE
    if t.dtype == torch.float64:
        return FLOAT64
    if t.dtype == torch.bfloat16:
        return BF16
    raise TypeError(f"unsupported dtype {t.dtype}")


class Comm:
    """pc_comm_t.  Use Comm.from_process_group (one process per GPU) or
    local_comms (several ranks in this process, e.g. virtual ranks on one GPU)."""

    def __init__(self, handle: int, keepalive=()):
        self.handle = handle
        self._keep = keepalive
        r, s, w = C.c_int32(), C.c_int32(), C.c_int32()
        check(_lib.pc().pc_comm_rank(handle, C.byref(r)), "pc_comm_rank")
        check(_lib.pc().pc_comm_size(handle, C.byref(s)), "pc_comm_size")
        check(_lib.pc().pc_comm_engine_warps(handle, C.byref(w)), "pc_comm_engine_warps")
        self.rank, self.size, self.engine_warps = r.value, s.value, w.value
        check(_lib.pc().pc_comm_overlap_warps(handle, C.byref(w)), "pc_comm_overlap_warps")
        self.overlap_warps = w.value
        self.requests: list[Request] = []

    @staticmethod
    def create(rank: int, size: int, device: int, allgather: Callable[[bytes], bytes] | None = None) -> "Comm":
        """allgather(bytes) -> bytes of size*len; run under the caller's group."""
        keep = ()
        fnptr = None
        if size > 1:
            def _cb(send, nbytes, recv, ctx):
                try:
                    data = C.string_at(send, nbytes)
                    out = allgather(data)
                    assert len(out) == nbytes * size
                    C.memmove(recv, out, len(out))
                    return 0
                except Exception as exc:  # never raise through C
                    print(f"[pc] allgather callback failed: {exc!r}")
                    return -1
            fnptr = _lib.AGFN(_cb)
            keep = (fnptr,)
        h = C.c_void_p()
        check(_lib.pc().pc_comm_create(rank, size, device, C.cast(fnptr, C.c_void_p) if fnptr else None, None,
                                       C.byref(h)), "pc_comm_create")
        return Comm(h.value, keep)

    @staticmethod
    def from_process_group(device: int, group=None) -> "Comm":
        import torch
        import torch.distributed as dist
        rank, size = dist.get_rank(group), dist.get_world_size(group)
        backend = dist.get_backend(group)

        def ag(data: bytes) -> bytes:
            t = torch.frombuffer(bytearray(data), dtype=torch.uint8)
            if backend == "nccl":
                t = t.cuda(device)
            out = [torch.empty_like(t) for _ in range(size)]
            dist.all_gather(out, t, group=group)
            return b"".join(bytes(o.cpu().numpy().tobytes()) for o in out)

        return Comm.create(rank, size, device, ag)

    def destroy(self):
        if self.handle:
            for r in list(self.requests):
                r.free()
            check(_lib.pc().pc_comm_destroy(self.handle), "pc_comm_destroy")
            self.handle = 0


class LocalGroup:
    def __init__(self, size: int):
        h = C.c_void_p()
        check(_lib.pc().pc_local_group_create(size, C.byref(h)), "pc_local_group_create")
        self.handle = h.value
        self.size = size

    def ctx(self, rank: int) -> int:
        return _lib.pc().pc_local_group_ctx(self.handle, rank)

    def destroy(self):
        if self.handle:
            _lib.pc().pc_local_group_destroy(self.handle)
            self.handle = 0


def run_ranks(fns: Sequence[Callable[[], object]]) -> list:
    """Run one callable per rank on its own thread (the blocking bootstrap
    all-gather of local groups needs every rank to arrive)."""
    out = [None] * len(fns)
    errs: list[BaseException] = []

    def go(i):
        try:
            out[i] = fns[i]()
        except BaseException as exc:  # propagate to the caller
            errs.append(exc)

    ts = [threading.Thread(target=go, args=(i,)) for i in range(len(fns))]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    if errs:
        raise errs[0]
    return out


def local_comms(size: int, devices: int | Sequence[int] = 0) -> tuple[LocalGroup, list[Comm]]:
    """`size` ranks living in this process (virtual ranks when they share a
    device; devices=-1 gives host-only "dry" comms)."""
    if isinstance(devices, int):
        devices = [devices] * size
    g = LocalGroup(size)
    fn = C.cast(_lib.pc().pc_local_allgather, C.c_void_p)

    def mk(r):
        def f():
            h = C.c_void_p()
            check(_lib.pc().pc_comm_create(r, size, devices[r], fn, g.ctx(r), C.byref(h)), "pc_comm_create")
            return Comm(h.value, (g,))
        return f

    comms = run_ranks([mk(r) for r in range(size)])
    return g, comms


class Prequest:
    """pc_prequest_t as opaque bytes (passed by pointer to launchers that pass
    it by value to kernels)."""

    def __init__(self):
        n = _lib.pc().pc_prequest_size()
        self.buf = C.create_string_buffer(n)

    @property
    def ptr(self) -> int:
        return C.addressof(self.buf)


class Request:
    def __init__(self, comm: Comm, handle: int, kind: int, nbytes: int, partitions: int):
        self.comm = comm
        self.handle = handle
        self.kind = kind
        self.nbytes = nbytes
        self.partitions = partitions
        self.preq: Prequest | None = None
        comm.requests.append(self)

    # -- epoch
    def start(self, stream=None):
        check(_lib.pc().pc_start(self.handle, _stream(stream)), "pc_start")

    def pbuf_prepare(self, stream=None):
        check(_lib.pc().pc_pbuf_prepare(self.handle, _stream(stream)), "pc_pbuf_prepare")

    def prequest_create(self, gran: int = GRAN_BLOCK, aggregation: int = 1, copy: int = COPY_INLINE) -> Prequest:
        p = Prequest()
        check(_lib.pc().pc_prequest_create(self.handle, gran, aggregation, copy, p.ptr), "pc_prequest_create")
        self.preq = p
        return p

    # -- completion
    def wait(self):
        check(_lib.pc().pc_wait(self.handle), "pc_wait")

    def wait_on_stream(self, stream=None):
        check(_lib.pc().pc_wait_on_stream(self.handle, _stream(stream)), "pc_wait_on_stream")

    def test(self) -> bool:
        f = C.c_int32()
        check(_lib.pc().pc_test(self.handle, C.byref(f)), "pc_test")
        return bool(f.value)

    def parrived(self, partition: int) -> bool:
        f = C.c_int32()
        check(_lib.pc().pc_parrived(self.handle, partition, C.byref(f)), "pc_parrived")
        return bool(f.value)

    def pready(self, partition: int, stream=None):
        check(_lib.pc().pc_pready(partition, self.handle, _stream(stream)), "pc_pready")

    def pready_range(self, lo: int, hi: int, stream=None):
        check(_lib.pc().pc_pready_range(lo, hi, self.handle, _stream(stream)), "pc_pready_range")

    # -- introspection
    def info(self) -> dict:
        a, s, w = C.c_int32(), C.c_int32(), C.c_int32()
        q = C.c_int64()
        check(_lib.pc().pc_request_info(self.handle, C.byref(a), C.byref(s), C.byref(q), C.byref(w)), "info")
        return {"algo": a.value, "algo_name": {1: "ring", 2: "rd", 3: "direct", 4: "direct_push", 5: "ll"}.get(a.value, "?"), "slices": s.value,
                "slice_elems": q.value, "engine_warps": w.value}

    def match(self) -> tuple[int, int]:
        p, i = C.c_int32(), C.c_int32()
        check(_lib.pc().pc_request_match(self.handle, C.byref(p), C.byref(i)), "pc_request_match")
        return p.value, i.value

    WORDS = {"flags": 0, "sent": 1, "cnt": 2, "ready": 3, "done": 4, "rtr": 5, "epoch": 6, "layout": 7, "err": 8}

    def words(self, which: str, offset: int, n: int):
        """Read control words (debug/tests): flags, sent, cnt, ready, done, rtr, epoch."""
        import numpy as np
        out = np.zeros(max(n, 1), dtype=np.uint32)
        check(_lib.pc().pc_request_words(self.handle, self.WORDS[which], offset, n, out.ctypes.data),
              "pc_request_words")
        return out[:n]

    def peer_buffer(self, j: int = 0) -> int:
        """pc_request_peer_buffer: peer-mapped address of a peer's receive
        buffer (send: the receiver's; DIRECT collective: peer (r+1+j) mod P)."""
        p = C.c_void_p()
        check(_lib.pc().pc_request_peer_buffer(self.handle, j, C.byref(p)), "pc_request_peer_buffer")
        return p.value or 0

    def set_overlap(self, on: bool = True):
        """pc_request_set_overlap: fork the engine at the epoch's control calls
        (default, overlaps the producer) or at the wait (no overlap)."""
        check(_lib.pc().pc_request_set_overlap(self.handle, int(on)), "pc_request_set_overlap")

    def set_timing(self, on: bool = True):
        check(_lib.pc().pc_request_set_timing(self.handle, int(on)), "pc_request_set_timing")

    def engine_times(self, max_n: int = 65536):
        """Durations (ms) of the engine launches since the last call (timing on)."""
        import numpy as np
        out = np.zeros(max_n, dtype=np.float32)
        n = check(_lib.pc().pc_request_engine_times(self.handle, out.ctypes.data, max_n), "engine_times")
        return out[:n]

    def error(self) -> tuple[int, int]:
        c, p = C.c_int32(), C.c_int32()
        check(_lib.pc().pc_request_error(self.handle, C.byref(c), C.byref(p)), "pc_request_error")
        return c.value, p.value

    def free(self):
        if self.handle:
            h = C.c_void_p(self.handle)
            check(_lib.pc().pc_request_free(C.byref(h)), "pc_request_free")
            self.handle = 0
            if self in self.comm.requests:
                self.comm.requests.remove(self)


def _handles(reqs):
    arr = (C.c_void_p * len(reqs))(*[q.handle for q in reqs])
    return arr


def waitall_on_stream(reqs, stream=None):
    """MPI_Waitall, stream-ordered: the p2p waits of all requests in one kernel."""
    check(_lib.pc().pc_waitall_on_stream(len(reqs), _handles(reqs), _stream(stream)), "pc_waitall_on_stream")


def startall(reqs, stream=None):
    """MPI_Startall: one kernel advances every request's epoch."""
    check(_lib.pc().pc_startall(len(reqs), _handles(reqs), _stream(stream)), "pc_startall")


def epoch_all(reqs, pready: bool = False, stream=None):
    """pc_epoch_all: Start + Pbuf_prepare (+ Pready of every partition of
    allreduce-kind requests) of already-exchanged requests in ONE kernel."""
    check(_lib.pc().pc_epoch_all(len(reqs), _handles(reqs), 1 if pready else 0, _stream(stream)), "pc_epoch_all")


def pbuf_prepare_all(reqs, stream=None):
    """Ready-to-receive of already-exchanged requests in one kernel."""
    check(_lib.pc().pc_pbuf_prepare_all(len(reqs), _handles(reqs), _stream(stream)), "pc_pbuf_prepare_all")


def preadyall(reqs, stream=None):
    """Host Pready of every partition of every request, one kernel."""
    check(_lib.pc().pc_preadyall(len(reqs), _handles(reqs), _stream(stream)), "pc_preadyall")


def psend_init(buf, partitions: int, count: int, dtype: int, dest: int, tag: int, comm: Comm) -> Request:
    h = C.c_void_p()
    check(_lib.pc().pc_psend_init(_ptr(buf), partitions, count, dtype, dest, tag, comm.handle, C.byref(h)),
          "pc_psend_init")
    es = ESIZE[dtype]
    return Request(comm, h.value, KIND_PSEND, partitions * count * es, partitions)


def precv_init(buf, partitions: int, count: int, dtype: int, source: int, tag: int, comm: Comm) -> Request:
    h = C.c_void_p()
    check(_lib.pc().pc_precv_init(_ptr(buf), partitions, count, dtype, source, tag, comm.handle, C.byref(h)),
          "pc_precv_init")
    es = ESIZE[dtype]
    return Request(comm, h.value, KIND_PRECV, partitions * count * es, partitions)


def pallreduce_init(sendbuf, recvbuf, partitions: int, count: int, dtype: int, op: int, algo: int,
                    comm: Comm) -> Request:
    h = C.c_void_p()
    check(_lib.pc().pc_pallreduce_init(_ptr(sendbuf), _ptr(recvbuf), partitions, count, dtype, op, algo,
                                       comm.handle, C.byref(h)), "pc_pallreduce_init")
    return Request(comm, h.value, KIND_PALLREDUCE, partitions * count * ESIZE[dtype], partitions)


def preduce_scatter_init(sendbuf, recvbuf, partitions: int, count: int, dtype: int, op: int, comm: Comm) -> Request:
    """Partitioned reduce-scatter (pc.h): sendbuf partitions x P x count, recvbuf partitions x count."""
    h = C.c_void_p()
    check(_lib.pc().pc_preduce_scatter_init(_ptr(sendbuf), _ptr(recvbuf), partitions, count, dtype, op,
                                            comm.handle, C.byref(h)), "pc_preduce_scatter_init")
    return Request(comm, h.value, KIND_PALLREDUCE, partitions * count * ESIZE[dtype], partitions)


def pallgather_init(sendbuf, recvbuf, partitions: int, count: int, dtype: int, comm: Comm) -> Request:
    """Partitioned allgather (pc.h): sendbuf partitions x count, recvbuf P x partitions x count."""
    h = C.c_void_p()
    check(_lib.pc().pc_pallgather_init(_ptr(sendbuf), _ptr(recvbuf), partitions, count, dtype, comm.handle,
                                       C.byref(h)), "pc_pallgather_init")
    return Request(comm, h.value, KIND_PALLREDUCE, partitions * count * ESIZE[dtype], partitions)


def pbcast_init(buf, partitions: int, count: int, dtype: int, root: int, comm: Comm) -> Request:
    """Partitioned broadcast (pc.h): the root's Pready(u) delivers buf[u] to every rank."""
    h = C.c_void_p()
    check(_lib.pc().pc_pbcast_init(_ptr(buf), partitions, count, dtype, root, comm.handle, C.byref(h)),
          "pc_pbcast_init")
    return Request(comm, h.value, KIND_PALLREDUCE, partitions * count * ESIZE[dtype], partitions)


# ------------------------------------------------------------------ pure host logic
def launch_count() -> int:
    """Kernels libpc launched in this process so far."""
    return int(_lib.pc().pc_launch_count())


def schedule_ring(P: int, r: int):
    import numpy as np
    out = np.zeros((max(2 * (P - 1), 1), 5), dtype=np.int32)
    n = check(_lib.pc().pc_schedule_ring(P, r, out.ctypes.data_as(_lib.PI32)), "pc_schedule_ring")
    return out[:n]


def schedule_rd(P: int, r: int):
    import numpy as np
    out = np.zeros((8, 5), dtype=np.int32)
    n = check(_lib.pc().pc_schedule_rd(P, r, out.ctypes.data_as(_lib.PI32)), "pc_schedule_rd")
    return out[:n]


def chunk_bounds(L: int, P: int):
    import numpy as np
    out = np.zeros(P + 1, dtype=np.int64)
    check(_lib.pc().pc_chunk_bounds(L, P, out.ctypes.data_as(_lib.PI64)), "pc_chunk_bounds")
    return out
