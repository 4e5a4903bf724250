"""Launchers for libpcapps.so: producer / application kernels compiled against
include/pc_device.cuh (the way a user kernel calls pc_pready / pc_parrived).
Argument marshalling only."""
from __future__ import annotations

import ctypes as C

from . import _lib
from .runtime import Prequest, _ptr, _stream

GRAN_NONE, GRAN_THREAD, GRAN_WARP, GRAN_BLOCK = -1, 0, 1, 2
GRAN_BLOCK_PUT = 3  # block granularity, Kernel Copy from registers (pc_pready_block_put, R35)


def _ok(rc, what):
    if rc != 0:
        raise RuntimeError(f"{what} launch failed ({rc})")


def vecadd(A, B, Cout, n: int, gran: int, preq: Prequest | None, stream=None, persistent: bool = False):
    """C = A + B (fp32, 8 B per thread, 1024-thread blocks) with pc_pready at
    `gran` (thread: partition = thread, warp: = warp, block: = block;
    block_put: = block, each thread's result assigned to the peer from its
    registers).
    persistent: the same partitions and Pready calls from one CTA per
    resident slot walking the logical blocks (next block's operands
    prefetched), instead of one CTA per logical block."""
    fn = _lib.apps().pcapp_vecadd_persistent if persistent else _lib.apps().pcapp_vecadd
    _ok(fn(_ptr(A), _ptr(B), _ptr(Cout), n, gran, preq.ptr if preq else None, _stream(stream)), "vecadd")


def pready_cost(A, B, Cout, threads: int, gran: int, preq: Prequest, out_ns, stream=None):
    """Fig 3 analogue: one block of `threads` threads computes C = A + B and
    Preadies at `gran`; out_ns (int64 device tensor, 1 element) receives the
    block's Pready cost from %globaltimer."""
    _ok(_lib.apps().pcapp_pready_cost(_ptr(A), _ptr(B), _ptr(Cout), threads, gran, preq.ptr, _ptr(out_ns),
                                      _stream(stream)), "pready_cost")


def produce(dst, src, partitions: int, part_bytes: int, gran: int, preq: Prequest, order_stride: int = 1,
            blocks: int = 0, stream=None):
    _ok(_lib.apps().pcapp_produce(_ptr(dst), _ptr(src), partitions, part_bytes, gran, order_stride, blocks,
                                  preq.ptr, _stream(stream)), "produce")


def produce_put(dst, src, partitions: int, part_bytes: int, elem_bytes: int, preq: Prequest, threads: int = 256,
                blocks: int = 0, stream=None):
    """Copy src -> dst partition by partition, handing each thread's element
    (elem_bytes = 4 / 8 / 16) to pc_pready_block_put (R35); part_bytes <=
    threads * elem_bytes."""
    _ok(_lib.apps().pcapp_produce_put(_ptr(dst), _ptr(src), partitions, part_bytes, elem_bytes, threads, blocks,
                                      preq.ptr, _stream(stream)), "produce_put")


def bce_grad(p, y, g, partitions: int, L: int, nf: float, preq: Prequest | None = None, order_stride: int = 1,
             blocks: int = 0, stream=None):
    """DL proxy producer (R28): g = (p - y) / ((p (1 - p)) n) over partitions of L
    fp32 elements, one block per partition; with ``preq`` each partition is
    Preadied (block granularity) into the partitioned allreduce that reads g."""
    _ok(_lib.apps().pcapp_bce_grad(_ptr(p), _ptr(y), _ptr(g), partitions, L, nf, order_stride, blocks,
                                   preq.ptr if preq is not None else None, _stream(stream)), "bce_grad")


def bce_grad_multi(ps, ys, gs, partitions: int, L: int, nf: float, preqs=None, blocks: int = 0, stream=None,
                   coop: bool = False):
    """bce_grad of every co-located rank in ONE launch, blocks interleaved
    (partition u of all ranks side by side), so an INLINE allreduce fold of u
    reads the ranks' just-written partitions from L2; preqs: one Prequest per
    rank (or None: no Pready).  coop: pc_pready_block_coop (R36) — the P
    blocks of a partition each fold one slice of it (every CTA resident)."""
    n = len(ps)
    arr = lambda xs: (C.c_void_p * n)(*[_ptr(x) for x in xs])  # noqa: E731
    qa = (C.c_void_p * n)(*[q.ptr for q in preqs]) if preqs is not None else None
    _ok(_lib.apps().pcapp_bce_grad_multi(n, arr(ps), arr(ys), arr(gs), partitions, L, nf, blocks, qa,
                                         1 if coop else 0, _stream(stream)), "bce_grad_multi")


def peer_copy(srcs, dsts, nbytes: int, blocks: int = 0, stream=None):
    """Bare peer copies (no library): len(srcs) concurrent copies of nbytes
    each, srcs[j] -> dsts[j] (int addresses or tensors; one side peer-mapped)."""
    n = len(srcs)
    sa = (C.c_void_p * n)(*[_ptr(x) for x in srcs])
    da = (C.c_void_p * n)(*[_ptr(x) for x in dsts])
    _ok(_lib.apps().pcapp_peer_copy(n, sa, da, nbytes, blocks, _stream(stream)), "peer_copy")


def memcpy_async(dst, src, nbytes: int, stream=None):
    """cudaMemcpyAsync(cudaMemcpyDefault) of nbytes (dst / src: tensors or
    int addresses, e.g. a peer-mapped buffer) on `stream`."""
    _ok(_lib.apps().pcapp_memcpy_async(_ptr(dst), _ptr(src), nbytes, _stream(stream)), "memcpy_async")


def overlap_probe(preqs, partitions: int, spin_ms: int, out_ns, stream=None):
    """a6 concurrency probe, one launch for the co-located ranks (block b =
    rank b's producer with preqs[b]): Pready(0), spin (<= spin_ms) until
    Parrived(0), then Pready the rest.  out_ns: int64 device tensor [P, 4] =
    %globaltimer at entry, after Pready(0), when Parrived(0) was seen (0:
    timed out), at exit."""
    n = len(preqs)
    arr = (C.c_void_p * n)(*[q.ptr for q in preqs])
    _ok(_lib.apps().pcapp_overlap_probe(arr, n, partitions, spin_ms, _ptr(out_ns), _stream(stream)),
        "overlap_probe")


def check_recv(preq: Prequest, recvbuf, out, partitions: int, part_bytes: int, status, blocks: int = 64,
               stream=None):
    _ok(_lib.apps().pcapp_check_recv(preq.ptr, _ptr(recvbuf), _ptr(out), partitions, part_bytes, blocks,
                                     _ptr(status), _stream(stream)), "check_recv")


def pingpong(sendq: Prequest, recvq: Prequest, side: int, iters: int, gran: int, out_ns, stream=None):
    _ok(_lib.apps().pcapp_pingpong(sendq.ptr, recvq.ptr, side, iters, gran, _ptr(out_ns), _stream(stream)),
        "pingpong")


def bare_pingpong(my_flag, peer_flag, side: int, iters: int, base: int, out_ns, stream=None):
    _ok(_lib.apps().pcapp_bare_pingpong(_ptr(my_flag), _ptr(peer_flag), side, iters, base, _ptr(out_ns),
                                        _stream(stream)), "bare_pingpong")


def pingpong_pair(sendA: Prequest, recvA: Prequest, sendB: Prequest, recvB: Prequest, iters: int, gran: int,
                  out_ns, stream=None, rt_ns=None):
    """Both sides in one launch (virtual ranks on one GPU).  rt_ns (optional,
    int64[iters]) receives every round-trip time seen by side 0."""
    _ok(_lib.apps().pcapp_pingpong_pair(sendA.ptr, recvA.ptr, sendB.ptr, recvB.ptr, iters, gran, _ptr(out_ns),
                                        _ptr(rt_ns), _stream(stream)), "pingpong_pair")


def bare_pingpong_pair(flagA, flagB, iters: int, base: int, out_ns, stream=None, scope: int = 2):
    """Flag ping-pong with no library (latency floor).  scope 0: relaxed GPU
    scope, 1: release/acquire GPU scope, 2: release/acquire system scope."""
    _ok(_lib.apps().pcapp_bare_pingpong_pair(_ptr(flagA), _ptr(flagB), iters, base, _ptr(out_ns), scope,
                                             _stream(stream)), "bare_pingpong_pair")


# --------------------------------------------------------------------------- Jacobi (a8)
T, B, L, R = 0, 1, 2, 3
_SEND_TAG = {T: 1, B: 2, L: 3, R: 4}   # tag = side of the SENDER the data leaves from
_RECV_TAG = {T: 2, B: 1, L: 4, R: 3}   # halo on my side d comes from the neighbour's opposite side
STRIP = 128  # mode 0 (warp tiles): columns per tile
JACOBI_MODES = {"warp": 0, "rows": 1}


def jacobi_strip(lx: int, mode: int) -> int:
    """Columns per tile: 128 for warp tiles; for the CTA row pipeline the
    widest of 1024/512/256/128 that divides lx (4 KiB rows per CTA at 16384^2)."""
    if mode == 0:
        return STRIP
    for w in (1024, 512, 256, 128):
        if lx % w == 0:
            return w
    raise ValueError("lx must be a multiple of 128")


class JacobiSolver:
    """2D Jacobi over a Py x Px decomposition with intra-kernel partitioned
    halo exchange.  `comms` holds the ranks this process
    drives (all P virtual ranks, or the single rank of a multi-GPU process);
    `ranks` are their comm ranks.  One epoch = one solve of `iters` iterations:
    every halo partition is (iteration slot, edge segment), readied once."""

    def __init__(self, comms, ranks, N: int, Py: int, Px: int, iters: int, H: int = 64, device: int = 0,
                 kernel: str | None = None, traditional: bool = False):
        import os

        import torch
        from . import runtime as rt
        self.torch, self.rt = torch, rt
        self.N, self.Py, self.Px, self.K, self.H = N, Py, Px, iters, H
        assert N % Py == 0 and N % Px == 0
        self.ly, self.lx = N // Py, N // Px
        self.kernel = kernel or os.environ.get("PC_JACOBI_KERNEL", "rows")
        self.mode = JACOBI_MODES[self.kernel]
        assert self.lx % STRIP == 0 and self.ly % H == 0, "lx must be a multiple of 128, ly of H"
        self.W = jacobi_strip(self.lx, self.mode)
        # traditional = the Listing 1 baseline (C4 comparison (i)): no partitioned
        # requests; kernel -> cudaStreamSynchronize -> peer copies of the edges
        self.traditional = traditional
        assert not traditional or self.mode == 1, "the traditional baseline uses the rows kernel"
        self.comms, self.ranks = comms, ranks
        dev = torch.device("cuda", device)
        self.dev = dev
        self.local = []
        for comm, r in zip(comms, ranks):
            py, px = divmod(r, Px)
            nb = {T: (py - 1) * Px + px if py > 0 else -1, B: (py + 1) * Px + px if py < Py - 1 else -1,
                  L: py * Px + px - 1 if px > 0 else -1, R: py * Px + px + 1 if px < Px - 1 else -1}
            st = {"r": r, "py": py, "px": px, "nb": nb, "comm": comm,
                  "grid": [torch.zeros(self.ly * self.lx, device=dev) for _ in range(2)],
                  "send": {}, "halo": {}, "sreq": {}, "rreq": {}, "sq": {}, "rq": {}}
            for d, q in nb.items():
                if q < 0:
                    continue
                seg = self.W if d in (T, B) else H
                nseg = (self.lx if d in (T, B) else self.ly) // seg
                parts = (iters + 1) * nseg
                st["send"][d] = torch.zeros(parts * seg, device=dev)
                st["halo"][d] = torch.zeros(parts * seg, device=dev)
                if traditional:
                    continue
                st["sreq"][d] = rt.psend_init(st["send"][d], parts, seg, rt.FLOAT32, q, _SEND_TAG[d], comm)
                st["rreq"][d] = rt.precv_init(st["halo"][d], parts, seg, rt.FLOAT32, q, _RECV_TAG[d], comm)
            self.local.append(st)
        self.desc = None
        self.epochs = 0

    def set_initial(self, a0):
        """a0: full N x N host array (numpy) or None for the perf init (top edge 1)."""
        import numpy as np
        torch = self.torch
        for st in self.local:
            blk = a0[st["py"] * self.ly:(st["py"] + 1) * self.ly, st["px"] * self.lx:(st["px"] + 1) * self.lx]
            st["grid"][0].copy_(torch.from_numpy(np.ascontiguousarray(blk, dtype=np.float32).reshape(-1)))
            st["grid"][1].copy_(st["grid"][0])

    def result(self):
        """Gather the local blocks after the last solve into an N x N array."""
        import numpy as np
        out = np.zeros((self.N, self.N), dtype=np.float32)
        for st in self.local:
            g = st["grid"][self.K & 1].cpu().numpy().reshape(self.ly, self.lx)
            out[st["py"] * self.ly:(st["py"] + 1) * self.ly, st["px"] * self.lx:(st["px"] + 1) * self.lx] = g
        return out

    def _reqs(self, st):
        return list(st["sreq"].values()) + list(st["rreq"].values())

    def _build_desc(self):
        import ctypes as C
        torch = self.torch
        lib = _lib.apps()
        sz = lib.pcapp_jacobi_rank_size()
        raw = bytearray(sz * len(self.local))
        starts = []
        blocks = 0
        for i, st in enumerate(self.local):
            has = (C.c_int * 4)(*[1 if st["nb"][d] >= 0 else 0 for d in range(4)])
            sendp = (C.c_void_p * 4)(*[st["send"][d].data_ptr() if d in st["send"] else 0 for d in range(4)])
            halop = (C.c_void_p * 4)(*[st["halo"][d].data_ptr() if d in st["halo"] else 0 for d in range(4)])
            sqp = (C.c_void_p * 4)(*[st["sq"][d].ptr if d in st["sq"] else 0 for d in range(4)])
            rqp = (C.c_void_p * 4)(*[st["rq"][d].ptr if d in st["rq"] else 0 for d in range(4)])
            buf = C.create_string_buffer(sz)
            rc = lib.pcapp_jacobi_describe2(buf, st["grid"][0].data_ptr(), st["grid"][1].data_ptr(), self.ly,
                                            self.lx, self.H, st["py"] * self.ly, st["px"] * self.lx, self.N,
                                            has, sendp, halop, sqp, rqp, self.mode, self.W)
            if rc != 0:
                raise RuntimeError("pcapp_jacobi_describe failed")
            if self.traditional:
                _ok(lib.pcapp_jacobi_set_traditional(buf, 1), "jacobi traditional")
            raw[i * sz:(i + 1) * sz] = buf.raw
            starts.append(blocks)
            tiles = (self.ly // self.H) * (self.lx // self.W)
            blocks += (tiles + 7) // 8 if self.mode == 0 else tiles
        self.desc = torch.frombuffer(raw, dtype=torch.uint8).to(self.dev)
        self.starts = torch.tensor(starts, dtype=torch.int32, device=self.dev)
        self.blocks = blocks

    def solve(self, stream, first_prepare=None):
        """One epoch: start + pbuf_prepare every request, the init push, K
        iteration launches, then wait_on_stream (senders before receivers).
        first_prepare(list_of_request_lists) runs the blocking first
        pbuf_prepare across ranks (threads for co-located ranks)."""
        lib = _lib.apps()
        if self.traditional:
            return self._solve_traditional(stream)
        for st in self.local:
            for q in self._reqs(st):
                q.start(stream)
        if self.epochs == 0:
            lists = [self._reqs(st) for st in self.local]
            if first_prepare is not None:
                first_prepare(lists)
            else:
                for lst in lists:
                    for q in lst:
                        q.pbuf_prepare(stream)
            for st in self.local:
                for d, q in st["sreq"].items():
                    st["sq"][d] = q.prequest_create(self.rt.GRAN_WARP, 1, self.rt.COPY_INLINE)
                for d, q in st["rreq"].items():
                    st["rq"][d] = q.prequest_create(self.rt.GRAN_WARP, 1, self.rt.COPY_INLINE)
            self._build_desc()
        else:
            for st in self.local:
                for q in self._reqs(st):
                    q.pbuf_prepare(stream)
        s = stream.cuda_stream if hasattr(stream, "cuda_stream") else (stream or 0)
        n = len(self.local)
        launch = lambda k, init: lib.pcapp_jacobi_launch2(self.desc.data_ptr(), self.starts.data_ptr(), n,
                                                          self.blocks, k, init, self.mode, self.W, self.H, s)
        _ok(launch(0, 1), "jacobi init")
        for k in range(self.K):
            _ok(launch(k, 0), "jacobi iter")
        for st in self.local:
            for q in st["sreq"].values():
                q.wait_on_stream(stream)
        for st in self.local:
            for q in st["rreq"].values():
                q.wait_on_stream(stream)
        self.epochs += 1

    def _solve_traditional(self, stream):
        """The Listing 1 baseline (C4 comparison (i)): every iteration is
        kernel -> cudaStreamSynchronize -> device-to-device copies of the staged
        edges into the neighbours' halo slots (cudaMemcpyAsync; a peer copy
        across GPUs), the next kernel stream-ordered after the copies.  Needs
        every rank in this process."""
        torch = self.torch
        assert len(self.local) == self.Py * self.Px, "traditional baseline: all ranks in this process"
        lib = _lib.apps()
        if self.desc is None:
            self._build_desc()
        s = stream.cuda_stream if hasattr(stream, "cuda_stream") else (stream or 0)
        n = len(self.local)
        by_rank = {st["r"]: st for st in self.local}
        opp = {T: B, B: T, L: R, R: L}

        def exchange(j):
            with torch.cuda.stream(stream):
                for st in self.local:
                    for d, q in st["nb"].items():
                        if q < 0:
                            continue
                        m = self.lx if d in (T, B) else self.ly
                        by_rank[q]["halo"][opp[d]][j * m:(j + 1) * m].copy_(st["send"][d][j * m:(j + 1) * m])

        for k in range(-1, self.K):
            _ok(lib.pcapp_jacobi_launch2(self.desc.data_ptr(), self.starts.data_ptr(), n, self.blocks, max(k, 0),
                                         1 if k < 0 else 0, self.mode, self.W, self.H, s), "jacobi traditional")
            stream.synchronize()  # Listing 1: the host waits for the kernel before sending
            exchange(k + 1)
        self.epochs += 1

    def errors(self):
        return [q.error() for st in self.local for q in self._reqs(st) if q.error()[0] != 0]

    def free(self):
        for st in self.local:
            for q in self._reqs(st):
                q.free()


class DLProxy:
    """The paper's DL kernel (§VI-D2) on co-located ranks: every
    step each rank computes its BCE gradient (``bce_grad``) and the ranks
    allreduce it with one persistent partitioned allreduce; ``pc_startall`` and
    ``pc_pbuf_prepare_all`` are inside the step, as in a training loop.  Each
    rank's producer runs on its own stream (as each GPU would run its own),
    after the epoch's control kernels on the control stream ``ctl``.

    mode "pready": the producer Preadies each partition from the kernel
                   (block granularity); the engine — forked at the epoch's
                   pbuf_prepare, enqueued at the wait — reduces each partition
                   as soon as every rank has produced it, while the producers
                   still run (§8(a) a6);
    mode "serial": producer kernels, then the collective (host-side Pready of
                   every partition, the MPI_Allreduce-after-the-kernel flow).
    ``overlap=False`` forks the engine at the wait (pc_request_set_overlap):
    the Pready mode without producer/engine concurrency.  ``copy=COPY_INLINE``
    (DIRECT schedule): no engine — the producer block whose Pready completes a
    partition on the last rank folds it for every rank (reading R33).
    Inputs: ``p`` (predictions), ``y`` (targets), fp32, one tensor per rank."""

    def __init__(self, comms, partitions: int, L: int, algo: int, p, y, overlap: bool = True, copy: int | None = None,
                 multi: bool = False, coop: bool = False):
        import torch

        from . import runtime as rt

        self.P, self.Np, self.L = len(comms), partitions, L
        self.p, self.y = p, y
        n = partitions * L
        self.nf = float(n)
        self.g = [torch.empty(max(n, 4), device=p[0].device) for _ in range(self.P)]
        self.out = [torch.empty(max(n, 4), device=p[0].device) for _ in range(self.P)]
        self.reqs = [rt.pallreduce_init(self.g[r], self.out[r], partitions, L, rt.FLOAT32, rt.SUM, algo, comms[r])
                     for r in range(self.P)]
        self.overlap = overlap
        if not overlap:
            for q in self.reqs:
                q.set_overlap(False)
        from .runtime import COPY_ENGINE
        # copy: COPY_ENGINE (the engine reduces) or COPY_INLINE (DIRECT only:
        # the producer block completing a partition on the last rank folds it,
        # reading R33)
        self.copy = COPY_ENGINE if copy is None else copy
        self.preqs = None
        self.ctl = torch.cuda.Stream()
        self.pst = [torch.cuda.Stream() for _ in range(self.P)]
        self.ev_ctl = torch.cuda.Event()
        self.ev_p = [torch.cuda.Event() for _ in range(self.P)]
        # multi: every rank's producer in ONE launch on the control stream,
        # partition u of all ranks side by side (bce_grad_multi)
        self.multi = multi or coop
        self.coop = coop  # multi + pc_pready_block_coop (INLINE copy, R36)

    def step(self, mode: str = "pready", order_stride: int = 1):
        from . import runtime as rt

        st = self.ctl
        if self.preqs is None:  # first epoch: exchange + mapping (collective over the ranks)
            for q in self.reqs:
                q.start(st)
            rt.run_ranks([(lambda q=q: q.pbuf_prepare(st)) for q in self.reqs])
            self.preqs = [q.prequest_create(rt.GRAN_BLOCK, 1, self.copy) for q in self.reqs]
        else:
            rt.startall(self.reqs, st)
            rt.pbuf_prepare_all(self.reqs, st)
        if self.multi:
            bce_grad_multi(self.p, self.y, self.g, self.Np, self.L, self.nf,
                           self.preqs if mode == "pready" else None, stream=st, coop=self.coop)
            if mode == "serial":
                rt.preadyall(self.reqs, st)
            for q in self.reqs:
                q.wait_on_stream(st)
            return
        self.ev_ctl.record(st)
        for r in range(self.P):
            self.pst[r].wait_event(self.ev_ctl)
            bce_grad(self.p[r], self.y[r], self.g[r], self.Np, self.L, self.nf,
                     self.preqs[r] if mode == "pready" else None, order_stride, stream=self.pst[r])
            self.ev_p[r].record(self.pst[r])
        if mode == "serial" or not self.overlap:  # the collective (or its fork point) after the kernels
            for r in range(self.P):
                st.wait_event(self.ev_p[r])
        if mode == "serial":
            rt.preadyall(self.reqs, st)
        for q in self.reqs:  # (enqueues the engine: after every producer in host order)
            q.wait_on_stream(st)
        if mode != "serial" and self.overlap:  # join the producers' tails before the next epoch
            for r in range(self.P):
                st.wait_event(self.ev_p[r])

    def errors(self):
        return [(r, q.error()) for r, q in enumerate(self.reqs) if q.error()[0] != 0]

    def free(self):
        for q in self.reqs:
            q.free()
