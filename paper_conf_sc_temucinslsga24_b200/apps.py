"""Launchers for libpcapps.so: producer / application kernels compiled against
include/pc_device.cuh (the way a user kernel calls pc_pready / pc_parrived).
Argument marshalling only."""
from __future__ import annotations

import ctypes as C

from . import _lib
from .runtime import Prequest, _ptr, _stream

GRAN_NONE, GRAN_THREAD, GRAN_WARP, GRAN_BLOCK = -1, 0, 1, 2


def _ok(rc, what):
    if rc != 0:
        raise RuntimeError(f"{what} launch failed ({rc})")


def vecadd(A, B, Cout, n: int, gran: int, preq: Prequest | None, stream=None):
    """C = A + B (fp32, 8 B per thread, 1024-thread blocks) with pc_pready at
    `gran` (thread: partition = thread, warp: = warp, block: = block)."""
    _ok(_lib.apps().pcapp_vecadd(_ptr(A), _ptr(B), _ptr(Cout), n, gran, preq.ptr if preq else None,
                                 _stream(stream)), "vecadd")


def produce(dst, src, partitions: int, part_bytes: int, gran: int, preq: Prequest, order_stride: int = 1,
            blocks: int = 0, stream=None):
    _ok(_lib.apps().pcapp_produce(_ptr(dst), _ptr(src), partitions, part_bytes, gran, order_stride, blocks,
                                  preq.ptr, _stream(stream)), "produce")


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


def bare_pingpong_pair(flagA, flagB, iters: int, base: int, out_ns, stream=None):
    _ok(_lib.apps().pcapp_bare_pingpong_pair(_ptr(flagA), _ptr(flagB), iters, base, _ptr(out_ns),
                                             _stream(stream)), "bare_pingpong_pair")
