"""Helpers for the GPU parity tests: virtual ranks on one device.

Every rank of a comm lives in this process and drives its own torch stream;
ranks that share the GPU address each other's buffers directly (no IPC), so the
whole multi-rank protocol (flags, RTR, engines, release/acquire) runs on one
B200.  The bootstrap all-gather (comm creation and the first pbuf_prepare)
needs one host thread per rank (run_ranks)."""
from __future__ import annotations

import contextlib
import os

import numpy as np
import torch

import paper_conf_sc_temucinslsga24_b200 as pc


def dev():
    return torch.device("cuda", 0)


@contextlib.contextmanager
def comms(P: int, timeout_ms: int = 5000):
    old = os.environ.get("PC_TIMEOUT_MS")
    os.environ["PC_TIMEOUT_MS"] = str(timeout_ms)
    try:
        g, cs = pc.local_comms(P, 0)
    finally:
        if old is None:
            os.environ.pop("PC_TIMEOUT_MS")
        else:
            os.environ["PC_TIMEOUT_MS"] = old
    try:
        yield cs
    finally:
        torch.cuda.synchronize()
        for c in cs:
            c.destroy()
        g.destroy()


def to_dev(a: np.ndarray) -> torch.Tensor:
    return torch.from_numpy(np.ascontiguousarray(a)).to(dev())


def alloc_like(a: np.ndarray) -> torch.Tensor:
    return torch.empty(a.shape, dtype=torch.from_numpy(a[:0]).dtype, device=dev())


def first_prepare(reqs, streams):
    """First pbuf_prepare of a batch: blocking exchange, one thread per rank.
    reqs[r] is the list of rank r's requests to prepare."""
    def mk(r):
        def f():
            for q in reqs[r]:
                q.pbuf_prepare(streams[r])
        return f
    pc.run_ranks([mk(r) for r in range(len(reqs))])
