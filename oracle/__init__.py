"""CPU oracle for the partitioned-communication hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package.  The product path
(``paper_conf_sc_temucinslsga24_b200``, ``libpc.so``) never imports it and shares
no code with it.  See ``oracle.cpp`` for what each function follows in the paper
(PAPER.md line citations) and DESIGN.md §"Readings of the paper" for R1..R23.

Functions (numpy in, numpy out):
  p2p(...)                O1  partitioned send/recv with aggregation + RTR
  allreduce_def_i32(...)  O2  plain definition, int32 (sum wraps, max, min)
  allreduce_def_f64(...)  O2  plain definition, fp32 inputs summed in fp64
  pallreduce(...)         O3/O4/O6  Alg 1 (ring), RD or DIRECT schedule + Alg 2, P threads
  bf16_round / bf16_op    R27 bf16 arithmetic (bit patterns as uint16)
  bce_grad(p, y, n)       O7  DL proxy producer (R28)
  alg1_table(P, r)        Alg 1 step tuples
  ring_fold_f32 / rd_tree_f32   closed forms of O3 / O4 (pinned against them)
  jacobi_seq / jacobi_decomp    O5
  reduce_scatter_def(...) O8  partitioned reduce-scatter, plain definition (rank-order fold, R25)
  allgather_def(...)      O9  partitioned allgather, plain definition (concatenation)
  bcast_def(...)          O10 partitioned broadcast, plain definition (copy of the root's buffer)
  xpart_arrived(...)      O11 MPI-4 different send/recv partitionings: which receive
                              partitions are complete, by byte coverage (R30)
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None

INT32, FLOAT32, FLOAT64, BF16 = 0, 1, 3, 4  # bf16 arrays are carried as uint16 bit patterns
SUM, MAX, MIN = 0, 1, 2
RING, RD, DIRECT = 1, 2, 3


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "oracle.cpp")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["make", "-s", "-C", _HERE, "liboracle.so"])
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        _lib = C.CDLL(_SO)
        P = C.c_void_p
        i32, i64, u64 = C.c_int, C.c_int64, C.c_uint64
        _lib.orc_p2p.argtypes = [P, P, i32, i64, i32, i32, i32, P, i32, i32, u64, P]
        _lib.orc_allreduce_def_i32.argtypes = [i32, i64, P, i32, P]
        _lib.orc_allreduce_def_f64.argtypes = [i32, i64, P, P, P]
        _lib.orc_pallreduce.argtypes = [i32, i32, i32, i64, i32, i32, i32, i32, P, P, P, u64, P, P]
        _lib.orc_pallreduce_direct.argtypes = [i32, i32, i64, i32, i32, i32, i32, P, P, P, u64, P, P]
        _lib.orc_alg1_table.argtypes = [i32, i32, P]
        _lib.orc_bf16_round.argtypes = [i64, P, P]
        _lib.orc_bce_grad.argtypes = [i64, P, P, C.c_float, P]
        _lib.orc_bf16_op.argtypes = [i32, i64, P, P, P]
        _lib.orc_ring_fold_f32.argtypes = [i32, i64, P, P, P]
        _lib.orc_rd_tree_f32.argtypes = [i32, i64, P, P]
        _lib.orc_jacobi_seq.argtypes = [i32, i32, i32, P, P]
        _lib.orc_jacobi_decomp.argtypes = [i32, i32, i32, i32, i32, P, P]
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


class OracleError(RuntimeError):
    pass


def _check(rc: int, what: str):
    if rc < 0:
        raise OracleError(f"{what} failed with {rc}")
    return rc


def p2p(send: np.ndarray, partitions: int, agg: int, orders: np.ndarray, workers: int = 4,
        use_rtr: bool = True, recv_delay_us: int = 0, jitter_seed: int = 1):
    """send: (epochs, total_bytes) uint8.  Returns (consumed, arrivals[epochs, n_transport])."""
    send = np.ascontiguousarray(send, dtype=np.uint8)
    epochs, total = send.shape
    assert total % partitions == 0
    nt = (partitions + agg - 1) // agg
    consumed = np.zeros_like(send)
    arrivals = np.zeros((epochs, nt), dtype=np.uint32)
    orders = np.ascontiguousarray(orders, dtype=np.int32).reshape(epochs, partitions)
    _check(lib().orc_p2p(_p(send), _p(consumed), partitions, total // partitions, agg, workers, epochs,
                         _p(orders), int(use_rtr), recv_delay_us, jitter_seed, _p(arrivals)), "orc_p2p")
    return consumed, arrivals


def allreduce_def_i32(x: np.ndarray, op: int = SUM) -> np.ndarray:
    """x: (P, n) int32 -> (n,) int32."""
    x = np.ascontiguousarray(x, dtype=np.int32)
    P, n = x.shape
    y = np.zeros(n, dtype=np.int32)
    _check(lib().orc_allreduce_def_i32(P, n, _p(x), op, _p(y)), "def_i32")
    return y


def allreduce_def_f64(x: np.ndarray):
    """x: (P, n) float32 -> (fp64 sum, fp64 sum|x|)."""
    x = np.ascontiguousarray(x, dtype=np.float32)
    P, n = x.shape
    y = np.zeros(n, dtype=np.float64)
    a = np.zeros(n, dtype=np.float64)
    _check(lib().orc_allreduce_def_f64(P, n, _p(x), _p(y), _p(a)), "def_f64")
    return y, a


def n_steps(algo: int, P: int) -> int:
    if algo == RING:
        return 2 * (P - 1)
    if algo == DIRECT:
        return 2
    k = 0
    while (1 << k) < P:
        k += 1
    return k


def pallreduce(x: np.ndarray, partitions: int, algo: int = RING, op: int = SUM, inplace: bool = False,
               orders: np.ndarray | None = None, jitter_seed: int = 1):
    """x: (epochs, P, Np*L) int32, float32, float64 or uint16 (= bf16 bit
    patterns, reading R27) (or (P, Np*L) for one epoch).

    Returns (y, reduces, arrivals): y has x's shape and holds each rank's recvbuf
    after its MPI_Wait; reduces/arrivals are (P, Np, max(nsteps,1)) counts from
    the last epoch."""
    squeeze = x.ndim == 2
    if squeeze:
        x = x[None]
    dtype = _DTYPES[x.dtype.type]
    x = np.ascontiguousarray(x)
    epochs, P, n = x.shape
    assert n % partitions == 0
    L = n // partitions
    if orders is None:
        orders = np.tile(np.arange(partitions, dtype=np.int32), (epochs, P, 1))
    orders = np.ascontiguousarray(orders, dtype=np.int32).reshape(epochs, P, partitions)
    ns = max(n_steps(algo, P), 1)
    y = np.zeros_like(x)
    red = np.zeros((P, partitions, ns), dtype=np.uint32)
    arr = np.zeros((P, partitions, ns), dtype=np.uint32)
    if algo == DIRECT:
        _check(lib().orc_pallreduce_direct(P, partitions, L, dtype, op, epochs, int(inplace), _p(x), _p(y),
                                           _p(orders), jitter_seed, _p(red), _p(arr)), "orc_pallreduce_direct")
    else:
        _check(lib().orc_pallreduce(algo, P, partitions, L, dtype, op, epochs, int(inplace), _p(x), _p(y),
                                    _p(orders), jitter_seed, _p(red), _p(arr)), "orc_pallreduce")
    return (y[0] if squeeze else y), red, arr


_DTYPES = {np.int32: INT32, np.float32: FLOAT32, np.float64: FLOAT64, np.uint16: BF16}


def bce_grad(p: np.ndarray, y: np.ndarray, n: float) -> np.ndarray:
    """O7 (R28): fp32 gradient of the mean BCE w.r.t. the predictions."""
    p = np.ascontiguousarray(p, dtype=np.float32)
    y = np.ascontiguousarray(y, dtype=np.float32)
    g = np.zeros_like(p)
    _check(lib().orc_bce_grad(p.size, _p(p), _p(y), float(n), _p(g)), "bce_grad")
    return g


def bf16_round(x: np.ndarray) -> np.ndarray:
    """float64 values -> nearest bf16 (ties to even), as uint16 bit patterns (R27)."""
    x = np.ascontiguousarray(x, dtype=np.float64)
    out = np.zeros(x.shape, dtype=np.uint16)
    _check(lib().orc_bf16_round(x.size, _p(x), _p(out)), "bf16_round")
    return out


def bf16_op(a: np.ndarray, b: np.ndarray, op: int = SUM) -> np.ndarray:
    """Elementwise a (+) b of bf16 bit patterns (uint16), correctly rounded (R27)."""
    a = np.ascontiguousarray(a, dtype=np.uint16)
    b = np.ascontiguousarray(b, dtype=np.uint16)
    out = np.zeros(a.shape, dtype=np.uint16)
    _check(lib().orc_bf16_op(op, a.size, _p(a), _p(b), _p(out)), "bf16_op")
    return out


def bf16_to_f64(b: np.ndarray) -> np.ndarray:
    """Exact decode of bf16 bit patterns (the upper half of an fp32)."""
    return (np.asarray(b, dtype=np.uint16).astype(np.uint32) << 16).view(np.float32).astype(np.float64)


def alg1_table(P: int, r: int) -> np.ndarray:
    """(2(P-1), 5) int32 rows (I, R, op, O, A)."""
    out = np.zeros((max(2 * (P - 1), 1), 5), dtype=np.int32)
    n = _check(lib().orc_alg1_table(P, r, _p(out)), "alg1_table")
    return out[:n]


def ring_fold_f32(x: np.ndarray, start: np.ndarray) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.float32)
    P, n = x.shape
    start = np.ascontiguousarray(start, dtype=np.int32)
    out = np.zeros(n, dtype=np.float32)
    _check(lib().orc_ring_fold_f32(P, n, _p(x), _p(start), _p(out)), "ring_fold")
    return out


def rd_tree_f32(x: np.ndarray) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.float32)
    P, n = x.shape
    out = np.zeros(n, dtype=np.float32)
    _check(lib().orc_rd_tree_f32(P, n, _p(x), _p(out)), "rd_tree")
    return out


def chunk_ids(L: int, P: int, partitions: int, esize: int = 4) -> np.ndarray:
    """Chunk id of every element of an (Np*L) buffer under reading R4
    (q = ceil(L/(vP))*v elements per chunk, v = 16/esize)."""
    v = 16 // esize
    q = -(-L // (v * P)) * v if L > 0 else v
    j = np.arange(L)
    c = np.minimum(j // max(q, 1), P - 1).astype(np.int32)
    return np.tile(c, partitions)


def jacobi_seq(a0: np.ndarray, iters: int) -> np.ndarray:
    a0 = np.ascontiguousarray(a0, dtype=np.float32)
    ny, nx = a0.shape
    out = np.zeros_like(a0)
    _check(lib().orc_jacobi_seq(ny, nx, iters, _p(a0), _p(out)), "jacobi_seq")
    return out


def jacobi_decomp(a0: np.ndarray, iters: int, Py: int, Px: int) -> np.ndarray:
    a0 = np.ascontiguousarray(a0, dtype=np.float32)
    ny, nx = a0.shape
    out = np.zeros_like(a0)
    _check(lib().orc_jacobi_decomp(ny, nx, Py, Px, iters, _p(a0), _p(out)), "jacobi_decomp")
    return out


# --------------------------------------------------------------------------- NEXT-3 collectives
# Plain definitions (generic schedule P:L151-L155, MPI_Op P:L155).
def _op(a: np.ndarray, b: np.ndarray, op: int) -> np.ndarray:
    """One element-wise a ⊕ b in the element type: int32 sum wraps mod 2^32;
    fp32/fp64 one IEEE op (RN-even; max/min = IEEE maxNum/minNum like
    std::fmax in oracle.cpp); bf16 (uint16 bit patterns) via the R27 oracle."""
    if a.dtype == np.uint16:
        return bf16_op(a, b, op)
    if a.dtype == np.int32:
        if op == SUM:
            return (a.view(np.uint32) + b.view(np.uint32)).view(np.int32)
        return np.maximum(a, b) if op == MAX else np.minimum(a, b)
    if op == SUM:
        return a + b  # numpy float32 / float64 add: one IEEE op, round to nearest even
    return np.fmax(a, b) if op == MAX else np.fmin(a, b)


def reduce_scatter_def(x: np.ndarray, partitions: int, op: int = SUM) -> np.ndarray:
    """O8.  x: (P, partitions * P * count), rank k's send buffer: partition u =
    P blocks of count, block d destined to rank d.  Returns y: (P, partitions *
    count), y[d][u] = x[0][u][d] ⊕ x[1][u][d] ⊕ ... ⊕ x[P-1][u][d], folded left
    in rank order (reading R25 — the DIRECT schedule's association)."""
    x = np.ascontiguousarray(x)
    P = x.shape[0]
    count = x.shape[1] // (partitions * P)
    assert count * partitions * P == x.shape[1]
    blocks = x.reshape(P, partitions, P, count)  # [source k][u][destination d][i]
    y = np.empty((P, partitions, count), dtype=x.dtype)
    for d in range(P):
        acc = blocks[0, :, d, :].copy()
        for k in range(1, P):
            acc = _op(acc, blocks[k, :, d, :], op)
        y[d] = acc
    return y.reshape(P, partitions * count)


def allgather_def(x: np.ndarray) -> np.ndarray:
    """O9.  x: (P, n) send buffers.  Every rank's receive buffer is the rank-
    major concatenation x[0] | x[1] | ... | x[P-1] (MPI_Allgather).  Returns
    (P, P * n)."""
    x = np.ascontiguousarray(x)
    P = x.shape[0]
    return np.tile(x.reshape(1, -1), (P, 1))


def bcast_def(x: np.ndarray, root: int) -> np.ndarray:
    """O10.  x: (P, n) buffers before the broadcast; afterwards every rank holds
    the root's buffer."""
    x = np.ascontiguousarray(x)
    return np.tile(x[root][None], (x.shape[0], 1))


def xpart_arrived(send_partitions: int, send_part_bytes: int, agg: int, recv_partitions: int,
                  recv_part_bytes: int, readied: np.ndarray) -> np.ndarray:
    """O11 (reading R30; MPI-4 partitioned semantics cited at P:L46: a receive
    partition has arrived once every one of its bytes has).  The sender's user
    partitions are grouped g = agg at a time into transport partitions, and a
    transport partition's bytes move (and are announced) only once all of its
    user partitions are readied.  readied: bool
    [send_partitions], the user partitions Preadied so far.  Returns bool
    [recv_partitions]: receive partition p is complete iff every byte of
    [p * recv_part_bytes, (p + 1) * recv_part_bytes) lies in a complete
    transport partition.  Brute force over bytes — small cases only."""
    total = send_partitions * send_part_bytes
    assert total == recv_partitions * recv_part_bytes
    readied = np.asarray(readied, dtype=bool)
    moved = np.zeros(total, dtype=bool)
    for t0 in range(0, send_partitions, agg):
        members = range(t0, min(t0 + agg, send_partitions))
        if all(readied[u] for u in members):
            for u in members:
                moved[u * send_part_bytes:(u + 1) * send_part_bytes] = True
    return np.array([bool(moved[p * recv_part_bytes:(p + 1) * recv_part_bytes].all())
                     for p in range(recv_partitions)], dtype=bool)
