#pragma once
// libpc device engines (sm_100a) — templated engine bodies shared by the
// per-(dtype, op) instantiation units.
//
//  ring_engine   partitioned allreduce, Alg 1 schedule progressed
//                on the GPU: the host Progression Engine of Alg 2
//                and its per-step reduce kernel + cudaStreamSynchronize
//                 are replaced by warps that wait on a flag,
//                reduce the arriving slice in registers and forward it to the
//                next rank in the same pass (the "computation inside the device
//                call" the paper proposes).
//  rd_engine     the same over a recursive-doubling schedule (north_star).
//  p2p_engine    ENGINE copy mode of partitioned send: poll local ready flags,
//                push slices over NVLink, publish the receiver's flag.
//  wait_words    stream-ordered MPI_Wait for send/recv requests.
//
// Unit of work = (user partition u, slice s) handled by ONE warp through all
// steps of the schedule ("each partition independently executes that
// schedule").  Warps take units in increasing order, x = gw, gw+W, ...
// with W identical on every rank (agreed at comm creation), so the dependency
// (unit x, step i) at rank r -> (unit x, step i-1) at rank r-1 can never form a
// cycle while all engine warps are resident.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <atomic>

#include "pc_device.cuh"
#include "pc_ops.cuh"
#include "pc_internal.h"

// engine.cuh is included by kernels.cu (control kernels, p2p engine, the
// dtype/op switch) and by engine_inst.cu, which is compiled once per
// (dtype, op) pair (-DPC_DT, -DPC_OP) so the 12 engine instantiations build in
// parallel.

namespace pc {
namespace {

using namespace pc_detail;

#ifndef PC_ENGINE_UNROLL
#define PC_ENGINE_UNROLL 8
#endif
constexpr int kU = PC_ENGINE_UNROLL;
#ifndef PC_DIRECT_FV
#define PC_DIRECT_FV 2
#endif  // 16-B vectors in flight per operand per lane
#ifndef PC_DIRECT_MINB
#define PC_DIRECT_MINB 1
#endif  // min CTAs per SM of the DIRECT engines: 1 = up to 255 registers, so all
        // P * PC_DIRECT_FV loads of a lane stay in registers (at 2 CTAs the
        // 128-register cap spills FV = 2; measured: FV 1 @ 2 CTAs 0.92 of HBM,
        // FV 2 @ 1 CTA 0.99, FV 4 @ 1 CTA 0.90)

// Engine-side bounded spin: the awaited event is a whole slice step of the
// upstream rank (tens of microseconds), so back off with __nanosleep early and
// keep the L2 free of polling traffic.
__device__ __forceinline__ bool engine_spin(const uint32_t *p, uint32_t target, int32_t *err, uint32_t tmo, int part,
                                            bool SYS) {
  uint32_t v = SYS ? ld_acquire_sys(p) : ld_acquire_gpu(p);
  if (reached(v, target)) return true;
  const uint64_t t0 = globaltimer();
  uint32_t ns = 64, n = 0;
  for (;;) {
    __nanosleep(ns);
    if (ns < 1024) ns <<= 1;
    v = SYS ? ld_acquire_sys(p) : ld_acquire_gpu(p);
    if (reached(v, target)) return true;
    if ((++n & 15) == 0) {
      if (aborted(err)) return false;
      if (tmo && globaltimer() - t0 > (uint64_t)tmo * 1000000ull) {
        set_error(err, PC_DEV_ERR_TIMEOUT, part);
        return false;
      }
    }
  }
}

// Warp-wide bounded wait on a flag word; lane 0 polls, the warp follows.
// sys: acquire at system scope (word written from another GPU).
__device__ __forceinline__ bool warp_wait(const uint32_t *p, uint32_t target, int32_t *err, uint32_t tmo, int part,
                                          bool sys) {
  bool ok = true;
  if ((threadIdx.x & 31) == 0) ok = engine_spin(p, target, err, tmo, part, sys);
  ok = __shfl_sync(0xffffffffu, ok, 0);
  __syncwarp();
  return ok;
}

// Publish: every lane's (peer) stores are made visible at the request's scope
// (system scope for a peer on another GPU), then lane 0 stores the epoch into
// the consumer's flag.
__device__ __forceinline__ void warp_signal(uint32_t *flag, uint32_t e, bool sys) {
  fence_release(sys);
  __syncwarp();
  if ((threadIdx.x & 31) == 0) st_relaxed_sys(flag, e);
}

// ⊕ and its 16-B vector form: include/pc_ops.cuh (shared with the INLINE
// allreduce fold of pc_device.cuh)
using pc_ops::Op;
using pc_ops::vop;

// out1[k] (and out2[k]) = local[k] ⊕ incoming[k], k < n elements, by one warp.
// All operands of one call sit at the same element offset of 16-B aligned
// buffers, so they share one misalignment: a scalar head of < 4 elements
// brings them to a 16-B boundary, the body runs on 16-B vectors (kU in flight
// per operand per lane), a scalar tail finishes.  (Gradient buffers of
// arbitrary tensor sizes, C3, make unaligned partitions the common case.)
template <int DT, int OP>
__device__ __forceinline__ void warp_reduce(void *out1, void *out2, const void *local, const void *incoming,
                                            int64_t n) {
  using O = Op<DT, OP>;
  using T = typename O::T;
  const uint32_t lane = threadIdx.x & 31;
  const T *a = reinterpret_cast<const T *>(local);
  const T *b = reinterpret_cast<const T *>(incoming);
  T *o1 = reinterpret_cast<T *>(out1);
  T *o2 = reinterpret_cast<T *>(out2);
  constexpr int64_t EPV = 16 / sizeof(T);
  const uintptr_t m = reinterpret_cast<uintptr_t>(out1) & 15;
  const bool same = ((reinterpret_cast<uintptr_t>(local) & 15) == m) &&
                    ((reinterpret_cast<uintptr_t>(incoming) & 15) == m) &&
                    (!out2 || (reinterpret_cast<uintptr_t>(out2) & 15) == m) && (m % sizeof(T)) == 0;
  int64_t head = same ? (int64_t)(((16 - m) & 15) / sizeof(T)) : n;
  if (head > n) head = n;
  for (int64_t k = lane; k < head; k += 32) {
    const T r = O::f(__ldcg(a + k), __ldcg(b + k));
    o1[k] = r;
    if (o2) o2[k] = r;
  }
  int64_t done = head;
  if (same && n > head) {
    const int64_t nv = (n - head) / EPV;
    const uint4 *av = reinterpret_cast<const uint4 *>(a + head);
    const uint4 *bv = reinterpret_cast<const uint4 *>(b + head);
    uint4 *o1v = reinterpret_cast<uint4 *>(o1 + head);
    uint4 *o2v = o2 ? reinterpret_cast<uint4 *>(o2 + head) : nullptr;
    int64_t k = lane;
    for (; k + 32 * (kU - 1) < nv; k += 32 * kU) {
      uint4 x[kU], y[kU];
#pragma unroll
      for (int j = 0; j < kU; ++j) x[j] = __ldcg(av + k + 32 * j);
#pragma unroll
      for (int j = 0; j < kU; ++j) y[j] = __ldcg(bv + k + 32 * j);
#pragma unroll
      for (int j = 0; j < kU; ++j) {
        const uint4 r = vop<DT, OP>(x[j], y[j]);
        o1v[k + 32 * j] = r;
        if (o2v) o2v[k + 32 * j] = r;
      }
    }
    for (; k < nv; k += 32) {
      const uint4 r = vop<DT, OP>(__ldcg(av + k), __ldcg(bv + k));
      o1v[k] = r;
      if (o2v) o2v[k] = r;
    }
    done = head + nv * EPV;
  }
  for (int64_t k = done + lane; k < n; k += 32) {
    const T r = O::f(__ldcg(a + k), __ldcg(b + k));
    o1[k] = r;
    if (o2) o2[k] = r;
  }
}

__device__ __forceinline__ void warp_copy(void *dst, const void *src, int64_t nbytes) {
  const uint32_t lane = threadIdx.x & 31;
  const uintptr_t m = reinterpret_cast<uintptr_t>(dst) & 15;
  if (m && (reinterpret_cast<uintptr_t>(src) & 15) == m && nbytes > (int64_t)(16 - m)) {
    // shared misalignment: copy a head up to the 16-B boundary, then vectors
    const int64_t h = (int64_t)(16 - m);
    copy_bytes(reinterpret_cast<uint8_t *>(dst), reinterpret_cast<const uint8_t *>(src), (uint64_t)h, lane, 32);
    dst = reinterpret_cast<uint8_t *>(dst) + h;
    src = reinterpret_cast<const uint8_t *>(src) + h;
    nbytes -= h;
  }
  if (((reinterpret_cast<uintptr_t>(dst) | reinterpret_cast<uintptr_t>(src)) & 15) == 0) {
    const int64_t nv = nbytes >> 4;
    const uint4 *s4 = reinterpret_cast<const uint4 *>(src);
    uint4 *d4 = reinterpret_cast<uint4 *>(dst);
    int64_t k = lane;
    for (; k + 32 * (kU - 1) < nv; k += 32 * kU) {
      uint4 x[kU];
#pragma unroll
      for (int j = 0; j < kU; ++j) x[j] = __ldcg(s4 + k + 32 * j);
#pragma unroll
      for (int j = 0; j < kU; ++j) d4[k + 32 * j] = x[j];
    }
    for (; k < nv; k += 32) d4[k] = __ldcg(s4 + k);
    const int64_t done = nv << 4;
    if (done < nbytes) copy_bytes(reinterpret_cast<uint8_t *>(dst) + done, reinterpret_cast<const uint8_t *>(src) + done,
                                  (uint64_t)(nbytes - done), lane, 32);
    return;
  }
  copy_bytes(reinterpret_cast<uint8_t *>(dst), reinterpret_cast<const uint8_t *>(src), (uint64_t)nbytes, lane, 32);
}

// src -> dst0 and dsts[0 .. nd-1] at the same byte offset (the allgather
// push): every source vector is loaded ONCE and stored nd+1 times.  The
// destinations share one misalignment (same offset of 16-B aligned buffers);
// if the source does not, fall back to one warp_copy per destination.
// skip: one index of dsts not written (-1: none); U source vectors per lane
// in flight.
template <int MAXD, int U = 4>
__device__ __forceinline__ void warp_copy_multi(uint8_t *dst0, uint8_t *const *dsts, int nd, int64_t doff,
                                                const uint8_t *src, int64_t nbytes, int skip = -1) {
  const uint32_t lane = threadIdx.x & 31;
  const uintptr_t m = reinterpret_cast<uintptr_t>(dst0 + doff) & 15;
  if ((reinterpret_cast<uintptr_t>(src) & 15) != m) {
    warp_copy(dst0 + doff, src, nbytes);
    for (int j = 0; j < nd; ++j)
      if (j != skip) warp_copy(dsts[j] + doff, src, nbytes);
    return;
  }
  int64_t h = (int64_t)((16 - m) & 15);
  if (h > nbytes) h = nbytes;
  for (int64_t b = lane; b < h; b += 32) {
    const uint8_t v = src[b];
    dst0[doff + b] = v;
    for (int j = 0; j < nd; ++j)
      if (j != skip) dsts[j][doff + b] = v;
  }
  const int64_t nv = (nbytes - h) >> 4;
  const uint4 *s4 = reinterpret_cast<const uint4 *>(src + h);
  int64_t k = lane;
  for (; k + 32 * (U - 1) < nv; k += 32 * U) {
    uint4 x[U];
#pragma unroll
    for (int v = 0; v < U; ++v) x[v] = __ldcg(s4 + k + 32 * v);
#pragma unroll
    for (int v = 0; v < U; ++v) {
      reinterpret_cast<uint4 *>(dst0 + doff + h)[k + 32 * v] = x[v];
#pragma unroll
      for (int j = 0; j < MAXD; ++j)
        if (j < nd && j != skip) reinterpret_cast<uint4 *>(dsts[j] + doff + h)[k + 32 * v] = x[v];
    }
  }
  for (; k < nv; k += 32) {
    const uint4 x = __ldcg(s4 + k);
    reinterpret_cast<uint4 *>(dst0 + doff + h)[k] = x;
#pragma unroll
    for (int j = 0; j < MAXD; ++j)
      if (j < nd && j != skip) reinterpret_cast<uint4 *>(dsts[j] + doff + h)[k] = x;
  }
  for (int64_t b = h + (nv << 4) + lane; b < nbytes; b += 32) {
    const uint8_t v = src[b];
    dst0[doff + b] = v;
    for (int j = 0; j < nd; ++j)
      if (j != skip) dsts[j][doff + b] = v;
  }
}

__device__ __forceinline__ int modp(int a, int p) { return ((a % p) + p) % p; }

// ---------------------------------------------------------------------------
// Ring (Alg 1).  Paper indexing: at step i rank r sends chunk R_i = r - i and
// receives chunk A_i = r - i - 1 (mod P).  Fused engine step E_i (i >= 1)
// consumes the arrival of step i-1 (chunk A_{i-1} = R_i) and sends step i:
//   1 <= i <= P-2 : acc = send[c] ⊕ staging[c]  -> O.staging[c]        (RS)
//   i  = P-1      : acc = send[c] ⊕ staging[c]  -> recv[c], O.recv[c]  (final)
//   P <= i <= 2P-3:        recv[c]              -> O.recv[c]           (AG)
// E_0 sends send[r] -> O.staging[r]; completion waits for step 2P-3.
// Operand order local ⊕ incoming (reading R5); flags are per (u, step, slice)
// (reading R3) and hold epoch values, so they are never reset.
// ---------------------------------------------------------------------------
// Alg 2 on a warp: the warp owns up to kMaxActive units and
// sweeps them round-robin, polling each unit's next dependency once and
// performing the step of every unit that is ready — exactly the per-partition
// state machine of Alg 2, with the progression thread replaced by the warp.
// A slow upstream unit therefore never idles the warp while another of its
// units can advance.  Dependencies form a DAG over (unit, step, rank), so
// progress only needs every engine warp to be resident.
constexpr int kMaxActive = 8;

__device__ __forceinline__ bool warp_poll(const uint32_t *p, uint32_t target, bool sys) {
  bool ok = false;
  if ((threadIdx.x & 31) == 0) ok = reached(sys ? ld_acquire_sys(p) : ld_acquire_gpu(p), target);
  return __shfl_sync(0xffffffffu, ok, 0);
}

// Warp-wide bounded wait until words[0 .. n-1] (n <= 32) have all reached
// target: lane j polls word j, so the n acquires are in flight together (one
// round trip per poll instead of n sequential waits).
__device__ __forceinline__ bool warp_wait_all(const uint32_t *words, int n, uint32_t target, int32_t *err,
                                              uint32_t tmo, bool sys) {
  const uint32_t lane = threadIdx.x & 31;
  bool mine = lane >= (uint32_t)n;
  const uint64_t t0 = globaltimer();
  uint32_t k = 0;
  for (;;) {
    if (!mine) mine = reached(sys ? ld_acquire_sys(words + lane) : ld_acquire_gpu(words + lane), target);
    if (__all_sync(0xffffffffu, mine)) return true;
    if ((++k & 63) == 0) {
      int stop = 0;
      if (lane == 0) {
        if (aborted(err)) {
          stop = 1;
        } else if (tmo && globaltimer() - t0 > (uint64_t)tmo * 1000000ull) {
          set_error(err, PC_DEV_ERR_TIMEOUT, -1);
          stop = 1;
        }
      }
      if (__shfl_sync(0xffffffffu, stop, 0)) return false;
      if (k > 1024) __nanosleep(256);
    }
  }
}

// Idle backoff shared by the sweeping engines; false on abort / timeout.
struct Idle {
  uint64_t since = 0;
  uint32_t ns = 0, spins = 0;
  __device__ __forceinline__ void progressed() {
    since = 0;
    ns = 0;
    spins = 0;
  }
  __device__ __forceinline__ bool wait(int32_t *err, uint32_t tmo, int part) {
    if (since == 0) since = globaltimer();
    // poll back-to-back first (a hop of a small message is ~1 us away), then
    // back off so long waits (large slices upstream) leave the L2 alone
    if (++spins > 64) {
      ns = ns ? (ns < 512 ? ns * 2 : 512) : 32;
      __nanosleep(ns);
    }
    if (aborted(err)) return false;
    if (tmo && globaltimer() - since > (uint64_t)tmo * 1000000ull) {
      if ((threadIdx.x & 31) == 0) set_error(err, PC_DEV_ERR_TIMEOUT, part);
      return false;
    }
    return true;
  }
};

template <int DT, int OP>
__device__ __forceinline__ void ring_step(const RingArgs &a, int u, int s, int i, uint32_t e) {
  const int P = a.P, r = a.r, NS = 2 * (P - 1);
  const int64_t es = sizeof(typename Op<DT, OP>::T);
  const int64_t base = (int64_t)u * a.L;
  const int64_t fbase = (int64_t)u * NS * a.ns + s;  // flag (u, i, s) = fbase + i * ns
  const int c = modp(r - i, P);                     // R_i = A_{i-1}
  const int64_t c_lo = min((int64_t)c * a.q, a.L), c_hi = min((int64_t)(c + 1) * a.q, a.L);
  const int64_t lo = c_lo + (int64_t)s * a.qs, hi = min(lo + a.qs, c_hi);
  const int64_t n = hi > lo ? hi - lo : 0;
  const int64_t off = (base + lo) * es;
  if (n) {
    if (i == 0)  // E_0: the user's Pready of S_0
      warp_copy(a.o_staging + off, a.sendbuf + off, n * es);
    else if (i <= P - 2)
      warp_reduce<DT, OP>(a.o_staging + off, nullptr, a.sendbuf + off, a.staging + off, n);
    else if (i == P - 1)
      warp_reduce<DT, OP>(a.recvbuf + off, a.o_recvbuf + off, a.sendbuf + off, a.staging + off, n);
    else
      warp_copy(a.o_recvbuf + off, a.recvbuf + off, n * es);
  }
  warp_signal(a.o_flags + fbase + (int64_t)i * a.ns, e, a.sys);
}

template <int DT, int OP>
__device__ __forceinline__ void ring_body(const RingArgs &a, const int gw, const int W) {
  const int P = a.P, NS = 2 * (P - 1);
  const uint32_t e = *(const volatile uint32_t *)a.epoch;  // device epoch word (graph-replayable)
  const int64_t es = sizeof(typename Op<DT, OP>::T);
  if (gw >= a.nunits) return;
  if (P == 1) {
    for (int x = gw; x < a.nunits; x += W) {
      const int u = x / a.ns, s = x % a.ns;
      if (!warp_wait(a.ready + u, e, a.err, a.timeout_ms, u, false)) return;
      const int64_t base = (int64_t)u * a.L, lo = (int64_t)s * a.qs, hi = min(lo + a.qs, a.L);
      if (hi > lo && a.sendbuf != a.recvbuf)
        warp_copy(a.recvbuf + (base + lo) * es, a.sendbuf + (base + lo) * es, (hi - lo) * es);
      __syncwarp();
      if ((threadIdx.x & 31) == 0) red_add_release_gpu(a.done + u, 1);
    }
    return;
  }
  // the consumer's ready-to-receive (written by a stream memop, never by an engine)
  if (!warp_wait(a.rtr, e, a.err, a.timeout_ms, -1, a.sys)) return;
  for (int j0 = 0; gw + j0 * W < a.nunits; j0 += kMaxActive) {
    int step[kMaxActive];
    int remaining = 0;
#pragma unroll
    for (int j = 0; j < kMaxActive; ++j) {
      const bool mine = gw + (j0 + j) * W < a.nunits;
      step[j] = mine ? 0 : NS + 1;
      remaining += mine;
    }
    Idle idle;
    while (remaining) {
      bool progressed = false;
#pragma unroll
      for (int j = 0; j < kMaxActive; ++j) {
        if (step[j] > NS) continue;
        const int x = gw + (j0 + j) * W;
        const int u = x / a.ns, s = x % a.ns;
        const int i = step[j];
        const uint32_t *dep = i == 0 ? a.ready + u : a.flags + ((int64_t)u * NS + (i - 1)) * a.ns + s;
        if (!warp_poll(dep, e, i != 0 && a.sys)) continue;
        progressed = true;
        if (i < NS) {
          ring_step<DT, OP>(a, u, s, i, e);
          step[j] = i + 1;
        } else {  // arrival of the last AG step: partition slice final here
          if ((threadIdx.x & 31) == 0) red_add_release_gpu(a.done + u, 1);
          step[j] = NS + 1;
          --remaining;
        }
      }
      if (progressed)
        idle.progressed();
      else if (!idle.wait(a.err, a.timeout_ms, gw))
        return;
    }
  }
}

// ---------------------------------------------------------------------------
// Recursive doubling: step k exchanges the whole slice with partner r ^ 2^k
// (its staging slot k); acc_{k+1} = acc_k ⊕ in_k is written to recv (the
// accumulator) and pushed to the next partner in the same pass.
// ---------------------------------------------------------------------------
template <int DT, int OP>
__device__ __forceinline__ void rd_body(const RdArgs &a, const int gw, const int W) {
  const int NS = a.nsteps;
  const uint32_t e = *(const volatile uint32_t *)a.epoch;  // device epoch word (graph-replayable)
  const int64_t es = sizeof(typename Op<DT, OP>::T);
  const int64_t stride = (int64_t)a.Np * a.L * es;  // bytes per staging slot
  uint32_t rtr_ok = 0;
  for (int x = gw; x < a.nunits; x += W) {
    const int u = x / a.ns, s = x % a.ns;
    const int64_t lo = (int64_t)s * a.qs, hi = min(lo + a.qs, a.L);
    const int64_t n = hi > lo ? hi - lo : 0;
    const int64_t off = ((int64_t)u * a.L + lo) * es;
    if (!warp_wait(a.ready + u, e, a.err, a.timeout_ms, u, false)) return;
    if (NS == 0) {
      if (n && a.sendbuf != a.recvbuf) warp_copy(a.recvbuf + off, a.sendbuf + off, n * es);
      __syncwarp();
      if ((threadIdx.x & 31) == 0) red_add_release_gpu(a.done + u, 1);
      continue;
    }
    auto fidx = [&](int k) { return ((int64_t)u * NS + k) * a.ns + s; };
    if (!(rtr_ok & 1u)) {
      if (!warp_wait(a.rtr + 0, e, a.err, a.timeout_ms, -1, a.sys)) return;
      rtr_ok |= 1u;
    }
    if (n) warp_copy(a.p_staging[0] + off, a.sendbuf + off, n * es);
    warp_signal(a.p_flags[0] + fidx(0), e, a.sys);
    for (int k = 0; k < NS; ++k) {
      if (!warp_wait(a.flags + fidx(k), e, a.err, a.timeout_ms, u, a.sys)) return;
      const uint8_t *acc = (k == 0) ? a.sendbuf : a.recvbuf;
      const uint8_t *in = a.staging + (int64_t)k * stride;
      if (k < NS - 1) {
        if (!(rtr_ok & (1u << (k + 1)))) {
          if (!warp_wait(a.rtr + k + 1, e, a.err, a.timeout_ms, -1, a.sys)) return;
          rtr_ok |= 1u << (k + 1);
        }
        if (n) warp_reduce<DT, OP>(a.recvbuf + off, a.p_staging[k + 1] + off, acc + off, in + off, n);
        warp_signal(a.p_flags[k + 1] + fidx(k + 1), e, a.sys);
      } else {
        if (n) warp_reduce<DT, OP>(a.recvbuf + off, nullptr, acc + off, in + off, n);
        __syncwarp();
      }
    }
    if ((threadIdx.x & 31) == 0) red_add_release_gpu(a.done + u, 1);
  }
}

// ---------------------------------------------------------------------------
// Direct two-step schedule (generic schedule with neighbour
// sets), PULL transport: the reduce step reads its P inputs
// straight from the peers' send buffers with peer loads over NVSwitch (no
// staging copy: per rank S bytes read + S written, vs. the ring's 2(P-1)/P·S
// over the links plus staging round trips in HBM).  Unit (u, slice s):
//   step 0 (after the user's Pready of u): announce "my partition u is final"
//          to every owner (release: the producer's writes, acquired through
//          ready[u], are ordered before the owner's reads) — bump each
//          owner's phase-0 counter for slice s;
//   step 1 (all P-1 phase-0 arrivals): fold the P contributions of my chunk
//          in rank order (reading R25) in registers, loading peer k's slice
//          from its send buffer, store the final slice locally and into every
//          peer's recvbuf, bump their phase-1 counters;
//   step 2 (all P-1 phase-1 arrivals): slice final everywhere -> done[u].
// A peer reuses its send buffer only after its own pc_wait, which needs every
// owner's phase-1 signal, issued after that owner's loads: no WAR hazard.
// ---------------------------------------------------------------------------
__device__ __forceinline__ void red_add_scope(uint32_t *p, uint32_t v, bool sys) {
  if (sys)
    asm volatile("red.relaxed.sys.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
  else
    asm volatile("red.relaxed.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// recvbuf[e0 .. e0+n) of this rank and of every peer = fold over ranks
// k = 0..P-1 (rank order, reading R25) of rank k's sendbuf[e0 ..), read with
// peer loads (PULL).  All operands sit at the same element offset of 16-B
// aligned buffers: scalar head, 16-B body, scalar tail.  Buffer pointers come
// straight from the kernel parameters (no pointer arrays on the stack).
// A: DirectArgs or CollArgs (sendbuf, p_sendbuf, recvbuf, p_recvbuf, P, r).
// Sources at element offset s0 of every rank's send buffer, destination at d0
// of this rank's recvbuf and (TO_PEERS) of every peer's.  When the sources and
// the destination do not share a 16-B misalignment the whole range takes the
// scalar path.
// L2 prefetch by the TMA engine (cp.async.bulk.prefetch.L2): bytes the warp
// will load soon are requested without registers or shared memory, so a thin
// warp (one 16-B vector per operand in registers) still keeps kPfAhead blocks
// of kPfBytes per source in flight.  16-B aligned, size a multiple of 16.
constexpr int64_t kPfBytes = 4096;
#ifndef PC_PF_AHEAD
#define PC_PF_AHEAD 2
#endif
constexpr int kPfAhead = PC_PF_AHEAD;
__device__ __forceinline__ void prefetch_l2(const void *p, int64_t bytes) {
  if (bytes <= 0) return;
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"((uint32_t)bytes) : "memory");
}

// MAXP: the largest P the call handles (P <= MAXP): the register arrays are
// sized by it, so a small comm can keep FV * 8 / MAXP vectors per operand in
// flight for the same registers (direct_body picks MAXP from P).
template <int DT, int OP, bool TO_PEERS = true, int FV = PC_DIRECT_FV, bool PF = false, int MAXP = kMaxDirect,
          typename A>
__device__ __forceinline__ void warp_fold_pull(const A &a, int64_t s0, int64_t d0, int64_t n) {
  using O = Op<DT, OP>;
  using T = typename O::T;
  const int P = a.P, r = a.r;
  const uint32_t lane = threadIdx.x & 31;
  constexpr int64_t EPV = 16 / sizeof(T);
  auto src = [&](int k) -> const T * {
    return reinterpret_cast<const T *>(k == r ? a.sendbuf : a.p_sendbuf[(k - r - 1 + P) % P]) + s0;
  };
  const int64_t e0 = d0;
  T *out_local = reinterpret_cast<T *>(a.recvbuf) + e0;
  const uintptr_t m = reinterpret_cast<uintptr_t>(out_local) & 15;
  int64_t head = (int64_t)(((16 - m) & 15) / sizeof(T));
  if ((reinterpret_cast<uintptr_t>(src(r)) & 15) != m) head = n;  // no common misalignment
  if (head > n) head = n;
  auto scalar = [&](int64_t k) {
    T acc = __ldcg(src(0) + k);
    for (int j = 1; j < P; ++j) acc = O::f(acc, __ldcg(src(j) + k));
    out_local[k] = acc;
    if (TO_PEERS)
      for (int j = 0; j < P - 1; ++j) (reinterpret_cast<T *>(a.p_recvbuf[j]) + e0)[k] = acc;
  };
  for (int64_t k = lane; k < head; k += 32) scalar(k);
  const int64_t nv = (n - head) / EPV;
  // all P * kFV loads of a lane are issued before the first add (the fold
  // itself stays in rank order): one round trip per kFV vectors, not P
  constexpr int kFV = FV;
  auto store_all = [&](int64_t vk, uint4 acc) {
    const int64_t eo = head + EPV * vk;
    *reinterpret_cast<uint4 *>(out_local + eo) = acc;
    if (TO_PEERS) {
#pragma unroll
      for (int j = 0; j < kMaxDirect - 1; ++j)
        if (j < P - 1) *reinterpret_cast<uint4 *>(reinterpret_cast<T *>(a.p_recvbuf[j]) + e0 + eo) = acc;
    }
  };
  // PF: lane j < P prefetches source j's 16-B body in blocks of kPfBytes,
  // kPfAhead blocks ahead of the loads (same-GPU peers only: a.sys == 0)
  constexpr int64_t kPfV = kPfBytes / 16;  // vectors per prefetch block
  const bool pf = PF && !a.sys && (int)lane < P;
  auto pf_block = [&](int64_t b) {
    const int64_t v0 = b * kPfV;
    if (v0 < nv)
      prefetch_l2(reinterpret_cast<const uint4 *>(src((int)lane) + head) + v0, (min(nv - v0, kPfV)) * 16);
  };
  if (pf)
    for (int b = 0; b < kPfAhead; ++b) pf_block(b);
  int64_t k = lane;
  for (; k + 32 * (kFV - 1) < nv; k += 32 * kFV) {
    if (pf && ((k - lane) % kPfV) == 0) pf_block((k - lane) / kPfV + kPfAhead);
    uint4 x[MAXP][kFV];
#pragma unroll
    for (int j = 0; j < MAXP; ++j)
      if (j < P) {
        const uint4 *sj = reinterpret_cast<const uint4 *>(src(j) + head);
#pragma unroll
        for (int v = 0; v < kFV; ++v) x[j][v] = __ldcg(sj + k + 32 * v);
      }
#pragma unroll
    for (int v = 0; v < kFV; ++v) {
      uint4 acc = x[0][v];
#pragma unroll
      for (int j = 1; j < MAXP; ++j)
        if (j < P) acc = vop<DT, OP>(acc, x[j][v]);
      store_all(k + 32 * v, acc);
    }
  }
  for (; k < nv; k += 32) {
    uint4 x[MAXP];
#pragma unroll
    for (int j = 0; j < MAXP; ++j)
      if (j < P) x[j] = __ldcg(reinterpret_cast<const uint4 *>(src(j) + head) + k);
    uint4 acc = x[0];
#pragma unroll
    for (int j = 1; j < MAXP; ++j)
      if (j < P) acc = vop<DT, OP>(acc, x[j]);
    store_all(k, acc);
  }
  for (int64_t kk = head + nv * EPV + lane; kk < n; kk += 32) scalar(kk);
}

// ---------------------------------------------------------------------------
// Bulk-copy PULL fold (DIRECT allreduce, same-GPU peers): the P source chunks
// of 512 B (one 16-B vector per lane) reach this warp's shared-memory stage by
// cp.async.bulk (the TMA engine), completing on the stage's mbarrier, so the
// loads in flight are no longer bounded by registers (the register version
// holds P vectors per lane and spills at 2).  Two stages per warp: while the
// warp folds stage s (rank order, R25) and stores the result to every rank's
// recvbuf, stage s^1's P copies are in flight.
// ---------------------------------------------------------------------------
#ifndef PC_DIRECT_BULK
#define PC_DIRECT_BULK 0  // measured 0.80-0.87 of HBM vs 0.99 for the register fold
#endif
#ifndef PC_BULK_STAGES
#define PC_BULK_STAGES 2
#endif
#ifndef PC_BULK_CHUNK
#define PC_BULK_CHUNK 512
#endif
constexpr int kBulkStages = PC_BULK_STAGES;
constexpr int kBulkChunk = PC_BULK_CHUNK;  // bytes per source per stage (a multiple of 512)
constexpr int kBulkWarpBytes = (kBulkStages * kMaxDirect * kBulkChunk + 8 * kBulkStages + 127) / 128 * 128;
constexpr size_t kBulkSmem = (size_t)(kEngineBlock / 32) * kBulkWarpBytes;  // a CTA's bulk stages
constexpr size_t kDirectSmem = PC_DIRECT_BULK ? kBulkSmem : 0;
// The thin (overlap) DIRECT engines: one 16-B vector per operand in flight in
// registers (PC_THIN_FV), or the bulk-copy fold (PC_THIN_BULK: the P source
// chunks staged in shared memory by cp.async.bulk, so the bytes in flight are
// not bounded by the 128-register budget; same-GPU peers only).
#ifndef PC_THIN_FV
#define PC_THIN_FV 1
#endif
#ifndef PC_THIN_BULK
#define PC_THIN_BULK 0
#endif
constexpr size_t kThinSmem = PC_THIN_BULK ? kBulkSmem : 0;

struct WarpBulk {
  uint8_t *stage;     // [kBulkStages][kMaxDirect][kBulkChunk]
  uint64_t *bar;      // [kBulkStages]
  uint32_t phase;     // bit s: parity of stage s's next completion
};

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void warp_bulk_init(WarpBulk &wb, uint8_t *smem) {
  const int wib = threadIdx.x >> 5;
  wb.stage = smem + (size_t)wib * kBulkWarpBytes;
  wb.bar = reinterpret_cast<uint64_t *>(wb.stage + kBulkStages * kMaxDirect * kBulkChunk);
  wb.phase = 0;
  if ((threadIdx.x & 31) == 0) {
    for (int s = 0; s < kBulkStages; ++s)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(wb.bar + s)) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
}

// lane 0: P bulk copies of `bytes` each into stage st, one mbarrier transaction
template <typename SrcFn>
__device__ __forceinline__ void bulk_issue(WarpBulk &wb, int st, int P, SrcFn src, uint32_t bytes) {
  const uint32_t bar = smem_u32(wb.bar + st);
  asm volatile("{\n .reg .b64 s;\n mbarrier.arrive.expect_tx.shared::cta.b64 s, [%0], %1;\n}" ::"r"(bar),
               "r"(bytes * (uint32_t)P)
               : "memory");
  for (int j = 0; j < P; ++j)
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(wb.stage + ((size_t)st * kMaxDirect + j) * kBulkChunk)),
                 "l"(src(j)), "r"(bytes), "r"(bar)
                 : "memory");
}

__device__ __forceinline__ void bulk_wait(WarpBulk &wb, int st) {
  const uint32_t bar = smem_u32(wb.bar + st), par = (wb.phase >> st) & 1u;
  asm volatile("{\n .reg .pred p;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W_%=;\n}" ::"r"(
                   bar),
               "r"(par)
               : "memory");
  wb.phase ^= 1u << st;
}

// As warp_fold_pull<.., TO_PEERS=true>, with the 16-B body moved by bulk copies.
template <int DT, int OP, typename A>
__device__ __forceinline__ void warp_fold_pull_bulk(const A &a, int64_t s0, int64_t d0, int64_t n, WarpBulk &wb) {
  using O = Op<DT, OP>;
  using T = typename O::T;
  const int P = a.P, r = a.r;
  const uint32_t lane = threadIdx.x & 31;
  constexpr int64_t EPV = 16 / sizeof(T);
  auto src = [&](int k) -> const T * {
    return reinterpret_cast<const T *>(k == r ? a.sendbuf : a.p_sendbuf[(k - r - 1 + P) % P]) + s0;
  };
  T *out_local = reinterpret_cast<T *>(a.recvbuf) + d0;
  const uintptr_t m = reinterpret_cast<uintptr_t>(out_local) & 15;
  if ((reinterpret_cast<uintptr_t>(src(r)) & 15) != m) {  // no common misalignment: register path
    warp_fold_pull<DT, OP, true>(a, s0, d0, n);
    return;
  }
  int64_t head = (int64_t)(((16 - m) & 15) / sizeof(T));
  if (head > n) head = n;
  auto scalar = [&](int64_t k) {
    T acc = __ldcg(src(0) + k);
    for (int j = 1; j < P; ++j) acc = O::f(acc, __ldcg(src(j) + k));
    out_local[k] = acc;
    for (int j = 0; j < P - 1; ++j) (reinterpret_cast<T *>(a.p_recvbuf[j]) + d0)[k] = acc;
  };
  for (int64_t k = lane; k < head; k += 32) scalar(k);
  constexpr int64_t VPC = kBulkChunk / 16;  // 16-B vectors per chunk per source
  const int64_t nv = (n - head) / EPV;      // 16-B vectors of the body
  const int64_t nch = (nv + VPC - 1) / VPC; // chunks per source
  auto chunk_src = [&](int64_t c) {
    return [=](int j) { return reinterpret_cast<const void *>(src(j) + head + c * VPC * EPV); };
  };
  auto chunk_bytes = [&](int64_t c) { return (uint32_t)((nv - c * VPC < VPC ? nv - c * VPC : VPC) * 16); };
  if (nch > 0 && lane == 0) {
    asm volatile("fence.proxy.async.global;" ::: "memory");  // producers' generic writes -> bulk reads
    for (int64_t c = 0; c < nch && c < kBulkStages; ++c) bulk_issue(wb, (int)c, P, chunk_src(c), chunk_bytes(c));
  }
  for (int64_t c = 0; c < nch; ++c) {
    const int st = (int)(c % kBulkStages);
    bulk_wait(wb, st);
#pragma unroll
    for (int64_t v = 0; v < VPC / 32; ++v) {
      const int64_t vk = c * VPC + v * 32 + lane;
      if (vk < nv) {
        const uint4 *sv =
            reinterpret_cast<const uint4 *>(wb.stage + (size_t)st * kMaxDirect * kBulkChunk) + v * 32 + lane;
        uint4 acc = sv[0];
#pragma unroll
        for (int j = 1; j < kMaxDirect; ++j)
          if (j < P) acc = vop<DT, OP>(acc, sv[j * VPC]);
        const int64_t eo = head + EPV * vk;
        *reinterpret_cast<uint4 *>(out_local + eo) = acc;
#pragma unroll
        for (int j = 0; j < kMaxDirect - 1; ++j)
          if (j < P - 1) *reinterpret_cast<uint4 *>(reinterpret_cast<T *>(a.p_recvbuf[j]) + d0 + eo) = acc;
      }
    }
    __syncwarp();
    if (c + kBulkStages < nch && lane == 0) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // our generic reads of the stage -> refill
      bulk_issue(wb, st, P, chunk_src(c + kBulkStages), chunk_bytes(c + kBulkStages));
    }
  }
  for (int64_t kk = head + nv * EPV + lane; kk < n; kk += 32) scalar(kk);
}

// Rank-order fold of one slice with rank-indexed source pointers S[k] and
// destinations D[0] (own recvbuf), D[1..P-1] (peers), all at the same byte
// offset: scalar head / 16-B body (FV vectors per operand in flight) / tail.
template <int DT, int OP, int FV>
__device__ __forceinline__ void warp_fold_ptrs(const uint8_t *const (&S)[kMaxDirect], uint8_t *const (&D)[kMaxDirect],
                                               int P, int64_t n) {
  using O = Op<DT, OP>;
  using T = typename O::T;
  const uint32_t lane = threadIdx.x & 31;
  constexpr int64_t EPV = 16 / sizeof(T);
  const uintptr_t m = reinterpret_cast<uintptr_t>(D[0]) & 15;
  int64_t head = (int64_t)(((16 - m) & 15) / sizeof(T));
  bool common = true;  // every source and destination shares D[0]'s misalignment (PUSH: the
#pragma unroll         // 16-B aligned staging slots may not): else the scalar path
  for (int j = 0; j < kMaxDirect; ++j)
    if (j < P)
      common = common && (reinterpret_cast<uintptr_t>(S[j]) & 15) == m && (reinterpret_cast<uintptr_t>(D[j]) & 15) == m;
  if (!common) head = n;
  if (head > n) head = n;
  auto scalar = [&](int64_t k) {
    T acc = __ldcg(reinterpret_cast<const T *>(S[0]) + k);
#pragma unroll
    for (int j = 1; j < kMaxDirect; ++j)
      if (j < P) acc = O::f(acc, __ldcg(reinterpret_cast<const T *>(S[j]) + k));
#pragma unroll
    for (int j = 0; j < kMaxDirect; ++j)
      if (j < P) reinterpret_cast<T *>(D[j])[k] = acc;
  };
  for (int64_t k = lane; k < head; k += 32) scalar(k);
  const int64_t nv = (n - head) / EPV;
  int64_t k = lane;
  for (; k + 32 * (FV - 1) < nv; k += 32 * FV) {
    uint4 x[kMaxDirect][FV];
#pragma unroll
    for (int j = 0; j < kMaxDirect; ++j)
      if (j < P) {
#pragma unroll
        for (int v = 0; v < FV; ++v)
          x[j][v] = __ldcg(reinterpret_cast<const uint4 *>(reinterpret_cast<const T *>(S[j]) + head) + k + 32 * v);
      }
#pragma unroll
    for (int v = 0; v < FV; ++v) {
      uint4 acc = x[0][v];
#pragma unroll
      for (int j = 1; j < kMaxDirect; ++j)
        if (j < P) acc = vop<DT, OP>(acc, x[j][v]);
#pragma unroll
      for (int j = 0; j < kMaxDirect; ++j)
        if (j < P) reinterpret_cast<uint4 *>(reinterpret_cast<T *>(D[j]) + head)[k + 32 * v] = acc;
    }
  }
  for (; k < nv; k += 32) {
    uint4 acc = __ldcg(reinterpret_cast<const uint4 *>(reinterpret_cast<const T *>(S[0]) + head) + k);
    uint4 x[kMaxDirect];
#pragma unroll
    for (int j = 1; j < kMaxDirect; ++j)
      if (j < P) x[j] = __ldcg(reinterpret_cast<const uint4 *>(reinterpret_cast<const T *>(S[j]) + head) + k);
#pragma unroll
    for (int j = 1; j < kMaxDirect; ++j)
      if (j < P) acc = vop<DT, OP>(acc, x[j]);
#pragma unroll
    for (int j = 0; j < kMaxDirect; ++j)
      if (j < P) reinterpret_cast<uint4 *>(reinterpret_cast<T *>(D[j]) + head)[k] = acc;
  }
  for (int64_t kk = head + nv * EPV + lane; kk < n; kk += 32) scalar(kk);
}

template <int DT, int OP, int FV = PC_DIRECT_FV, bool PF = false, bool PUSH = false, bool BULK = PC_DIRECT_BULK,
          int MAXP = kMaxDirect>
__device__ __forceinline__ void direct_body(const DirectArgs &a, const int gw, const int W, uint8_t *smem) {
  const int P = a.P, r = a.r;
  const uint32_t e = *(const volatile uint32_t *)a.epoch;
  const int64_t es = sizeof(typename Op<DT, OP>::T);
  if (gw >= a.nunits) return;
  if (P == 1) {
    for (int x = gw; x < a.nunits; x += W) {
      const int u = x / a.ns, s = x % a.ns;
      if (!warp_wait(a.ready + u, e, a.err, a.timeout_ms, u, false)) return;
      const int64_t base = (int64_t)u * a.L, lo = (int64_t)s * a.qs, hi = min(lo + a.qs, a.L);
      if (hi > lo && a.sendbuf != a.recvbuf)
        warp_copy(a.recvbuf + (base + lo) * es, a.sendbuf + (base + lo) * es, (hi - lo) * es);
      __syncwarp();
      if ((threadIdx.x & 31) == 0) red_add_release_gpu(a.done + u, 1);
    }
    return;
  }
  WarpBulk wb{};
  if (BULK && !a.sys) warp_bulk_init(wb, smem);
  // every peer has posted ready-to-receive (all P-1 words polled at once)
  if (!warp_wait_all(a.rtr, P - 1, e, a.err, a.timeout_ms, a.sys)) return;
  const uint32_t target = e * (uint32_t)(P - 1);
  for (int j0 = 0; gw + j0 * W < a.nunits; j0 += kMaxActive) {
    int step[kMaxActive];
    int remaining = 0;
#pragma unroll
    for (int j = 0; j < kMaxActive; ++j) {
      const bool mine = gw + (j0 + j) * W < a.nunits;
      step[j] = mine ? 0 : 3;
      remaining += mine;
    }
    Idle idle;
    while (remaining) {
      bool progressed = false;
#pragma unroll
      for (int jj = 0; jj < kMaxActive; ++jj) {
        if (step[jj] > 2) continue;
        const int x = gw + (j0 + jj) * W;
        const int u = x / a.ns, s = x % a.ns;
        const int i = step[jj];
        const uint32_t *dep = i == 0 ? a.ready + u : a.cnt + ((int64_t)u * 2 + (i - 1)) * a.ns + s;
        if (!warp_poll(dep, i == 0 ? e : target, i != 0 && a.sys)) continue;
        progressed = true;
        const int64_t base = (int64_t)u * a.L;
        if (i == 0) {
          if (PUSH) {  // PUSH: my slice s of chunk o -> owner o's staging slot [u][r] (peer stores)
            for (int j = 0; j < P - 1; ++j) {
              const int o = (r + 1 + j) % P;
              const int64_t o_lo = min((int64_t)o * a.q, a.L), o_hi = min((int64_t)(o + 1) * a.q, a.L);
              const int64_t lo = o_lo + (int64_t)s * a.qs, hi = min(lo + a.qs, o_hi);
              if (hi > lo)
                warp_copy(const_cast<uint8_t *>(a.p_sendbuf[j]) + (((int64_t)u * P + r) * a.q + (int64_t)s * a.qs) * es,
                          a.sendbuf + (base + lo) * es, (hi - lo) * es);
            }
          }
          fence_release(a.sys);
          __syncwarp();
          if ((threadIdx.x & 31) == 0)
            for (int j = 0; j < P - 1; ++j) red_add_scope(a.p_cnt[j] + ((int64_t)u * 2 + 0) * a.ns + s, 1, a.sys);
          step[jj] = 1;
        } else if (i == 1) {
          const int64_t c_lo = min((int64_t)r * a.q, a.L), c_hi = min((int64_t)(r + 1) * a.q, a.L);
          const int64_t lo = c_lo + (int64_t)s * a.qs, hi = min(lo + a.qs, c_hi);
          if (PUSH && hi > lo) {  // PUSH: every source is local (my send buffer / my staging slots)
            const uint8_t *S[kMaxDirect];
            uint8_t *D[kMaxDirect];
#pragma unroll
            for (int k = 0; k < kMaxDirect; ++k) {
              S[k] = nullptr;
              D[k] = nullptr;
              if (k < P) {
                S[k] = k == r ? a.sendbuf + (base + lo) * es
                              : a.staging + (((int64_t)u * P + k) * a.q + (int64_t)s * a.qs) * es;
                D[k] = (k == 0 ? a.recvbuf : a.p_recvbuf[k - 1]) + (base + lo) * es;
              }
            }
            warp_fold_ptrs<DT, OP, FV>(S, D, P, hi - lo);
          } else if (!PUSH && hi > lo) {
            if (BULK && !a.sys)
              warp_fold_pull_bulk<DT, OP>(a, base + lo, base + lo, hi - lo, wb);
            else  // MAXP < 8: fewer sources, FV * 8 / MAXP vectors per operand in flight, same registers
              warp_fold_pull<DT, OP, true, FV * kMaxDirect / MAXP, PF, MAXP>(a, base + lo, base + lo, hi - lo);
          }
          fence_release(a.sys);
          __syncwarp();
          if ((threadIdx.x & 31) == 0)
            for (int j = 0; j < P - 1; ++j) red_add_scope(a.p_cnt[j] + ((int64_t)u * 2 + 1) * a.ns + s, 1, a.sys);
          step[jj] = 2;
        } else {
          if ((threadIdx.x & 31) == 0) red_add_release_gpu(a.done + u, 1);
          step[jj] = 3;
          --remaining;
        }
      }
      if (progressed)
        idle.progressed();
      else if (!idle.wait(a.err, a.timeout_ms, gw))
        return;
    }
  }
}

// ---------------------------------------------------------------------------
// One-shot LL allreduce (PC_ALGO_LL, small messages).  Unit = user partition
// u.  Step 0 (the user's Pready of u): the warp stores partition u as 16-B
// lines {4 B data, e, 4 B data, e} into slot [e & 1][r][u] of EVERY peer's
// line area — no fence, no flag: each 8-B half carries the epoch, so a line is
// its own arrival flag.  Step 1: every line of u from all P-1 peers carries
// epoch e -> fold the P contributions in rank order (R25; my own from my send
// buffer) and store the result into MY recvbuf only -> done[u].  One hop.
// Parity slot e&1 was last read by the peer in epoch e-2; this rank completing
// e-1 needed the peer's e-1 lines, pushed by the peer's engine e-1, which runs
// after its engine e-2 finished reading — so no ready-to-receive is needed.
// ---------------------------------------------------------------------------
template <int DT, int OP>
__device__ __forceinline__ uint64_t vop8(uint64_t a, uint64_t b) {
  using O = Op<DT, OP>;
  using T = typename O::T;
  constexpr int EPW = 8 / sizeof(T);
  uint64_t r;
  T *pr = reinterpret_cast<T *>(&r);
  const T *pa = reinterpret_cast<const T *>(&a);
  const T *pb = reinterpret_cast<const T *>(&b);
#pragma unroll
  for (int j = 0; j < EPW; ++j) pr[j] = O::f(pa[j], pb[j]);
  return r;
}

// Unit = (partition u, slice s) of 32 * kLLPerLane lines: each lane owns at
// most kLLPerLane lines of the slice, loads them from all P-1 sources at once
// (every load in flight together), validates, and folds straight from the
// registers.
constexpr int kLLPerLane = 2;
constexpr int64_t kLLSlice = 32 * kLLPerLane;  // lines per unit

template <int DT, int OP>
__device__ __forceinline__ void ll_body(const DirectArgs &a, const int gw, const int W) {
  const int P = a.P, r = a.r;
  const uint32_t e = *(const volatile uint32_t *)a.epoch;
  const uint32_t lane = threadIdx.x & 31;
  const int64_t es = sizeof(typename Op<DT, OP>::T);
  const uint64_t pb = (uint64_t)a.L * es;  // bytes per partition
  const int64_t Lp = a.ll_lines;           // lines per partition
  const int64_t par = e & 1;
  auto line = [&](const uint8_t *area, int k, int u, int64_t j) {  // line (parity, source k, partition u, j)
    return area + ((((par * P + k) * (int64_t)a.Np + u) * Lp + j) << 4);
  };
  if (gw >= a.nunits) return;
  for (int j0 = 0; gw + j0 * W < a.nunits; j0 += kMaxActive) {
    int step[kMaxActive];
    int remaining = 0;
#pragma unroll
    for (int j = 0; j < kMaxActive; ++j) {
      const bool mine = gw + (j0 + j) * W < a.nunits;
      step[j] = mine ? 0 : 2;
      remaining += mine;
    }
    Idle idle;
    while (remaining) {
      bool progressed = false;
#pragma unroll 1
      for (int jj = 0; jj < kMaxActive; ++jj) {
        if (step[jj] > 1) continue;
        const int x = gw + (j0 + jj) * W;
        const int u = x / a.ns;
        const int64_t k0 = (int64_t)(x % a.ns) * kLLSlice;
        const uint8_t *src = a.sendbuf + (uint64_t)u * pb;
        if (step[jj] == 0) {
          if (!warp_poll(a.ready + u, e, false)) continue;
#pragma unroll
          for (int t = 0; t < kLLPerLane; ++t) {  // push: my lines of the slice to every peer
            const int64_t k = k0 + t * 32 + lane;
            if (k >= Lp) continue;
            const uint32_t nb = ll_nbytes(pb, (uint32_t)k);
            const uint64_t v = nb ? ld_payload8(src + 8 * k, nb) : 0;
            const uint64_t lo = (v & 0xffffffffull) | ((uint64_t)e << 32), hi = (v >> 32) | ((uint64_t)e << 32);
            for (int j = 0; j < P - 1; ++j)
              st_ll(const_cast<uint8_t *>(line(a.p_sendbuf[j], r, u, k)), lo, hi, a.sys);
          }
          step[jj] = 1;
          progressed = true;
        } else {
          // every source's lines in flight at once, then one validity vote
          ulonglong2 ln[kMaxDirect][kLLPerLane];
          bool ok = true;
#pragma unroll
          for (int q = 0; q < kMaxDirect; ++q)
#pragma unroll
            for (int t = 0; t < kLLPerLane; ++t) {
              const int64_t k = k0 + t * 32 + lane;
              ln[q][t] = make_ulonglong2(0, 0);
              if (q < P && q != r && k < Lp) ln[q][t] = ld_ll(line(a.staging, q, u, k), a.sys);
            }
#pragma unroll
          for (int q = 0; q < kMaxDirect; ++q)
#pragma unroll
            for (int t = 0; t < kLLPerLane; ++t) {
              const int64_t k = k0 + t * 32 + lane;
              if (q < P && q != r && k < Lp)
                ok = ok && (uint32_t)(ln[q][t].x >> 32) == e && (uint32_t)(ln[q][t].y >> 32) == e;
            }
          if (!__all_sync(0xffffffffu, ok)) continue;
#pragma unroll
          for (int t = 0; t < kLLPerLane; ++t) {  // fold in rank order, store my result
            const int64_t k = k0 + t * 32 + lane;
            const uint32_t nb = k < Lp ? ll_nbytes(pb, (uint32_t)k) : 0u;
            if (!nb) continue;
            uint64_t acc = 0;
#pragma unroll
            for (int q = 0; q < kMaxDirect; ++q) {
              if (q >= P) continue;
              const uint64_t v = q == r ? ld_payload8(src + 8 * k, nb)
                                        : (ln[q][t].x & 0xffffffffull) | (ln[q][t].y << 32);
              acc = q == 0 ? v : vop8<DT, OP>(acc, v);
            }
            st_payload8(a.recvbuf + (uint64_t)u * pb + 8 * k, acc, nb);
          }
          __syncwarp();
          if (lane == 0) red_add_release_gpu(a.done + u, 1);
          step[jj] = 2;
          --remaining;
          progressed = true;
        }
      }
      if (progressed)
        idle.progressed();
      else if (!idle.wait(a.err, a.timeout_ms, gw))
        return;
    }
  }
}

template <int DT, int OP>
__global__ void __launch_bounds__(kEngineBlock) ll_engine(DirectArgs a) {
  ll_body<DT, OP>(a, (blockIdx.x * blockDim.x + threadIdx.x) >> 5, (gridDim.x * blockDim.x) >> 5);
}
template <int DT, int OP>
__global__ void __launch_bounds__(kEngineBlock) ll_engine_group(DirectGroupArgs g) {
  int k = 0;
  while (k + 1 < g.n && (int)blockIdx.x >= g.block_start[k + 1]) ++k;
  const int b = blockIdx.x - g.block_start[k];
  const int nb = (k + 1 < g.n ? g.block_start[k + 1] : (int)gridDim.x) - g.block_start[k];
  ll_body<DT, OP>(g.a[k], (b * blockDim.x + threadIdx.x) >> 5, (nb * blockDim.x) >> 5);
}

// ---------------------------------------------------------------------------
// Batched DIRECT engine: MPI_Waitall over many partitioned allreduces of one
// GPU in ONE launch (one request per gradient tensor).
// Entries (request t, local rank j) live in a device table (DirectArgs are
// epoch-invariant; each unit reads its request's epoch word).  Global units
// are ordered [t][x][j] — a logical unit's local ranks are adjacent — and
// every warp takes its global units in increasing order, so the smallest
// incomplete logical unit is active on every rank whatever the width
// (deadlock freedom).  Same steps and bits as direct_body.
// ---------------------------------------------------------------------------
__device__ __forceinline__ bool warp_poll_all(const uint32_t *words, int n, uint32_t target, bool sys) {
  const uint32_t lane = threadIdx.x & 31;
  bool mine = lane >= (uint32_t)n || reached(sys ? ld_acquire_sys(words + lane) : ld_acquire_gpu(words + lane), target);
  return __all_sync(0xffffffffu, mine);
}

template <int DT, int OP, int FV>
__device__ __forceinline__ void direct_batch_body(const DirectBatchArgs b, const int gw, const int W) {
  const int R = b.R;
  const int total = b.ubase[b.nreq];
  for (int j0 = 0; gw + j0 * W < total; j0 += kMaxActive) {
    int step[kMaxActive], ent[kMaxActive], unit[kMaxActive];
    uint32_t ep[kMaxActive];
    int remaining = 0;
#pragma unroll
    for (int jj = 0; jj < kMaxActive; ++jj) {
      const int g = gw + (j0 + jj) * W;
      step[jj] = 3;
      ent[jj] = 0;
      unit[jj] = 0;
      ep[jj] = 0;
      if (g < total) {
        int lo = 0, hi = b.nreq;  // request t: ubase[t] <= g < ubase[t + 1]
        while (hi - lo > 1) {
          const int mid = (lo + hi) >> 1;
          if (b.ubase[mid] <= g) lo = mid; else hi = mid;
        }
        const int off = g - b.ubase[lo];
        ent[jj] = lo * R + off % R;
        unit[jj] = off / R;
        ep[jj] = *(const volatile uint32_t *)b.tab[ent[jj]].epoch;
        step[jj] = 0;
        ++remaining;
      }
    }
    Idle idle;
    while (remaining) {
      bool progressed = false;
#pragma unroll
      for (int jj = 0; jj < kMaxActive; ++jj) {
        if (step[jj] > 2) continue;
        const DirectArgs &a = b.tab[ent[jj]];
        const int P = a.P, r = a.r, ns = a.ns, sys = a.sys;
        const int u = unit[jj] / ns, s = unit[jj] % ns;
        const int i = step[jj];
        const uint32_t e = ep[jj];
        if (i == 0) {  // the user's Pready of u, and every peer's ready-to-receive
          if (!warp_poll(a.ready + u, e, false) || !warp_poll_all(a.rtr, P - 1, e, sys)) continue;
        } else if (!warp_poll(a.cnt + ((int64_t)u * 2 + (i - 1)) * ns + s, e * (uint32_t)(P - 1), sys)) {
          continue;
        }
        progressed = true;
        if (i == 0) {
          fence_release(sys);
          __syncwarp();
          if ((threadIdx.x & 31) == 0)
            for (int j = 0; j < P - 1; ++j) red_add_scope(a.p_cnt[j] + ((int64_t)u * 2 + 0) * ns + s, 1, sys);
          step[jj] = 1;
        } else if (i == 1) {
          const int64_t es = sizeof(typename Op<DT, OP>::T);
          const int64_t c_lo = min((int64_t)r * a.q, a.L), c_hi = min((int64_t)(r + 1) * a.q, a.L);
          const int64_t lo = c_lo + (int64_t)s * a.qs, hi = min(lo + a.qs, c_hi);
          if (hi > lo) {
            const int64_t boff = ((int64_t)u * a.L + lo) * es;
            const uint8_t *S[kMaxDirect];
            uint8_t *D[kMaxDirect];
#pragma unroll
            for (int k = 0; k < kMaxDirect; ++k) {  // rank-indexed sources, D[0] = own recvbuf
              S[k] = nullptr;
              D[k] = nullptr;
              if (k < P) {
                S[k] = (k == r ? a.sendbuf : a.p_sendbuf[(k - r - 1 + P) % P]) + boff;
                D[k] = (k == 0 ? a.recvbuf : a.p_recvbuf[k - 1]) + boff;
              }
            }
            warp_fold_ptrs<DT, OP, FV>(S, D, P, hi - lo);
          }
          fence_release(sys);
          __syncwarp();
          if ((threadIdx.x & 31) == 0)
            for (int j = 0; j < P - 1; ++j) red_add_scope(a.p_cnt[j] + ((int64_t)u * 2 + 1) * ns + s, 1, sys);
          step[jj] = 2;
        } else {
          if ((threadIdx.x & 31) == 0) red_add_release_gpu(a.done + u, 1);
          step[jj] = 3;
          --remaining;
        }
      }
      if (progressed)
        idle.progressed();
      else if (!idle.wait(b.err, b.timeout_ms, gw))
        return;
    }
  }
}

template <int DT, int OP>
__global__ void __launch_bounds__(kEngineBlock, PC_DIRECT_MINB) direct_engine_batch(DirectBatchArgs b) {
  direct_batch_body<DT, OP, PC_DIRECT_FV>(b, (blockIdx.x * blockDim.x + threadIdx.x) >> 5,
                                          (gridDim.x * blockDim.x) >> 5);
}
template <int DT, int OP>
__global__ void __launch_bounds__(kEngineBlock, 2) direct_engine_batch_thin(DirectBatchArgs b) {
  direct_batch_body<DT, OP, 1>(b, (blockIdx.x * blockDim.x + threadIdx.x) >> 5, (gridDim.x * blockDim.x) >> 5);
}

// ---------------------------------------------------------------------------
// Partitioned reduce-scatter / allgather / broadcast: the two
// halves of the DIRECT schedule and its one-to-all special case, same unit
// sweep (Alg 2 on a warp).  Unit (u, slice s) of one block of `count` elements.
//  REDUCE_SCATTER (sendbuf [u][P blocks], recvbuf [u][count]), PULL:
//    0: ready[u] -> announce to every peer (phase-0 counter)
//    1: P-1 announcements -> fold block r of partition u over all ranks in rank
//       order (peer loads) into my recvbuf[u]; tell every peer "done reading"
//    2: P-1 "done reading" -> done[u]  (my send buffer is reusable)
//  ALLGATHER (sendbuf [u][count], recvbuf [rank][u][count]), PUSH:
//    0: ready[u] -> copy my block to recvbuf[r][u] here and at every peer,
//       fence, per-source arrival flag + phase-0 counter at every peer
//    1: P-1 arrivals of partition u -> done[u]
//  BCAST (buf [u][count]): root: ready[u] -> announce to every peer
//    (phase-0 counter) -> all P-1 parts read (phase-1) -> done[u];
//    non-root kk (of P-1): root's announcement -> read part kk of the root's
//    slice ONCE (peer loads) and store it into every receiver's buf -> bump
//    the root's and every receiver's phase-1 counter -> (all P-1 parts of my
//    slice arrived) done[u].  The root's slice leaves it once (S, not (P-1) S)
//  (ALLGATHER pushes each vector once to all P buffers: warp_copy_multi)
// ---------------------------------------------------------------------------
template <int DT, int OP, int MAXP = kMaxDirect>
__device__ __forceinline__ void coll_body(const CollArgs &a, const int gw, const int W) {
  const int P = a.P, r = a.r;
  const uint32_t e = *(const volatile uint32_t *)a.epoch;
  const int64_t es = a.es;
  if (gw >= a.nunits) return;
  const bool rs = a.coll == PC_COLL_REDUCE_SCATTER, ag = a.coll == PC_COLL_ALLGATHER;
  const bool bc = a.coll == PC_COLL_BCAST, root = bc && r == a.root;
  // writers into peers' buffers need every peer's ready-to-receive
  // (allgather pushes; broadcast receivers forward their part to the others)
  if (P > 1 && (ag || (bc && !root)) && !warp_wait_all(a.rtr, P - 1, e, a.err, a.timeout_ms, a.sys)) return;
  const uint32_t target = e * (uint32_t)(P - 1);
  for (int j0 = 0; gw + j0 * W < a.nunits; j0 += kMaxActive) {
    int step[kMaxActive];
    int remaining = 0;
#pragma unroll
    for (int j = 0; j < kMaxActive; ++j) {
      const bool mine = gw + (j0 + j) * W < a.nunits;
      step[j] = mine ? 0 : 3;
      remaining += mine;
    }
    Idle idle;
    while (remaining) {
      bool progressed = false;
#pragma unroll
      for (int jj = 0; jj < kMaxActive; ++jj) {
        if (step[jj] > 2) continue;
        const int x = gw + (j0 + jj) * W;
        const int u = x / a.ns, s = x % a.ns;
        const int i = step[jj];
        const int64_t lo = (int64_t)s * a.qs, hi = min(lo + a.qs, a.count), n = hi > lo ? hi - lo : 0;
        const uint32_t *cnt_u = a.cnt + (int64_t)u * 2 * a.ns + s;  // phase p at cnt_u[p * ns]
        bool finished = false;
        if (P == 1) {  // one rank: the result is the input
          if (!warp_poll(a.ready + u, e, false)) continue;
          if (n && !bc) {
            const int64_t so = rs ? (int64_t)u * a.count + lo : (int64_t)u * a.count + lo;
            warp_copy(a.recvbuf + so * es, a.sendbuf + so * es, n * es);
          }
          if (ag && (threadIdx.x & 31) == 0) st_release_gpu(a.srcflags + (int64_t)u * a.ns + s, e);
          finished = true;
        } else if (bc && !root && P == 2) {  // one receiver: copy the root's slice, tell the root
          if (!warp_poll(cnt_u, e, a.sys)) continue;
          const int64_t off = ((int64_t)u * a.count + lo) * es;
          if (n) warp_copy(a.recvbuf + off, a.p_recvbuf[0] + off, n * es);
          fence_release(a.sys);  // our reads of the root's slice are done before it may reuse it
          __syncwarp();
          if ((threadIdx.x & 31) == 0) red_add_scope(a.p_cnt[0] + ((int64_t)u * 2 + 1) * a.ns + s, 1, a.sys);
          finished = true;
        } else if (bc && !root && i == 0) {
          // split receive (scatter + allgather): once the root announced the
          // slice, receiver kk (of the P-1) reads part kk of it from the root
          // ONCE and stores it into every receiver's buffer; then it tells the
          // root (its part was read) and every receiver (the part arrived)
          if (!warp_poll(cnt_u, e, a.sys)) continue;
          const int jr = (a.root - r - 1 + P) % P;          // the root's peer index
          const int kk = (r - a.root - 1 + P) % P;          // my part, 0 .. P-2
          const int64_t epv = 16 / es > 0 ? 16 / es : 1;
          const int64_t pq = (((n + P - 2) / (P - 1)) + epv - 1) / epv * epv;
          const int64_t plo = min(lo + (int64_t)kk * pq, hi), phi = min(plo + pq, hi);
          const int64_t off = ((int64_t)u * a.count + plo) * es;
          if (phi > plo)
            warp_copy_multi<kMaxDirect - 1, 8>(a.recvbuf, a.p_recvbuf, P - 1, off, a.p_recvbuf[jr] + off,
                                               (phi - plo) * es, jr);
          fence_release(a.sys);  // my reads of the root and my stores to the receivers, then the signals
          __syncwarp();
          if ((threadIdx.x & 31) == 0)
            for (int j = 0; j < P - 1; ++j) red_add_scope(a.p_cnt[j] + ((int64_t)u * 2 + 1) * a.ns + s, 1, a.sys);
          if ((threadIdx.x & 31) == 0) red_add_scope(const_cast<uint32_t *>(cnt_u + a.ns), 1, a.sys);  // my own part
          step[jj] = 1;
        } else if (bc && !root) {  // every part of my slice arrived (P-1 receivers, me included)
          if (!warp_poll(cnt_u + a.ns, target, a.sys)) continue;
          finished = true;
        } else if (i == 0) {
          if (!warp_poll(a.ready + u, e, false)) continue;
          const int64_t off = ((int64_t)u * a.count + lo) * es;  // my block (AG, BCAST)
          if (ag) {
            const int64_t doff = (((int64_t)r * a.Np + u) * a.count + lo) * es;
            if (n) warp_copy_multi<kMaxDirect - 1>(a.recvbuf, a.p_recvbuf, P - 1, doff, a.sendbuf + off, n * es);
          }
          // (broadcast root: nothing to copy — the peers PULL the slice)
          fence_release(a.sys);
          __syncwarp();
          if ((threadIdx.x & 31) == 0) {
            for (int j = 0; j < P - 1; ++j) {
              if (ag) st_relaxed_sys(a.p_srcflags[j] + ((int64_t)r * a.Np + u) * a.ns + s, e);
              red_add_scope(a.p_cnt[j] + (int64_t)u * 2 * a.ns + s, 1, a.sys);
            }
            if (ag) st_release_gpu(a.srcflags + ((int64_t)r * a.Np + u) * a.ns + s, e);
          }
          step[jj] = 1;
        } else if (i == 1 && root) {  // every peer has pulled the slice
          if (!warp_poll(cnt_u + a.ns, target, a.sys)) continue;
          finished = true;
        } else if (i == 1) {
          if (!warp_poll(cnt_u, target, a.sys)) continue;
          if (rs) {
            if (n)
              warp_fold_pull<DT, OP, false, PC_DIRECT_FV * kMaxDirect / MAXP, false, MAXP>(
                  a, ((int64_t)u * P + r) * a.count + lo, (int64_t)u * a.count + lo, n);
            fence_release(a.sys);
            __syncwarp();
            if ((threadIdx.x & 31) == 0)
              for (int j = 0; j < P - 1; ++j) red_add_scope(a.p_cnt[j] + ((int64_t)u * 2 + 1) * a.ns + s, 1, a.sys);
            step[jj] = 2;
          } else {
            finished = true;
          }
        } else {  // RS step 2: every peer finished reading my partition u
          if (!warp_poll(cnt_u + a.ns, target, a.sys)) continue;
          finished = true;
        }
        progressed = true;
        if (finished) {
          __syncwarp();
          if ((threadIdx.x & 31) == 0) red_add_release_gpu(a.done + u, 1);
          step[jj] = 3;
          --remaining;
        }
      }
      if (progressed)
        idle.progressed();
      else if (!idle.wait(a.err, a.timeout_ms, gw))
        return;
    }
  }
}

// MAXP as for the DIRECT engines: the reduce-scatter fold keeps 8 / MAXP
// times more loads in flight for small comms.
template <int DT, int OP, int MAXP = kMaxDirect>
__global__ void __launch_bounds__(kEngineBlock, PC_DIRECT_MINB) coll_engine(CollArgs a) {
  coll_body<DT, OP, MAXP>(a, (blockIdx.x * blockDim.x + threadIdx.x) >> 5, (gridDim.x * blockDim.x) >> 5);
}
template <int DT, int OP, int MAXP = kMaxDirect>
__global__ void __launch_bounds__(kEngineBlock, PC_DIRECT_MINB) coll_engine_group(CollGroupArgs g) {
  int k = 0;
  while (k + 1 < g.n && (int)blockIdx.x >= g.block_start[k + 1]) ++k;
  const int b = blockIdx.x - g.block_start[k];
  const int nb = (k + 1 < g.n ? g.block_start[k + 1] : (int)gridDim.x) - g.block_start[k];
  coll_body<DT, OP, MAXP>(g.a[k], (b * blockDim.x + threadIdx.x) >> 5, (nb * blockDim.x) >> 5);
}

// MAXP: the comm size bound of the instantiation (P <= MAXP): 8, or 4 / 2
// for small comms, which keep 2x / 4x more vectors per operand in flight
// for the same registers (the launcher picks it from P).
template <int DT, int OP, int MAXP = kMaxDirect>
__global__ void __launch_bounds__(kEngineBlock, PC_DIRECT_MINB) direct_engine(DirectArgs a) {
  extern __shared__ __align__(128) uint8_t dsmem[];
  direct_body<DT, OP, PC_DIRECT_FV, false, false, PC_DIRECT_BULK, MAXP>(
      a, (blockIdx.x * blockDim.x + threadIdx.x) >> 5, (gridDim.x * blockDim.x) >> 5, dsmem);
}
template <int DT, int OP, int MAXP = kMaxDirect>
__global__ void __launch_bounds__(kEngineBlock, PC_DIRECT_MINB) direct_engine_group(DirectGroupArgs g) {
  int k = 0;
  while (k + 1 < g.n && (int)blockIdx.x >= g.block_start[k + 1]) ++k;
  const int b = blockIdx.x - g.block_start[k];
  const int nb = (k + 1 < g.n ? g.block_start[k + 1] : (int)gridDim.x) - g.block_start[k];
  extern __shared__ __align__(128) uint8_t dsmem[];
  direct_body<DT, OP, PC_DIRECT_FV, false, false, PC_DIRECT_BULK, MAXP>(
      g.a[k], (b * blockDim.x + threadIdx.x) >> 5, (nb * blockDim.x) >> 5, dsmem);
}

// "Thin" DIRECT engines for the overlap case (the engine runs beside the
// user's producer kernels): 2 CTAs per SM (<= 128 registers) and
// one 16-B vector per operand in flight, so an SM holding an engine CTA still
// has half its registers and 56 warp slots for producer blocks (a fat CTA
// leaves ~11 K registers: no 512-thread producer block fits beside it).
template <int DT, int OP>
__global__ void __launch_bounds__(kEngineBlock, 2) direct_engine_thin(DirectArgs a) {
  extern __shared__ __align__(128) uint8_t tsmem[];
  direct_body<DT, OP, PC_THIN_FV, !PC_THIN_BULK, false, PC_THIN_BULK>(
      a, (blockIdx.x * blockDim.x + threadIdx.x) >> 5, (gridDim.x * blockDim.x) >> 5, tsmem);
}
template <int DT, int OP>
__global__ void __launch_bounds__(kEngineBlock, 2) direct_engine_group_thin(DirectGroupArgs g) {
  int k = 0;
  while (k + 1 < g.n && (int)blockIdx.x >= g.block_start[k + 1]) ++k;
  const int b = blockIdx.x - g.block_start[k];
  const int nb = (k + 1 < g.n ? g.block_start[k + 1] : (int)gridDim.x) - g.block_start[k];
  extern __shared__ __align__(128) uint8_t tsmem[];
  direct_body<DT, OP, PC_THIN_FV, !PC_THIN_BULK, false, PC_THIN_BULK>(
      g.a[k], (b * blockDim.x + threadIdx.x) >> 5, (nb * blockDim.x) >> 5, tsmem);
}

// DIRECT, PUSH variant (PC_ALGO_DIRECT_PUSH): separate kernels, so the PULL
// kernels carry none of its registers.
template <int DT, int OP>
__global__ void __launch_bounds__(kEngineBlock, PC_DIRECT_MINB) direct_engine_push(DirectArgs a) {
  direct_body<DT, OP, PC_DIRECT_FV, false, true>(a, (blockIdx.x * blockDim.x + threadIdx.x) >> 5,
                                                 (gridDim.x * blockDim.x) >> 5, nullptr);
}
template <int DT, int OP>
__global__ void __launch_bounds__(kEngineBlock, PC_DIRECT_MINB) direct_engine_group_push(DirectGroupArgs g) {
  int k = 0;
  while (k + 1 < g.n && (int)blockIdx.x >= g.block_start[k + 1]) ++k;
  const int b = blockIdx.x - g.block_start[k];
  const int nb = (k + 1 < g.n ? g.block_start[k + 1] : (int)gridDim.x) - g.block_start[k];
  direct_body<DT, OP, PC_DIRECT_FV, false, true>(g.a[k], (b * blockDim.x + threadIdx.x) >> 5,
                                                 (nb * blockDim.x) >> 5, nullptr);
}

// Single-rank launches (one rank per GPU / process).
template <int DT, int OP>
__global__ void __launch_bounds__(kEngineBlock) ring_engine(RingArgs a) {
  ring_body<DT, OP>(a, (blockIdx.x * blockDim.x + threadIdx.x) >> 5, (gridDim.x * blockDim.x) >> 5);
}
template <int DT, int OP>
__global__ void __launch_bounds__(kEngineBlock) rd_engine(RdArgs a) {
  rd_body<DT, OP>(a, (blockIdx.x * blockDim.x + threadIdx.x) >> 5, (gridDim.x * blockDim.x) >> 5);
}

// Grouped launches: the engines of every rank that shares this GPU inside one
// process (virtual ranks) run as ONE kernel, so they are co-resident by
// construction and no engine can sit behind another in a hardware queue
// (DESIGN.md §"Virtual ranks").  Block b belongs to the rank whose block range
// contains it; warps are numbered within that rank exactly as in the
// single-rank launch.
template <int DT, int OP>
__global__ void __launch_bounds__(kEngineBlock) ring_engine_group(RingGroupArgs g) {
  int k = 0;
  while (k + 1 < g.n && (int)blockIdx.x >= g.block_start[k + 1]) ++k;
  const int b = blockIdx.x - g.block_start[k];
  const int nb = (k + 1 < g.n ? g.block_start[k + 1] : (int)gridDim.x) - g.block_start[k];
  ring_body<DT, OP>(g.a[k], (b * blockDim.x + threadIdx.x) >> 5, (nb * blockDim.x) >> 5);
}
template <int DT, int OP>
__global__ void __launch_bounds__(kEngineBlock) rd_engine_group(RdGroupArgs g) {
  int k = 0;
  while (k + 1 < g.n && (int)blockIdx.x >= g.block_start[k + 1]) ++k;
  const int b = blockIdx.x - g.block_start[k];
  const int nb = (k + 1 < g.n ? g.block_start[k + 1] : (int)gridDim.x) - g.block_start[k];
  rd_body<DT, OP>(g.a[k], (b * blockDim.x + threadIdx.x) >> 5, (nb * blockDim.x) >> 5);
}

}  // namespace

extern std::atomic<uint64_t> g_launches;

inline int grid_for(int warps, int nunits) {
  int w = warps < nunits ? warps : nunits;
  if (w < 1) w = 1;
  return (w * 32 + kEngineBlock - 1) / kEngineBlock;
}

// Launchers of the six engine kernels for one (dtype, op).  Declared here,
// defined and explicitly instantiated only in engine_inst.cu (one TU per
// (dtype, op)), so kernels.cu never compiles an engine body.
template <int DT, int OP>
struct EngineLaunch {
  static int ring(const RingArgs &a, int warps, cudaStream_t s);
  static int rd(const RdArgs &a, int warps, cudaStream_t s);
  static int direct(const DirectArgs &a, int warps, cudaStream_t s, bool thin);
  static int ring_group(const RingGroupArgs &h, int blocks, cudaStream_t s);
  static int rd_group(const RdGroupArgs &h, int blocks, cudaStream_t s);
  static int direct_group(const DirectGroupArgs &h, int blocks, cudaStream_t s, bool thin);
  static int direct_batch(const DirectBatchArgs &b, int blocks, cudaStream_t s, bool thin);
  static int coll(const CollArgs &a, int warps, cudaStream_t s);
  static int coll_group(const CollGroupArgs &h, int blocks, cudaStream_t s);
  static int occupancy(int *ctas);
  static int occupancy_direct(int *ctas);
  static int preload();  // load every engine kernel now (lazy module loading, see kernels.cu)
};

// The small-comm (MAXP = 4, 2) DIRECT / collective kernels of one (dtype, op):
// defined in engine_small.cu, a translation unit of their own (built for the
// gradient types' SUM only), so the long compiles run in parallel.
template <int DT, int OP>
struct SmallCommLaunch {
  static int direct(const DirectArgs &a, int grid, cudaStream_t s, int maxp);
  static int direct_group(const DirectGroupArgs &h, int blocks, cudaStream_t s, int maxp);
  static int coll(const CollArgs &a, int grid, cudaStream_t s, int maxp);
  static int coll_group(const CollGroupArgs &h, int blocks, cudaStream_t s, int maxp);
  static int preload();
};
template <int DT, int OP>
constexpr bool kSmallCommKernels = (DT == 1 || DT == 4) && OP == 0;

}  // namespace pc
