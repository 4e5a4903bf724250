/*
 * include/pc_device.cuh — device bindings of libpc (sm_100a).
 *
 *   PC_DEVICE int  pc_pready      (int partition, pc_prequest_t preq);  any thread
 *   PC_DEVICE int  pc_pready_warp (int partition, pc_prequest_t preq);  warp-collective
 *   PC_DEVICE int  pc_warp_begin(pc_prequest_t preq, pc_warp_state *st);     warp-collective
 *   PC_DEVICE int  pc_pready_warp (int partition, pc_prequest_t preq, st);  warp-collective (checked once)
 *   PC_DEVICE int  pc_pready_block(int partition, pc_prequest_t preq);  block-collective
 *   PC_DEVICE int  pc_pready_block_put<T>(int partition, pc_prequest_t preq,
 *                                         uint64_t idx, const T &v);     block-collective
 *   PC_DEVICE int  pc_put_begin<T>(pc_prequest_t preq, pc_put_state *st, int batch = 1);  block-collective
 *   PC_DEVICE int  pc_pready_block_put<T>(partition, preq, idx, v, st);     block-collective
 *   PC_DEVICE void pc_put_end(pc_prequest_t preq, pc_put_state &st);       block-collective
 *   PC_DEVICE int  pc_pready_block(int partition, pc_prequest_t preq, pc_put_state &st);  (checked once)
 *   PC_DEVICE int  pc_pready_block_coop(int partition, pc_prequest_t preq);  block-collective (R36,
 *                  INLINE allreduce, -DPC_INLINE_ALLREDUCE)
 *   PC_DEVICE int  pc_parrived    (pc_prequest_t preq, int partition);
 *   PC_DEVICE int  pc_wait_arrived(pc_prequest_t preq, int partition);
 *   PC_DEVICE int  pc_parrived_warp / pc_wait_arrived_warp(preq, partition);  warp-collective
 *
 * Paper: MPIX_Pready / MPIX_Pready_{thread,warp,block} / MPIX_Parrived
 * (Listing 2; §IV-A4).  PC_DEVICE plays the role of
 * MPIX_Device.
 *
 * pc_pready* semantics: "user partition `partition` of the send buffer is
 * final for the current epoch".  Call at most once per partition per epoch.
 *   - Aggregation: user partition p belongs to transport
 *     partition t = p / g.  Contributors increment a never-reset GPU-global
 *     counter cnt[t] (target e*g_t, wrap-aware); thread-granularity callers are
 *     first combined per warp with __match_any_sync so one atomic covers every
 *     lane of the warp that targets the same t (the library-side aggregation
 *     the paper recommends).
 *   - INLINE copy ("Kernel Copy"): every caller pushes ITS OWN
 *     partition's bytes to the receiver's buffer (16-byte vector stores over
 *     NVLink, after checking the ready-to-receive word, Pbuf_prepare P:L62),
 *     fences at the request's scope, then counts; the contribution that
 *     completes t releases the receiver's flag[t] = e (the completion the
 *     paper sent through the host, done here on the device).
 *   - ENGINE copy: the completing contributor only release-stores ready[t] = e;
 *     library engine warps move the data.
 *   - HOST copy (the paper's Progression Engine): the completing
 *     contributor release-stores hready[t] = e into pinned host memory; the
 *     library's host progression thread copies and signals.
 *   - Allreduce requests: marks user partition u ready (step S_0 is the
 *     user's Pready); the library engine runs the schedule.
 * Returns 0, or a PC_ERR_* code that is also recorded in the sticky error word
 * (bad partition, duplicate Pready detected by counter overshoot).
 *
 * pc_pready_block_put (MPIX extension, reading R35): pc_pready_block for a
 * block whose thread k has written element idx_k (of type T, 4/8/16 B) of the
 * partition and still holds it in registers: the INLINE Kernel Copy assigns
 * v straight to the receiver ("an assignment statement") instead of
 * re-reading the partition from L2 after the barrier.  The caller writes its
 * send buffer as usual and its threads together cover every element of the
 * partition (idx = UINT64_MAX: this thread holds none).  Every other copy
 * mode, request kind or alignment falls back to pc_pready_block (the send
 * buffer already holds the data).  Persistent producers call
 * pc_put_begin<T>(preq, &st) once per CTA before their loop and then
 * pc_pready_block_put(partition, preq, idx, v, st): {epoch, ready-to-receive}
 * is checked once, and each Pready is the raw chain — assign from registers,
 * barrier, release, flag.
 *
 * INLINE allreduce (pc_prequest_create(..., PC_COPY_INLINE) on a DIRECT
 * allreduce, reading R33): the Pready that completes a partition on the last
 * rank folds it for every rank.  The fold is compiled into these bindings only
 * in translation units built with -DPC_INLINE_ALLREDUCE (kernels that Pready
 * into such a request), so producers of other requests keep their register
 * allocation; elsewhere a Pready on an INLINE allreduce reports PC_DEV_ERR_ARG.
 *
 * pc_parrived: 1 iff the partition is complete in this epoch (receive: its
 * bytes are in recvbuf; allreduce: its final result is in recvbuf).
 * It is an ld.acquire.sys of a flag in the caller's OWN memory (written
 * remotely by the producer), not a host round trip.  Other threads
 * of the block must synchronise with the polling thread before they read the
 * partition.
 */
#ifndef PC_DEVICE_CUH_
#define PC_DEVICE_CUH_

#include <stdint.h>

#include "pc_ops.cuh"
#include "pc_prequest.h"

typedef struct pc_prequest_s pc_prequest_t;

#define PC_DEVICE __device__ __forceinline__
/* Paths a Pready rarely takes (a spin on a ready-to-receive word that is not
 * there yet, an error, a partition of more than 16 B per thread): out of line,
 * so the common path of a producer capped at 32 registers (two 1024-thread
 * CTAs per SM) does not spill for them. */
#define PC_COLD static __device__ __noinline__

#ifndef PC_DEV_ERR_ARG
#define PC_DEV_ERR_ARG (-1)
#define PC_DEV_ERR_TIMEOUT (-5)
#define PC_DEV_ERR_DEVICE (-6)
#endif

namespace pc_detail {

PC_DEVICE uint32_t ld_acquire_sys(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
PC_DEVICE uint32_t ld_acquire_gpu(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
/* {p[0], p[1]} in one system-scope acquire (the epoch word and the RTR word
 * are adjacent in the control block: one L2 round trip for both). */
PC_DEVICE uint2 ld_acquire_sys_v2(const uint32_t *p) {
  uint2 v;
  asm volatile("ld.acquire.sys.global.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(p) : "memory");
  return v;
}
PC_DEVICE uint2 ld_acquire_gpu_v2(const uint32_t *p) {
  uint2 v;
  asm volatile("ld.acquire.gpu.global.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(p) : "memory");
  return v;
}
PC_DEVICE void st_relaxed_gpu(uint32_t *p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
PC_DEVICE uint32_t ld_relaxed_sys(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
PC_DEVICE uint4 ld_relaxed_gpu_v4(const uint4 *p) {
  uint4 v;
  asm volatile("ld.relaxed.gpu.global.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p)
               : "memory");
  return v;
}
PC_DEVICE uint4 ld_relaxed_sys_v4(const uint4 *p) {
  uint4 v;
  asm volatile("ld.relaxed.sys.global.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p)
               : "memory");
  return v;
}
PC_DEVICE void st_release_sys(uint32_t *p, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
PC_DEVICE void st_relaxed_sys(uint32_t *p, uint32_t v) {
  asm volatile("st.relaxed.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
PC_DEVICE void st_release_gpu(uint32_t *p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
PC_DEVICE uint32_t atom_add_acq_rel_gpu(uint32_t *p, uint32_t v) {
  uint32_t old;
  asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
  return old;
}
PC_DEVICE uint32_t atom_add_acq_rel_sys(uint32_t *p, uint32_t v) {
  uint32_t old;
  asm volatile("atom.acq_rel.sys.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
  return old;
}
PC_DEVICE void red_add_release_gpu(uint32_t *p, uint32_t v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
PC_DEVICE void fence_sys() { asm volatile("fence.acq_rel.sys;" ::: "memory"); }
PC_DEVICE void fence_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
/* Acquire-release fence at the scope the request needs: system scope when a
 * peer is another GPU (NVLink), GPU scope when every peer shares this GPU.
 * (Kept for completeness; the library's acquires after relaxed loads use
 * fence_acquire, its releases fence_release.) */
PC_DEVICE void fence_scope(uint32_t sys) {
  if (sys)
    fence_sys();
  else
    fence_gpu();
}
/* Release fence (PTX fence.release): with the strong (relaxed) flag store
 * that follows it, a release pattern — every memory operation before it (and,
 * cumulatively, those ordered before it by a barrier) is visible at `scope`
 * before the flag.  Same MEMBAR as fence.acq_rel without the L1 invalidation
 * (profiles/r02_c2_floor.jsonl: st.release-style signalling 185 -> 170 us at
 * 256 MiB).  Every Pready / engine signal releases; none acquires. */
PC_DEVICE void fence_release(uint32_t sys) {
  if (sys)
    asm volatile("fence.release.sys;" ::: "memory");
  else
    asm volatile("fence.release.gpu;" ::: "memory");
}
/* Acquire fence (PTX fence.acquire): after relaxed loads of flag words, the
 * acquire pattern for every one of them — only the L1 invalidation in the
 * SASS (CCTL.IVALL), no MEMBAR: a wait that reads many flags relaxed and
 * then acquires once pays no store drain. */
PC_DEVICE void fence_acquire(uint32_t sys) {
  if (sys)
    asm volatile("fence.acquire.sys;" ::: "memory");
  else
    asm volatile("fence.acquire.gpu;" ::: "memory");
}
PC_DEVICE uint32_t ld_acquire_scope(const uint32_t *p, uint32_t sys) {
  return sys ? ld_acquire_sys(p) : ld_acquire_gpu(p);
}
PC_DEVICE uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
PC_DEVICE uint32_t lane_id() {
  uint32_t l;
  asm("mov.u32 %0, %%laneid;" : "=r"(l));
  return l;
}
/* wrap-aware "v has reached target" for monotonically increasing u32 words */
PC_DEVICE bool reached(uint32_t v, uint32_t target) { return (int32_t)(v - target) >= 0; }

PC_COLD void set_error(int32_t *err, int32_t code, int32_t part) {
  if (atomicCAS(err, 0, code) == 0) {
    err[1] = part;
    __threadfence_system();
  }
}
PC_DEVICE bool aborted(const int32_t *err) { return *(const volatile int32_t *)err != 0; }

/* Spin until *p has reached `target`.  SYS: acquire at system scope (word
 * written by another GPU); else GPU scope.  Bounded: after timeout_ms sets the
 * sticky error word and returns false; also returns false as soon as another
 * thread has set an error (so one failure drains every waiter instead of
 * hanging the device). */
template <bool SYS>
PC_COLD bool spin_geq(const uint32_t *p, uint32_t target, int32_t *err, uint32_t timeout_ms, int32_t part) {
  uint32_t v = SYS ? ld_acquire_sys(p) : ld_acquire_gpu(p);
  if (reached(v, target)) return true;
  const uint64_t t0 = globaltimer();
  uint32_t n = 0, ns = 0;
  for (;;) {
    if (ns) __nanosleep(ns);
    v = SYS ? ld_acquire_sys(p) : ld_acquire_gpu(p);
    if (reached(v, target)) return true;
    ++n;
    if (n > 512) ns = ns ? (ns < 512 ? ns * 2 : 512) : 32;
    if ((n & 127) == 0) {
      if (aborted(err)) return false;
      if (timeout_ms && globaltimer() - t0 > (uint64_t)timeout_ms * 1000000ull) {
        set_error(err, PC_DEV_ERR_TIMEOUT, part);
        return false;
      }
    }
  }
}

/* Cooperative byte copy by `n` participants (participant index `idx`):
 * 16-byte vector loads (L2, .cg) and stores when both pointers are 16-B
 * aligned, 4 independent vectors in flight per participant; 4-byte and
 * 1-byte fallbacks otherwise.  dst may be a peer-mapped (NVLink) address. */
PC_DEVICE void copy_bytes(uint8_t *dst, const uint8_t *src, uint64_t nbytes, uint32_t idx, uint32_t n) {
  const uintptr_t mis = reinterpret_cast<uintptr_t>(dst) & 15;
  if (mis && (reinterpret_cast<uintptr_t>(src) & 15) == mis && nbytes > 16 - mis) {
    // shared misalignment: bytes up to the 16-B boundary, then vectors
    const uint64_t h = 16 - mis;
    for (uint64_t b = idx; b < h; b += n) dst[b] = src[b];
    dst += h;
    src += h;
    nbytes -= h;
  }
  if (((reinterpret_cast<uintptr_t>(dst) | reinterpret_cast<uintptr_t>(src)) & 15) == 0) {
    const uint64_t nv = nbytes >> 4;
    const uint4 *s = reinterpret_cast<const uint4 *>(src);
    uint4 *d = reinterpret_cast<uint4 *>(dst);
    uint64_t k = idx;
    for (; k + 3ull * n < nv; k += 4ull * n) {
      uint4 a = __ldcg(s + k), b = __ldcg(s + k + n), c = __ldcg(s + k + 2 * n), e = __ldcg(s + k + 3 * n);
      d[k] = a;
      d[k + n] = b;
      d[k + 2 * n] = c;
      d[k + 3 * n] = e;
    }
    for (; k < nv; k += n) d[k] = __ldcg(s + k);
    for (uint64_t b = (nv << 4) + idx; b < nbytes; b += n) dst[b] = src[b];
  } else if (((reinterpret_cast<uintptr_t>(dst) | reinterpret_cast<uintptr_t>(src) | nbytes) & 3) == 0) {
    const uint32_t *s = reinterpret_cast<const uint32_t *>(src);
    uint32_t *d = reinterpret_cast<uint32_t *>(dst);
    for (uint64_t k = idx; k < (nbytes >> 2); k += n) d[k] = __ldcg(s + k);
  } else {
    for (uint64_t b = idx; b < nbytes; b += n) dst[b] = src[b];
  }
}

PC_COLD void copy_bytes_cold(uint8_t *dst, const uint8_t *src, uint64_t nbytes, uint32_t idx, uint32_t n) {
  copy_bytes(dst, src, nbytes, idx, n);
}

PC_DEVICE uint32_t epoch_of(const pc_prequest_t &q) { return *(const volatile uint32_t *)q.epoch; }

PC_DEVICE uint32_t transport_size(const pc_prequest_t &q, int t) {
  const int rem = q.partitions - t * q.agg;
  return (uint32_t)(rem < q.agg ? rem : q.agg);
}

/* Count `add` contributions to transport partition t; returns true for the
 * single contribution that completes t in epoch e.  Flags a duplicate Pready
 * (counter already at/over the target) in the sticky error word.  With g = 1
 * every Pready completes its own transport partition: no counter (the
 * latency-critical path; duplicate detection needs g > 1). */
/* Two-level counting for large g (reading R32): with g >= 4 * kSubAgg the
 * user partitions of a transport partition count first into sub-counters of
 * kSubAgg consecutive partitions (words cnt[ntransport ...], unused by the
 * one-level layout: ntransport * (1 + ceil(g / kSubAgg)) <= N_p), and only
 * the contribution completing a sub-group adds its size to cnt[t] — a
 * whole-buffer transport partition of 1 M warp Preadies no longer funnels
 * 1 M atomics into one word.  The acq_rel atomics chain the releases. */
constexpr int kSubAgg = 256;
PC_DEVICE bool sub_agg(const pc_prequest_t &q) { return q.agg >= 4 * kSubAgg; }
/* The counter a contribution of partition p goes to first: lanes that share
 * it are combined into one update (thread granularity). */
PC_DEVICE int counter_key(const pc_prequest_t &q, int p) {
  const int t = p / q.agg;
  if (!sub_agg(q)) return t;
  return t * ((q.agg + kSubAgg - 1) / kSubAgg) + (p - t * q.agg) / kSubAgg;
}

PC_DEVICE bool contribute(const pc_prequest_t &q, int t, uint32_t add, uint32_t e, int part) {
  if (q.agg == 1) return true;
  if (sub_agg(q)) {
    const int sl = (part - t * q.agg) / kSubAgg;
    const int rest = (int)transport_size(q, t) - sl * kSubAgg;
    const uint32_t ssz = (uint32_t)(rest < kSubAgg ? rest : kSubAgg);
    const uint32_t old = atom_add_acq_rel_gpu(q.cnt + q.ntransport + counter_key(q, part), add);
    const int32_t d = (int32_t)(e * ssz - old);
    if (d <= 0) {
      set_error(q.err, PC_DEV_ERR_DEVICE, part);
      return false;
    }
    if (d > (int32_t)add) return false;  // sub-group not complete yet
    add = ssz;                           // carry the whole sub-group to cnt[t]
  }
  const uint32_t target = e * transport_size(q, t);
  const uint32_t old = atom_add_acq_rel_gpu(q.cnt + t, add);
  const int32_t d = (int32_t)(target - old);
  if (d <= 0) {
    set_error(q.err, PC_DEV_ERR_DEVICE, part);
    return false;
  }
  return d <= (int32_t)add;
}

/* ENGINE / HOST copy: the completing contributor marks transport partition t
 * ready for the mover — the library's engine warps (GPU-scope flag) or the
 * host progression thread (system-scope store into pinned host memory, after
 * which the host may read the partition's bytes). */
PC_DEVICE void mark_ready(const pc_prequest_t &q, int t, uint32_t e) {
  if (q.copy == 3)
    st_release_sys(q.hready + t, e);
  else
    st_release_gpu(q.ready + t, e);
}

/* MPI-4 partitionings that differ between the two sides (reading R30).
 * Send side: the receive partitions [*p0, *p1] that transport partition t's
 * bytes overlap.  Receive side: how many send transport partitions (of g user
 * partitions of peer_part_bytes each) overlap receive partition p. */
PC_DEVICE void xp_recv_span(int t, int partitions, int agg, uint64_t part_bytes, uint64_t peer_part_bytes,
                            uint64_t *p0, uint64_t *p1) {
  const uint64_t tb = (uint64_t)agg * part_bytes, total = (uint64_t)partitions * part_bytes;
  const uint64_t lo = (uint64_t)t * tb, hi = lo + tb < total ? lo + tb : total;
  *p0 = lo / peer_part_bytes;
  *p1 = (hi - 1) / peer_part_bytes;
}
PC_DEVICE uint32_t xp_need(uint64_t p, uint64_t part_bytes, uint32_t g, uint64_t peer_part_bytes) {
  const uint64_t tb = (uint64_t)g * peer_part_bytes;
  const uint64_t lo = p * part_bytes, hi = lo + part_bytes;
  return (uint32_t)((hi - 1) / tb - lo / tb + 1);
}
PC_DEVICE void red_add_relaxed_sys(uint32_t *p, uint32_t v) {
  asm volatile("red.relaxed.sys.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
/* The receiver-side arrival signal of transport partition t (after the
 * pushes are fenced): equal partitionings store flag[t] = e; different ones
 * add 1 to the counter of every receive partition t overlaps (the receiver
 * waits for e * xp_need). */
PC_DEVICE void signal_transport(uint32_t *peer_flags, int t, uint32_t e, uint32_t xpart, int partitions, int agg,
                                uint64_t part_bytes, uint64_t peer_part_bytes) {
  if (!xpart) {
    st_relaxed_sys(peer_flags + t, e);
    return;
  }
  uint64_t p0, p1;
  xp_recv_span(t, partitions, agg, part_bytes, peer_part_bytes, &p0, &p1);
  for (uint64_t p = p0; p <= p1; ++p) red_add_relaxed_sys(peer_flags + p, 1);
}
PC_DEVICE void signal_transport(const pc_prequest_t &q, int t, uint32_t e) {
  signal_transport(q.peer_flags, t, e, q.xpart, q.partitions, q.agg, q.part_bytes, q.peer_part_bytes);
}

/* Publish transport partition t once this contributor's own bytes are in
 * place ("Kernel Copy": every contributor assigns its data to the
 * peer address, counters aggregate, then the partition is marked).  The
 * caller has already fenced its pushes at the request's scope.  g = 1: the
 * contribution is the whole transport partition, flag it directly; g > 1: the
 * acq_rel counter add orders every other contributor's (fenced) pushes before
 * the completing contributor, which fences again and flags. */
PC_DEVICE void publish(const pc_prequest_t &q, int t, uint32_t add, uint32_t e, int part) {
  if (q.agg == 1) {
    signal_transport(q, t, e);
    st_relaxed_gpu(q.sent + t, e);
    return;
  }
  if (contribute(q, t, add, e, part)) {
    fence_release(q.sys_scope);
    signal_transport(q, t, e);
    st_relaxed_gpu(q.sent + t, e);
  }
}

/* The fence a contributor issues after its pushes, before publish().  With
 * g > 1 at GPU scope the contribution's atom.acq_rel.gpu is itself the
 * (cumulative) release of those pushes, so the fence is dropped; g = 1
 * (publish stores the flag directly) and system scope keep it. */
PC_DEVICE void fence_before_publish(const pc_prequest_t &q) {
  if (q.agg == 1 || q.sys_scope) fence_release(q.sys_scope);
}

/* {epoch, rtr[0]} in one acquire at the request's scope (adjacent words). */
PC_DEVICE uint2 epoch_rtr(const pc_prequest_t &q) {
  return q.sys_scope ? ld_acquire_sys_v2(q.epoch) : ld_acquire_gpu_v2(q.epoch);
}

/* The epoch alone, relaxed: for a Pready that moves no bytes (flag-only
 * partitions, ENGINE mode) there is no receiver buffer to protect, so no
 * ready-to-receive check and no acquire (an acquire also invalidates L1). */
PC_DEVICE uint32_t epoch_relaxed(const pc_prequest_t &q) { return ld_relaxed_sys(q.epoch); }

/* ------------------------------------------------------------ LL lines
 * PC_COPY_LL: payload byte 8j..8j+7 of user partition p travels in line j =
 * {d0, e, d1, e} (d0/d1 = payload bytes 0-3 / 4-7, little endian), stored as
 * ONE st.relaxed.v2.u64 whose two 8-byte elements are each single-copy atomic:
 * a reader that sees e in both halves has this epoch's 8 bytes.  Lines live in
 * the receiver's control block, [epoch parity][partition][line]. */
PC_DEVICE void st_ll(uint8_t *dst, uint64_t lo, uint64_t hi, uint32_t sys) {
  if (sys)
    asm volatile("st.relaxed.sys.global.v2.u64 [%0], {%1, %2};" ::"l"(dst), "l"(lo), "l"(hi) : "memory");
  else
    asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(dst), "l"(lo), "l"(hi) : "memory");
}
PC_DEVICE ulonglong2 ld_ll(const uint8_t *src, uint32_t sys) {
  ulonglong2 v;
  if (sys)
    asm volatile("ld.relaxed.sys.global.v2.u64 {%0, %1}, [%2];" : "=l"(v.x), "=l"(v.y) : "l"(src) : "memory");
  else
    asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(v.x), "=l"(v.y) : "l"(src) : "memory");
  return v;
}
/* n (1..8) payload bytes at s, little endian, zero-padded */
PC_DEVICE uint64_t ld_payload8(const uint8_t *s, uint32_t n) {
  const uintptr_t a = reinterpret_cast<uintptr_t>(s);
  if (n == 8 && (a & 7) == 0) return *reinterpret_cast<const uint64_t *>(s);
  if ((a & 3) == 0 && (n & 3) == 0) {
    const uint64_t lo = *reinterpret_cast<const uint32_t *>(s);
    return n == 8 ? lo | ((uint64_t)(*reinterpret_cast<const uint32_t *>(s + 4)) << 32) : lo;
  }
  uint64_t v = 0;
  for (uint32_t b = 0; b < n; ++b) v |= (uint64_t)s[b] << (8 * b);
  return v;
}
PC_DEVICE void st_payload8(uint8_t *d, uint64_t v, uint32_t n) {
  const uintptr_t a = reinterpret_cast<uintptr_t>(d);
  if (n == 8 && (a & 7) == 0) {
    *reinterpret_cast<uint64_t *>(d) = v;
  } else if ((a & 3) == 0 && (n & 3) == 0) {
    *reinterpret_cast<uint32_t *>(d) = (uint32_t)v;
    if (n == 8) *reinterpret_cast<uint32_t *>(d + 4) = (uint32_t)(v >> 32);
  } else {
    for (uint32_t b = 0; b < n; ++b) d[b] = (uint8_t)(v >> (8 * b));
  }
}
PC_DEVICE uint32_t ll_nbytes(uint64_t part_bytes, uint32_t j) {
  const uint64_t o = 8ull * j;
  return o < part_bytes ? (uint32_t)(part_bytes - o < 8 ? part_bytes - o : 8) : 0u;
}

/* Sender: participant idx of n pushes lines idx, idx+n, ... of partition p and
 * returns the epoch.  The first payload load is issued BEFORE the epoch read so
 * the two round trips overlap, and neither is an acquire.  Ready-to-receive is
 * not checked here: the line area of parity e&1 was last read by the receiver
 * in epoch e-2, and the sender's completion of epoch e-1 (pc_wait / pc_test /
 * pc_wait_on_stream) already acquired rtr >= e-1, i.e. the receiver had
 * finished epoch e-2 — the stream order from that wait to this epoch's kernels
 * carries the ordering (R29). */
PC_DEVICE uint32_t ll_push(const pc_prequest_t &q, int p, uint32_t idx, uint32_t n) {
  const uint32_t nl = q.ll_lines;
  const uint64_t pb = q.part_bytes;
  const uint8_t *src = q.sbuf + (uint64_t)p * pb;
  uint64_t d = 0;
  if (idx < nl) {
    const uint32_t nb = ll_nbytes(pb, idx);
    if (nb) d = ld_payload8(src + 8ull * idx, nb);
  }
  const uint32_t e = epoch_relaxed(q);
  uint8_t *dst = q.peer_ll + ((uint64_t)(e & 1) * (uint64_t)q.partitions + (uint64_t)p) * nl * 16ull;
  const uint64_t eh = (uint64_t)e << 32;
  for (uint32_t j = idx; j < nl; j += n) {
    if (j != idx) {
      const uint32_t nb = ll_nbytes(pb, j);
      d = nb ? ld_payload8(src + 8ull * j, nb) : 0;
    }
    st_ll(dst + 16ull * j, (d & 0xffffffffull) | eh, (d >> 32) | eh, q.sys_scope);
  }
  return e;
}

/* Receiver: 1 iff every line of partition p carries epoch e; then the payload
 * is unpacked into recvbuf (by the calling thread). */
PC_DEVICE bool ll_consume(const pc_prequest_t &q, int p, uint32_t e) {
  const uint32_t nl = q.ll_lines;
  const uint64_t pb = q.part_bytes;
  const uint8_t *lines = q.ll + ((uint64_t)(e & 1) * (uint64_t)q.partitions + (uint64_t)p) * nl * 16ull;
  uint8_t *dst = q.rbuf + (uint64_t)p * pb;
  for (uint32_t j0 = 0; j0 < nl; j0 += 8) {
    const uint32_t m = nl - j0 < 8 ? nl - j0 : 8;
    ulonglong2 v[8];
#pragma unroll
    for (uint32_t k = 0; k < 8; ++k)
      if (k < m) v[k] = ld_ll(lines + 16ull * (j0 + k), q.sys_scope);
#pragma unroll
    for (uint32_t k = 0; k < 8; ++k)
      if (k < m && ((uint32_t)(v[k].x >> 32) != e || (uint32_t)(v[k].y >> 32) != e)) return false;
#pragma unroll
    for (uint32_t k = 0; k < 8; ++k)
      if (k < m) {
        const uint32_t nb = ll_nbytes(pb, j0 + k);
        if (nb) st_payload8(dst + 8ull * (j0 + k), (v[k].x & 0xffffffffull) | (v[k].y << 32), nb);
      }
  }
  return true;
}

/* Warp-collective receiver (all 32 lanes): lane l loads lines l, l+32, l+64,
 * l+96 of the partition in one round trip, the warp votes, every lane unpacks
 * its lines.  Returns the same value on every lane. */
PC_DEVICE bool ll_consume_warp(const pc_prequest_t &q, int p, uint32_t e, uint32_t lane) {
  const uint32_t nl = q.ll_lines;
  const uint64_t pb = q.part_bytes;
  const uint8_t *lines = q.ll + ((uint64_t)(e & 1) * (uint64_t)q.partitions + (uint64_t)p) * nl * 16ull;
  uint8_t *dst = q.rbuf + (uint64_t)p * pb;
  for (uint32_t j0 = 0; j0 < nl; j0 += 128) {
    ulonglong2 v[4];
    bool ok = true;
#pragma unroll
    for (uint32_t k = 0; k < 4; ++k) {
      const uint32_t j = j0 + 32 * k + lane;
      if (j < nl) v[k] = ld_ll(lines + 16ull * j, q.sys_scope);
    }
#pragma unroll
    for (uint32_t k = 0; k < 4; ++k) {
      const uint32_t j = j0 + 32 * k + lane;
      if (j < nl) ok = ok && (uint32_t)(v[k].x >> 32) == e && (uint32_t)(v[k].y >> 32) == e;
    }
    if (!__all_sync(0xffffffffu, ok)) return false;
#pragma unroll
    for (uint32_t k = 0; k < 4; ++k) {
      const uint32_t j = j0 + 32 * k + lane;
      const uint32_t nb = j < nl ? ll_nbytes(pb, j) : 0u;
      if (nb) st_payload8(dst + 8ull * j, (v[k].x & 0xffffffffull) | (v[k].y << 32), nb);
    }
  }
  return true;
}

/* Sender completion accounting of an LL Pready (the receiver needs no flag). */
PC_DEVICE void ll_account(const pc_prequest_t &q, int t, uint32_t add, uint32_t e, int part) {
  if (contribute(q, t, add, e, part)) st_relaxed_gpu(q.sent + t, e);
}

}  // namespace pc_detail

/* ------------------------------------------------------------------ Pready */

/* ------------------------------------------------------------ INLINE allreduce
 * (reading R33: "the Pready could also trigger the computation", the
 * paper's Kernel Copy applied to the collective).  Every rank's Pready of user
 * partition u adds 1 to u's arrival counter in rank 0's control block
 * (acq_rel: the caller's data writes are released; the last arrival acquires
 * every rank's).  The contribution that completes u (target e*P) — the last
 * rank to produce u — checks that every peer posted ready-to-receive for
 * epoch e (implied by causality: each peer's Pready of u follows its
 * Pbuf_prepare), folds u over the P send buffers in rank order (R25: the
 * DIRECT schedule's bits, oracle O6), stores the result into all P recvbufs,
 * fences once and writes done[u] = e on every rank.  No engine, no spinning
 * kernel: the reduction runs in the producer block that completed the data,
 * while the data is still in L2. */
namespace pc_detail {

PC_DEVICE bool ar_arrive(const pc_prequest_t &q, int u, uint32_t e) {
  uint32_t *c = q.ar_tab->cnt + u;
  const uint32_t old = q.sys_scope ? atom_add_acq_rel_sys(c, 1u) : atom_add_acq_rel_gpu(c, 1u);
  const int32_t d = (int32_t)(e * (uint32_t)q.nranks - old);
  if (d <= 0) {  // more than P arrivals in this epoch: a duplicate Pready
    set_error(q.err, PC_DEV_ERR_DEVICE, u);
    return false;
  }
  return d == 1;
}

/* Every peer posted ready-to-receive for epoch e: the P-1 words are read
 * relaxed, all in flight at once (acquire loads would serialise), then one
 * fence gives the acquire; only a word still behind is spun on. */
PC_DEVICE bool ar_rtr_ok(const pc_prequest_t &q, int u, uint32_t e) {
  const uint32_t *w = q.ar_tab->rtr;
  uint32_t v[PC_AR_MAX - 1];
#pragma unroll
  for (int j = 0; j < PC_AR_MAX - 1; ++j)
    if (j < q.nranks - 1) v[j] = ld_relaxed_sys(w + j);
#pragma unroll
  for (int j = 0; j < PC_AR_MAX - 1; ++j)
    if (j < q.nranks - 1 && !reached(v[j], e)) {
      const bool ok = q.sys_scope ? spin_geq<true>(w + j, e, q.err, q.timeout_ms, u)
                                  : spin_geq<false>(w + j, e, q.err, q.timeout_ms, u);
      if (!ok) return false;
    }
  fence_acquire(q.sys_scope);  // the acquire pattern for the relaxed loads above
  return true;
}

template <int DT, int OP>
PC_DEVICE void ar_scalar(const pc_ar_tab_s *tab, int P, uint64_t b) {
  using O = pc_ops::Op<DT, OP>;
  using T = typename O::T;
  T acc = __ldcg(reinterpret_cast<const T *>(tab->send[0] + b));
  for (int k = 1; k < P; ++k) acc = O::f(acc, __ldcg(reinterpret_cast<const T *>(tab->send[k] + b)));
  for (int k = 0; k < P; ++k) *reinterpret_cast<T *>(tab->recv[k] + b) = acc;
}

template <int DT, int OP>
PC_DEVICE void ar_fold_t(const pc_ar_tab_s *tab, int P, uint64_t off, uint64_t nbytes, uint32_t idx,
                         uint32_t n) {
  using O = pc_ops::Op<DT, OP>;
  using T = typename O::T;
  // 16-B aligned bases (pc_pallreduce_init), the same offset in every buffer:
  // scalar head to the 16-B boundary, 16-B body, scalar tail
  uint64_t head = (16 - (off & 15)) & 15;
  if (head > nbytes) head = nbytes;
  const uint64_t nv = (nbytes - head) / 16;
  const uint64_t body_end = head + nv * 16;
  for (uint64_t b = (uint64_t)idx * sizeof(T); b < head; b += (uint64_t)n * sizeof(T))
    ar_scalar<DT, OP>(tab, P, off + b);
  for (uint64_t b = body_end + (uint64_t)idx * sizeof(T); b < nbytes; b += (uint64_t)n * sizeof(T))
    ar_scalar<DT, OP>(tab, P, off + b);
  const uint8_t *s0 = tab->send[0] + off + head, *s1 = tab->send[1] + off + head, *s2 = tab->send[2] + off + head,
                *s3 = tab->send[3] + off + head, *s4 = tab->send[4] + off + head, *s5 = tab->send[5] + off + head,
                *s6 = tab->send[6] + off + head, *s7 = tab->send[7] + off + head;
  // destination pointers in registers too (stores could alias the table, so a
  // pointer read inside the loop would be re-issued before every store)
  uint8_t *d0 = tab->recv[0] + off + head, *d1 = tab->recv[1] + off + head, *d2 = tab->recv[2] + off + head,
          *d3 = tab->recv[3] + off + head, *d4 = tab->recv[4] + off + head, *d5 = tab->recv[5] + off + head,
          *d6 = tab->recv[6] + off + head, *d7 = tab->recv[7] + off + head;
  for (uint64_t v = idx; v < nv; v += n) {
    const uint64_t o = v * 16;
    uint4 x0 = __ldcg(reinterpret_cast<const uint4 *>(s0 + o)), x1, x2, x3, x4, x5, x6, x7;
    if (P > 1) x1 = __ldcg(reinterpret_cast<const uint4 *>(s1 + o));
    if (P > 2) x2 = __ldcg(reinterpret_cast<const uint4 *>(s2 + o));
    if (P > 3) x3 = __ldcg(reinterpret_cast<const uint4 *>(s3 + o));
    if (P > 4) x4 = __ldcg(reinterpret_cast<const uint4 *>(s4 + o));
    if (P > 5) x5 = __ldcg(reinterpret_cast<const uint4 *>(s5 + o));
    if (P > 6) x6 = __ldcg(reinterpret_cast<const uint4 *>(s6 + o));
    if (P > 7) x7 = __ldcg(reinterpret_cast<const uint4 *>(s7 + o));
    uint4 acc = x0;  // rank order (R25)
    if (P > 1) acc = pc_ops::vop<DT, OP>(acc, x1);
    if (P > 2) acc = pc_ops::vop<DT, OP>(acc, x2);
    if (P > 3) acc = pc_ops::vop<DT, OP>(acc, x3);
    if (P > 4) acc = pc_ops::vop<DT, OP>(acc, x4);
    if (P > 5) acc = pc_ops::vop<DT, OP>(acc, x5);
    if (P > 6) acc = pc_ops::vop<DT, OP>(acc, x6);
    if (P > 7) acc = pc_ops::vop<DT, OP>(acc, x7);
    *reinterpret_cast<uint4 *>(d0 + o) = acc;
    if (P > 1) *reinterpret_cast<uint4 *>(d1 + o) = acc;
    if (P > 2) *reinterpret_cast<uint4 *>(d2 + o) = acc;
    if (P > 3) *reinterpret_cast<uint4 *>(d3 + o) = acc;
    if (P > 4) *reinterpret_cast<uint4 *>(d4 + o) = acc;
    if (P > 5) *reinterpret_cast<uint4 *>(d5 + o) = acc;
    if (P > 6) *reinterpret_cast<uint4 *>(d6 + o) = acc;
    if (P > 7) *reinterpret_cast<uint4 *>(d7 + o) = acc;
  }
}

/* Fold partition u by n cooperating participants (index idx).  Not inlined:
 * the fold's P-way loads would otherwise raise the register allocation of
 * every producer kernel that calls a Pready binding (a call on the rare
 * completing path costs nothing measurable). */
#ifdef PC_INLINE_ALLREDUCE
/* (scalars only: a reference to the caller's by-value request would make
 * every thread copy the whole pc_prequest_t into local memory) */
static __device__ __noinline__ void ar_fold_scalars(const pc_ar_tab_s *t, int P, int dtype, int op, uint64_t off,
                                                    uint64_t nb, uint32_t idx, uint32_t n) {
#define PC_AR_CASE(DTV)                                      \
  if (op == 0) ar_fold_t<DTV, 0>(t, P, off, nb, idx, n);   \
  else if (op == 1) ar_fold_t<DTV, 1>(t, P, off, nb, idx, n); \
  else ar_fold_t<DTV, 2>(t, P, off, nb, idx, n);
  switch (dtype) {
    case 0: PC_AR_CASE(0); break;
    case 1: PC_AR_CASE(1); break;
    case 3: PC_AR_CASE(3); break;
    default: PC_AR_CASE(4); break;
  }
#undef PC_AR_CASE
}
PC_DEVICE void ar_fold(const pc_prequest_t &q, int u, uint32_t idx, uint32_t n) {
  ar_fold_scalars(q.ar_tab, q.nranks, q.dtype, q.op, (uint64_t)u * q.part_bytes, q.part_bytes, idx, n);
}
#endif

/* After the fold (every participant's stores ordered before by a barrier):
 * one cumulative fence, then done[u] = e on every rank. */
PC_DEVICE void ar_publish(const pc_prequest_t &q, int u, uint32_t e) {
  fence_release(q.sys_scope);
  for (int k = 0; k < q.nranks; ++k) st_relaxed_sys(q.ar_tab->done[k] + u, e);
}
/* A fold of the whole partition by one participant: also advance u's slice
 * counter by P, so epochs folded this way and cooperative epochs (R36, P
 * slices of one each) keep the same target e * P on the same request. */
PC_DEVICE void ar_publish_all(const pc_prequest_t &q, int u, uint32_t e) {
  uint32_t *c2 = q.ar_tab->cnt + q.partitions + u;
  if (q.sys_scope)
    atom_add_acq_rel_sys(c2, (uint32_t)q.nranks);
  else
    atom_add_acq_rel_gpu(c2, (uint32_t)q.nranks);
  ar_publish(q, u, e);
}

}  // namespace pc_detail

/* Thread granularity: any subset of threads, each for its own partition.
 * INLINE: every lane pushes its own partition's bytes, lanes of the warp that
 * share a transport partition are combined (__match_any_sync) into one counter
 * update, the completing contribution flags it (P:L231's "aggregate to the
 * block level internally", done per warp).  ENGINE: count, the completing
 * contribution marks the transport partition ready for the engine. */
PC_DEVICE int pc_pready(int partition, pc_prequest_t preq) {
  using namespace pc_detail;
  if (partition < 0 || partition >= preq.partitions) {
    set_error(preq.err, PC_DEV_ERR_ARG, partition);
    return PC_DEV_ERR_ARG;
  }
  if (preq.kind == PC_KIND_PALLREDUCE) {
    if (!preq.ar_tab) {
      st_release_gpu(preq.ready + partition, epoch_of(preq));
      return 0;
    }
#ifdef PC_INLINE_ALLREDUCE
    const uint32_t e = epoch_of(preq);  // INLINE (R33): this thread alone folds if it completes u
    if (ar_arrive(preq, partition, e)) {
      if (!ar_rtr_ok(preq, partition, e)) return PC_DEV_ERR_TIMEOUT;
      ar_fold(preq, partition, 0, 1);
      ar_publish_all(preq, partition, e);
    }
    return 0;
#else
    set_error(preq.err, PC_DEV_ERR_ARG, partition);  // INLINE allreduce needs -DPC_INLINE_ALLREDUCE
    return PC_DEV_ERR_ARG;
#endif
  }
  const unsigned mask = __activemask();
  const uint32_t lane = lane_id();
  const uint32_t first = __ffs(mask) - 1;
  const int t = partition / preq.agg;
  const unsigned grp = __match_any_sync(mask, counter_key(preq, partition));
  const uint32_t leader = __ffs(grp) - 1;
  if (preq.copy == 2) {  // LL: this lane pushes its partition's lines itself
    const uint32_t e = ll_push(preq, partition, 0, 1);
    __syncwarp(mask);
    if (lane == leader) ll_account(preq, t, __popc(grp), e, partition);
    return 0;
  }
  uint32_t e = 0, rtr0 = 0;
  // INLINE partitions of 8 or 16 aligned bytes (the paper's 8 B per thread):
  // load the payload before the {epoch, rtr} acquire (round trips overlap)
  const uint64_t off0 = (uint64_t)partition * preq.part_bytes;
  const bool small = preq.copy == 0 && (preq.part_bytes == 8 || preq.part_bytes == 16) &&
                     ((reinterpret_cast<uintptr_t>(preq.sbuf + off0) | reinterpret_cast<uintptr_t>(preq.peer_rbuf + off0)) &
                      (preq.part_bytes - 1)) == 0;
  uint4 v = make_uint4(0, 0, 0, 0);
  if (small) {
    if (preq.part_bytes == 16) {
      v = __ldcg(reinterpret_cast<const uint4 *>(preq.sbuf + off0));
    } else {
      const uint2 h = __ldcg(reinterpret_cast<const uint2 *>(preq.sbuf + off0));
      v.x = h.x;
      v.y = h.y;
    }
  }
  if (lane == first) {
    if (preq.copy == 0 && preq.part_bytes) {
      const uint2 er = epoch_rtr(preq);
      e = er.x;
      rtr0 = er.y;
    } else {
      e = epoch_relaxed(preq);
    }
  }
  e = __shfl_sync(mask, e, first);
  if (preq.copy == 1 || preq.copy == 3) {  // ENGINE / HOST progression
    __syncwarp(mask);    // every lane's data writes are ordered before the leader's release
    if (lane == leader && contribute(preq, t, __popc(grp), e, partition)) mark_ready(preq, t, e);
    return 0;
  }
  if (preq.part_bytes) {
    bool ok = true;
    if (lane == first && !reached(rtr0, e)) ok = spin_geq<true>(preq.rtr, e, preq.err, preq.timeout_ms, partition);
    if (!__shfl_sync(mask, ok, first)) return PC_DEV_ERR_TIMEOUT;
    if (small) {
      if (preq.part_bytes == 16)
        *reinterpret_cast<uint4 *>(preq.peer_rbuf + off0) = v;
      else
        *reinterpret_cast<uint2 *>(preq.peer_rbuf + off0) = make_uint2(v.x, v.y);
    } else {
      copy_bytes_cold(preq.peer_rbuf + off0, preq.sbuf + off0, preq.part_bytes, 0, 1);
    }
  }
  // One fence per group, not per lane: __syncwarp orders the group's pushes
  // before the leader's fence, which is cumulative (the cooperative-groups
  // grid.sync pattern: barrier, then one thread's fence + signal).
  __syncwarp(mask);
  if (lane == leader) {
    if (preq.part_bytes) fence_before_publish(preq);
    publish(preq, t, __popc(grp), e, partition);
  }
  return 0;
}

/* Warp granularity: warp-collective — ALL 32 lanes of the warp call it with
 * the same partition (like __syncwarp()); one notification per warp (P:L137,
 * reading R11).  (__activemask() cannot be used to find the participants: with
 * independent thread scheduling a converged-looking warp may run this code as
 * several subsets, which would count the warp more than once.)  INLINE: the
 * warp pushes its partition with 16-B stores, then publishes. */
PC_DEVICE int pc_pready_warp(int partition, pc_prequest_t preq) {
  using namespace pc_detail;
  const unsigned full = 0xffffffffu;
  const uint32_t lane = lane_id();
  __syncwarp(full);  // every lane's data writes are ordered before lane 0's release
  if (partition < 0 || partition >= preq.partitions) {
    if (lane == 0) set_error(preq.err, PC_DEV_ERR_ARG, partition);
    return PC_DEV_ERR_ARG;
  }
  if (preq.kind == PC_KIND_PALLREDUCE) {
    if (!preq.ar_tab) {
      if (lane == 0) st_release_gpu(preq.ready + partition, epoch_of(preq));
      __syncwarp(full);
      return 0;
    }
#ifdef PC_INLINE_ALLREDUCE
    int st = 0;  // INLINE (R33): 1 = this warp completed u and folds it, -1 = RTR timeout
    uint32_t e = 0;
    if (lane == 0) {
      e = epoch_of(preq);
      st = ar_arrive(preq, partition, e) ? (ar_rtr_ok(preq, partition, e) ? 1 : -1) : 0;
    }
    st = __shfl_sync(full, st, 0);
    e = __shfl_sync(full, e, 0);
    if (st == 1) {
      ar_fold(preq, partition, lane, 32);
      __syncwarp(full);
      if (lane == 0) ar_publish_all(preq, partition, e);
    }
    __syncwarp(full);
    return st < 0 ? PC_DEV_ERR_TIMEOUT : 0;
#else
    if (lane == 0) set_error(preq.err, PC_DEV_ERR_ARG, partition);  // needs -DPC_INLINE_ALLREDUCE
    __syncwarp(full);
    return PC_DEV_ERR_ARG;
#endif
  }
  const int t = partition / preq.agg;
  if (preq.copy == 2) {  // LL: every lane loads its line, reads the epoch and stores (no broadcast)
    const uint32_t e = ll_push(preq, partition, lane, 32);
    __syncwarp(full);
    if (lane == 0) ll_account(preq, t, 1, e, partition);
    __syncwarp(full);
    return 0;
  }
  if (preq.copy == 1 || preq.copy == 3 || preq.part_bytes == 0) {  // no bytes for this warp to move
    if (lane == 0) {
      const uint32_t e = epoch_relaxed(preq);
      if (preq.copy == 1 || preq.copy == 3) {
        if (contribute(preq, t, 1, e, partition)) mark_ready(preq, t, e);
      } else {
        publish(preq, t, 1, e, partition);
      }
    }
    __syncwarp(full);
    return 0;
  }
  uint32_t e = 0;
  bool ok = true;
  const uint64_t off = (uint64_t)partition * preq.part_bytes;
  // Small aligned partition (<= one 16-B vector per lane): load the payload
  // BEFORE the {epoch, rtr} acquire so the two L2 round trips overlap (the
  // bytes are this kernel's own; only the peer store must follow the acquire).
  const uintptr_t al = reinterpret_cast<uintptr_t>(preq.sbuf + off) | reinterpret_cast<uintptr_t>(preq.peer_rbuf + off);
  const bool small16 = preq.part_bytes <= 512 && (preq.part_bytes & 15) == 0 && (al & 15) == 0;
  const bool small8 = !small16 && preq.part_bytes <= 256 && (preq.part_bytes & 7) == 0 && (al & 7) == 0;
  const bool small = small16 || small8;
  uint4 v = make_uint4(0, 0, 0, 0);
  if (small16 && 16ull * lane < preq.part_bytes) v = __ldcg(reinterpret_cast<const uint4 *>(preq.sbuf + off) + lane);
  if (small8 && 8ull * lane < preq.part_bytes) {
    const uint2 h = __ldcg(reinterpret_cast<const uint2 *>(preq.sbuf + off) + lane);
    v.x = h.x;
    v.y = h.y;
  }
  if (lane == 0) {
    const uint2 er = epoch_rtr(preq);
    e = er.x;
    if (!reached(er.y, e)) ok = spin_geq<true>(preq.rtr, e, preq.err, preq.timeout_ms, partition);
  }
  e = __shfl_sync(full, e, 0);
  if (!__shfl_sync(full, ok, 0)) return PC_DEV_ERR_TIMEOUT;
  if (small16) {
    if (16ull * lane < preq.part_bytes) reinterpret_cast<uint4 *>(preq.peer_rbuf + off)[lane] = v;
  } else if (small8) {
    if (8ull * lane < preq.part_bytes) reinterpret_cast<uint2 *>(preq.peer_rbuf + off)[lane] = make_uint2(v.x, v.y);
  } else {
    copy_bytes_cold(preq.peer_rbuf + off, preq.sbuf + off, preq.part_bytes, lane, 32);
  }
  __syncwarp(full);  // the warp's pushes, then ONE cumulative fence by lane 0
  if (lane == 0) {
    fence_before_publish(preq);
    publish(preq, t, 1, e, partition);
  }
  __syncwarp(full);
  return 0;
}

/* Warp granularity for a persistent warp (R35's check-once, warp form):
 * pc_warp_begin (warp-collective) checks {epoch, ready-to-receive} once per
 * warp per epoch — both fixed once reached — and the pc_pready_warp(...,
 * st) that follow (INLINE partitioned send, partitions of at most 16 B per
 * lane) push straight away and release the flag with one st.release: no
 * acquire round trip per message.  Any other request (or st.ok == 0) takes
 * the plain pc_pready_warp. */
struct pc_warp_state {
  uint32_t e;   /* the epoch pc_warp_begin found */
  uint32_t ok;  /* 1: checked; the fast path may be used */
};
PC_DEVICE int pc_warp_begin(pc_prequest_t preq, pc_warp_state *st) {
  using namespace pc_detail;
  const unsigned full = 0xffffffffu;
  const uint32_t lane = lane_id();
  st->e = 0;
  st->ok = 0;
  if (preq.kind == PC_KIND_PALLREDUCE || preq.copy != 0 || preq.part_bytes == 0 || preq.part_bytes > 512 ||
      (preq.part_bytes & 7) != 0)
    return PC_DEV_ERR_ARG;
  uint32_t e = 0;
  int ok = 1;
  if (lane == 0) {
    const uint2 er = epoch_rtr(preq);
    e = er.x;
    if (!reached(er.y, e)) ok = spin_geq<true>(preq.rtr, e, preq.err, preq.timeout_ms, -5);
  }
  e = __shfl_sync(full, e, 0);
  ok = __shfl_sync(full, ok, 0);
  __syncwarp(full);  // lane 0's acquire happens before every lane's later pushes
  if (!ok) return PC_DEV_ERR_TIMEOUT;
  st->e = e;
  st->ok = 1;
  return 0;
}

PC_DEVICE int pc_pready_warp(int partition, pc_prequest_t preq);

PC_DEVICE int pc_pready_warp(int partition, pc_prequest_t preq, const pc_warp_state &st) {
  using namespace pc_detail;
  const unsigned full = 0xffffffffu;
  if (!st.ok) return pc_pready_warp(partition, preq);
  const uint64_t off = (uint64_t)partition * preq.part_bytes;
  const uintptr_t al = reinterpret_cast<uintptr_t>(preq.sbuf + off) | reinterpret_cast<uintptr_t>(preq.peer_rbuf + off);
  const bool small16 = (preq.part_bytes & 15) == 0 && (al & 15) == 0;
  if (!small16 && (al & 7) != 0) return pc_pready_warp(partition, preq);
  const uint32_t lane = lane_id();
  __syncwarp(full);  // every lane's data writes are ordered before the pushes
  if (partition < 0 || partition >= preq.partitions) {
    if (lane == 0 && atomicCAS(preq.err, 0, PC_DEV_ERR_ARG) == 0) preq.err[1] = partition;
    return PC_DEV_ERR_ARG;
  }
  if (small16) {
    if (16ull * lane < preq.part_bytes)
      reinterpret_cast<uint4 *>(preq.peer_rbuf + off)[lane] = __ldcg(reinterpret_cast<const uint4 *>(preq.sbuf + off) + lane);
  } else if (8ull * lane < preq.part_bytes) {
    reinterpret_cast<uint2 *>(preq.peer_rbuf + off)[lane] = __ldcg(reinterpret_cast<const uint2 *>(preq.sbuf + off) + lane);
  }
  __syncwarp(full);  // the warp's pushes, then ONE release by lane 0
  if (lane == 0) {
    if (preq.agg == 1 && !preq.xpart) {  // the flag store itself releases
      if (preq.sys_scope)
        st_release_sys(preq.peer_flags + partition, st.e);
      else
        st_release_gpu(preq.peer_flags + partition, st.e);
      st_relaxed_gpu(preq.sent + partition, st.e);
    } else {
      fence_before_publish(preq);
      publish(preq, partition / preq.agg, 1, st.e, partition);
    }
  }
  __syncwarp(full);
  return 0;
}

/* Block granularity: every thread of the block calls it with the same
 * partition; __syncthreads() then one notification.  INLINE: the
 * block pushes its partition, then thread 0 publishes. */
PC_DEVICE int pc_pready_block(int partition, pc_prequest_t preq) {
  using namespace pc_detail;
  __shared__ uint32_t s_e;
  __shared__ int s_ok;
  const uint32_t tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  const uint32_t nthr = blockDim.x * blockDim.y * blockDim.z;
  if (partition < 0 || partition >= preq.partitions) {
    if (tid == 0) set_error(preq.err, PC_DEV_ERR_ARG, partition);
    return PC_DEV_ERR_ARG;
  }
  // INLINE Kernel Copy of a partition with bytes: thread 0 takes the epoch and
  // checks the receiver's ready-to-receive word BEFORE the data barrier (it
  // does not depend on the partition's bytes), so that one barrier publishes
  // both the data and {e, ok}.  (The previous call's readers of s_e / s_ok all
  // passed its closing barrier before thread 0 gets here.)
  const bool inl = preq.kind != PC_KIND_PALLREDUCE && preq.copy == 0 && preq.part_bytes != 0;
  const bool flag_only = preq.kind != PC_KIND_PALLREDUCE && (preq.copy == 1 || preq.copy == 3 || preq.part_bytes == 0);
  uint32_t e0 = 0;
  if (tid == 0) {
    if (inl) {
      const uint2 er = epoch_rtr(preq);
      s_e = er.x;
      s_ok = 1;
      if (!reached(er.y, er.x)) s_ok = spin_geq<true>(preq.rtr, er.x, preq.err, preq.timeout_ms, partition);
    } else if (flag_only) {
      e0 = epoch_relaxed(preq);  // (ENGINE / HOST / no bytes) its latency hides behind the barrier too
    }
  }
  __syncthreads();  // the block's data writes are complete
  if (preq.kind == PC_KIND_PALLREDUCE) {
    if (!preq.ar_tab) {
      if (tid == 0) st_release_gpu(preq.ready + partition, epoch_of(preq));
      return 0;
    }
#ifdef PC_INLINE_ALLREDUCE
    if (tid == 0) {  // INLINE (R33): s_ok 1 = this block completed u and folds it, -1 = RTR timeout
      const uint32_t e = epoch_of(preq);
      s_e = e;
      s_ok = ar_arrive(preq, partition, e) ? (ar_rtr_ok(preq, partition, e) ? 1 : -1) : 0;
    }
    __syncthreads();
    const int st = s_ok;
    if (st == 1) {
      ar_fold(preq, partition, tid, nthr);
      __syncthreads();  // every thread's stores, then ONE cumulative fence + the done words
      if (tid == 0) ar_publish_all(preq, partition, s_e);
    }
    __syncthreads();  // s_e / s_ok are reused by the block's next Pready
    return st < 0 ? PC_DEV_ERR_TIMEOUT : 0;
#else
    if (tid == 0) set_error(preq.err, PC_DEV_ERR_ARG, partition);  // needs -DPC_INLINE_ALLREDUCE
    return PC_DEV_ERR_ARG;
#endif
  }
  const int t = partition / preq.agg;
  if (preq.copy == 2) {  // LL: every thread pushes its lines
    const uint32_t e = ll_push(preq, partition, tid, nthr);
    __syncthreads();
    if (tid == 0) ll_account(preq, t, 1, e, partition);
    return 0;
  }
  if (flag_only) {  // no bytes for this block to move
    if (tid == 0) {
      const uint32_t e = e0;
      if (preq.copy == 1 || preq.copy == 3) {
        if (contribute(preq, t, 1, e, partition)) mark_ready(preq, t, e);
      } else {
        publish(preq, t, 1, e, partition);
      }
    }
    return 0;
  }
  // Partitions of at most one 16-B vector per thread (the paper's 8 KiB
  // block = 1024 threads x 8 B): one L2 read-back per thread (the user's
  // threads wrote the partition in any layout), then its push.
  const uint32_t e = s_e;
  if (!s_ok) return PC_DEV_ERR_TIMEOUT;
  const uint64_t off = (uint64_t)partition * preq.part_bytes;
  const uintptr_t al = reinterpret_cast<uintptr_t>(preq.sbuf + off) | reinterpret_cast<uintptr_t>(preq.peer_rbuf + off);
  const bool v16 = preq.part_bytes <= 16ull * nthr && (preq.part_bytes & 15) == 0 && (al & 15) == 0;
  const bool v8 = !v16 && preq.part_bytes <= 8ull * nthr && (preq.part_bytes & 7) == 0 && (al & 7) == 0;
  uint4 v = make_uint4(0, 0, 0, 0);
  if (v16 && 16ull * tid < preq.part_bytes) v = __ldcg(reinterpret_cast<const uint4 *>(preq.sbuf + off) + tid);
  if (v8 && 8ull * tid < preq.part_bytes) {
    const uint2 h = __ldcg(reinterpret_cast<const uint2 *>(preq.sbuf + off) + tid);
    v.x = h.x;
    v.y = h.y;
  }
  if (v16) {
    if (16ull * tid < preq.part_bytes) reinterpret_cast<uint4 *>(preq.peer_rbuf + off)[tid] = v;
  } else if (v8) {
    if (8ull * tid < preq.part_bytes) reinterpret_cast<uint2 *>(preq.peer_rbuf + off)[tid] = make_uint2(v.x, v.y);
  } else {
    copy_bytes_cold(preq.peer_rbuf + off, preq.sbuf + off, preq.part_bytes, tid, nthr);
  }
  __syncthreads();  // the block's pushes, then ONE cumulative fence by thread 0 (not one per thread)
  if (tid == 0) {
    fence_before_publish(preq);
    publish(preq, t, 1, e, partition);
  }
  return 0;
}

/* Block granularity from registers (R35): see the header comment.  Same
 * chain as the INLINE path of pc_pready_block minus the read-back: thread 0
 * checks {epoch, ready-to-receive} before the barrier that also orders the
 * block's send-buffer writes, every thread assigns its element to the
 * receiver, a second barrier, then ONE release fence and the flag. */
namespace pc_detail {
template <typename T>
PC_DEVICE bool put_eligible(const pc_prequest_t &q) {
  return q.kind != PC_KIND_PALLREDUCE && q.copy == 0 && q.part_bytes != 0 &&
         ((reinterpret_cast<uintptr_t>(q.peer_rbuf) | q.part_bytes) & (sizeof(T) - 1)) == 0;
}
/* The release of partition p after a barrier that ordered its assignments. */
PC_DEVICE void put_release(const pc_prequest_t &q, int partition, uint32_t e) {
  if (q.agg == 1 && !q.xpart) {  // the flag store itself releases (one MEMBAR, no separate fence)
    if (q.sys_scope)
      st_release_sys(q.peer_flags + partition, e);
    else
      st_release_gpu(q.peer_flags + partition, e);
    st_relaxed_gpu(q.sent + partition, e);
  } else {
    fence_before_publish(q);
    publish(q, partition / q.agg, 1, e, partition);
  }
}
/* The assignment, barrier, release and flag of a checked epoch. */
template <typename T>
PC_DEVICE void put_publish(int partition, const pc_prequest_t &q, uint64_t idx, const T &v, uint32_t e,
                           uint32_t tid) {
  if (idx < q.part_bytes / sizeof(T))
    *reinterpret_cast<T *>(q.peer_rbuf + (uint64_t)partition * q.part_bytes + idx * sizeof(T)) = v;
  __syncthreads();  // the block's pushes, then ONE cumulative release by thread 0
  if (tid == 0) put_release(q, partition, e);
}
}  // namespace pc_detail

template <typename T>
PC_DEVICE int pc_pready_block_put(int partition, pc_prequest_t preq, uint64_t idx, const T &v) {
  using namespace pc_detail;
  static_assert(sizeof(T) == 4 || sizeof(T) == 8 || sizeof(T) == 16, "element of 4, 8 or 16 bytes");
  if (!put_eligible<T>(preq)) return pc_pready_block(partition, preq);
  __shared__ uint32_t s_e;
  __shared__ int s_ok;
  const uint32_t tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  if (partition < 0 || partition >= preq.partitions) {
    if (tid == 0) set_error(preq.err, PC_DEV_ERR_ARG, partition);
    return PC_DEV_ERR_ARG;
  }
  if (tid == 0) {  // (the previous call's readers of s_e / s_ok passed its closing barrier)
    const uint2 er = epoch_rtr(preq);
    s_e = er.x;
    s_ok = 1;
    if (!reached(er.y, er.x)) s_ok = spin_geq<true>(preq.rtr, er.x, preq.err, preq.timeout_ms, partition);
  }
  __syncthreads();  // {e, ok} (the elements themselves are this thread's own registers)
  const uint32_t e = s_e;
  if (!s_ok) return PC_DEV_ERR_TIMEOUT;
  put_publish(partition, preq, idx, v, e, tid);
  return 0;
}

/* Persistent producers (R35): the {epoch, ready-to-receive} check once per
 * CTA per epoch, before its first pc_pready_block_put(..., st).  batch > 1:
 * the CTA releases its Preadies `batch` at a time — one barrier and one
 * warp-wide MEMBAR per batch instead of per logical block (lane k of warp 0
 * releases the k-th pending partition's flag); a flag is never set before
 * its partition's bytes are visible, only later; pc_put_end (block-
 * collective, after the CTA's last Pready) releases the rest.  Both are
 * fixed for the rest of the epoch once reached, so the later calls carry no
 * load and no barrier before the assignment — the raw chain (assign from
 * registers, barrier, release, flag) with nothing out of line in the loop.
 * Block-collective.  Returns 0 with st->ok = 1; PC_DEV_ERR_ARG with st->ok =
 * 0 when the request does not take the register path (not an INLINE
 * partitioned send, or misaligned for T: use pc_pready_block); or
 * PC_DEV_ERR_TIMEOUT. */
struct pc_put_state {
  uint32_t e;      /* the epoch pc_put_begin found */
  uint32_t ok;     /* 1: checked; the fast pc_pready_block_put may be used */
  uint32_t batch;  /* logical blocks per release (1 .. min(32, threads per block)) */
  uint32_t npend;  /* Preadies since the last release (the same in every thread) */
  int mine;        /* thread k < batch: the partition of the k-th pending Pready */
};

template <typename T>
PC_DEVICE int pc_put_begin(pc_prequest_t preq, pc_put_state *st, int batch = 1) {
  using namespace pc_detail;
  __shared__ uint32_t s_e;
  __shared__ int s_ok;
  const uint32_t tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  st->e = 0;
  st->ok = 0;
  const uint32_t nthr = blockDim.x * blockDim.y * blockDim.z;  // thread k < batch records pending Pready k
  const uint32_t cap = nthr < 32 ? nthr : 32;
  st->batch = batch < 1 ? 1u : ((uint32_t)batch > cap ? cap : (uint32_t)batch);
  st->npend = 0;
  st->mine = -1;
  if (!put_eligible<T>(preq)) return PC_DEV_ERR_ARG;
  if (tid == 0) {
    const uint2 er = epoch_rtr(preq);
    s_e = er.x;
    s_ok = 1;
    if (!reached(er.y, er.x)) s_ok = spin_geq<true>(preq.rtr, er.x, preq.err, preq.timeout_ms, -4);
  }
  __syncthreads();
  if (!s_ok) return PC_DEV_ERR_TIMEOUT;
  st->e = s_e;
  st->ok = 1;
  return 0;
}

template <typename T>
PC_DEVICE int pc_pready_block_put(int partition, pc_prequest_t preq, uint64_t idx, const T &v, pc_put_state &st) {
  static_assert(sizeof(T) == 4 || sizeof(T) == 8 || sizeof(T) == 16, "element of 4, 8 or 16 bytes");
  if (!st.ok) return PC_DEV_ERR_ARG;
  const uint32_t tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  if ((unsigned)partition >= (unsigned)preq.partitions) {  // (no out-of-line call in the loop)
    if (tid == 0 && atomicCAS(preq.err, 0, PC_DEV_ERR_ARG) == 0) preq.err[1] = partition;
    return PC_DEV_ERR_ARG;
  }
  if (st.batch == 1) {
    pc_detail::put_publish(partition, preq, idx, v, st.e, tid);
    return 0;
  }
  if (idx < preq.part_bytes / sizeof(T))
    *reinterpret_cast<T *>(preq.peer_rbuf + (uint64_t)partition * preq.part_bytes + idx * sizeof(T)) = v;
  if (tid == st.npend) st.mine = partition;
  if (++st.npend < st.batch) return 0;
  __syncthreads();  // the batch's assignments, then lane k of warp 0 releases pending partition k
  if (tid < st.npend) pc_detail::put_release(preq, st.mine, st.e);
  st.npend = 0;
  return 0;
}

/* The MPI-shaped block Pready in a persistent CTA, checked once: with a
 * state from pc_put_begin<uint8_t> (any size or alignment), the block's
 * partition is read back after the barrier and pushed as in pc_pready_block,
 * but {epoch, ready-to-receive} is not re-checked and the releases are
 * batched like pc_pready_block_put's (pc_put_end flushes). */
PC_DEVICE int pc_pready_block(int partition, pc_prequest_t preq, pc_put_state &st) {
  using namespace pc_detail;
  if (!st.ok) return pc_pready_block(partition, preq);
  const uint32_t tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  const uint32_t nthr = blockDim.x * blockDim.y * blockDim.z;
  if ((unsigned)partition >= (unsigned)preq.partitions) {
    if (tid == 0 && atomicCAS(preq.err, 0, PC_DEV_ERR_ARG) == 0) preq.err[1] = partition;
    return PC_DEV_ERR_ARG;
  }
  __syncthreads();  // the block's data writes are complete
  const uint64_t off = (uint64_t)partition * preq.part_bytes;
  const uintptr_t al = reinterpret_cast<uintptr_t>(preq.sbuf + off) | reinterpret_cast<uintptr_t>(preq.peer_rbuf + off);
  if (preq.part_bytes <= 16ull * nthr && (preq.part_bytes & 15) == 0 && (al & 15) == 0) {
    if (16ull * tid < preq.part_bytes)
      reinterpret_cast<uint4 *>(preq.peer_rbuf + off)[tid] = __ldcg(reinterpret_cast<const uint4 *>(preq.sbuf + off) + tid);
  } else if (preq.part_bytes <= 8ull * nthr && (preq.part_bytes & 7) == 0 && (al & 7) == 0) {
    if (8ull * tid < preq.part_bytes)
      reinterpret_cast<uint2 *>(preq.peer_rbuf + off)[tid] = __ldcg(reinterpret_cast<const uint2 *>(preq.sbuf + off) + tid);
  } else {
    copy_bytes_cold(preq.peer_rbuf + off, preq.sbuf + off, preq.part_bytes, tid, nthr);
  }
  if (tid == st.npend) st.mine = partition;
  if (++st.npend < st.batch) return 0;
  __syncthreads();  // the batch's pushes, then lane k of warp 0 releases pending partition k
  if (tid < st.npend) put_release(preq, st.mine, st.e);
  st.npend = 0;
  return 0;
}

/* Block-collective, after the CTA's last pc_pready_block_put of the epoch:
 * releases the partitions still pending in a batch. */
PC_DEVICE void pc_put_end(pc_prequest_t preq, pc_put_state &st) {
  if (!st.ok || st.npend == 0) return;
  const uint32_t tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  __syncthreads();
  if (tid < st.npend) pc_detail::put_release(preq, st.mine, st.e);
  st.npend = 0;
}

#ifdef PC_INLINE_ALLREDUCE
/* Cooperative INLINE allreduce (MPIX extension, reading R36): for producers
 * that run the P ranks' blocks of partition u side by side (one launch over
 * the co-located ranks, units (u, r) adjacent and all CTAs resident — the
 * caller's construction; the spin below is bounded by the request's timeout).
 * Block (u, r): its data writes, then one arrival on u's counter (acq_rel),
 * a wait until all P ranks arrived and every peer is ready to receive, then it
 * folds slice r of P of partition u (16-B aligned byte ranges) over the P
 * send buffers in rank order (R25: the same bits as O6 / the DIRECT engine)
 * into every rank's recv buffer; the block completing the last slice (a second
 * counter, the INLINE request's unused ready words in rank 0's control block)
 * writes done[u] = e on every rank.  Instead of one block folding P
 * partitions, P blocks fold one each — and the P partitions were just written
 * (L2).  Other request kinds: pc_pready_block. */
PC_DEVICE int pc_pready_block_coop(int partition, pc_prequest_t preq) {
  using namespace pc_detail;
  if (preq.kind != PC_KIND_PALLREDUCE || !preq.ar_tab) return pc_pready_block(partition, preq);
  __shared__ uint32_t s_e;
  __shared__ int s_ok, s_r;
  const uint32_t tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  const uint32_t nthr = blockDim.x * blockDim.y * blockDim.z;
  if (partition < 0 || partition >= preq.partitions) {
    if (tid == 0) set_error(preq.err, PC_DEV_ERR_ARG, partition);
    return PC_DEV_ERR_ARG;
  }
  const int P = preq.nranks;
  const pc_ar_tab_s *t = preq.ar_tab;
  __syncthreads();  // the block's data writes are complete
  if (tid == 0) {
    const uint32_t e = epoch_of(preq);
    s_e = e;
    int r = 0;
    for (int k = 0; k < P; ++k)
      if (t->send[k] == preq.sbuf) r = k;
    s_r = r;
    uint32_t *c = t->cnt + partition;
    const uint32_t old = preq.sys_scope ? atom_add_acq_rel_sys(c, 1u) : atom_add_acq_rel_gpu(c, 1u);
    const int32_t d = (int32_t)(e * (uint32_t)P - old);
    int ok = 1;
    if (d <= 0) {  // more than P arrivals in this epoch: a duplicate Pready
      set_error(preq.err, PC_DEV_ERR_DEVICE, partition);
      ok = 0;
    } else if (d > 1) {  // wait for the other ranks' blocks of u
      ok = preq.sys_scope ? spin_geq<true>(c, e * (uint32_t)P, preq.err, preq.timeout_ms, partition)
                          : spin_geq<false>(c, e * (uint32_t)P, preq.err, preq.timeout_ms, partition);
    }
    if (ok) ok = ar_rtr_ok(preq, partition, e) ? 1 : 0;
    s_ok = ok;
  }
  __syncthreads();
  const uint32_t e = s_e;
  const int r = s_r;
  if (!s_ok) return PC_DEV_ERR_TIMEOUT;
  const uint64_t chunk = ((preq.part_bytes + (uint64_t)P * 16 - 1) / ((uint64_t)P * 16)) * 16;
  const uint64_t lo = (uint64_t)r * chunk;
  const uint64_t hi = lo + chunk < preq.part_bytes ? lo + chunk : preq.part_bytes;
  if (lo < hi)
    ar_fold_scalars(t, P, preq.dtype, preq.op, (uint64_t)partition * preq.part_bytes + lo, hi - lo, tid, nthr);
  __syncthreads();  // every thread's stores, then ONE release + the slice count
  if (tid == 0) {
    fence_release(preq.sys_scope);
    uint32_t *c2 = t->cnt + preq.partitions + partition;
    const uint32_t old = preq.sys_scope ? atom_add_acq_rel_sys(c2, 1u) : atom_add_acq_rel_gpu(c2, 1u);
    const int32_t d = (int32_t)(e * (uint32_t)P - old);
    if (d <= 0)
      set_error(preq.err, PC_DEV_ERR_DEVICE, partition);
    else if (d == 1)
      ar_publish(preq, partition, e);  // (its release covers the other slices, acquired by the add)
  }
  __syncthreads();  // s_e / s_ok / s_r are reused by the block's next Pready
  return 0;
}
#endif

/* ---------------------------------------------------------------- Parrived */
/* Allgather receive partition u' = k * partitions + u (rank k's partition u):
 * all of its slices' arrival epochs (written by rank k after its pushes). */
namespace pc_detail {
PC_DEVICE bool ag_arrived(const pc_prequest_t &q, int up, uint32_t e) {
  for (uint32_t s = 0; s < q.done_mul; ++s)
    if (!reached(ld_acquire_scope(q.srcflags + (uint64_t)up * q.done_mul + s, q.sys_scope), e)) return false;
  return true;
}
}  // namespace pc_detail

PC_DEVICE int pc_parrived(pc_prequest_t preq, int partition) {
  using namespace pc_detail;
  const bool ag = preq.kind == PC_KIND_PALLREDUCE && preq.coll == 2;
  if (partition < 0 || partition >= (ag ? preq.nranks * preq.partitions : preq.partitions)) return 0;
  const uint32_t e = epoch_of(preq);
  if (ag) return ag_arrived(preq, partition, e) ? 1 : 0;
  if (preq.kind == PC_KIND_PALLREDUCE)  // INLINE: done[u] written by the folding rank (maybe another GPU)
    return reached(ld_acquire_scope(preq.done + partition, preq.sys_scope), e * preq.done_mul);
  if (preq.kind == PC_KIND_PSEND) {
    const int t = partition / preq.agg;
    return reached(ld_acquire_gpu(preq.sent + t), e);
  }
  const uint32_t g = *(const volatile uint32_t *)preq.layout;
  if (g == 0) return 0;  // sender has not published its transport layout yet
  if (g & PC_LAYOUT_LL) return ll_consume(preq, partition, e) ? 1 : 0;
  if (g & PC_LAYOUT_XP)
    return reached(ld_acquire_scope(preq.flags + partition, preq.sys_scope),
                   e * xp_need((uint64_t)partition, preq.part_bytes, g & PC_LAYOUT_G, preq.peer_part_bytes));
  return reached(ld_acquire_scope(preq.flags + partition / (int)g, preq.sys_scope), e);
}

/* Acquire-spin until pc_parrived(preq, partition) (bounded by timeout_ms).
 * The epoch and the transport layout are read once; the loop is a single
 * ld.acquire of the partition's flag (one L2 round trip per poll). */
PC_DEVICE int pc_wait_arrived(pc_prequest_t preq, int partition) {
  using namespace pc_detail;
  const bool ag = preq.kind == PC_KIND_PALLREDUCE && preq.coll == 2;
  if (partition < 0 || partition >= (ag ? preq.nranks * preq.partitions : preq.partitions)) return PC_DEV_ERR_ARG;
  const uint64_t t0 = globaltimer();
  const uint32_t e = epoch_of(preq);
  if (ag) {
    uint32_t n = 0;
    while (!ag_arrived(preq, partition, e)) {
      if ((++n & 127) == 0) {
        if (aborted(preq.err)) return PC_DEV_ERR_TIMEOUT;
        if (preq.timeout_ms && globaltimer() - t0 > (uint64_t)preq.timeout_ms * 1000000ull) {
          set_error(preq.err, PC_DEV_ERR_TIMEOUT, partition);
          return PC_DEV_ERR_TIMEOUT;
        }
        if (n > 4096) __nanosleep(128);
      }
    }
    return 0;
  }
  const uint32_t *w;
  uint32_t target = e;
  bool sys = false;
  if (preq.kind == PC_KIND_PALLREDUCE) {
    w = preq.done + partition;
    target = e * preq.done_mul;
  } else if (preq.kind == PC_KIND_PSEND) {
    w = preq.sent + partition / preq.agg;
  } else {
    uint32_t g;
    uint32_t n = 0;
    while ((g = *(const volatile uint32_t *)preq.layout) == 0) {  // sender not set up yet
      if ((++n & 127) == 0) {
        if (aborted(preq.err)) return PC_DEV_ERR_TIMEOUT;
        if (preq.timeout_ms && globaltimer() - t0 > (uint64_t)preq.timeout_ms * 1000000ull) {
          set_error(preq.err, PC_DEV_ERR_TIMEOUT, partition);
          return PC_DEV_ERR_TIMEOUT;
        }
        __nanosleep(256);
      }
    }
    if (g & PC_LAYOUT_LL) {  // poll the partition's lines themselves
      n = 0;
      while (!ll_consume(preq, partition, e)) {
        if ((++n & 127) == 0) {
          if (aborted(preq.err)) return PC_DEV_ERR_TIMEOUT;
          if (preq.timeout_ms && globaltimer() - t0 > (uint64_t)preq.timeout_ms * 1000000ull) {
            set_error(preq.err, PC_DEV_ERR_TIMEOUT, partition);
            return PC_DEV_ERR_TIMEOUT;
          }
          if (n > 4096) __nanosleep(128);
        }
      }
      return 0;
    }
    if (g & PC_LAYOUT_XP) {
      w = preq.flags + partition;
      target = e * xp_need((uint64_t)partition, preq.part_bytes, g & PC_LAYOUT_G, preq.peer_part_bytes);
    } else {
      w = preq.flags + partition / (int)g;
    }
    sys = preq.sys_scope != 0;
  }
  // no bytes to read after the flag -> a relaxed poll is enough
  const bool relaxed = preq.part_bytes == 0;
  uint32_t n = 0;
  while (!reached(relaxed ? ld_relaxed_sys(w) : (sys ? ld_acquire_sys(w) : ld_acquire_gpu(w)), target)) {
    if ((++n & 127) == 0) {
      if (aborted(preq.err)) return PC_DEV_ERR_TIMEOUT;
      if (preq.timeout_ms && globaltimer() - t0 > (uint64_t)preq.timeout_ms * 1000000ull) {
        set_error(preq.err, PC_DEV_ERR_TIMEOUT, partition);
        return PC_DEV_ERR_TIMEOUT;
      }
      if (n > 4096) __nanosleep(128);
    }
  }
  return 0;
}

/* Warp-collective Parrived / wait: all 32 lanes call it with the same
 * partition (like pc_pready_warp) and all get the result.  For an LL receive
 * the lanes poll and unpack the partition's lines together (one round trip per
 * poll for partitions up to 2 KiB of lines); otherwise lane 0 polls the flag.
 * After it returns, every lane may read the partition. */
PC_DEVICE int pc_parrived_warp(pc_prequest_t preq, int partition) {
  using namespace pc_detail;
  const uint32_t lane = lane_id();
  if (preq.kind == PC_KIND_PRECV && partition >= 0 && partition < preq.partitions) {
    const uint32_t g = *(const volatile uint32_t *)preq.layout;
    if (g & PC_LAYOUT_LL) return ll_consume_warp(preq, partition, epoch_of(preq), lane) ? 1 : 0;
  }
  int r = 0;
  if (lane == 0) r = pc_parrived(preq, partition);
  r = __shfl_sync(0xffffffffu, r, 0);
  return r;
}

PC_DEVICE int pc_wait_arrived_warp(pc_prequest_t preq, int partition) {
  using namespace pc_detail;
  const unsigned full = 0xffffffffu;
  const uint32_t lane = lane_id();
  if (preq.kind == PC_KIND_PRECV && partition >= 0 && partition < preq.partitions) {
    const uint32_t e = epoch_of(preq);
    uint32_t g = *(const volatile uint32_t *)preq.layout;
    if (g & PC_LAYOUT_LL) {
      const uint64_t t0 = globaltimer();
      uint32_t n = 0;
      while (!ll_consume_warp(preq, partition, e, lane)) {
        if ((++n & 127) == 0) {
          int stop = 0;
          if (lane == 0) {
            if (aborted(preq.err)) {
              stop = 1;
            } else if (preq.timeout_ms && globaltimer() - t0 > (uint64_t)preq.timeout_ms * 1000000ull) {
              set_error(preq.err, PC_DEV_ERR_TIMEOUT, partition);
              stop = 1;
            }
          }
          if (__shfl_sync(full, stop, 0)) return PC_DEV_ERR_TIMEOUT;
          if (n > 4096) __nanosleep(128);
        }
      }
      return 0;
    }
  }
  int r = 0;
  if (lane == 0) r = pc_wait_arrived(preq, partition);
  r = __shfl_sync(full, r, 0);
  return r;
}

#endif /* PC_DEVICE_CUH_ */
