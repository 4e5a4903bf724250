// libpcapps: application / producer kernels that USE the device bindings of
// pc_device.cuh the way a user kernel would (Listing 2).  They are
// the "compute" side of the paper's experiments:
//   vecadd       C = A + B, 8 B per thread, 1024-thread blocks, with
//                pc_pready at thread / warp / block granularity (P:L223,
//                P:L229; §VI-A)
//   (the collective producers produce / bce_grad / overlap_probe live in
//    apps_coll.cu, built with -DPC_INLINE_ALLREDUCE)
//   check_recv   receiver kernel that waits pc_parrived per partition and
//                consumes it (device Parrived)
//   pingpong     Pready->Parrived latency inside one persistent kernel per side
//   bare_pingpong  the same with raw flags and no library (latency floor)
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include "pc_device.cuh"

#define PCAPP_GRAN_NONE (-1)
#define PCAPP_GRAN_THREAD 0
#define PCAPP_GRAN_WARP 1
#define PCAPP_GRAN_BLOCK 2
#define PCAPP_GRAN_BLOCK_PUT 3  // block granularity, Kernel Copy from registers (pc_pready_block_put)

namespace {

template <int MINB, int gran>
__global__ void __launch_bounds__(1024, MINB) vecadd_kernel(const float2 *__restrict__ A, const float2 *__restrict__ B,
                                                            float2 *__restrict__ C, int64_t n2, pc_prequest_t preq) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  float2 c = make_float2(0.f, 0.f);
  if (i < n2) {
    const float2 a = A[i], b = B[i];
    c = make_float2(a.x + b.x, a.y + b.y);
    C[i] = c;
  }
  if (gran == PCAPP_GRAN_THREAD) {
    if (i < n2) pc_pready((int)i, preq);
  } else if (gran == PCAPP_GRAN_WARP) {
    pc_pready_warp((int)(i >> 5), preq);
  } else if (gran == PCAPP_GRAN_BLOCK) {
    pc_pready_block((int)blockIdx.x, preq);
  } else if (gran == PCAPP_GRAN_BLOCK_PUT) {
    pc_pready_block_put((int)blockIdx.x, preq, i < n2 ? (uint64_t)threadIdx.x : ~0ull, c);
  }
}

// The same C = A + B with the same partitions (logical block p = 1024 threads
// x 8 B, warp p*32 + w, thread i) and the same Pready calls, as a persistent
// kernel: one 1024-thread CTA per resident slot (2 per SM) walks the logical
// blocks p = blockIdx.x, + gridDim.x, ...  The operands are staged by TMA
// bulk copies (cp.async.bulk, one 8 KiB tile of A and of B per logical block)
// into a ring of kStages shared-memory stages, each completing on its own
// mbarrier, kStages - 1 logical blocks ahead — so the HBM loads overlap the
// Pready chain (barrier, push, the release thread 0 issues before the flag)
// without holding registers (a register prefetch spilled at the 32-register
// budget of 2 CTAs per SM, and the spill store waited for the load).  A warp
// arrives on the stage's "empty" mbarrier once it has read it; thread 32 (not
// thread 0, whose Pready releases: a MEMBAR issued by the thread that has
// bulk copies in flight waited for them, 305 -> xx us at 256 MiB) refills the
// stage after its own Pready.  A ragged last tile moves its 16-B-aligned part
// by TMA and the rest by plain loads.
constexpr int kStages = 4;
constexpr int kTile = 1024;  // float2 per logical block
constexpr size_t kStagedSmem = (size_t)2 * kStages * kTile * sizeof(float2) + 2 * kStages * sizeof(uint64_t);

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, uint32_t bytes) {
  asm volatile("{\n .reg .b64 st;\n mbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n}" ::"r"(smem_u32(b)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
  asm volatile("{\n .reg .b64 st;\n mbarrier.arrive.shared::cta.b64 st, [%0];\n}" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W_%=;\n}" ::"r"(
          smem_u32(b)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *b) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(b))
               : "memory");
}

template <int gran>
__global__ void __launch_bounds__(1024, 2) vecadd_persistent_kernel(const float2 *__restrict__ A,
                                                                    const float2 *__restrict__ B,
                                                                    float2 *__restrict__ C, int64_t n2,
                                                                    int64_t nblk, int batch, pc_prequest_t preq) {
  // 32-bit loop state (the launcher guarantees n2 < 2^31) and smem offsets
  // from one base: the loop carries few registers at the 32-register budget.
  extern __shared__ __align__(128) uint8_t smem[];
  constexpr uint32_t kTileBytes = kTile * sizeof(float2);
  constexpr uint32_t kFull = 2 * kStages * kTileBytes, kEmpty = kFull + kStages * 8;
  const uint32_t tid = threadIdx.x, base = smem_u32(smem);
  const int N2 = (int)n2, NB = (int)nblk, G = (int)gridDim.x;
  const int T = (NB - (int)blockIdx.x + G - 1) / G;  // logical blocks of this CTA
  constexpr uint32_t kIssuer = 32;  // the thread that issues the bulk copies
  auto bulk_bytes = [&](int p) -> uint32_t {
    const int rem = N2 - p * kTile;
    return (uint32_t)((rem < kTile ? rem : kTile) * 8) & ~15u;
  };
  auto issue = [&](int k) {  // thread kIssuer: tile k of this CTA into stage k % kStages
    const int p = (int)blockIdx.x + k * G;
    const uint32_t s = (uint32_t)(k % kStages), by = bulk_bytes(p);
    uint64_t *f = reinterpret_cast<uint64_t *>(smem + kFull) + s;
    mbar_expect_tx(f, 2 * by);
    if (by) {
      bulk_g2s(smem + s * kTileBytes, A + (int64_t)p * kTile, by, f);
      bulk_g2s(smem + (kStages + s) * kTileBytes, B + (int64_t)p * kTile, by, f);
    }
  };
  if (tid == 0) {
    for (int s = 0; s < kStages; ++s) {
      mbar_init(reinterpret_cast<uint64_t *>(smem + kFull) + s, 1);
      mbar_init(reinterpret_cast<uint64_t *>(smem + kEmpty) + s, 1024 / 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (tid == kIssuer)
    for (int k = 0; k < kStages && k < T; ++k) issue(k);
  pc_warp_state ws{0, 0};  // warp granularity: {epoch, ready-to-receive} checked once per warp
  if (gran == PCAPP_GRAN_WARP) pc_warp_begin(preq, &ws);
  pc_put_state bs{0, 0, 1, 0, -1};  // block granularity: checked once per CTA, releases batched
  if (gran == PCAPP_GRAN_BLOCK) pc_put_begin<uint8_t>(preq, &bs, batch);  // (bs.ok = 0: the plain Pready)
  for (int k = 0; k < T; ++k) {
    const int p = (int)blockIdx.x + k * G;
    const uint32_t s = (uint32_t)(k % kStages), par = (uint32_t)(k / kStages) & 1u;
    const int i = p * kTile + (int)tid;
    mbar_wait(reinterpret_cast<uint64_t *>(smem + kFull) + s, par);
    float2 c = make_float2(0.f, 0.f);
    if (8u * tid + 8u <= bulk_bytes(p)) {
      float2 a, b;
      asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(a.x), "=f"(a.y) : "r"(base + s * kTileBytes + 8u * tid));
      asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];"
                   : "=f"(b.x), "=f"(b.y)
                   : "r"(base + (kStages + s) * kTileBytes + 8u * tid));
      c = make_float2(a.x + b.x, a.y + b.y);
    } else if (i < N2) {  // ragged tail beyond the bulk copy
      const float2 a = __ldcs(A + i), b = __ldcs(B + i);
      c = make_float2(a.x + b.x, a.y + b.y);
    }
    __syncwarp();
    if ((tid & 31) == 0) mbar_arrive(reinterpret_cast<uint64_t *>(smem + kEmpty) + s);
    if (i < N2) C[i] = c;
    if (gran == PCAPP_GRAN_THREAD) {
      if (i < N2) pc_pready(i, preq);
    } else if (gran == PCAPP_GRAN_WARP) {
      pc_pready_warp(i >> 5, preq, ws);
    } else if (gran == PCAPP_GRAN_BLOCK) {
      pc_pready_block(p, preq, bs);
    }
    if (tid == kIssuer && k + kStages < T) {  // every warp has read stage s: refill it
      mbar_wait(reinterpret_cast<uint64_t *>(smem + kEmpty) + s, par);
      issue(k + kStages);
    }
  }
  if (gran == PCAPP_GRAN_BLOCK) pc_put_end(preq, bs);
}

// block_put from a persistent producer (R35): the paper's 8 KiB logical
// blocks, 1024 threads x 8 B, with pc_put_begin once per CTA and the
// register path of pc_pready_block_put per logical block — nothing out of
// line in the loop, so the operands of the NEXT logical block are prefetched
// into registers (no spill at 32 registers) and their HBM latency overlaps the
// Pready chain of this one (assign, barrier, thread 0's release + flag).
__global__ void __launch_bounds__(1024, 2) vecadd_put_persistent_kernel(const float2 *__restrict__ A,
                                                                        const float2 *__restrict__ B,
                                                                        float2 *__restrict__ C, int n2, int nblk,
                                                                        int batch, pc_prequest_t preq) {
  const int G = gridDim.x;
  int p = blockIdx.x;
  float2 a = make_float2(0.f, 0.f), b = a;
  int i = p * 1024 + (int)threadIdx.x;
  if (i < n2) {  // the first operands' HBM latency overlaps pc_put_begin's acquire
    a = __ldcs(A + i);
    b = __ldcs(B + i);
  }
  pc_put_state st;
  if (pc_put_begin<float2>(preq, &st, batch) != 0) return;  // (the launcher checked eligibility; timeout is recorded)
  for (; p < nblk; p += G, i += G * 1024) {
    const float2 c = make_float2(a.x + b.x, a.y + b.y);
    const int in = i + G * 1024;
    if (in < n2) {
      a = __ldcs(A + in);
      b = __ldcs(B + in);
    }
    if (i < n2) C[i] = c;
    pc_pready_block_put(p, preq, i < n2 ? (uint64_t)threadIdx.x : ~0ull, c, st);
  }
  pc_put_end(preq, st);
}

// pc_pready_block_put with 4-, 8- or 16-byte elements (test producer): each
// CTA copies its partitions src -> send buffer (one element of type T per
// thread, partition bytes <= blockDim * sizeof(T)) and hands the element it
// holds to pc_pready_block_put; partitions whose size or alignment does not
// suit T take the library's pc_pready_block fallback.
template <typename T>
__global__ void produce_put_kernel(uint8_t *__restrict__ dst, const uint8_t *__restrict__ src, int partitions,
                                   int64_t part_bytes, pc_prequest_t preq) {
  const uint64_t ne = (uint64_t)part_bytes / sizeof(T), tail = (uint64_t)part_bytes % sizeof(T);
  for (int p = blockIdx.x; p < partitions; p += gridDim.x) {
    const uint64_t off = (uint64_t)p * part_bytes;
    T v{};
    const bool mine = threadIdx.x < ne;
    if (mine) {
      memcpy(&v, src + off + (uint64_t)threadIdx.x * sizeof(T), sizeof(T));
      memcpy(dst + off + (uint64_t)threadIdx.x * sizeof(T), &v, sizeof(T));
    }
    if (threadIdx.x < tail) dst[off + ne * sizeof(T) + threadIdx.x] = src[off + ne * sizeof(T) + threadIdx.x];
    pc_pready_block_put(p, preq, mine ? (uint64_t)threadIdx.x : ~0ull, v);
  }
}

// Bare NVLink peer-copy floor (SURVEY §8(d) "Rooflines"): no
// library, no flags — n concurrent copies of `bytes` each (blockIdx.y = copy),
// 16-B vectors, 4 in flight per thread.  dst (push) or src (pull) is a
// peer-mapped address; the bench times every rank writing to / reading from
// its peers at once, the traffic pattern of the DIRECT schedule.
struct PeerCopyArgs {
  int n;
  uint64_t bytes;
  const uint8_t *src[8];
  uint8_t *dst[8];
};
__global__ void __launch_bounds__(512) peer_copy_kernel(PeerCopyArgs a) {
  const int j = blockIdx.y;
  const uint4 *s = reinterpret_cast<const uint4 *>(a.src[j]);
  uint4 *d = reinterpret_cast<uint4 *>(a.dst[j]);
  const uint64_t nv = a.bytes / 16, stride = (uint64_t)gridDim.x * blockDim.x;
  uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; k + 3 * stride < nv; k += 4 * stride) {
    const uint4 v0 = s[k], v1 = s[k + stride], v2 = s[k + 2 * stride], v3 = s[k + 3 * stride];
    d[k] = v0;
    d[k + stride] = v1;
    d[k + 2 * stride] = v2;
    d[k + 3 * stride] = v3;
  }
  for (; k < nv; k += stride) d[k] = s[k];
}

// Fig 3 analogue: ONE block of t threads computes C = A + B (8 B per
// thread) and marks it ready at thread / warp / block granularity; thread 0
// records %globaltimer around the Pready calls (after a block barrier on both
// sides), i.e. the cost of the block's Pready set including the INLINE copy,
// fences and flag stores.  Warp granularity needs t % 32 == 0.
__global__ void __launch_bounds__(1024) pready_cost_kernel(const float2 *__restrict__ A, const float2 *__restrict__ B,
                                   float2 *__restrict__ C, int gran, pc_prequest_t preq,
                                   unsigned long long *out_ns) {
  const int i = threadIdx.x;
  C[i] = make_float2(A[i].x + B[i].x, A[i].y + B[i].y);
  __syncthreads();
  unsigned long long t0 = 0;
  if (i == 0) t0 = pc_detail::globaltimer();
  __syncthreads();
  if (gran == PCAPP_GRAN_THREAD)
    pc_pready(i, preq);
  else if (gran == PCAPP_GRAN_WARP)
    pc_pready_warp(i >> 5, preq);
  else
    pc_pready_block(0, preq);
  __syncthreads();
  if (i == 0) *out_ns = pc_detail::globaltimer() - t0;
}

__global__ void check_recv_kernel(pc_prequest_t preq, const uint8_t *recvbuf, uint8_t *out, int partitions,
                                  int64_t part_bytes, int *status) {
  __shared__ int ok;
  for (int p = blockIdx.x; p < partitions; p += gridDim.x) {
    if (threadIdx.x == 0) ok = pc_wait_arrived(preq, p) == 0;
    __syncthreads();
    if (!ok) {
      if (threadIdx.x == 0) atomicAdd(status, 1);
      return;
    }
    const int64_t off = (int64_t)p * part_bytes;
    for (int64_t j = threadIdx.x; j < part_bytes; j += blockDim.x) out[off + j] = __ldcg(recvbuf + off + j);
    __syncthreads();
  }
}

// Ping-pong: side 0 readies partition k of its send request and waits for
// partition k of its receive request; side 1 mirrors.  One warp per side.
// Partition k is used once per epoch (MPI rule).  out_ns[0] = total ns on
// side 0 for `iters` round trips.
__global__ void pingpong_kernel(pc_prequest_t sendq, pc_prequest_t recvq, int side, int iters, int gran,
                                unsigned long long *out_ns) {
  pc_warp_state ws{0, 0};
  if (gran != PCAPP_GRAN_THREAD) pc_warp_begin(sendq, &ws);  // (st.ok = 0: the plain Pready)
  const uint64_t t0 = pc_detail::globaltimer();
  for (int k = 0; k < iters; ++k) {
    if (side == 1) {
      if (threadIdx.x == 0) pc_wait_arrived(recvq, k);
      __syncwarp();
    }
    if (gran == PCAPP_GRAN_THREAD) {
      if (threadIdx.x == 0) pc_pready(k, sendq);
    } else {
      pc_pready_warp(k, sendq, ws);
    }
    if (side == 0) {
      if (threadIdx.x == 0) pc_wait_arrived(recvq, k);
      __syncwarp();
    }
  }
  if (threadIdx.x == 0) out_ns[0] = pc_detail::globaltimer() - t0;
}

// Both sides in ONE launch (block 0 = side 0, block 1 = side 1): for virtual
// ranks sharing a GPU, so the two spinning sides are co-resident by
// construction.
__global__ void pingpong_pair_kernel(pc_prequest_t sendA, pc_prequest_t recvA, pc_prequest_t sendB,
                                     pc_prequest_t recvB, int iters, int gran, unsigned long long *out_ns,
                                     unsigned long long *rt_ns) {
  const int side = blockIdx.x;
  const pc_prequest_t &sq = side ? sendB : sendA;
  const pc_prequest_t &rq = side ? recvB : recvA;
  // warp granularity: {epoch, ready-to-receive} checked once per warp (the
  // receiver's Pbuf_prepare preceded this launch), then warp-collective
  // Pready and wait; thread: lane 0 alone
  pc_warp_state ws{0, 0};
  if (gran != PCAPP_GRAN_THREAD) pc_warp_begin(sq, &ws);  // (st.ok = 0: the plain Pready)
  const uint64_t t0 = pc_detail::globaltimer();
  uint64_t tk = t0;
  for (int k = 0; k < iters; ++k) {
    if (side == 1) {
      if (gran == PCAPP_GRAN_THREAD) {
        if (threadIdx.x == 0) pc_wait_arrived(rq, k);
      } else {
        pc_wait_arrived_warp(rq, k);
      }
      __syncwarp();
    }
    if (gran == PCAPP_GRAN_THREAD) {
      if (threadIdx.x == 0) pc_pready(k, sq);
    } else {
      pc_pready_warp(k, sq, ws);
    }
    if (side == 0) {
      if (gran == PCAPP_GRAN_THREAD) {
        if (threadIdx.x == 0) pc_wait_arrived(rq, k);
      } else {
        pc_wait_arrived_warp(rq, k);
      }
      if (threadIdx.x == 0) {
        const uint64_t t = pc_detail::globaltimer();
        if (rt_ns) rt_ns[k] = t - tk;  // one round trip = two Pready->Parrived hops
        tk = t;
      }
      __syncwarp();
    }
  }
  if (threadIdx.x == 0) out_ns[side] = pc_detail::globaltimer() - t0;
}

// The latency floor: the same ping-pong with two bare flags and no library.
// scope 0: relaxed GPU-scope loads/stores (the hardware floor for ranks that
// share a GPU), 1: release/acquire at GPU scope, 2: release/acquire at system
// scope (what a flag to another GPU costs).
__device__ __forceinline__ uint32_t bare_ld(const uint32_t *p, int scope) {
  uint32_t v;
  if (scope == 0)
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  else if (scope == 1)
    v = pc_detail::ld_acquire_gpu(p);
  else
    v = pc_detail::ld_acquire_sys(p);
  return v;
}
__device__ __forceinline__ void bare_st(uint32_t *p, uint32_t v, int scope) {
  if (scope == 0)
    pc_detail::st_relaxed_gpu(p, v);
  else if (scope == 1)
    pc_detail::st_release_gpu(p, v);
  else
    pc_detail::st_release_sys(p, v);
}

__global__ void bare_pingpong_pair_kernel(uint32_t *flagA, uint32_t *flagB, int iters, uint32_t base,
                                          unsigned long long *out_ns, int scope) {
  if (threadIdx.x != 0) return;
  const int side = blockIdx.x;
  uint32_t *mine = side ? flagB : flagA;
  uint32_t *peer = side ? flagA : flagB;
  const uint64_t t0 = pc_detail::globaltimer();
  for (int k = 1; k <= iters; ++k) {
    const uint32_t v = base + (uint32_t)k;
    if (side == 1)
      while (!pc_detail::reached(bare_ld(mine, scope), v)) {
      }
    bare_st(peer, v, scope);
    if (side == 0)
      while (!pc_detail::reached(bare_ld(mine, scope), v)) {
      }
  }
  out_ns[side] = pc_detail::globaltimer() - t0;
}


// Latency decomposition probe (tools/lat_probe.py): the pair ping-pong with
// the library wait and/or Pready replaced by raw flag operations.
//   WLIB: pc_wait_arrived (1) or a relaxed poll of flags[k] (0)
//   PLIB: pc_pready_warp (1), pc_pready by lane 0 (2), or raw: copy the
//         payload, fence at the request scope, store the peer flag (0)
template <int WLIB, int PLIB>
__global__ void lat_probe_pair_kernel(pc_prequest_t sendA, pc_prequest_t recvA, pc_prequest_t sendB,
                                      pc_prequest_t recvB, int iters, unsigned long long *out_ns) {
  const int side = blockIdx.x;
  const pc_prequest_t &sq = side ? sendB : sendA;
  const pc_prequest_t &rq = side ? recvB : recvA;
  const uint32_t e = pc_detail::epoch_of(sq);
  auto wait = [&](int k) {
    if (WLIB == 2) {
      pc_wait_arrived_warp(rq, k);
    } else if (threadIdx.x == 0) {
      if (WLIB) {
        pc_wait_arrived(rq, k);
      } else {
        while (!pc_detail::reached(pc_detail::ld_relaxed_sys(rq.flags + k), e)) {
        }
        if (rq.part_bytes) pc_detail::fence_gpu();
      }
    }
    __syncwarp();
  };
  auto ready = [&](int k) {
    if (PLIB == 1) {
      pc_pready_warp(k, sq);
    } else if (PLIB == 2) {
      if (threadIdx.x == 0) pc_pready(k, sq);
      __syncwarp();
    } else if (PLIB == 3) {  // lane 0: epoch_rtr + publish, no shuffles
      __syncwarp();
      if (threadIdx.x == 0) {
        const uint2 er = pc_detail::epoch_rtr(sq);
        pc_detail::publish(sq, k / sq.agg, 1, er.x, k);
      }
      __syncwarp();
    } else if (PLIB == 4) {  // + broadcast of e
      __syncwarp();
      uint32_t ee = 0;
      if (threadIdx.x == 0) ee = pc_detail::epoch_rtr(sq).x;
      ee = __shfl_sync(0xffffffffu, ee, 0);
      if (threadIdx.x == 0) pc_detail::publish(sq, k / sq.agg, 1, ee, k);
      __syncwarp();
    } else if (PLIB >= 10) {  // lane 0: epoch load variant + publish
      __syncwarp();
      if (threadIdx.x == 0) {
        uint32_t ee;
        if (PLIB == 10) ee = pc_detail::ld_acquire_gpu(sq.epoch);
        else if (PLIB == 11) ee = pc_detail::ld_acquire_sys(sq.epoch);
        else if (PLIB == 12) asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(ee) : "l"(sq.epoch) : "memory");
        else if (PLIB == 13) ee = pc_detail::ld_acquire_sys_v2(sq.epoch).x;
        else ee = pc_detail::ld_acquire_gpu_v2(sq.epoch).x;
        pc_detail::publish(sq, k / sq.agg, 1, ee, k);
      }
      __syncwarp();
    } else if (PLIB == 5) {  // relaxed epoch read by lane 0 + publish
      __syncwarp();
      if (threadIdx.x == 0) pc_detail::publish(sq, k / sq.agg, 1, pc_detail::ld_relaxed_sys(sq.epoch), k);
      __syncwarp();
    } else {
      if (sq.part_bytes) {
        const uint64_t off = (uint64_t)k * sq.part_bytes;
        pc_detail::copy_bytes(sq.peer_rbuf + off, sq.sbuf + off, sq.part_bytes, threadIdx.x, 32);
        pc_detail::fence_gpu();
        __syncwarp();
      }
      if (threadIdx.x == 0) {
        pc_detail::st_relaxed_sys(sq.peer_flags + k, e);
        pc_detail::st_relaxed_gpu(sq.sent + k, e);
      }
      __syncwarp();
    }
  };
  const uint64_t t0 = pc_detail::globaltimer();
  long long c_ready = 0, c_wait = 0;
  for (int k = 0; k < iters; ++k) {
    const long long c0 = clock64();
    if (side == 1) wait(k);
    const long long c1 = clock64();
    ready(k);
    const long long c2 = clock64();
    if (side == 0) wait(k);
    c_wait += c1 - c0;
    c_ready += c2 - c1;
  }
  if (threadIdx.x == 0) {
    out_ns[side] = pc_detail::globaltimer() - t0;
    out_ns[2 + 2 * side] = (unsigned long long)c_ready;  // SM cycles inside Pready
    out_ns[3 + 2 * side] = (unsigned long long)c_wait;   // SM cycles inside the side-1 wait
  }
}

// Flag ping-pong microbenchmark over memory-order variants (latency floor
// study): 0 st.release.sys/ld.acquire.sys, 1 relaxed.sys,
// 2 release/acquire.gpu, 3 relaxed.gpu, 4 fence.acq_rel.sys+st.relaxed.sys /
// ld.acquire.sys, 5 volatile.
template <int V>
__device__ __forceinline__ void vstore(uint32_t *p, uint32_t v) {
  if (V == 0) asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
  if (V == 1) asm volatile("st.relaxed.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
  if (V == 2) asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
  if (V == 3) asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
  if (V == 4) asm volatile("fence.acq_rel.sys;\n\tst.relaxed.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
  if (V == 5) asm volatile("st.volatile.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
template <int V>
__device__ __forceinline__ uint32_t vload(const uint32_t *p) {
  uint32_t v;
  if (V == 0 || V == 4) asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  if (V == 1) asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  if (V == 2) asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  if (V == 3) asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  if (V == 5) asm volatile("ld.volatile.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
template <int V>
__global__ void flag_variant_kernel(uint32_t *flagA, uint32_t *flagB, int iters, uint32_t base,
                                    unsigned long long *out_ns) {
  if (threadIdx.x != 0) return;
  const int side = blockIdx.x;
  uint32_t *mine = side ? flagB : flagA;
  uint32_t *peer = side ? flagA : flagB;
  const uint64_t t0 = pc_detail::globaltimer();
  for (int k = 1; k <= iters; ++k) {
    const uint32_t v = base + (uint32_t)k;
    if (side == 1)
      while (!pc_detail::reached(vload<V>(mine), v)) {
      }
    vstore<V>(peer, v);
    if (side == 0)
      while (!pc_detail::reached(vload<V>(mine), v)) {
      }
  }
  out_ns[side] = pc_detail::globaltimer() - t0;
}

// Latency floor: the same ping-pong with a bare flag and no library.
__global__ void bare_pingpong_kernel(uint32_t *my_flag, uint32_t *peer_flag, int side, int iters, uint32_t base,
                                     unsigned long long *out_ns) {
  if (threadIdx.x != 0) return;
  const uint64_t t0 = pc_detail::globaltimer();
  for (int k = 1; k <= iters; ++k) {
    const uint32_t v = base + (uint32_t)k;
    if (side == 1)
      while (!pc_detail::reached(pc_detail::ld_acquire_sys(my_flag), v)) {
      }
    pc_detail::st_release_sys(peer_flag, v);
    if (side == 0)
      while (!pc_detail::reached(pc_detail::ld_acquire_sys(my_flag), v)) {
      }
  }
  out_ns[0] = pc_detail::globaltimer() - t0;
}

}  // namespace

// Resident 1024-thread vecadd CTAs per SM the launch asks ptxas for (1: up to
// 64 registers per thread; 2: 32).  PCAPP_VECADD_MINB=1|2, default 2.
int minb() {
  static int v = 0;
  if (!v) {
    const char *e = getenv("PCAPP_VECADD_MINB");
    v = (e && e[0] == '1') ? 1 : 2;
  }
  return v;
}

// One instantiation per (CTAs per SM, granularity): a launch carries only the
// Pready path it calls, so the 32-register budget of 2 CTAs per SM is spent on
// that path alone.
using VecaddFn = void (*)(const float2 *, const float2 *, float2 *, int64_t, pc_prequest_t);
using VecaddPersFn = void (*)(const float2 *, const float2 *, float2 *, int64_t, int64_t, int, pc_prequest_t);
template <int MINB>
VecaddFn vecadd_fn(int gran) {
  switch (gran) {
    case PCAPP_GRAN_THREAD: return vecadd_kernel<MINB, PCAPP_GRAN_THREAD>;
    case PCAPP_GRAN_WARP: return vecadd_kernel<MINB, PCAPP_GRAN_WARP>;
    case PCAPP_GRAN_BLOCK: return vecadd_kernel<MINB, PCAPP_GRAN_BLOCK>;
    case PCAPP_GRAN_BLOCK_PUT: return vecadd_kernel<MINB, PCAPP_GRAN_BLOCK_PUT>;
    default: return vecadd_kernel<MINB, PCAPP_GRAN_NONE>;
  }
}
VecaddPersFn vecadd_pers_fn(int gran) {
  switch (gran) {
    case PCAPP_GRAN_THREAD: return vecadd_persistent_kernel<PCAPP_GRAN_THREAD>;
    case PCAPP_GRAN_WARP: return vecadd_persistent_kernel<PCAPP_GRAN_WARP>;
    case PCAPP_GRAN_BLOCK: return vecadd_persistent_kernel<PCAPP_GRAN_BLOCK>;
    default: return vecadd_persistent_kernel<PCAPP_GRAN_NONE>;
  }
}

// Logical blocks per release of the persistent register Kernel Copy producer
// (pc_put_begin batch; PCAPP_PUT_BATCH=1..32, default 4).
int put_batch() {  // (read at every launch: tests vary it)
  const char *e = getenv("PCAPP_PUT_BATCH");
  int v = e ? atoi(e) : 4;
  return v < 1 ? 1 : (v > 32 ? 32 : v);
}

extern "C" {

int pcapp_vecadd(const float *A, const float *B, float *C, int64_t n, int gran, const pc_prequest_t *preq,
                 cudaStream_t s) {
  if (n % 2 || gran < PCAPP_GRAN_NONE || gran > PCAPP_GRAN_BLOCK_PUT) return -1;
  const int64_t n2 = n / 2;
  const int64_t blocks = (n2 + 1023) / 1024;
  pc_prequest_t q{};
  if (preq) q = *preq;
  if (gran != PCAPP_GRAN_NONE && !preq) return -1;
  if (blocks < 1) return 0;
  const VecaddFn f = minb() == 2 ? vecadd_fn<2>(gran) : vecadd_fn<1>(gran);
  f<<<(unsigned)blocks, 1024, 0, s>>>((const float2 *)A, (const float2 *)B, (float2 *)C, n2, q);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_vecadd_persistent(const float *A, const float *B, float *C, int64_t n, int gran, const pc_prequest_t *preq,
                            cudaStream_t s) {
  if (n % 2 || gran < PCAPP_GRAN_NONE || gran > PCAPP_GRAN_BLOCK_PUT) return -1;
  if ((reinterpret_cast<uintptr_t>(A) | reinterpret_cast<uintptr_t>(B)) & 15) return -1;  // TMA: 16-B sources
  const int64_t n2 = n / 2;
  if (n2 + kTile >= (1ll << 31)) return -1;  // 32-bit element indices
  const int64_t nblk = (n2 + kTile - 1) / kTile;
  pc_prequest_t q{};
  if (preq) q = *preq;
  if (gran != PCAPP_GRAN_NONE && !preq) return -1;
  if (nblk < 1) return 0;
  const bool put_ok = q.kind != PC_KIND_PALLREDUCE && q.copy == 0 && q.part_bytes != 0 &&
                      ((reinterpret_cast<uintptr_t>(q.peer_rbuf) | q.part_bytes) & 7) == 0;
  if (gran == PCAPP_GRAN_BLOCK_PUT && put_ok) {
    int dev = 0, sms = 0, per = 0;
    if (cudaGetDevice(&dev) != cudaSuccess ||
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess ||
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, vecadd_put_persistent_kernel, 1024, 0) != cudaSuccess ||
        per < 1)
      return -2;
    const int64_t grid = nblk < (int64_t)sms * per ? nblk : (int64_t)sms * per;
    vecadd_put_persistent_kernel<<<(unsigned)grid, 1024, 0, s>>>((const float2 *)A, (const float2 *)B, (float2 *)C,
                                                                 (int)n2, (int)nblk, put_batch(), q);
    return cudaGetLastError() == cudaSuccess ? 0 : -2;
  }
  if (gran == PCAPP_GRAN_BLOCK_PUT) gran = PCAPP_GRAN_BLOCK;  // same partitions: the send buffer holds the data
  const VecaddPersFn f = vecadd_pers_fn(gran);
  int dev = 0, sms = 0, per = 0;  // resident 1024-thread CTAs of this instantiation
  if (cudaGetDevice(&dev) != cudaSuccess ||
      cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess ||
      cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kStagedSmem) != cudaSuccess ||
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, f, 1024, kStagedSmem) != cudaSuccess || per < 1)
    return -2;
  int64_t slots = (int64_t)sms * per;
  // ENGINE copy: the library's engine runs beside the producer on up to half
  // of the SMs (PC_OVERLAP_FRAC); a persistent grid over every slot would make
  // it wait for the producer's CTAs to retire, so leave it that half.
  if (preq && q.copy == 1 && slots > 1) slots /= 2;
  const int64_t grid = nblk < slots ? nblk : slots;
  f<<<(unsigned)grid, 1024, kStagedSmem, s>>>((const float2 *)A, (const float2 *)B, (float2 *)C, n2, nblk,
                                              put_batch(), q);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_produce_put(void *dst, const void *src, int partitions, int64_t part_bytes, int elem_bytes, int threads,
                      int blocks, const pc_prequest_t *preq, cudaStream_t s) {
  if (!preq || partitions < 1 || threads < 32 || threads > 1024 || part_bytes < 1) return -1;
  if ((uint64_t)part_bytes > (uint64_t)threads * (uint64_t)elem_bytes) return -1;  // one element per thread
  if (blocks <= 0) blocks = partitions < 592 ? partitions : 592;
  const pc_prequest_t q = *preq;
  uint8_t *d = (uint8_t *)dst;
  const uint8_t *sr = (const uint8_t *)src;
  switch (elem_bytes) {
    case 4: produce_put_kernel<uint32_t><<<blocks, threads, 0, s>>>(d, sr, partitions, part_bytes, q); break;
    case 8: produce_put_kernel<uint2><<<blocks, threads, 0, s>>>(d, sr, partitions, part_bytes, q); break;
    case 16: produce_put_kernel<uint4><<<blocks, threads, 0, s>>>(d, sr, partitions, part_bytes, q); break;
    default: return -1;
  }
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_pready_cost(const float *A, const float *B, float *C, int threads, int gran, const pc_prequest_t *preq,
                      unsigned long long *out_ns, cudaStream_t s) {
  if (threads < 1 || threads > 1024 || !preq || (gran == PCAPP_GRAN_WARP && threads % 32)) return -1;
  pready_cost_kernel<<<1, threads, 0, s>>>((const float2 *)A, (const float2 *)B, (float2 *)C, gran, *preq, out_ns);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_check_recv(const pc_prequest_t *preq, const void *recvbuf, void *out, int partitions, int64_t part_bytes,
                     int blocks, int *status, cudaStream_t s) {
  if (!preq) return -1;
  check_recv_kernel<<<blocks, 256, 0, s>>>(*preq, (const uint8_t *)recvbuf, (uint8_t *)out, partitions, part_bytes,
                                           status);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_pingpong(const pc_prequest_t *sendq, const pc_prequest_t *recvq, int side, int iters, int gran,
                   unsigned long long *out_ns, cudaStream_t s) {
  if (!sendq || !recvq) return -1;
  pingpong_kernel<<<1, 32, 0, s>>>(*sendq, *recvq, side, iters, gran, out_ns);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_bare_pingpong(uint32_t *my_flag, uint32_t *peer_flag, int side, int iters, uint32_t base,
                        unsigned long long *out_ns, cudaStream_t s) {
  bare_pingpong_kernel<<<1, 32, 0, s>>>(my_flag, peer_flag, side, iters, base, out_ns);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_pingpong_pair(const pc_prequest_t *sendA, const pc_prequest_t *recvA, const pc_prequest_t *sendB,
                        const pc_prequest_t *recvB, int iters, int gran, unsigned long long *out_ns,
                        unsigned long long *rt_ns, cudaStream_t s) {
  if (!sendA || !recvA || !sendB || !recvB) return -1;
  pingpong_pair_kernel<<<2, 32, 0, s>>>(*sendA, *recvA, *sendB, *recvB, iters, gran, out_ns, rt_ns);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_bare_pingpong_pair(uint32_t *flagA, uint32_t *flagB, int iters, uint32_t base, unsigned long long *out_ns,
                             int scope,
                             cudaStream_t s) {
  bare_pingpong_pair_kernel<<<2, 32, 0, s>>>(flagA, flagB, iters, base, out_ns, scope);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_flag_variant(uint32_t *flagA, uint32_t *flagB, int variant, int iters, uint32_t base,
                       unsigned long long *out_ns, cudaStream_t s) {
  switch (variant) {
    case 0: flag_variant_kernel<0><<<2, 32, 0, s>>>(flagA, flagB, iters, base, out_ns); break;
    case 1: flag_variant_kernel<1><<<2, 32, 0, s>>>(flagA, flagB, iters, base, out_ns); break;
    case 2: flag_variant_kernel<2><<<2, 32, 0, s>>>(flagA, flagB, iters, base, out_ns); break;
    case 3: flag_variant_kernel<3><<<2, 32, 0, s>>>(flagA, flagB, iters, base, out_ns); break;
    case 4: flag_variant_kernel<4><<<2, 32, 0, s>>>(flagA, flagB, iters, base, out_ns); break;
    default: flag_variant_kernel<5><<<2, 32, 0, s>>>(flagA, flagB, iters, base, out_ns); break;
  }
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}


int pcapp_lat_probe_pair(const pc_prequest_t *sendA, const pc_prequest_t *recvA, const pc_prequest_t *sendB,
                         const pc_prequest_t *recvB, int mode, int iters, unsigned long long *out_ns, cudaStream_t s) {
  if (!sendA || !recvA || !sendB || !recvB) return -1;
#define PCAPP_LP(W, P_) lat_probe_pair_kernel<W, P_><<<2, 32, 0, s>>>(*sendA, *recvA, *sendB, *recvB, iters, out_ns)
  switch (mode) {
    case 0: PCAPP_LP(1, 1); break;
    case 1: PCAPP_LP(0, 1); break;
    case 2: PCAPP_LP(1, 0); break;
    case 3: PCAPP_LP(0, 0); break;
    case 4: PCAPP_LP(1, 2); break;
    case 5: PCAPP_LP(0, 2); break;
    case 6: PCAPP_LP(1, 3); break;
    case 7: PCAPP_LP(1, 4); break;
    case 8: PCAPP_LP(1, 5); break;
    case 9: PCAPP_LP(2, 1); break;
    case 10: PCAPP_LP(1, 10); break;
    case 11: PCAPP_LP(1, 11); break;
    case 12: PCAPP_LP(1, 12); break;
    case 13: PCAPP_LP(1, 13); break;
    default: PCAPP_LP(1, 14); break;
  }
#undef PCAPP_LP
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_peer_copy(int n, const void *const *src, void *const *dst, uint64_t bytes, int blocks, cudaStream_t s) {
  if (n < 1 || n > 8 || (bytes & 15)) return -1;
  PeerCopyArgs a{};
  a.n = n;
  a.bytes = bytes;
  for (int j = 0; j < n; ++j) {
    a.src[j] = (const uint8_t *)src[j];
    a.dst[j] = (uint8_t *)dst[j];
  }
  if (blocks <= 0) blocks = 148 * 4 / n > 0 ? 148 * 4 / n : 1;
  peer_copy_kernel<<<dim3(blocks, n), 512, 0, s>>>(a);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

// cudaMemcpyAsync (cudaMemcpyDefault: peer-mapped destinations included) —
// the copy of the traditional model (Listing 1) in the bench's N > 1 legs.
int pcapp_memcpy_async(void *dst, const void *src, uint64_t bytes, cudaStream_t s) {
  return cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDefault, s) == cudaSuccess ? 0 : -2;
}

size_t pcapp_prequest_size(void) { return sizeof(pc_prequest_t); }

}  // extern "C"
