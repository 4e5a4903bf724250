// libpcapps, collective producers: the application kernels that Pready into
// partitioned COLLECTIVES (allreduce & co).  Built with -DPC_INLINE_ALLREDUCE
// so their Pready bindings carry the INLINE allreduce fold (reading R33); the
// p2p producers in apps.cu do not pay its registers.
//   produce        copy a prepared input into the send buffer partition by
//                  partition and Pready each one (allreduce producer, §VI-B)
//   bce_grad       DL proxy (§VI-D2; reading R28): gradient of the
//                  mean binary cross-entropy w.r.t. the predictions, one
//                  partition per block, pc_pready_block into a partitioned
//                  allreduce as soon as the partition's gradient is stored
//   overlap_probe  a6 concurrency probe (Pready(0), in-kernel Parrived(0), rest)
#ifndef PC_INLINE_ALLREDUCE
#error "apps_coll.cu is built with -DPC_INLINE_ALLREDUCE"
#endif
#include <cuda_runtime.h>
#include <stdint.h>

#include "pc_device.cuh"

#define PCAPP_GRAN_THREAD 0
#define PCAPP_GRAN_WARP 1
#define PCAPP_GRAN_BLOCK 2

namespace {

// Each block produces partitions p = blockIdx.x, +gridDim.x, ...: copies
// src -> dst for the partition, then marks it ready.
__global__ void __launch_bounds__(512) produce_kernel(uint8_t *__restrict__ dst, const uint8_t *__restrict__ src,
                                                     int partitions, int64_t part_bytes, int gran, int order_stride,
                                                     pc_prequest_t preq) {
  for (int k = blockIdx.x; k < partitions; k += gridDim.x) {
    // a permuted production order (order_stride coprime with partitions)
    const int p = (int)(((int64_t)k * order_stride) % partitions);
    const int64_t off = (int64_t)p * part_bytes;
    const uint4 *s4 = reinterpret_cast<const uint4 *>(src + off);
    uint4 *d4 = reinterpret_cast<uint4 *>(dst + off);
    const int64_t nv = ((((uintptr_t)(src + off)) | ((uintptr_t)(dst + off))) & 15) ? 0 : part_bytes / 16;
    for (int64_t j = threadIdx.x; j < nv; j += blockDim.x) d4[j] = s4[j];
    for (int64_t j = nv * 16 + threadIdx.x; j < part_bytes; j += blockDim.x) dst[off + j] = src[off + j];
    if (gran == PCAPP_GRAN_BLOCK) {
      pc_pready_block(p, preq);
    } else if (gran == PCAPP_GRAN_WARP) {
      __syncthreads();
      if (threadIdx.x < 32) pc_pready_warp(p, preq);
    } else {
      __syncthreads();
      if (threadIdx.x == 0) {
        __threadfence();
        pc_pready(p, preq);
      }
    }
  }
}

// Overlap probe (§8(a) a6, "each partition independently executes that
// schedule"): one block Preadies partition 0 of a partitioned collective, then
// (thread 0) spins until the collective reports partition 0 complete on this
// rank (device pc_parrived, at most spin_ms), then Preadies partitions 1.. and
// exits.  Partition 0 can only complete while this kernel is still running if
// the engine runs concurrently with it.  out[0..3] = %globaltimer at entry,
// after Pready(0), when Parrived(0) was seen (0 = never, timed out), at exit.
// Block b is rank b's producer (one launch for all co-located ranks, so the P
// spinning producers are co-resident by construction: separate launches on P
// streams may share a hardware queue and run one after another).
struct ProbeArgs {
  int n;
  pc_prequest_t q[8];
};
__global__ void overlap_probe_kernel(ProbeArgs a, int partitions, uint32_t spin_ms, unsigned long long *out_all) {
  const pc_prequest_t &preq = a.q[blockIdx.x];
  unsigned long long *out = out_all + 4 * blockIdx.x;
  __shared__ int s_arrived;
  if (threadIdx.x == 0) out[0] = pc_detail::globaltimer();
  pc_pready_block(0, preq);
  if (threadIdx.x == 0) {
    const unsigned long long t1 = pc_detail::globaltimer();
    out[1] = t1;
    int arrived = 0;
    for (;;) {
      if (pc_parrived(preq, 0)) {
        arrived = 1;
        break;
      }
      if (pc_detail::globaltimer() - t1 > (unsigned long long)spin_ms * 1000000ull) break;
      __nanosleep(200);
    }
    out[2] = arrived ? pc_detail::globaltimer() : 0ull;
    s_arrived = arrived;
  }
  __syncthreads();
  for (int p = 1; p < partitions; ++p) pc_pready_block(p, preq);
  __syncthreads();
  if (threadIdx.x == 0) out[3] = pc_detail::globaltimer();
}

// R28: g = (p - y) / ((p * (1 - p)) * n), five IEEE fp32 ops in this order
// (explicit _rn intrinsics: no contraction, IEEE division).
__device__ __forceinline__ float bce_g(float p, float y, float nf) {
  return __fdiv_rn(__fsub_rn(p, y), __fmul_rn(__fmul_rn(p, __fsub_rn(1.0f, p)), nf));
}

// Each block produces partitions k = blockIdx.x, +gridDim.x, ... in the order
// p = k * order_stride mod partitions; then Preadies it (block granularity).
// use_pready = 0: the plain kernel (the serialized baseline's producer).
__global__ void __launch_bounds__(512) bce_grad_kernel(const float *__restrict__ P, const float *__restrict__ Y,
                                                      float *__restrict__ G, int partitions, int64_t L, float nf,
                                                      int order_stride, int use_pready, pc_prequest_t preq) {
  for (int k = blockIdx.x; k < partitions; k += gridDim.x) {
    const int u = (int)(((int64_t)k * order_stride) % partitions);
    const int64_t off = (int64_t)u * L;
    const float *p = P + off, *y = Y + off;
    float *g = G + off;
    const bool vec = ((((uintptr_t)p) | ((uintptr_t)y) | ((uintptr_t)g)) & 15) == 0;
    const int64_t nv = vec ? L / 4 : 0;
    const float4 *p4 = reinterpret_cast<const float4 *>(p), *y4 = reinterpret_cast<const float4 *>(y);
    float4 *g4 = reinterpret_cast<float4 *>(g);
#pragma unroll 4
    for (int64_t j = threadIdx.x; j < nv; j += blockDim.x) {
      const float4 a = __ldcs(p4 + j), b = __ldcs(y4 + j);
      g4[j] = make_float4(bce_g(a.x, b.x, nf), bce_g(a.y, b.y, nf), bce_g(a.z, b.z, nf), bce_g(a.w, b.w, nf));
    }
    for (int64_t j = nv * 4 + threadIdx.x; j < L; j += blockDim.x) g[j] = bce_g(p[j], y[j], nf);
    if (use_pready) {
      pc_pready_block(u, preq);
    }
  }
}

// The DL proxy's producers of ALL co-located ranks in one launch, unit k =
// (partition u = k / P, rank r = k % P): the P blocks producing partition u
// run side by side, so the Pready that completes u (INLINE, R33) folds P
// gradient partitions that were just written and still sit in L2 instead of
// re-reading them from HBM (one launch also makes the ranks' blocks
// co-resident by construction).  Per rank the same arithmetic and the same
// Pready as bce_grad_kernel.
struct BceMultiArgs {
  int n;
  const float *p[8];
  const float *y[8];
  float *g[8];
  pc_prequest_t q[8];
};
__global__ void __launch_bounds__(512) bce_grad_multi_kernel(BceMultiArgs a, int partitions, int64_t L, float nf,
                                                            int use_pready) {
  // use_pready: 0 none, 1 pc_pready_block, 2 pc_pready_block_coop (R36)
  const int P = a.n;
  const int64_t units = (int64_t)partitions * P;
  for (int64_t k = blockIdx.x; k < units; k += gridDim.x) {
    const int u = (int)(k / P), r = (int)(k % P);
    const int64_t off = (int64_t)u * L;
    const float *p = a.p[r] + off, *y = a.y[r] + off;
    float *g = a.g[r] + off;
    const bool vec = ((((uintptr_t)p) | ((uintptr_t)y) | ((uintptr_t)g)) & 15) == 0;
    const int64_t nv = vec ? L / 4 : 0;
    const float4 *p4 = reinterpret_cast<const float4 *>(p), *y4 = reinterpret_cast<const float4 *>(y);
    float4 *g4 = reinterpret_cast<float4 *>(g);
#pragma unroll 4
    for (int64_t j = threadIdx.x; j < nv; j += blockDim.x) {
      const float4 x = __ldcs(p4 + j), t = __ldcs(y4 + j);
      g4[j] = make_float4(bce_g(x.x, t.x, nf), bce_g(x.y, t.y, nf), bce_g(x.z, t.z, nf), bce_g(x.w, t.w, nf));
    }
    for (int64_t j = nv * 4 + threadIdx.x; j < L; j += blockDim.x) g[j] = bce_g(p[j], y[j], nf);
    if (use_pready == 2)
      pc_pready_block_coop(u, a.q[r]);
    else if (use_pready)
      pc_pready_block(u, a.q[r]);
  }
}

}  // namespace

extern "C" {

int pcapp_produce(void *dst, const void *src, int partitions, int64_t part_bytes, int gran, int order_stride,
                  int blocks, const pc_prequest_t *preq, cudaStream_t s) {
  if (!preq || partitions < 1) return -1;
  if (blocks <= 0) blocks = partitions < 1184 ? partitions : 1184;
  produce_kernel<<<blocks, 512, 0, s>>>((uint8_t *)dst, (const uint8_t *)src, partitions, part_bytes, gran,
                                        order_stride < 1 ? 1 : order_stride, *preq);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_bce_grad(const float *p, const float *y, float *g, int partitions, int64_t L, float nf, int order_stride,
                   int blocks, const pc_prequest_t *preq, cudaStream_t s) {
  if (partitions < 1 || L < 0) return -1;
  if (blocks <= 0) blocks = partitions < 1184 ? partitions : 1184;
  pc_prequest_t q{};
  if (preq) q = *preq;
  bce_grad_kernel<<<blocks, 512, 0, s>>>(p, y, g, partitions, L, nf, order_stride < 1 ? 1 : order_stride,
                                         preq ? 1 : 0, q);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_bce_grad_multi(int n, const float *const *p, const float *const *y, float *const *g, int partitions,
                         int64_t L, float nf, int blocks, const pc_prequest_t *const *preqs, int coop,
                         cudaStream_t s) {
  if (n < 1 || n > 8 || partitions < 1 || L < 0 || !p || !y || !g) return -1;
  BceMultiArgs a{};
  a.n = n;
  for (int r = 0; r < n; ++r) {
    a.p[r] = p[r];
    a.y[r] = y[r];
    a.g[r] = g[r];
    if (preqs) a.q[r] = *preqs[r];
  }
  const int64_t units = (int64_t)partitions * n;
  if (coop && preqs) {
    // the P blocks of a partition wait for one another: every CTA resident,
    // and a multiple of n so the ranks' blocks of u are always in one wave
    int dev = 0, sms = 0, per = 0;
    if (cudaGetDevice(&dev) != cudaSuccess ||
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess ||
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, bce_grad_multi_kernel, 512, 0) != cudaSuccess || per < 1)
      return -2;
    int64_t cap = (int64_t)sms * per;
    cap -= cap % n;
    if (blocks <= 0 || blocks > cap) blocks = (int)cap;
    blocks -= blocks % n;
    if (blocks < n) return -1;
  } else if (blocks <= 0) {
    blocks = units < 1184 ? (int)units : 1184;
  }
  bce_grad_multi_kernel<<<blocks, 512, 0, s>>>(a, partitions, L, nf, preqs ? (coop ? 2 : 1) : 0);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

// preqs: n prequests (one per co-located rank); out: n x 4 stamps
int pcapp_overlap_probe(const pc_prequest_t *const *preqs, int n, int partitions, uint32_t spin_ms,
                        unsigned long long *out, cudaStream_t s) {
  if (!preqs || n < 1 || n > 8 || partitions < 1) return -1;
  ProbeArgs a{};
  a.n = n;
  for (int i = 0; i < n; ++i) a.q[i] = *preqs[i];
  overlap_probe_kernel<<<n, 128, 0, s>>>(a, partitions, spin_ms, out);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

}  // extern "C"
