// C2 floor probe (no library): what the block-granularity Kernel Copy costs
// on top of the vector add, per producer shape, on one B200 (peer = another
// HBM buffer of the same GPU).  nvcc -gencode arch=compute_100a,code=sm_100a
// -O3 -o c2_floor c2_floor.cu && ./c2_floor [MiB]
//   nonpers        C = A + B, one 1024-thread CTA per 8 KiB block
//   nonpers+push   + every thread stores its result to the peer buffer too,
//                  barrier, thread 0 fence.acq_rel.gpu + flag
//   pers           persistent CTAs (2 per SM), next block's operands prefetched
//   pers+push      + push, barrier, thread 0 fence + flag (the others run on)
//   pers+push/rel  + push, barrier, thread 0 st.release.gpu flag
//   pers+push/nof  + push, no fence or flag (upper bound)
//   copy           cudaMemcpyAsync D2D of C (the traditional copy)
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e_)); exit(1); } } while (0)

__global__ void __launch_bounds__(1024) nonpers(const float2 *A, const float2 *B, float2 *C, float2 *R,
                                                uint32_t *flag, int64_t n2, int mode, uint32_t e) {
  const int64_t i = (int64_t)blockIdx.x * 1024 + threadIdx.x;
  float2 c = make_float2(0.f, 0.f);
  if (i < n2) {
    const float2 a = A[i], b = B[i];
    c = make_float2(a.x + b.x, a.y + b.y);
    C[i] = c;
  }
  if (mode == 0) return;
  __shared__ uint32_t s_e;
  if (mode >= 5 && threadIdx.x == 0) {  // library-like: {epoch, rtr} acquire before the data barrier
    uint32_t ep, rtr;
    asm volatile("ld.acquire.gpu.global.v2.u32 {%0, %1}, [%2];" : "=r"(ep), "=r"(rtr) : "l"(flag + gridDim.x) : "memory");
    s_e = ep + rtr;
  }
  if (mode >= 4) {  // library-like: barrier, then read the partition back from L2
    __syncthreads();
    if (i < n2) c = __ldcg(C + i);
  }
  if (mode == 6) c.x += (float)(s_e & 0);
  if (i < n2) R[i] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    if (mode == 1)
      asm volatile("fence.acq_rel.gpu;" ::: "memory");
    else
      asm volatile("fence.release.gpu;" ::: "memory");
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(flag + blockIdx.x), "r"(e) : "memory");
  }
}

__global__ void __launch_bounds__(1024, 2) pers(const float2 *A, const float2 *B, float2 *C, float2 *R,
                                                 uint32_t *flag, int64_t n2, int64_t nblk, int mode, uint32_t e) {
  int64_t p = blockIdx.x;
  float2 a = make_float2(0.f, 0.f), b = a;
  {
    const int64_t i = p * 1024 + threadIdx.x;
    if (p < nblk && i < n2) { a = __ldcs(A + i); b = __ldcs(B + i); }
  }
  for (; p < nblk; p += gridDim.x) {
    const int64_t i = p * 1024 + threadIdx.x;
    const float2 c = make_float2(a.x + b.x, a.y + b.y);
    const int64_t in = i + (int64_t)gridDim.x * 1024;
    if (p + gridDim.x < nblk && in < n2) { a = __ldcs(A + in); b = __ldcs(B + in); }
    if (i < n2) C[i] = c;
    if (mode == 0) continue;
    if (i < n2) R[i] = c;
    if (mode == 3) continue;
    __syncthreads();
    if (threadIdx.x == 0) {
      if (mode == 1) {
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
        asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(flag + p), "r"(e) : "memory");
      } else {
        asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(flag + p), "r"(e) : "memory");
      }
    }
  }
}


// TMA-staged persistent variant (the library's vecadd_persistent_kernel shape)
constexpr int kSt = 4;
__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__global__ void __launch_bounds__(1024, 2) pers_tma(const float2 *A, const float2 *B, float2 *C, float2 *R,
                                                     uint32_t *flag, int n2, int nblk, int mode, uint32_t e, int issuer) {
  extern __shared__ __align__(128) uint8_t sm[];
  float2 *sA = (float2 *)sm, *sB = sA + kSt * 1024;
  uint64_t *full = (uint64_t *)(sB + kSt * 1024), *empty = full + kSt;
  const int tid = threadIdx.x, G = gridDim.x, T = (nblk - (int)blockIdx.x + G - 1) / G;
  auto issue = [&](int k) {
    const int p = blockIdx.x + k * G, s = k % kSt;
    asm volatile("{\n .reg .b64 st;\n mbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n}" ::"r"(su32(full + s)), "r"(16384) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(su32(sA + s * 1024)), "l"(A + (int64_t)p * 1024), "r"(8192), "r"(su32(full + s)) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(su32(sB + s * 1024)), "l"(B + (int64_t)p * 1024), "r"(8192), "r"(su32(full + s)) : "memory");
  };
  if (tid == 0) {
    for (int s = 0; s < kSt; ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(full + s)), "r"(1) : "memory");
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(empty + s)), "r"(32) : "memory");
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (tid == issuer) for (int k = 0; k < kSt && k < T; ++k) issue(k);
  for (int k = 0; k < T; ++k) {
    const int p = blockIdx.x + k * G, s = k % kSt;
    const uint32_t par = (k / kSt) & 1;
    asm volatile("{\n .reg .pred q;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 q, [%0], %1;\n @!q bra W_%=;\n}" ::"r"(su32(full + s)), "r"(par) : "memory");
    const float2 a = sA[s * 1024 + tid], b = sB[s * 1024 + tid];
    const float2 c = make_float2(a.x + b.x, a.y + b.y);
    __syncwarp();
    if ((tid & 31) == 0) asm volatile("{\n .reg .b64 st;\n mbarrier.arrive.shared::cta.b64 st, [%0];\n}" ::"r"(su32(empty + s)) : "memory");
    const int i = p * 1024 + tid;
    C[i] = c;
    if (mode >= 1) {
      R[i] = c;
      if (mode <= 2) {
        __syncthreads();
        if (tid == 0) {
          if (mode == 1) asm volatile("fence.release.gpu;\n\tst.relaxed.gpu.global.u32 [%0], %1;" ::"l"(flag + p), "r"(e) : "memory");
          else asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(flag + p), "r"(e) : "memory");
        }
      }
    }
    if (tid == issuer && k + kSt < T) {
      asm volatile("{\n .reg .pred q;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 q, [%0], %1;\n @!q bra W_%=;\n}" ::"r"(su32(empty + s)), "r"(par) : "memory");
      issue(k + kSt);
    }
  }
}

int main(int argc, char **argv) {
  const int64_t mib = argc > 1 ? atoll(argv[1]) : 256;
  const int64_t n = mib << 18, n2 = n / 2, nblk = (n2 + 1023) / 1024;
  float2 *A, *B, *C, *R;
  uint32_t *flag;
  CK(cudaMalloc(&A, n * 4));
  CK(cudaMalloc(&B, n * 4));
  CK(cudaMalloc(&C, n * 4));
  CK(cudaMalloc(&R, n * 4));
  CK(cudaMalloc(&flag, nblk * 4 + 64));
  CK(cudaMemset(flag, 0, nblk * 4 + 64));
  CK(cudaMemset(A, 0, n * 4));
  CK(cudaMemset(B, 0, n * 4));
  int sms = 0, per = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, pers, 1024, 0));
  const int64_t grid = nblk < (int64_t)sms * per ? nblk : (int64_t)sms * per;
  const size_t smt = (size_t)2 * kSt * 1024 * 8 + 2 * kSt * 8;
  CK(cudaFuncSetAttribute(pers_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smt));
  int pert = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&pert, pers_tma, 1024, smt));
  const int64_t gridt = nblk < (int64_t)sms * pert ? nblk : (int64_t)sms * pert;
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  const int it = 20;
  uint32_t ep = 1;
  auto run = [&](const char *name, int kind) {
    for (int w = 0; w < 3 + it; ++w) {
      if (w == 3) CK(cudaEventRecord(e0));
      switch (kind) {
        case 0: nonpers<<<nblk, 1024>>>(A, B, C, R, flag, n2, 0, ep++); break;
        case 1: nonpers<<<nblk, 1024>>>(A, B, C, R, flag, n2, 1, ep++); break;
        case 2: pers<<<grid, 1024>>>(A, B, C, R, flag, n2, nblk, 0, ep++); break;
        case 3: pers<<<grid, 1024>>>(A, B, C, R, flag, n2, nblk, 1, ep++); break;
        case 4: pers<<<grid, 1024>>>(A, B, C, R, flag, n2, nblk, 2, ep++); break;
        case 5: pers<<<grid, 1024>>>(A, B, C, R, flag, n2, nblk, 3, ep++); break;
        case 6: CK(cudaMemcpyAsync(R, C, n * 4, cudaMemcpyDeviceToDevice)); break;
        case 7:
          nonpers<<<nblk, 1024>>>(A, B, C, R, flag, n2, 0, ep++);
          CK(cudaMemcpyAsync(R, C, n * 4, cudaMemcpyDeviceToDevice));
          break;
        case 9: nonpers<<<nblk, 1024>>>(A, B, C, R, flag, n2, 3, ep++); break;
        case 10: nonpers<<<nblk, 1024>>>(A, B, C, R, flag, n2, 4, ep++); break;
        case 11: nonpers<<<nblk, 1024>>>(A, B, C, R, flag, n2, 6, ep++); break;
        case 12: case 13: case 14: case 15: case 16:
          pers_tma<<<gridt, 1024, smt>>>(A, B, C, R, flag, (int)n2, (int)nblk, kind == 12 ? 0 : kind == 13 ? 1 : kind == 14 ? 2 : kind == 15 ? 3 : 1, ep++, kind == 16 ? 0 : 32);
          break;
        case 8:
          pers<<<grid, 1024>>>(A, B, C, R, flag, n2, nblk, 0, ep++);
          CK(cudaMemcpyAsync(R, C, n * 4, cudaMemcpyDeviceToDevice));
          break;
      }
    }
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    CK(cudaGetLastError());
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    const double us = ms * 1e3 / it;
    printf("{\"probe\": \"c2_floor\", \"MiB\": %lld, \"variant\": \"%s\", \"us\": %.2f, \"grid\": %lld}\n",
           (long long)mib, name, us, (long long)((kind >= 2 && kind <= 5) || kind == 8 ? grid : nblk));
  };
  run("nonpers", 0);
  run("nonpers+push(fence)", 1);
  run("pers", 2);
  run("pers+push(fence)", 3);
  run("pers+push(st.release)", 4);
  run("pers+push(no flag)", 5);
  run("copy", 6);
  run("nonpers->copy", 7);
  run("pers->copy", 8);
  run("nonpers+push(fence.release)", 9);
  run("nonpers+readback+push(fence.release)", 10);
  run("nonpers+epoch_acquire+readback+push(fence.release)", 11);
  run("pers_tma", 12);
  run("pers_tma+push(fence.release)", 13);
  run("pers_tma+push(st.release)", 14);
  run("pers_tma+push(no flag)", 15);
  run("pers_tma+push(fence.release, issuer=tid0)", 16);
  return 0;
}
