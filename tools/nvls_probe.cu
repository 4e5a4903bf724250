// tools/nvls_probe.cu — does this box support NVLink SHARP multicast objects
// (cuMulticastCreate / multimem.* PTX)?  Probe for SURVEY NEXT-1 (ii).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/nvls_probe tools/nvls_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdio.h>

#define CK(x) do { CUresult r_ = (x); if (r_ != CUDA_SUCCESS) { const char *s_; cuGetErrorString(r_, &s_); \
  printf("%s -> %d (%s)\n", #x, (int)r_, s_); return 1; } } while (0)

__global__ void mm_kernel(float *mc, float *out, int n) {
  int i = (blockIdx.x * blockDim.x + threadIdx.x) * 4;
  if (i + 4 > n) return;
  float a, b, c, d;
  asm volatile("multimem.ld_reduce.relaxed.sys.global.add.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(a), "=f"(b), "=f"(c), "=f"(d) : "l"(mc + i) : "memory");
  out[i] = a; out[i + 1] = b; out[i + 2] = c; out[i + 3] = d;
  asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1,%2,%3,%4};"
               :: "l"(mc + i), "f"(a + 1.f), "f"(b + 1.f), "f"(c + 1.f), "f"(d + 1.f) : "memory");
}

int main() {
  CK(cuInit(0));
  int ndev = 0; cudaGetDeviceCount(&ndev);
  CUdevice dev; CK(cuDeviceGet(&dev, 0));
  int mc = 0; CK(cuDeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev));
  printf("devices %d multicast_supported %d\n", ndev, mc);
  cudaSetDevice(0); cudaFree(0);
  if (!mc) return 0;
  CUmulticastObjectProp prop = {};
  size_t gran = 0;
  CUmemGenericAllocationHandle mch;
  const CUmemAllocationHandleType hts[3] = {CU_MEM_HANDLE_TYPE_NONE, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR,
                                           CU_MEM_HANDLE_TYPE_FABRIC};
  bool ok = false;
  for (int nd = 1; nd <= 2 && !ok; ++nd)
    for (int h = 0; h < 3 && !ok; ++h) {
      prop = CUmulticastObjectProp{};
      prop.numDevices = nd; prop.size = 2 << 20; prop.handleTypes = hts[h];
      CUresult g = cuMulticastGetGranularity(&gran, &prop, CU_MULTICAST_GRANULARITY_RECOMMENDED);
      CUresult c = cuMulticastCreate(&mch, &prop);
      printf("numDevices %d handle %d: granularity rc %d (%zu) create rc %d\n", nd, (int)hts[h], (int)g, gran, (int)c);
      ok = c == CUDA_SUCCESS && nd == 1;
    }
  if (!ok) return 0;
  CK(cuMulticastAddDevice(mch, dev));
  CUmemAllocationProp ap = {}; ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE; ap.location.id = 0;
  CUmemGenericAllocationHandle ph; CK(cuMemCreate(&ph, prop.size, &ap, 0));
  CK(cuMulticastBindMem(mch, 0, ph, 0, prop.size, 0));
  CUdeviceptr uc, mcp; CK(cuMemAddressReserve(&uc, prop.size, gran, 0, 0)); CK(cuMemMap(uc, prop.size, 0, ph, 0));
  CK(cuMemAddressReserve(&mcp, prop.size, gran, 0, 0)); CK(cuMemMap(mcp, prop.size, 0, mch, 0));
  CUmemAccessDesc ad = {}; ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE; ad.location.id = 0;
  ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  CK(cuMemSetAccess(uc, prop.size, &ad, 1)); CK(cuMemSetAccess(mcp, prop.size, &ad, 1));
  int n = 1 << 16; float h[4] = {1.5f, 2.5f, -3.f, 4.f};
  for (int i = 0; i < n; i += 4) cudaMemcpy((float *)uc + i, h, 16, cudaMemcpyHostToDevice);
  float *out; cudaMalloc(&out, n * 4);
  mm_kernel<<<n / 4 / 256, 256>>>((float *)mcp, out, n);
  cudaError_t e = cudaDeviceSynchronize();
  printf("kernel: %s\n", cudaGetErrorString(e));
  float o[4], u[4]; cudaMemcpy(o, out, 16, cudaMemcpyDeviceToHost); cudaMemcpy(u, (float *)uc, 16, cudaMemcpyDeviceToHost);
  printf("ld_reduce %g %g %g %g  after st %g %g %g %g\n", o[0], o[1], o[2], o[3], u[0], u[1], u[2], u[3]);
  return 0;
}
