// One (dtype, op) instantiation of the engine launchers declared in
// engine.cuh; the Makefile compiles this file 12 times with
// -DPC_DT=<0|1|3|4> -DPC_OP=<0|1|2>.
#include "engine.cuh"

#if !defined(PC_DT) || !defined(PC_OP)
#error "compile with -DPC_DT=<dtype> -DPC_OP=<op>"
#endif

namespace pc {

// The small-comm instantiations (MAXP 4 / 2, engine.cuh) exist for the
// gradient types' SUM only (fp32, bf16; SmallCommLaunch in engine_small.cu):
// every other (dtype, op) runs the MAXP = 8 kernels for any P (correct, fewer
// loads in flight) — it keeps the library's build time and size in bounds.

template <int DT, int OP>
int EngineLaunch<DT, OP>::ring(const RingArgs &a, int warps, cudaStream_t s) {
  ring_engine<DT, OP><<<grid_for(warps, a.nunits), kEngineBlock, 0, s>>>(a);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

template <int DT, int OP>
int EngineLaunch<DT, OP>::rd(const RdArgs &a, int warps, cudaStream_t s) {
  rd_engine<DT, OP><<<grid_for(warps, a.nunits), kEngineBlock, 0, s>>>(a);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

// The DIRECT engines take kDirectSmem of dynamic shared memory (bulk-copy
// stages, engine.cuh): opt in once per kernel.
template <typename K>
static int direct_smem_attr(K kernel) {
  static bool done = false;
  if (!done && kDirectSmem > 48 * 1024) {
    PC_CUDA(cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kDirectSmem));
    done = true;
  }
  return 0;
}

template <int DT, int OP>
int EngineLaunch<DT, OP>::direct(const DirectArgs &a, int warps, cudaStream_t s, bool thin) {
  if (a.ll) {
    ll_engine<DT, OP><<<grid_for(warps, a.nunits), kEngineBlock, 0, s>>>(a);
    g_launches++;
    PC_CUDA(cudaGetLastError());
    return 0;
  }
  if (a.push) {
    direct_engine_push<DT, OP><<<grid_for(warps, a.nunits), kEngineBlock, 0, s>>>(a);
    g_launches++;
    PC_CUDA(cudaGetLastError());
    return 0;
  }
  if (thin) {
    if (kThinSmem > 48 * 1024)
      PC_CUDA(cudaFuncSetAttribute(direct_engine_thin<DT, OP>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)kThinSmem));
    direct_engine_thin<DT, OP><<<grid_for(warps, a.nunits), kEngineBlock, kThinSmem, s>>>(a);
    g_launches++;
    PC_CUDA(cudaGetLastError());
    return 0;
  }
  if (int rc = direct_smem_attr(direct_engine<DT, OP>)) return rc;
  const int grid = grid_for(warps, a.nunits);
  if constexpr (kSmallCommKernels<DT, OP>) {
    if (a.P <= 4) {
      return SmallCommLaunch<DT, OP>::direct(a, grid, s, a.P <= 2 ? 2 : 4);
    } else {
      direct_engine<DT, OP><<<grid, kEngineBlock, kDirectSmem, s>>>(a);
    }
  } else {
    direct_engine<DT, OP><<<grid, kEngineBlock, kDirectSmem, s>>>(a);
  }
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

template <int DT, int OP>
int EngineLaunch<DT, OP>::ring_group(const RingGroupArgs &h, int blocks, cudaStream_t s) {
  ring_engine_group<DT, OP><<<blocks, kEngineBlock, 0, s>>>(h);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

template <int DT, int OP>
int EngineLaunch<DT, OP>::rd_group(const RdGroupArgs &h, int blocks, cudaStream_t s) {
  rd_engine_group<DT, OP><<<blocks, kEngineBlock, 0, s>>>(h);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

template <int DT, int OP>
int EngineLaunch<DT, OP>::direct_group(const DirectGroupArgs &h, int blocks, cudaStream_t s, bool thin) {
  if (h.a[0].ll) {
    ll_engine_group<DT, OP><<<blocks, kEngineBlock, 0, s>>>(h);
    g_launches++;
    PC_CUDA(cudaGetLastError());
    return 0;
  }
  if (h.a[0].push) {
    direct_engine_group_push<DT, OP><<<blocks, kEngineBlock, 0, s>>>(h);
    g_launches++;
    PC_CUDA(cudaGetLastError());
    return 0;
  }
  if (thin) {
    if (kThinSmem > 48 * 1024)
      PC_CUDA(cudaFuncSetAttribute(direct_engine_group_thin<DT, OP>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)kThinSmem));
    direct_engine_group_thin<DT, OP><<<blocks, kEngineBlock, kThinSmem, s>>>(h);
    g_launches++;
    PC_CUDA(cudaGetLastError());
    return 0;
  }
  if (int rc = direct_smem_attr(direct_engine_group<DT, OP>)) return rc;
  if constexpr (kSmallCommKernels<DT, OP>) {
    if (h.a[0].P <= 4) {
      return SmallCommLaunch<DT, OP>::direct_group(h, blocks, s, h.a[0].P <= 2 ? 2 : 4);
    } else {
      direct_engine_group<DT, OP><<<blocks, kEngineBlock, kDirectSmem, s>>>(h);
    }
  } else {
    direct_engine_group<DT, OP><<<blocks, kEngineBlock, kDirectSmem, s>>>(h);
  }
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

template <int DT, int OP>
int EngineLaunch<DT, OP>::direct_batch(const DirectBatchArgs &b, int blocks, cudaStream_t s, bool thin) {
  if (thin)
    direct_engine_batch_thin<DT, OP><<<blocks, kEngineBlock, 0, s>>>(b);
  else
    direct_engine_batch<DT, OP><<<blocks, kEngineBlock, 0, s>>>(b);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

template <int DT, int OP>
int EngineLaunch<DT, OP>::occupancy(int *ctas) {
  int a = 0, b = 0;
  PC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&a, ring_engine<DT, OP>, kEngineBlock, 0));
  PC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, rd_engine<DT, OP>, kEngineBlock, 0));
  *ctas = a < b ? a : b;
  return 0;
}

// The DIRECT engines run fewer, fatter CTAs (PC_DIRECT_MINB): their own
// capacity, with their shared-memory stages when PC_DIRECT_BULK.
template <int DT, int OP>
int EngineLaunch<DT, OP>::occupancy_direct(int *ctas) {
  int a = 0, b = 0;
  if (int rc = direct_smem_attr(direct_engine_group<DT, OP>)) return rc;
  if (int rc = direct_smem_attr(direct_engine<DT, OP>)) return rc;
  PC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&a, direct_engine_group<DT, OP>, kEngineBlock, kDirectSmem));
  PC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, direct_engine<DT, OP>, kEngineBlock, kDirectSmem));
  *ctas = a < b ? a : b;
  // the collective engines (reduce-scatter PULL fold) use the same fat CTAs
  PC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&a, coll_engine<DT, OP>, kEngineBlock, 0));
  PC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, coll_engine_group<DT, OP>, kEngineBlock, 0));
  *ctas = *ctas < a ? *ctas : a;
  *ctas = *ctas < b ? *ctas : b;
  return 0;
}

template <int DT, int OP>
int EngineLaunch<DT, OP>::coll(const CollArgs &a, int warps, cudaStream_t s) {
  const int grid = grid_for(warps, a.nunits);
  if constexpr (kSmallCommKernels<DT, OP>) {
    if (a.P <= 4) {
      return SmallCommLaunch<DT, OP>::coll(a, grid, s, a.P <= 2 ? 2 : 4);
    } else {
      coll_engine<DT, OP><<<grid, kEngineBlock, 0, s>>>(a);
    }
  } else {
    coll_engine<DT, OP><<<grid, kEngineBlock, 0, s>>>(a);
  }
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

template <int DT, int OP>
int EngineLaunch<DT, OP>::coll_group(const CollGroupArgs &h, int blocks, cudaStream_t s) {
  if constexpr (kSmallCommKernels<DT, OP>) {
    if (h.a[0].P <= 4) {
      return SmallCommLaunch<DT, OP>::coll_group(h, blocks, s, h.a[0].P <= 2 ? 2 : 4);
    } else {
      coll_engine_group<DT, OP><<<blocks, kEngineBlock, 0, s>>>(h);
    }
  } else {
    coll_engine_group<DT, OP><<<blocks, kEngineBlock, 0, s>>>(h);
  }
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

template <int DT, int OP>
int EngineLaunch<DT, OP>::preload() {
  cudaFuncAttributes fa;
  PC_CUDA(cudaFuncGetAttributes(&fa, ring_engine<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, rd_engine<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, direct_engine<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, ring_engine_group<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, rd_engine_group<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, direct_engine_group<DT, OP>));
  if constexpr (kSmallCommKernels<DT, OP>) {
    if (int rc = SmallCommLaunch<DT, OP>::preload()) return rc;
  }
  PC_CUDA(cudaFuncGetAttributes(&fa, direct_engine_thin<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, direct_engine_group_thin<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, direct_engine_batch<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, direct_engine_push<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, ll_engine<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, ll_engine_group<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, direct_engine_group_push<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, direct_engine_batch_thin<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, coll_engine<DT, OP>));
  PC_CUDA(cudaFuncGetAttributes(&fa, coll_engine_group<DT, OP>));

  return 0;
}

template struct EngineLaunch<PC_DT, PC_OP>;

}  // namespace pc
