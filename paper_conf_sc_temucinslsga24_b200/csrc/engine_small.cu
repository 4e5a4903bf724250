// The small-comm (MAXP = 4, 2) DIRECT allreduce and collective kernels of
// one (dtype, op): more 16-B loads per operand in flight for P <= 4 in the
// same registers (engine.cuh warp_fold_pull).  Built only for the gradient
// types' SUM (Makefile: -DPC_DT=1|4 -DPC_OP=0).
#include "engine.cuh"

#if !defined(PC_DT) || !defined(PC_OP)
#error "compile with -DPC_DT=<dtype> -DPC_OP=<op>"
#endif

namespace pc {

template <int DT, int OP>
int SmallCommLaunch<DT, OP>::direct(const DirectArgs &a, int grid, cudaStream_t s, int maxp) {
  if (maxp <= 2)
    direct_engine<DT, OP, 2><<<grid, kEngineBlock, kDirectSmem, s>>>(a);
  else
    direct_engine<DT, OP, 4><<<grid, kEngineBlock, kDirectSmem, s>>>(a);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

template <int DT, int OP>
int SmallCommLaunch<DT, OP>::direct_group(const DirectGroupArgs &h, int blocks, cudaStream_t s, int maxp) {
  if (maxp <= 2)
    direct_engine_group<DT, OP, 2><<<blocks, kEngineBlock, kDirectSmem, s>>>(h);
  else
    direct_engine_group<DT, OP, 4><<<blocks, kEngineBlock, kDirectSmem, s>>>(h);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

template <int DT, int OP>
int SmallCommLaunch<DT, OP>::coll(const CollArgs &a, int grid, cudaStream_t s, int maxp) {
  if (maxp <= 2)
    coll_engine<DT, OP, 2><<<grid, kEngineBlock, 0, s>>>(a);
  else
    coll_engine<DT, OP, 4><<<grid, kEngineBlock, 0, s>>>(a);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

template <int DT, int OP>
int SmallCommLaunch<DT, OP>::coll_group(const CollGroupArgs &h, int blocks, cudaStream_t s, int maxp) {
  if (maxp <= 2)
    coll_engine_group<DT, OP, 2><<<blocks, kEngineBlock, 0, s>>>(h);
  else
    coll_engine_group<DT, OP, 4><<<blocks, kEngineBlock, 0, s>>>(h);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

template <int DT, int OP>
int SmallCommLaunch<DT, OP>::preload() {
  cudaFuncAttributes fa;
  PC_CUDA(cudaFuncGetAttributes(&fa, direct_engine<DT, OP, 4>));
  PC_CUDA(cudaFuncGetAttributes(&fa, direct_engine<DT, OP, 2>));
  PC_CUDA(cudaFuncGetAttributes(&fa, direct_engine_group<DT, OP, 4>));
  PC_CUDA(cudaFuncGetAttributes(&fa, direct_engine_group<DT, OP, 2>));
  PC_CUDA(cudaFuncGetAttributes(&fa, coll_engine<DT, OP, 4>));
  PC_CUDA(cudaFuncGetAttributes(&fa, coll_engine<DT, OP, 2>));
  PC_CUDA(cudaFuncGetAttributes(&fa, coll_engine_group<DT, OP, 4>));
  PC_CUDA(cudaFuncGetAttributes(&fa, coll_engine_group<DT, OP, 2>));
  return 0;
}

template struct SmallCommLaunch<PC_DT, PC_OP>;

}  // namespace pc
