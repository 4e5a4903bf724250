/*
 * include/pc_ops.cuh — the reduction operators ⊕ of the partitioned
 * collectives (MPI_Op, §IV-B1), shared by the library's engines
 * (csrc/engine.cuh) and the INLINE allreduce fold of the device bindings
 * (pc_device.cuh, reading R33).  Readings R5 / R27:
 *   int32  : SUM wraps mod 2^32, MAX / MIN;
 *   fp32   : one IEEE op, round to nearest even, no contraction (__fadd_rn);
 *   fp64   : one IEEE binary64 op (__dadd_rn);
 *   bf16   : the bf16 nearest (ties to even) to the exact result: decode to
 *            fp32, one fp32 op, round once (exact because 24 >= 2*8+2).
 * DT codes follow pc_dtype_t (0 INT32, 1 FLOAT32, 3 FLOAT64, 4 BF16); OP codes
 * pc_op_t (0 SUM, 1 MAX, 2 MIN).  vop applies ⊕ lane-wise to a 16-B vector.
 */
#ifndef PC_OPS_CUH_
#define PC_OPS_CUH_

#include <cuda_bf16.h>
#include <stdint.h>

namespace pc_ops {

template <int DT, int OP>
struct Op;
template <int OP>
struct Op<0, OP> {  // int32: sum wraps mod 2^32
  using T = int32_t;
  static __device__ __forceinline__ int32_t f(int32_t a, int32_t b) {
    if (OP == 0) return (int32_t)((uint32_t)a + (uint32_t)b);
    if (OP == 1) return a > b ? a : b;
    return a < b ? a : b;
  }
};
template <int OP>
struct Op<1, OP> {  // fp32: one IEEE add, round to nearest even, no contraction
  using T = float;
  static __device__ __forceinline__ float f(float a, float b) {
    if (OP == 0) return __fadd_rn(a, b);
    if (OP == 1) return fmaxf(a, b);
    return fminf(a, b);
  }
};
template <int OP>
struct Op<3, OP> {  // fp64 (the paper's `double` buffers)
  using T = double;
  static __device__ __forceinline__ double f(double a, double b) {
    if (OP == 0) return __dadd_rn(a, b);
    if (OP == 1) return fmax(a, b);
    return fmin(a, b);
  }
};
template <int OP>
struct Op<4, OP> {  // bf16 storage (uint16 bits); each op is one correctly rounded bf16 result:
  using T = uint16_t;  // a + b of two bf16 values is exact in fp32 or the small one is below half an ulp
  static __device__ __forceinline__ float up(uint16_t v) { return __uint_as_float((uint32_t)v << 16); }
  static __device__ __forceinline__ uint16_t dn(float f) { return __bfloat16_as_ushort(__float2bfloat16_rn(f)); }
  static __device__ __forceinline__ uint16_t f(uint16_t a, uint16_t b) {
    if (OP == 0) return dn(__fadd_rn(up(a), up(b)));
    if (OP == 1) return dn(fmaxf(up(a), up(b)));
    return dn(fminf(up(a), up(b)));
  }
};

template <int DT, int OP>
__device__ __forceinline__ uint4 vop(uint4 a, uint4 b) {
  using O = Op<DT, OP>;
  using T = typename O::T;
  constexpr int EPV = 16 / sizeof(T);
  uint4 r;
  T *ra = reinterpret_cast<T *>(&r);
  const T *pa = reinterpret_cast<const T *>(&a);
  const T *pb = reinterpret_cast<const T *>(&b);
#pragma unroll
  for (int j = 0; j < EPV; ++j) ra[j] = O::f(pa[j], pb[j]);
  return r;
}

// fp32 SUM on sm_100: packed add.rn.f32x2 (SASS FADD2) — two IEEE
// round-to-nearest-even adds per instruction, bit-identical to __fadd_rn
// lane by lane (no .ftz: subnormals kept), half the FADD issue slots of the
// scalar form (the thin overlap engines are issue-bound).
template <>
__device__ __forceinline__ uint4 vop<1, 0>(uint4 a, uint4 b) {
#if defined(__CUDA_ARCH__) && __CUDA_ARCH__ >= 1000
  unsigned long long lo, hi;
  asm("add.rn.f32x2 %0, %1, %2;"
      : "=l"(lo)
      : "l"(((unsigned long long)a.y << 32) | a.x), "l"(((unsigned long long)b.y << 32) | b.x));
  asm("add.rn.f32x2 %0, %1, %2;"
      : "=l"(hi)
      : "l"(((unsigned long long)a.w << 32) | a.z), "l"(((unsigned long long)b.w << 32) | b.z));
  return make_uint4((uint32_t)lo, (uint32_t)(lo >> 32), (uint32_t)hi, (uint32_t)(hi >> 32));
#else
  return make_uint4(__float_as_uint(__fadd_rn(__uint_as_float(a.x), __uint_as_float(b.x))),
                    __float_as_uint(__fadd_rn(__uint_as_float(a.y), __uint_as_float(b.y))),
                    __float_as_uint(__fadd_rn(__uint_as_float(a.z), __uint_as_float(b.z))),
                    __float_as_uint(__fadd_rn(__uint_as_float(a.w), __uint_as_float(b.w))));
#endif
}

}  // namespace pc_ops

#endif /* PC_OPS_CUH_ */
