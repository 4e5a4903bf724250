// Jacobi solver with intra-kernel partitioned halo exchange (SURVEY §8(a) a8,
// P:L304; stencil per DESIGN.md reading R17, decomposition per R18).
//
// Each rank owns an ly x lx block of the global N x N grid (boundary rows and
// columns of the global grid are Dirichlet-fixed).  One kernel launch per
// iteration; a warp owns a tile of H rows x 128 columns (one float4 per lane)
// and slides down it keeping up/centre/down rows in registers, so every grid
// element is read once and written once per iteration (HBM-bound: 8 B per
// cell update).  Tiles on the block edge:
//   * before computing, wait for the halo partition they read
//     (pc_wait_arrived on the receive request; one partition = one tile's
//     edge segment of one iteration),
//   * while computing, also write their edge values into the send staging
//     buffer, and after the tile, pc_pready_warp() that segment — the
//     INLINE push lands in the neighbour's halo buffer over NVLink.
// Partition numbering: (slot j, segment s) -> j * nseg + s, with slot j = the
// iteration that READS it (slot 0 = initial halos, pushed by jacobi_init);
// iteration k reads slot k and fills slot k+1.  One epoch covers the whole
// solve, so halo buffers are never overwritten while in use (no RTR needed
// inside the solve, reading R18).
#include <cuda_runtime.h>
#include <stdint.h>

#include "pc_device.cuh"

namespace {

constexpr int kStrip = 128;  // columns per warp tile (32 lanes x float4)
#ifndef PC_JACOBI_MINB
#define PC_JACOBI_MINB 4  // 4 CTAs x 8 warps per SM: enough loads in flight for HBM (measured, tools/jacobi_variants.sh)
#endif
#ifndef PC_JACOBI_RB
#define PC_JACOBI_RB 4
#endif
constexpr int kRB = PC_JACOBI_RB;  // rows loaded together per batch (tile height H % kRB == 0)
enum { T = 0, B = 1, L = 2, R = 3 };

struct JacobiRank {
  float *grid[2];   // ly x lx, row-major, pitch lx
  int ly, lx, H;    // local block, tile height
  int gy0, gx0, N;  // global offset of the block, global size (boundary included)
  int has[4];       // neighbour exists on side T/B/L/R
  float *sendbuf[4];      // staging of my edge on side d, (K+1) slots
  const float *halo[4];   // halo received on side d, (K+1) slots
  pc_prequest_t sq[4];    // send request towards side d
  pc_prequest_t rq[4];    // receive request for the halo on side d
  int nsegR, nsegC;       // segments per slot: row halos (lx/128), column halos (ly/H)
  int tiles;              // (ly/H) * (lx/128)
};

__device__ __forceinline__ float stencil(float up, float dn, float lf, float rt) {
  return __fmul_rn(0.25f, __fadd_rn(__fadd_rn(up, dn), __fadd_rn(lf, rt)));
}

__device__ __forceinline__ float4 ld4(const float *p) { return __ldcg(reinterpret_cast<const float4 *>(p)); }

__device__ void tile_iter(const JacobiRank &d, int tile, int k) {
  const int lane = threadIdx.x & 31;
  const int nstrip = d.lx / kStrip;
  const int rb = tile / nstrip, sx = tile % nstrip;
  const int r0 = rb * d.H, x0 = sx * kStrip + 4 * lane;
  const float *a = d.grid[k & 1];
  float *b = d.grid[(k + 1) & 1];
  const int lx = d.lx, ly = d.ly;
  const bool top = rb == 0 && d.has[T], bot = (r0 + d.H == ly) && d.has[B];
  const bool left = sx == 0 && d.has[L], right = (sx == nstrip - 1) && d.has[R];
  // Parrived: the halo segments this tile reads (slot k)
  if (lane == 0) {
    if (top) pc_wait_arrived(d.rq[T], k * d.nsegR + sx);
    if (bot) pc_wait_arrived(d.rq[B], k * d.nsegR + sx);
    if (left) pc_wait_arrived(d.rq[L], k * d.nsegC + rb);
    if (right) pc_wait_arrived(d.rq[R], k * d.nsegC + rb);
  }
  __syncwarp();
  const float *hT = d.halo[T] + (size_t)k * lx, *hB = d.halo[B] + (size_t)k * lx;
  const float *hL = d.halo[L] + (size_t)k * ly, *hR = d.halo[R] + (size_t)k * ly;
  float4 cur = ld4(a + (size_t)r0 * lx + x0);
  float4 up;
  if (r0 > 0) up = ld4(a + (size_t)(r0 - 1) * lx + x0);
  else if (top) up = ld4(hT + x0);
  else up = cur;  // global boundary row: not used
  const int gx = d.gx0 + x0;
  const bool colfix0 = gx == 0, colfix3 = gx + 3 == d.N - 1;
  // Rows in batches of kRB: the kRB next rows (and the lane-0 / lane-31 edge
  // scalars) are loaded together so each warp keeps kRB 512-B loads in flight.
  for (int r = r0; r < r0 + d.H; r += kRB) {
    float4 nx[kRB];
    float le[kRB], re[kRB];
#pragma unroll
    for (int j = 0; j < kRB; ++j) {
      const int rr = r + 1 + j;
      nx[j] = rr < ly ? ld4(a + (size_t)rr * lx + x0) : (d.has[B] ? ld4(hB + x0) : cur);
    }
#pragma unroll
    for (int j = 0; j < kRB; ++j) {
      const int rr = r + j;
      le[j] = 0.f;
      re[j] = 0.f;
      if (lane == 0) le[j] = x0 > 0 ? __ldcg(a + (size_t)rr * lx + x0 - 1) : (d.has[L] ? __ldcg(hL + rr) : 0.f);
      if (lane == 31) re[j] = x0 + 4 < lx ? __ldcg(a + (size_t)rr * lx + x0 + 4) : (d.has[R] ? __ldcg(hR + rr) : 0.f);
    }
#pragma unroll
    for (int j = 0; j < kRB; ++j) {
      const int rr = r + j;
      const float4 dn = nx[j];
      float lf = __shfl_up_sync(0xffffffffu, cur.w, 1);
      float rt = __shfl_down_sync(0xffffffffu, cur.x, 1);
      if (lane == 0) lf = le[j];
      if (lane == 31) rt = re[j];
      const int gy = d.gy0 + rr;
      float4 o;
      if (gy == 0 || gy == d.N - 1) {
        o = cur;  // Dirichlet row
      } else {
        o.x = colfix0 ? cur.x : stencil(up.x, dn.x, lf, cur.y);
        o.y = stencil(up.y, dn.y, cur.x, cur.z);
        o.z = stencil(up.z, dn.z, cur.y, cur.w);
        o.w = colfix3 ? cur.w : stencil(up.w, dn.w, cur.z, rt);
      }
      *reinterpret_cast<float4 *>(b + (size_t)rr * lx + x0) = o;
      // edge staging for the neighbours (slot k+1)
      if (rr == 0 && d.has[T]) *reinterpret_cast<float4 *>(d.sendbuf[T] + (size_t)(k + 1) * lx + x0) = o;
      if (rr == ly - 1 && d.has[B]) *reinterpret_cast<float4 *>(d.sendbuf[B] + (size_t)(k + 1) * lx + x0) = o;
      if (left && lane == 0) d.sendbuf[L][(size_t)(k + 1) * ly + rr] = o.x;
      if (right && lane == 31) d.sendbuf[R][(size_t)(k + 1) * ly + rr] = o.w;
      up = cur;
      cur = dn;
    }
  }
  // Pready: push my edge segments of slot k+1 (INLINE copy by this warp)
  if (top) pc_pready_warp((k + 1) * d.nsegR + sx, d.sq[T]);
  if (bot) pc_pready_warp((k + 1) * d.nsegR + sx, d.sq[B]);
  if (left) pc_pready_warp((k + 1) * d.nsegC + rb, d.sq[L]);
  if (right) pc_pready_warp((k + 1) * d.nsegC + rb, d.sq[R]);
}

// Slot 0: push the initial edges (the halos iteration 0 reads).
__device__ void tile_init(const JacobiRank &d, int tile) {
  const int lane = threadIdx.x & 31;
  const int nstrip = d.lx / kStrip;
  const int rb = tile / nstrip, sx = tile % nstrip;
  const int r0 = rb * d.H, x0 = sx * kStrip + 4 * lane;
  const float *a = d.grid[0];
  const int lx = d.lx, ly = d.ly;
  const bool top = rb == 0 && d.has[T], bot = (r0 + d.H == ly) && d.has[B];
  const bool left = sx == 0 && d.has[L], right = (sx == nstrip - 1) && d.has[R];
  if (top) *reinterpret_cast<float4 *>(d.sendbuf[T] + x0) = ld4(a + x0);
  if (bot) *reinterpret_cast<float4 *>(d.sendbuf[B] + x0) = ld4(a + (size_t)(ly - 1) * lx + x0);
  for (int r = r0 + lane; r < r0 + d.H; r += 32) {
    if (left) d.sendbuf[L][r] = __ldcg(a + (size_t)r * lx);
    if (right) d.sendbuf[R][r] = __ldcg(a + (size_t)r * lx + lx - 1);
  }
  __syncwarp();
  if (top) pc_pready_warp(sx, d.sq[T]);
  if (bot) pc_pready_warp(sx, d.sq[B]);
  if (left) pc_pready_warp(rb, d.sq[L]);
  if (right) pc_pready_warp(rb, d.sq[R]);
}

// One launch covers the tiles of `nranks` ranks (all co-located ranks of a
// process on this GPU, or a single rank): block b -> rank via block_start.
__global__ void __launch_bounds__(256, PC_JACOBI_MINB) jacobi_kernel(const JacobiRank *__restrict__ ranks, const int *block_start,
                                                    int nranks, int k, int init) {
  int q = 0;
  while (q + 1 < nranks && (int)blockIdx.x >= block_start[q + 1]) ++q;
  const JacobiRank &d = ranks[q];
  const int tile = (blockIdx.x - block_start[q]) * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (tile >= d.tiles) return;
  if (init)
    tile_init(d, tile);
  else
    tile_iter(d, tile, k);
}

}  // namespace

extern "C" {

size_t pcapp_jacobi_rank_size(void) { return sizeof(JacobiRank); }

// ranks: device array of nranks JacobiRank descriptors (layout: see
// pcapp_jacobi_describe); block_start: device array of nranks ints.
int pcapp_jacobi_launch(const void *ranks, const int *block_start, int nranks, int total_blocks, int k, int init,
                        cudaStream_t s) {
  jacobi_kernel<<<total_blocks, 256, 0, s>>>((const JacobiRank *)ranks, block_start, nranks, k, init);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

// Fill one host-side descriptor (the caller copies the array to the device).
int pcapp_jacobi_describe(void *out, float *grid0, float *grid1, int ly, int lx, int H, int gy0, int gx0, int N,
                          const int *has, float *const *sendbuf, const float *const *halo,
                          const pc_prequest_t *const *sq, const pc_prequest_t *const *rq) {
  if (lx % kStrip || ly % H || H < kRB || H % kRB) return -1;
  JacobiRank d{};
  d.grid[0] = grid0;
  d.grid[1] = grid1;
  d.ly = ly;
  d.lx = lx;
  d.H = H;
  d.gy0 = gy0;
  d.gx0 = gx0;
  d.N = N;
  for (int i = 0; i < 4; ++i) {
    d.has[i] = has[i];
    d.sendbuf[i] = sendbuf[i];
    d.halo[i] = halo[i];
    if (has[i]) {
      d.sq[i] = *sq[i];
      d.rq[i] = *rq[i];
    }
  }
  d.nsegR = lx / kStrip;
  d.nsegC = ly / H;
  d.tiles = (ly / H) * (lx / kStrip);
  *(JacobiRank *)out = d;
  return 0;
}

}  // extern "C"
