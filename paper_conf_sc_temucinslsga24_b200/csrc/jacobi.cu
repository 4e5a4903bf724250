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
  int nsegR, nsegC;       // segments per slot: row halos (lx/W), column halos (ly/H)
  int tiles;              // (ly/H) * (lx/W): warps (mode 0) or CTAs (mode 1)
  int W;                  // columns per tile: 128 (mode 0, one warp) or the CTA strip (mode 1)
  int mode;               // 0 warp tiles (register sliding window), 1 CTA row pipeline (bulk copies)
  int trad;               // 1: traditional baseline (Listing 1): no Parrived / Pready in the kernel;
                          //    the host copies the staged edges between launches
};

__device__ __forceinline__ float stencil(float up, float dn, float lf, float rt) {
  return __fmul_rn(0.25f, __fadd_rn(__fadd_rn(up, dn), __fadd_rn(lf, rt)));
}

__device__ __forceinline__ float4 ld4(const float *p) { return __ldcg(reinterpret_cast<const float4 *>(p)); }

// Halo Parrived / Pready are kept out of line so the protocol's registers do
// not spill the stencil loop (ptxas: 0 spills with the 64-register cap).
__device__ __noinline__ void halo_wait(const JacobiRank &d, bool top, bool bot, bool left, bool right, int sx, int rb,
                                       int k) {
  if (top) pc_wait_arrived(d.rq[T], k * d.nsegR + sx);
  if (bot) pc_wait_arrived(d.rq[B], k * d.nsegR + sx);
  if (left) pc_wait_arrived(d.rq[L], k * d.nsegC + rb);
  if (right) pc_wait_arrived(d.rq[R], k * d.nsegC + rb);
}

__device__ __noinline__ void edge_pready(const JacobiRank &d, bool top, bool bot, bool left, bool right, int sx,
                                         int rb, int slot) {
  if (top) pc_pready_warp(slot * d.nsegR + sx, d.sq[T]);
  if (bot) pc_pready_warp(slot * d.nsegR + sx, d.sq[B]);
  if (left) pc_pready_warp(slot * d.nsegC + rb, d.sq[L]);
  if (right) pc_pready_warp(slot * d.nsegC + rb, d.sq[R]);
}

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
  if (lane == 0 && (top | bot | left | right)) halo_wait(d, top, bot, left, right, sx, rb, k);
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
  if (top | bot | left | right) edge_pready(d, top, bot, left, right, sx, rb, k + 1);
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

// ---------------------------------------------------------------------------
// Mode 1: CTA row pipeline.  A CTA of W/4 threads owns a tile of H rows x W
// columns (W up to 1024: 4 KiB contiguous per row, one float4 per thread) and
// slides down it.  Rows reach shared memory by bulk copies (cp.async.bulk, the
// TMA engine: one instruction per row, no per-lane address math) into a ring
// of NR row slots, each completing on its own mbarrier; thread 0 keeps the
// ring NR rows ahead, refilling after every batch of TB rows.  A row slot
// holds 4 pad floats on each side, so the left/right neighbours of the strip
// edge come with the row (or, on the rank edge, from the column halo, also
// bulk-copied).  Every grid element is read from HBM once and written once.
// ---------------------------------------------------------------------------
#ifndef PC_JACOBI_NR
#define PC_JACOBI_NR 16
#endif
constexpr int kNR = PC_JACOBI_NR;

__device__ __forceinline__ uint32_t smem_addr(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, uint32_t bytes) {
  asm volatile("{\n .reg .b64 st;\n mbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n}" ::"r"(smem_addr(b)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *b) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_addr(dst)),
               "l"(src), "r"(bytes), "r"(smem_addr(b))
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W_%=;\n}" ::"r"(
          smem_addr(b)),
      "r"(parity)
      : "memory");
}

__host__ __device__ constexpr size_t rows_smem_bytes(int W, int H) {
  return (size_t)kNR * (W + 8) * 4 + (size_t)2 * H * 4 + (size_t)(2 * kNR + 1) * 8;
}

__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
  asm volatile("{\n .reg .b64 st;\n mbarrier.arrive.shared::cta.b64 st, [%0];\n}" ::"r"(smem_addr(b)) : "memory");
}

// Warp-specialised: W/128 consumer warps compute (thread t owns columns
// 4t..4t+3 of the strip) and one producer warp keeps the ring full.  Slot s
// has a "full" barrier (1 arrival + the copy's bytes) and an "empty" barrier
// (one arrival per consumer warp once it has read the row), so no CTA-wide
// barrier sits on the row loop.
__device__ void tile_rows_iter(const JacobiRank &d, int tile, int k, uint8_t *smem) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int W = d.W, RW = W + 8, H = d.H, lx = d.lx, ly = d.ly;
  const int ncw = W / 128;  // consumer warps; warp ncw is the producer
  const int nstrip = lx / W;
  const int rb = tile / nstrip, sx = tile % nstrip;
  const int r0 = rb * H, x0 = sx * W;
  const bool top = rb == 0 && d.has[T], bot = (r0 + H == ly) && d.has[B];
  const bool left = sx == 0 && d.has[L], right = (sx == nstrip - 1) && d.has[R];
  const float *a = d.grid[k & 1];
  float *b = d.grid[(k + 1) & 1];
  float *ring = reinterpret_cast<float *>(smem);
  float *colL = ring + (size_t)kNR * RW, *colR = colL + H;
  uint64_t *full = reinterpret_cast<uint64_t *>(colR + H), *empty = full + kNR, *colbar = empty + kNR;
  const int nrows = H + 2;  // ring row j = local row r0 - 1 + j
  if (tid == 0) {
    for (int j = 0; j < kNR; ++j) {
      mbar_init(full + j, 1);
      mbar_init(empty + j, ncw);
    }
    mbar_init(colbar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == ncw) {  // ---------------- producer
    if (lane == 0) {
      const float *hT = d.halo[T] + (size_t)k * lx, *hB = d.halo[B] + (size_t)k * lx;
      const float *hL = d.halo[L] + (size_t)k * ly, *hR = d.halo[R] + (size_t)k * ly;
      auto halo_row = [&](int j) {
        const int r = r0 - 1 + j;
        return (r < 0 && d.has[T]) || (r >= ly && d.has[B]);
      };
      auto issue = [&](int j) {
        int r = r0 - 1 + j;
        float *dst = ring + (size_t)(j % kNR) * RW;
        const float *src;
        int off, n;
        if (halo_row(j)) {
          src = (r < 0 ? hT : hB) + x0, off = 4, n = W;
        } else {
          // outside the grid without a neighbour: the unused neighbour of a
          // Dirichlet row, any row will do
          r = r < 0 ? 0 : (r >= ly ? ly - 1 : r);
          const int lp = x0 > 0 ? 4 : 0, rp = x0 + W < lx ? 4 : 0;
          src = a + (size_t)r * lx + x0 - lp, off = 4 - lp, n = W + lp + rp;
        }
        mbar_expect_tx(full + j % kNR, (uint32_t)n * 4);
        bulk_g2s(dst + off, src, (uint32_t)n * 4, full + j % kNR);
      };
      const int first = min(kNR, nrows);
      for (int j = 0; j < first; ++j)  // grid rows first: they need no arrival
        if (!halo_row(j)) issue(j);
      // Parrived: the halo segments this tile reads (slot k), then their copies
      if ((top | bot | left | right) && !d.trad) {
        halo_wait(d, top, bot, left, right, sx, rb, k);
        asm volatile("fence.proxy.async.global;" ::: "memory");
      }
      for (int j = 0; j < first; ++j)
        if (halo_row(j)) issue(j);
      if (left | right) {
        mbar_expect_tx(colbar, (uint32_t)((left + right) * H * 4));
        if (left) bulk_g2s(colL, hL + r0, H * 4, colbar);
        if (right) bulk_g2s(colR, hR + r0, H * 4, colbar);
      }
      for (int j = kNR; j < nrows; ++j) {
        mbar_wait(empty + j % kNR, (uint32_t)(j / kNR - 1) & 1);
        issue(j);
      }
    }
  } else {  // ---------------- consumers
    const int c = 4 * tid;
    if (left | right) mbar_wait(colbar, 0);
    const int gx = d.gx0 + x0 + c;
    const bool colfix0 = gx == 0, colfix3 = gx + 3 == d.N - 1;
    const bool edgeL = tid == 0 && x0 == 0, edgeR = tid == W / 4 - 1 && x0 + W == lx;
    auto row = [&](int j) { return ring + (size_t)(j % kNR) * RW + 4; };
    auto release = [&](int j) {
      __syncwarp();
      if (lane == 0) mbar_arrive(empty + j % kNR);
    };
    mbar_wait(full + 0, 0);
    float4 up = *reinterpret_cast<const float4 *>(row(0) + c);
    release(0);
    mbar_wait(full + 1 % kNR, (1 / kNR) & 1);
    float4 cur = *reinterpret_cast<const float4 *>(row(1) + c);
    float lp = lane == 0 ? row(1)[c - 1] : 0.f, rp = lane == 31 ? row(1)[c + 4] : 0.f;
    release(1);
    float *sT = top ? d.sendbuf[T] + (size_t)(k + 1) * lx + x0 + c : nullptr;
    float *sB = bot ? d.sendbuf[B] + (size_t)(k + 1) * lx + x0 + c : nullptr;
    float *sL = (left && tid == 0) ? d.sendbuf[L] + (size_t)(k + 1) * ly : nullptr;
    float *sR = (right && edgeR) ? d.sendbuf[R] + (size_t)(k + 1) * ly : nullptr;
    float *out = b + (size_t)r0 * lx + x0 + c;
    const int gy0 = d.gy0 + r0, Nm1 = d.N - 1;
    for (int i = 1; i <= H; ++i, out += lx) {
      const int jn = i + 1;
      mbar_wait(full + jn % kNR, (uint32_t)(jn / kNR) & 1);
      const float *dr = row(jn);
      const float4 dn = *reinterpret_cast<const float4 *>(dr + c);
      const float dl = lane == 0 ? dr[c - 1] : 0.f, drt = lane == 31 ? dr[c + 4] : 0.f;
      release(jn);
      float lf = __shfl_up_sync(0xffffffffu, cur.w, 1);
      float rt = __shfl_down_sync(0xffffffffu, cur.x, 1);
      if (lane == 0) lf = lp;
      if (lane == 31) rt = rp;
      if (edgeL) lf = left ? colL[i - 1] : 0.f;
      if (edgeR) rt = right ? colR[i - 1] : 0.f;
      const int gy = gy0 + i - 1;
      float4 o;
      if (gy == 0 || gy == Nm1) {
        o = cur;  // Dirichlet row
      } else {
        o.x = colfix0 ? cur.x : stencil(up.x, dn.x, lf, cur.y);
        o.y = stencil(up.y, dn.y, cur.x, cur.z);
        o.z = stencil(up.z, dn.z, cur.y, cur.w);
        o.w = colfix3 ? cur.w : stencil(up.w, dn.w, cur.z, rt);
      }
      *reinterpret_cast<float4 *>(out) = o;
      if (sT && i == 1) *reinterpret_cast<float4 *>(sT) = o;  // local row 0
      if (sB && i == H) *reinterpret_cast<float4 *>(sB) = o;  // local row ly - 1
      if (sL) sL[r0 + i - 1] = o.x;
      if (sR) sR[r0 + i - 1] = o.w;
      up = cur;
      cur = dn;
      lp = dl;
      rp = drt;
    }
  }
  // Pready: push my edge segments of slot k+1 (INLINE copy by warp 0)
  if ((top | bot | left | right) && !d.trad) {
    __syncthreads();
    if (warp == 0) edge_pready(d, top, bot, left, right, sx, rb, k + 1);
  }
}

__device__ void tile_rows_init(const JacobiRank &d, int tile) {
  const int tid = threadIdx.x, nth = blockDim.x;
  const int W = d.W, H = d.H, lx = d.lx, ly = d.ly;
  const int nstrip = lx / W;
  const int rb = tile / nstrip, sx = tile % nstrip;
  const int r0 = rb * H, x0 = sx * W, c = 4 * tid;
  const float *a = d.grid[0];
  const bool top = rb == 0 && d.has[T], bot = (r0 + H == ly) && d.has[B];
  const bool left = sx == 0 && d.has[L], right = (sx == nstrip - 1) && d.has[R];
  if (top && c < W) *reinterpret_cast<float4 *>(d.sendbuf[T] + x0 + c) = ld4(a + x0 + c);
  if (bot && c < W) *reinterpret_cast<float4 *>(d.sendbuf[B] + x0 + c) = ld4(a + (size_t)(ly - 1) * lx + x0 + c);
  for (int r = r0 + tid; r < r0 + H; r += nth) {
    if (left) d.sendbuf[L][r] = __ldcg(a + (size_t)r * lx);
    if (right) d.sendbuf[R][r] = __ldcg(a + (size_t)r * lx + lx - 1);
  }
  if ((top | bot | left | right) && !d.trad) {
    __syncthreads();
    if (tid < 32) edge_pready(d, top, bot, left, right, sx, rb, 0);
  }
}

__global__ void __launch_bounds__(288) jacobi_rows_kernel(const JacobiRank *__restrict__ ranks,
                                                          const int *block_start, int nranks, int k, int init) {
  extern __shared__ __align__(128) uint8_t smem[];
  int q = 0;
  while (q + 1 < nranks && (int)blockIdx.x >= block_start[q + 1]) ++q;
  const JacobiRank &d = ranks[q];
  const int tile = blockIdx.x - block_start[q];
  if (tile >= d.tiles) return;
  if (init)
    tile_rows_init(d, tile);
  else
    tile_rows_iter(d, tile, k, smem);
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
// mode 0: blocks of 256 threads (8 warp tiles); mode 1: one CTA of W/4
// threads per tile with rows_smem_bytes(W, H) of dynamic shared memory.
int pcapp_jacobi_launch2(const void *ranks, const int *block_start, int nranks, int total_blocks, int k, int init,
                         int mode, int W, int H, cudaStream_t s) {
  if (mode == 0) {
    jacobi_kernel<<<total_blocks, 256, 0, s>>>((const JacobiRank *)ranks, block_start, nranks, k, init);
  } else {
    const size_t sm = rows_smem_bytes(W, H);
    static size_t configured = 0;
    if (sm > configured) {
      if (cudaFuncSetAttribute(jacobi_rows_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm) !=
          cudaSuccess)
        return -2;
      configured = sm;
    }
    jacobi_rows_kernel<<<total_blocks, W / 4 + 32, sm, s>>>((const JacobiRank *)ranks, block_start, nranks, k, init);
  }
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

int pcapp_jacobi_launch(const void *ranks, const int *block_start, int nranks, int total_blocks, int k, int init,
                        cudaStream_t s) {
  return pcapp_jacobi_launch2(ranks, block_start, nranks, total_blocks, k, init, 0, kStrip, 0, s);
}

// Fill one host-side descriptor (the caller copies the array to the device).
// mode 0: W must be 128 (one warp tile), H % kRB == 0; mode 1: W in
// {128, 256, 512, 1024} dividing lx, H % 4 == 0 (16-B column-halo copies).
int pcapp_jacobi_describe2(void *out, float *grid0, float *grid1, int ly, int lx, int H, int gy0, int gx0, int N,
                           const int *has, float *const *sendbuf, const float *const *halo,
                           const pc_prequest_t *const *sq, const pc_prequest_t *const *rq, int mode, int W) {
  if (mode == 0 && (W != kStrip || H < kRB || H % kRB)) return -1;
  if (mode == 1 && ((W != 128 && W != 256 && W != 512 && W != 1024) || H < 4 || H % 4)) return -1;
  if (mode != 0 && mode != 1) return -1;
  if (lx % W || ly % H) return -1;
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
    if (has[i] && sq[i] && rq[i]) {
      d.sq[i] = *sq[i];
      d.rq[i] = *rq[i];
    }
  }
  d.nsegR = lx / W;
  d.nsegC = ly / H;
  d.tiles = (ly / H) * (lx / W);
  d.W = W;
  d.mode = mode;
  *(JacobiRank *)out = d;
  return 0;
}

// Traditional baseline switch on a filled descriptor (mode 1 only): the
// kernel neither waits for halos nor Preadies its edges.
int pcapp_jacobi_set_traditional(void *desc, int trad) {
  JacobiRank *d = (JacobiRank *)desc;
  if (trad && d->mode != 1) return -1;
  d->trad = trad;
  return 0;
}

int pcapp_jacobi_describe(void *out, float *grid0, float *grid1, int ly, int lx, int H, int gy0, int gx0, int N,
                          const int *has, float *const *sendbuf, const float *const *halo,
                          const pc_prequest_t *const *sq, const pc_prequest_t *const *rq) {
  return pcapp_jacobi_describe2(out, grid0, grid1, ly, lx, H, gy0, gx0, N, has, sendbuf, halo, sq, rq, 0, kStrip);
}

}  // extern "C"
