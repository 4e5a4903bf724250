// libpc device kernels (sm_100a): ENGINE-mode p2p copy, stream-ordered waits,
// epoch / ready-to-receive control kernels, host-binding Pready kernels, and
// the (dtype, op) switch onto the allreduce engines of engine.cuh (compiled
// per instantiation in engine_inst.cu).
#include "engine.cuh"

namespace pc {
namespace {

using namespace pc_detail;

// ---------------------------------------------------------------------------
// ENGINE copy mode of partitioned send: unit = (transport partition t, slice s).
// ---------------------------------------------------------------------------
// Each warp sweeps up to kMaxActive of its units at a time (Alg 2 style):
// every unit found ready in a sweep is copied, then ONE fence publishes the
// whole set — with block-sized transport partitions (8 KiB) a fence per unit
// was most of the engine's time.  A transport partition of one slice needs
// no slice counter: its warp alone completes it.
__global__ void __launch_bounds__(kEngineBlock) p2p_engine(P2pEngineArgs a) {
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int W = (gridDim.x * blockDim.x) >> 5;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t e = *(const volatile uint32_t *)a.epoch;  // device epoch word (graph-replayable)
  bool rtr_ok = false;
  // Small transport partitions (one slice of <= 512 B, 8-B aligned: thread /
  // warp granularity): each LANE owns a unit — 32 ready flags polled at once,
  // each lane copies its own unit with 16-B (or 8-B) vectors, one warp-wide release,
  // then every lane signals its own unit (the 8-unit warp-cooperative sweep
  // below spent a poll round trip per 8 units of a few hundred bytes).
  const uint64_t ub = (uint64_t)a.agg * a.part_bytes;
  const uintptr_t bal = reinterpret_cast<uintptr_t>(a.sbuf) | reinterpret_cast<uintptr_t>(a.peer_rbuf);
  const bool v16 = (ub & 15) == 0 && (bal & 15) == 0;  // else 8-B vectors (thread granularity: 8-B units)
  if (a.ns == 1 && !a.xpart && ub <= 512 && (ub & 7) == 0 && (bal & 7) == 0) {
    for (int j0 = 0; gw + j0 * W < a.nunits; j0 += 32) {
      const int x = gw + (j0 + (int)lane) * W;  // this lane's unit = transport partition x
      uint32_t pending = __ballot_sync(0xffffffffu, x < a.nunits);
      Idle idle;
      while (pending) {
        const bool rdy = ((pending >> lane) & 1u) && reached(ld_acquire_gpu(a.ready + x), e);
        const uint32_t ready = __ballot_sync(0xffffffffu, rdy) & pending;
        if (!ready) {
          if (!idle.wait(a.err, a.timeout_ms, gw)) return;
          continue;
        }
        idle.progressed();
        if (!rtr_ok) {
          if (!warp_wait(a.rtr, e, a.err, a.timeout_ms, -1, a.sys)) return;
          rtr_ok = true;
        }
        if (rdy) {
          const int rem = a.partitions - x * a.agg;
          const uint64_t len = (uint64_t)(rem < a.agg ? rem : a.agg) * a.part_bytes;
          const uint8_t *src = a.sbuf + (uint64_t)x * ub;
          uint8_t *dst = a.peer_rbuf + (uint64_t)x * ub;
          uint64_t b = 0;
          if (v16)
            for (; b + 16 <= len; b += 16)
              *reinterpret_cast<uint4 *>(dst + b) = __ldcg(reinterpret_cast<const uint4 *>(src + b));
          for (; b + 8 <= len; b += 8)
            *reinterpret_cast<uint2 *>(dst + b) = __ldcg(reinterpret_cast<const uint2 *>(src + b));
          for (; b < len; ++b) dst[b] = src[b];  // a ragged last transport partition
        }
        fence_release(a.sys);  // each lane's copies, before its own signal
        if (rdy) {
          signal_transport(a.peer_flags, x, e, 0u, a.partitions, a.agg, a.part_bytes, a.peer_part_bytes);
          st_relaxed_gpu(a.sent + x, e);
        }
        __syncwarp();
        pending &= ~ready;
      }
    }
    return;
  }
  for (int j0 = 0; gw + j0 * W < a.nunits; j0 += kMaxActive) {
    uint32_t pending = 0;
#pragma unroll
    for (int j = 0; j < kMaxActive; ++j)
      if (gw + (j0 + j) * W < a.nunits) pending |= 1u << j;
    Idle idle;
    while (pending) {
      // poll: lane j looks at unit j's ready flag (all polls in flight together)
      bool rdy = false;
      if (lane < (uint32_t)kMaxActive && ((pending >> lane) & 1u)) {
        const int t = (gw + (j0 + (int)lane) * W) / a.ns;
        rdy = reached(ld_acquire_gpu(a.ready + t), e);
      }
      const uint32_t ready = __ballot_sync(0xffffffffu, rdy) & pending;
      if (!ready) {
        if (!idle.wait(a.err, a.timeout_ms, gw)) return;
        continue;
      }
      idle.progressed();
      if (!rtr_ok) {
        if (!warp_wait(a.rtr, e, a.err, a.timeout_ms, -1, a.sys)) return;
        rtr_ok = true;
      }
      for (int j = 0; j < kMaxActive; ++j) {
        if (!((ready >> j) & 1u)) continue;
        const int x = gw + (j0 + j) * W;
        const int t = x / a.ns, s = x % a.ns;
        const int rem = a.partitions - t * a.agg;
        const uint64_t len = (uint64_t)(rem < a.agg ? rem : a.agg) * a.part_bytes;
        const uint64_t off = (uint64_t)t * a.agg * a.part_bytes;
        const uint64_t slo = (uint64_t)s * a.slice_bytes;
        const uint64_t n = slo < len ? min(a.slice_bytes, len - slo) : 0;
        if (n) warp_copy(a.peer_rbuf + off + slo, a.sbuf + off + slo, (int64_t)n);
      }
      fence_release(a.sys);  // one cumulative fence for every copy of this sweep
      __syncwarp();
      if (lane == 0) {
        for (int j = 0; j < kMaxActive; ++j) {
          if (!((ready >> j) & 1u)) continue;
          const int t = (gw + (j0 + j) * W) / a.ns;
          const bool last = a.ns == 1 || atom_add_acq_rel_gpu(a.donecnt + t, 1) + 1 == e * (uint32_t)a.ns;
          if (last && a.ns > 1) fence_release(a.sys);  // the other slices' copies (acquired by the add) too
          if (last) {
            signal_transport(a.peer_flags, t, e, a.xpart, a.partitions, a.agg, a.part_bytes, a.peer_part_bytes);
            st_relaxed_gpu(a.sent + t, e);  // (after the fence: the copies are delivered)
          }
        }
      }
      __syncwarp();
      pending &= ~ready;
    }
  }
}

// Bulk wait until words[0 .. n-1] have all reached `target` (participant idx
// of nthr, grid-stride): relaxed 16-B loads of 4 words each — one round trip
// for the whole range once everything has arrived, instead of one dependent
// acquire per word — a bounded acquire spin only on words still behind, then
// one acquire fence per participant for the words it saw relaxed (the
// "ld.relaxed; fence.acquire" pattern: an L1 invalidation, no MEMBAR).  Words is 4-B aligned.
__device__ __forceinline__ bool wait_words_range(const uint32_t *w, int n, uint32_t target, int sys, int32_t *err,
                                                 uint32_t tmo, uint32_t idx, uint32_t nthr) {
  int head = (int)(((16u - (uint32_t)(reinterpret_cast<uintptr_t>(w) & 15u)) & 15u) >> 2);
  if (head > n) head = n;
  auto spin = [&](int i) {
    return sys ? spin_geq<true>(w + i, target, err, tmo, i) : spin_geq<false>(w + i, target, err, tmo, i);
  };
  for (int i = (int)idx; i < head; i += (int)nthr)
    if (!spin(i)) return false;
  const int nv = (n - head) >> 2;
  const uint4 *v = reinterpret_cast<const uint4 *>(w + head);
  bool relaxed = false;
  for (int k = (int)idx; k < nv; k += (int)nthr) {
    const uint4 x = sys ? ld_relaxed_sys_v4(v + k) : ld_relaxed_gpu_v4(v + k);
    relaxed = true;
    const uint32_t xs[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
    for (int j = 0; j < 4; ++j)
      if (!reached(xs[j], target) && !spin(head + 4 * k + j)) return false;
  }
  for (int i = head + 4 * nv + (int)idx; i < n; i += (int)nthr)
    if (!spin(i)) return false;
  if (relaxed) fence_acquire(sys);
  return true;
}

__device__ __forceinline__ void wait_words_body(const uint32_t *words, int n, const uint32_t *epoch, uint32_t mul,
                                                const uint32_t *layout, int partitions, int32_t *err, uint32_t tmo,
                                                int sys, const uint32_t *rtr, uint32_t bid, uint32_t nb) {
  __shared__ int s_n;
  const uint32_t target = *(const volatile uint32_t *)epoch * mul;
  // LL sender: its epoch completes only once the receiver posted ready-to-
  // receive for this epoch (acquire), i.e. finished reading epoch e-1's lines,
  // whose parity epoch e+1 reuses (ll_push, R29)
  if (rtr && bid == 0 && threadIdx.x == 32) spin_geq<true>(rtr, target, err, tmo, -3);
  if (threadIdx.x == 0) {
    int nn = n;
    if (layout) {
      // receiver: the sender publishes g at pc_prequest_create
      const uint64_t t0 = globaltimer();
      uint32_t g;
      while ((g = *(const volatile uint32_t *)layout) == 0) {
        if (aborted(err)) break;
        if (tmo && globaltimer() - t0 > (uint64_t)tmo * 1000000ull) {
          set_error(err, PC_DEV_ERR_TIMEOUT, -2);
          break;
        }
        __nanosleep(256);
      }
      nn = g ? (partitions + (int)g - 1) / (int)g : 0;
    }
    s_n = nn;
  }
  __syncthreads();
  wait_words_range(words, s_n, target, sys, err, tmo, bid * blockDim.x + threadIdx.x, nb * blockDim.x);
}

__global__ void wait_words_kernel(const uint32_t *words, int n, const uint32_t *epoch, uint32_t mul,
                                  const uint32_t *layout, int partitions, int32_t *err, uint32_t tmo, int sys,
                                  const uint32_t *rtr) {
  wait_words_body(words, n, epoch, mul, layout, partitions, err, tmo, sys, rtr, blockIdx.x, gridDim.x);
}

// Receive-side MPI_Wait / MPI_Test for a request whose sender may push LL
// lines (PC_COPY_LL): the layout word tells which protocol the sender chose.
// LL: every thread owns lines i = (p, j) of the grid-stride range, waits (or,
// in test mode, checks once) until the line carries this epoch in both halves
// and unpacks its payload bytes into recvbuf.  Flags: block 0 waits on the
// transport flags exactly as wait_words_kernel.  Test mode (pending != null):
// no spinning; every line / flag not there yet adds 1 to *pending.
// (block `bid` of the `nb` blocks serving this request)
__device__ __forceinline__ void recv_wait_body(const pc_prequest_t &q, int32_t *pending, uint32_t bid, uint32_t nb) {
  __shared__ uint32_t s_g;
  const uint32_t e = *(const volatile uint32_t *)q.epoch;
  if (threadIdx.x == 0) {
    const uint64_t t0 = globaltimer();
    uint32_t g;
    while ((g = *(const volatile uint32_t *)q.layout) == 0) {  // the sender publishes g at pc_prequest_create
      if (pending || aborted(q.err)) break;
      if (q.timeout_ms && globaltimer() - t0 > (uint64_t)q.timeout_ms * 1000000ull) {
        set_error(q.err, PC_DEV_ERR_TIMEOUT, -2);
        break;
      }
      __nanosleep(256);
    }
    s_g = g;
  }
  __syncthreads();
  const uint32_t g = s_g;
  if (g == 0) {
    if (pending && bid == 0 && threadIdx.x == 0) atomicAdd(pending, 1);
    return;
  }
  if (g & PC_LAYOUT_LL) {
    const uint32_t nl = q.ll_lines;
    const uint64_t nlines = (uint64_t)q.partitions * nl;
    const uint8_t *base = q.ll + (uint64_t)(e & 1) * nlines * 16ull;
    const uint64_t t0 = globaltimer();
    for (uint64_t i = (uint64_t)bid * blockDim.x + threadIdx.x; i < nlines; i += (uint64_t)nb * blockDim.x) {
      ulonglong2 v = ld_ll(base + 16ull * i, q.sys_scope);
      uint32_t n = 0;
      while ((uint32_t)(v.x >> 32) != e || (uint32_t)(v.y >> 32) != e) {
        if (pending) break;
        if ((++n & 127) == 0) {
          if (aborted(q.err)) return;
          if (q.timeout_ms && globaltimer() - t0 > (uint64_t)q.timeout_ms * 1000000ull) {
            set_error(q.err, PC_DEV_ERR_TIMEOUT, (int)(i / nl));
            return;
          }
          __nanosleep(128);
        }
        v = ld_ll(base + 16ull * i, q.sys_scope);
      }
      if ((uint32_t)(v.x >> 32) != e || (uint32_t)(v.y >> 32) != e) {
        atomicAdd(pending, 1);
        continue;
      }
      const uint64_t p = i / nl;
      const uint32_t j = (uint32_t)(i % nl);
      const uint32_t nb = ll_nbytes(q.part_bytes, j);
      if (nb) st_payload8(q.rbuf + p * q.part_bytes + 8ull * j, (v.x & 0xffffffffull) | (v.y << 32), nb);
    }
    return;
  }
  // equal partitionings: one flag per send transport partition (target e);
  // different ones (R30): one counter per receive partition (e * overlaps)
  const bool xp = (g & PC_LAYOUT_XP) != 0;
  const int nt = xp ? q.partitions : (q.partitions + (int)g - 1) / (int)g;
  if (!xp && !pending) {  // MPI_Wait, uniform target: the bulk wait over every block
    wait_words_range(q.flags, nt, e, q.sys_scope, q.err, q.timeout_ms, bid * blockDim.x + threadIdx.x,
                     nb * blockDim.x);
    return;
  }
  for (int i = (int)(bid * blockDim.x + threadIdx.x); i < nt; i += (int)(nb * blockDim.x)) {
    const uint32_t target = xp ? e * xp_need((uint64_t)i, q.part_bytes, g & PC_LAYOUT_G, q.peer_part_bytes) : e;
    if (pending) {
      if (!reached(ld_acquire_scope(q.flags + i, q.sys_scope), target)) atomicAdd(pending, 1);
      continue;
    }
    bool ok = q.sys_scope ? spin_geq<true>(q.flags + i, target, q.err, q.timeout_ms, i)
                          : spin_geq<false>(q.flags + i, target, q.err, q.timeout_ms, i);
    if (!ok) break;
  }
}

__global__ void recv_wait_kernel(pc_prequest_t q, int32_t *pending) { recv_wait_body(q, pending, blockIdx.x, gridDim.x); }

// pc_waitall_on_stream: request k's wait runs on its own block range (block
// ranges are uniform per block, so the bodies' barriers are block-uniform).
__global__ void wait_all_kernel(WaitAllArgs a) {
  int k = 0;
  while (k + 1 < a.n && (int)blockIdx.x >= a.block_start[k + 1]) ++k;
  const pc_prequest_t &q = a.q[k];
  const uint32_t bid = blockIdx.x - a.block_start[k], nb = a.block_start[k + 1] - a.block_start[k];
  if (q.kind == PC_KIND_PSEND) {
    wait_words_body(q.sent, q.ntransport, q.epoch, 1, nullptr, q.partitions, q.err, q.timeout_ms, 0,
                    q.copy == PC_COPY_LL ? q.rtr : nullptr, bid, nb);
  } else {
    recv_wait_body(q, nullptr, bid, nb);
  }
}

// Host pc_parrived of a receive request: the device binding, run by one thread
// (for LL it also unpacks the partition's lines into recvbuf).
__global__ void parrived_kernel(pc_prequest_t q, int partition, int32_t *out) {
  out[0] = pc_parrived(q, partition);
}

__global__ void set_word_kernel(uint32_t *addr, uint32_t v) { st_release_sys(addr, v); }

// pc_start: the epoch lives on the device and is advanced in stream order, so
// a captured CUDA graph replays correct epochs (the host never writes it).
__global__ void epoch_bump_kernel(uint32_t *epoch) { *epoch = *epoch + 1; }

__global__ void ctl_kernel(CtlArgs a) {
  const int i = threadIdx.x;
  if (i >= a.n) return;
  uint32_t *ep = const_cast<uint32_t *>(a.epoch[i]);
  if (!a.dst[i]) {
    *ep = *ep + 1;
  } else {
    const uint32_t e = *(const volatile uint32_t *)ep;
    if (a.sys[i])
      st_release_sys(a.dst[i], e);
    else
      st_release_gpu(a.dst[i], e);
  }
}

// pc_pbuf_prepare: ready-to-receive = this rank's current epoch, written into
// every producer's RTR slot (remote stores; release so that everything this
// rank did to the buffers before is ordered first).
__global__ void rtr_kernel(RtrArgs a) {
  const uint32_t e = *(const volatile uint32_t *)a.epoch;
  for (int i = 0; i < a.n; ++i) {
    if (a.sys)
      st_release_sys(a.dst[i], e);
    else
      st_release_gpu(a.dst[i], e);
  }
}

__global__ void pready_all_kernel(PreadyAllArgs a) {
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int W = (gridDim.x * blockDim.x) >> 5;
  int base = 0;
  for (int k = 0; k < a.n; ++k) {
    const int np = a.q[k].partitions;
    // global index base + j is taken by warp (base + j) mod W
    for (int j = ((gw - base) % W + W) % W; j < np; j += W) pc_pready_warp(j, a.q[k]);
    base += np;
  }
}

// One block: (1) every request's epoch e <- e + 1, (2) every ready-to-receive
// write of the new epoch into the producers' RTR words, (3) optionally the
// user's Pready (S_0) of every partition of every allreduce-kind request.
// Barriers order the phases (all in one block, so CTA-scope visibility).
__global__ void __launch_bounds__(1024) epoch_all_kernel(EpochAllArgs a) {
  __shared__ uint32_t esh[kMaxPreadyAll];  // the new epochs: no dependent global reload per RTR / request
  const int t = threadIdx.x;
  if (t < a.n) {
    const uint32_t e = a.epoch[t][0] + 1;
    a.epoch[t][0] = e;
    esh[t] = e;
  }
  __syncthreads();
  if (t < a.nrtr) {
    const uint32_t e = esh[a.rtr_req[t]];
    if ((a.rtr_sysmask >> t) & 1)
      st_release_sys(a.rtr_dst[t], e);
    else
      st_release_gpu(a.rtr_dst[t], e);
  }
  if (!a.pready) return;
  // S_0 of every partition: ready[u] = e.  No fences: the user's data was
  // written by kernels earlier in stream order, and the only reader of
  // ready[] is this rank's engine, launched after this kernel in stream order
  // (kernel boundaries order both), so plain stores spread over the block
  // replace one release per partition.
  for (int k = 0; k < a.n; ++k) {
    const uint32_t e = esh[k];
    uint32_t *ready = a.ready[k];
    for (int j = t; j < a.partitions[k]; j += blockDim.x) st_relaxed_gpu(ready + j, e);
  }
}

// pc_epoch_all over any number of requests: the three barrier-ordered
// phases of epoch_all_kernel with the lists in device memory.  The new epochs
// are kept in shared memory (no dependent global loads per RTR / Pready);
// every thread owns whole requests for the Pready of small ones, the block
// sweeps the few large ones together.
constexpr int kEpochBatchSmem = 8192;
__global__ void __launch_bounds__(1024) epoch_batch_kernel(EpochBatchArgs a) {
  __shared__ uint32_t esh[kEpochBatchSmem];
  const int t = threadIdx.x;
  for (int i = t; i < a.n; i += blockDim.x) {
    uint32_t *ep = a.ent[i].epoch;
    const uint32_t e = *ep + 1;
    *ep = e;
    if (i < kEpochBatchSmem) esh[i] = e;
  }
  __syncthreads();
  auto epoch = [&](int i) -> uint32_t {
    return i < kEpochBatchSmem ? esh[i] : *(const volatile uint32_t *)a.ent[i].epoch;
  };
  // ready-to-receive: one fence per thread at the strongest scope it stores
  // at, then relaxed stores (the earlier consumers of each recvbuf finished
  // in earlier kernels of this stream)
  bool fsys = false, fgpu = false;
  for (int k = t; k < a.nrtr; k += blockDim.x) {
    const RtrEnt r = a.rtr[k];
    if (r.sys) {
      if (!fsys) fence_release(1);
      fsys = true;
      st_relaxed_sys(r.dst, epoch(r.req));
    } else {
      if (!fgpu && !fsys) fence_release(0);
      fgpu = true;
      st_relaxed_gpu(r.dst, epoch(r.req));
    }
  }
  if (!a.pready) return;
  for (int i = t; i < a.n; i += blockDim.x) {  // S_0 of every partition (ordering as in epoch_all_kernel)
    const EpochEnt en = a.ent[i];
    if (!en.ready || en.partitions > kEpochSmallParts) continue;
    const uint32_t e = epoch(i);
    for (int j = 0; j < en.partitions; ++j) st_relaxed_gpu(en.ready + j, e);
  }
  for (int b = 0; b < a.nbig; ++b) {
    const int i = a.big[b];
    const EpochEnt en = a.ent[i];
    const uint32_t e = epoch(i);
    for (int j = t; j < en.partitions; j += blockDim.x) st_relaxed_gpu(en.ready + j, e);
  }
}

__global__ void pready_range_kernel(pc_prequest_t q, int lo, int hi) {
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int W = (gridDim.x * blockDim.x) >> 5;
  for (int p = lo + gw; p <= hi; p += W) pc_pready_warp(p, q);
}

}  // namespace


// (dtype, op) -> the EngineLaunch instantiation compiled in engine_inst.cu
template <typename F>
static int dispatch(int dtype, int op, F f) {
  using std::integral_constant;
#define PC_DISPATCH_OPS(DTV)                                                                    \
  do {                                                                                          \
    if (op == PC_OP_SUM) return f(EngineLaunch<DTV, 0>());                                      \
    if (op == PC_OP_MAX) return f(EngineLaunch<DTV, 1>());                                      \
    return f(EngineLaunch<DTV, 2>());                                                           \
  } while (0)
  switch (dtype) {
    case PC_INT32: PC_DISPATCH_OPS(0);
    case PC_FLOAT32: PC_DISPATCH_OPS(1);
    case PC_FLOAT64: PC_DISPATCH_OPS(3);
    case PC_BF16: PC_DISPATCH_OPS(4);
    default: return PC_ERR_ARG;
  }
#undef PC_DISPATCH_OPS
}

std::atomic<uint64_t> g_launches{0};

int launch_ring_engine(const RingArgs &a, int warps, cudaStream_t s) {
  return dispatch(a.dtype, a.op, [&](auto E) { return decltype(E)::ring(a, warps, s); });
}

int launch_rd_engine(const RdArgs &a, int warps, cudaStream_t s) {
  return dispatch(a.dtype, a.op, [&](auto E) { return decltype(E)::rd(a, warps, s); });
}

int launch_direct_engine(const DirectArgs &a, int warps, cudaStream_t s, bool thin) {
  return dispatch(a.dtype, a.op, [&](auto E) { return decltype(E)::direct(a, warps, s, thin); });
}

// allgather / broadcast move bytes only: any instantiation serves (fp32 sum)
static int coll_dtype(const CollArgs &a) { return a.coll == PC_COLL_REDUCE_SCATTER ? a.dtype : PC_FLOAT32; }
static int coll_op(const CollArgs &a) { return a.coll == PC_COLL_REDUCE_SCATTER ? a.op : PC_OP_SUM; }

int launch_coll_engine(const CollArgs &a, int warps, cudaStream_t s) {
  return dispatch(coll_dtype(a), coll_op(a), [&](auto E) { return decltype(E)::coll(a, warps, s); });
}

int launch_coll_engine_group(const CollGroupArgs &g, int warps, cudaStream_t s) {
  CollGroupArgs h = g;
  int blocks = 0;
  for (int k = 0; k < g.n; ++k) {
    h.block_start[k] = blocks;
    blocks += grid_for(warps, g.a[k].nunits);
  }
  return dispatch(coll_dtype(g.a[0]), coll_op(g.a[0]), [&](auto E) { return decltype(E)::coll_group(h, blocks, s); });
}

int launch_ring_engine_group(const RingGroupArgs &g, int warps, cudaStream_t s) {
  RingGroupArgs h = g;
  int blocks = 0;
  for (int k = 0; k < g.n; ++k) {
    h.block_start[k] = blocks;
    blocks += grid_for(warps, g.a[k].nunits);
  }
  return dispatch(g.a[0].dtype, g.a[0].op, [&](auto E) { return decltype(E)::ring_group(h, blocks, s); });
}

int launch_rd_engine_group(const RdGroupArgs &g, int warps, cudaStream_t s) {
  RdGroupArgs h = g;
  int blocks = 0;
  for (int k = 0; k < g.n; ++k) {
    h.block_start[k] = blocks;
    blocks += grid_for(warps, g.a[k].nunits);
  }
  return dispatch(g.a[0].dtype, g.a[0].op, [&](auto E) { return decltype(E)::rd_group(h, blocks, s); });
}

int launch_direct_engine_group(const DirectGroupArgs &g, int warps, cudaStream_t s, bool thin) {
  DirectGroupArgs h = g;
  int blocks = 0;
  for (int k = 0; k < g.n; ++k) {
    h.block_start[k] = blocks;
    blocks += grid_for(warps, g.a[k].nunits);
  }
  return dispatch(g.a[0].dtype, g.a[0].op, [&](auto E) { return decltype(E)::direct_group(h, blocks, s, thin); });
}

int launch_direct_engine_batch(const DirectBatchArgs &b, int dtype, int op, int blocks, cudaStream_t s, bool thin) {
  return dispatch(dtype, op, [&](auto E) { return decltype(E)::direct_batch(b, blocks, s, thin); });
}

int launch_p2p_engine(const P2pEngineArgs &a, int warps, cudaStream_t s) {
  p2p_engine<<<grid_for(warps, a.nunits), kEngineBlock, 0, s>>>(a);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

int launch_wait_words(const uint32_t *words, int n, const uint32_t *epoch, uint32_t mul, const uint32_t *layout,
                      int partitions, int32_t *err, uint32_t timeout_ms, cudaStream_t s, bool sys,
                      const uint32_t *rtr) {
  // (a receiver's n is an upper bound: the sender's g may aggregate)
  wait_words_kernel<<<wait_words_blocks(n), 256, 0, s>>>(words, n, epoch, mul, layout, partitions, err, timeout_ms,
                                                         sys ? 1 : 0, rtr);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

// Flag words of a request: at most one 256-thread block per 1024 words, at
// most one block per SM (spinning blocks never fill the GPU: DESIGN.md §7).
int wait_words_blocks(int n) {
  static int sms = 0;  // (one device per process in this library's use; B200: 148)
  if (!sms) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) !=
                                                   cudaSuccess || sms < 1)
      sms = 148;
  }
  const int b = (n + 1023) / 1024;
  return b < 1 ? 1 : (b > sms ? sms : b);
}

int recv_wait_blocks(const pc_prequest_t &q) {
  int blocks = wait_words_blocks(q.partitions);
  if (q.ll_lines) {
    const int64_t lines = (int64_t)q.partitions * q.ll_lines;
    blocks = (int)((lines + 255) / 256);
    if (blocks > 4 * 148) blocks = 4 * 148;
    if (blocks < 1) blocks = 1;
  }
  return blocks;
}

int launch_wait_all(const WaitAllArgs &a, cudaStream_t s) {
  wait_all_kernel<<<a.block_start[a.n], 256, 0, s>>>(a);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

int launch_recv_wait(const pc_prequest_t &q, int32_t *pending, cudaStream_t s) {
  recv_wait_kernel<<<recv_wait_blocks(q), 256, 0, s>>>(q, pending);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

int launch_parrived(const pc_prequest_t &q, int partition, int32_t *out, cudaStream_t s) {
  parrived_kernel<<<1, 1, 0, s>>>(q, partition, out);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

int launch_ctl(const CtlArgs &a, cudaStream_t s) {
  if (a.n <= 0) return 0;
  ctl_kernel<<<1, kMaxCtl, 0, s>>>(a);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

int launch_epoch_bump(uint32_t *epoch, cudaStream_t s) {
  epoch_bump_kernel<<<1, 1, 0, s>>>(epoch);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

int launch_rtr(const RtrArgs &a, cudaStream_t s) {
  rtr_kernel<<<1, 1, 0, s>>>(a);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

// Stream-ordered wait for *addr >= value (fallback for cuStreamWaitValue32):
// one thread, bounded by tmo_ms (then it gives up; the caller's request has
// its own timeouts downstream).
__global__ void wait_value_kernel(const uint32_t *addr, uint32_t value, int sys, uint32_t tmo_ms) {
  const uint64_t t0 = globaltimer();
  while (!reached(sys ? ld_acquire_sys(addr) : ld_acquire_gpu(addr), value)) {
    if (tmo_ms && globaltimer() - t0 > (uint64_t)tmo_ms * 1000000ull) return;
    __nanosleep(256);
  }
}

int launch_wait_value(const uint32_t *addr, uint32_t value, cudaStream_t s, bool sys, uint32_t tmo_ms) {
  wait_value_kernel<<<1, 1, 0, s>>>(addr, value, sys ? 1 : 0, tmo_ms);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

// Progression engine (PC_COPY_HOST): after the stream-ordered copy of
// transport partitions [t, t+n), publish their arrival at the receiver and
// their completion at the sender.
__global__ void pe_signal_kernel(uint32_t *peer_flags, uint32_t *sent, int n, uint32_t v, int sys) {
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    if (sys)
      st_release_sys(peer_flags + i, v);
    else
      st_release_gpu(peer_flags + i, v);
    st_release_gpu(sent + i, v);
  }
}

// With lazy module loading (the CUDA 12 default) the FIRST launch of a kernel
// may wait for the device to go idle while it loads — fatal when that launch
// comes from the progress thread while the user's wait kernels spin on the
// very flags it is about to write.  Load the progress thread's kernels up
// front (pc_prequest_create, before any epoch runs).
// Every library kernel, loaded at pc_comm_create: no first launch may then
// stall behind kernels that spin on the work it is about to do (engines and
// waits are launched while producers and waits of other ranks run).
int kernels_preload() {
  cudaFuncAttributes fa;
  PC_CUDA(cudaFuncGetAttributes(&fa, p2p_engine));
  PC_CUDA(cudaFuncGetAttributes(&fa, wait_words_kernel));
  PC_CUDA(cudaFuncGetAttributes(&fa, recv_wait_kernel));
  PC_CUDA(cudaFuncGetAttributes(&fa, wait_all_kernel));
  PC_CUDA(cudaFuncGetAttributes(&fa, parrived_kernel));
  PC_CUDA(cudaFuncGetAttributes(&fa, set_word_kernel));
  PC_CUDA(cudaFuncGetAttributes(&fa, epoch_bump_kernel));
  PC_CUDA(cudaFuncGetAttributes(&fa, ctl_kernel));
  PC_CUDA(cudaFuncGetAttributes(&fa, rtr_kernel));
  PC_CUDA(cudaFuncGetAttributes(&fa, pready_all_kernel));
  PC_CUDA(cudaFuncGetAttributes(&fa, epoch_all_kernel));
  PC_CUDA(cudaFuncGetAttributes(&fa, epoch_batch_kernel));
  PC_CUDA(cudaFuncGetAttributes(&fa, pready_range_kernel));
  if (int rc = pe_kernels_preload()) return rc;
  for (int dt : {PC_INT32, PC_FLOAT32, PC_FLOAT64, PC_BF16})
    for (int op : {PC_OP_SUM, PC_OP_MAX, PC_OP_MIN})
      if (int rc = dispatch(dt, op, [&](auto E) { return decltype(E)::preload(); })) return rc;
  return 0;
}

int pe_kernels_preload() {
  cudaFuncAttributes fa;
  PC_CUDA(cudaFuncGetAttributes(&fa, pe_signal_kernel));
  PC_CUDA(cudaFuncGetAttributes(&fa, wait_value_kernel));
  return 0;
}

int launch_pe_signal(uint32_t *peer_flags, uint32_t *sent, int n, uint32_t v, bool sys, cudaStream_t s) {
  pe_signal_kernel<<<1, 256, 0, s>>>(peer_flags, sent, n, v, sys ? 1 : 0);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

int launch_set_word(uint32_t *addr, uint32_t value, cudaStream_t s) {
  set_word_kernel<<<1, 1, 0, s>>>(addr, value);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

int launch_pready_all(const PreadyAllArgs &a, cudaStream_t s) {
  int total = 0;
  for (int k = 0; k < a.n; ++k) total += a.q[k].partitions;
  int blocks = (total + 7) / 8;
  if (blocks > 148) blocks = 148;
  if (blocks < 1) blocks = 1;
  pready_all_kernel<<<blocks, 256, 0, s>>>(a);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

int launch_epoch_batch(const EpochBatchArgs &a, cudaStream_t s) {
  epoch_batch_kernel<<<1, 1024, 0, s>>>(a);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

int launch_epoch_all(const EpochAllArgs &a, cudaStream_t s) {
  epoch_all_kernel<<<1, 1024, 0, s>>>(a);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

int launch_pready_range(pc_prequest_t q, int lo, int hi, cudaStream_t s) {
  const int n = hi - lo + 1;
  int blocks = (n + 7) / 8;
  if (blocks > 148) blocks = 148;
  if (blocks < 1) blocks = 1;
  pready_range_kernel<<<blocks, 256, 0, s>>>(q, lo, hi);
  g_launches++;
  PC_CUDA(cudaGetLastError());
  return 0;
}

uint64_t launch_count() { return g_launches.load(); }

int engine_occupancy_ctas_per_sm(int *ctas) { return EngineLaunch<1, 0>::occupancy(ctas); }
int direct_occupancy_ctas_per_sm(int *ctas) { return EngineLaunch<1, 0>::occupancy_direct(ctas); }

}  // namespace pc
