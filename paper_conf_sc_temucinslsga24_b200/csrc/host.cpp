// libpc host runtime: comm bootstrap, request lifecycle, matching, schedules.
//
// Paper mapping (§IV-A/§IV-B):
//   pc_psend_init / pc_precv_init   MPI_Psend_init / MPI_Precv_init:
//                                   record parameters only (non-blocking)
//   pc_start                        MPI_Start: new epoch, stream-ordered
//   pc_pbuf_prepare                 MPIX_Pbuf_prepare: first
//                                   call = setup_t exchange + registration (here:
//                                   all-gather of request records + CUDA IPC
//                                   handles); every call = ready-to-receive
//   pc_prequest_create              MPIX_Prequest_create
//   pc_pallreduce_init              MPIX_Pallreduce_init (Alg 1)
//   pc_wait                         MPI_Wait (Alg 2 P:L178 runs on the GPU)
#include <cuda.h>
#include <cuda_runtime.h>
#include <unistd.h>

#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <string>
#include <tuple>

#include "pc_internal.h"

namespace pc {

static bool env_flag(const char *n) {
  const char *v = getenv(n);
  return v && *v && strcmp(v, "0") != 0;
}
static double env_double(const char *n, double dflt) {
  const char *v = getenv(n);
  return v && *v ? atof(v) : dflt;
}
static long env_long(const char *n, long dflt) {
  const char *v = getenv(n);
  if (!v || !*v) return dflt;
  return strtol(v, nullptr, 0);
}

void logf(const char *fmt, ...) {
  if (!env_flag("PC_DEBUG")) return;
  va_list ap;
  va_start(ap, fmt);
  fprintf(stderr, "[pc] ");
  vfprintf(stderr, fmt, ap);
  fprintf(stderr, "\n");
  va_end(ap);
}

int cuda_err(cudaError_t e, const char *what) {
  fprintf(stderr, "[pc] CUDA error %d (%s) in %s\n", (int)e, cudaGetErrorString(e), what);
  return e == cudaErrorMemoryAllocation ? PC_ERR_NOMEM : PC_ERR_CUDA;
}

// ------------------------------------------------------------------ driver entry points
typedef CUresult (*PFN_getAddrRange)(CUdeviceptr *, size_t *, CUdeviceptr);
typedef CUresult (*PFN_writeValue32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
static PFN_getAddrRange g_getAddrRange = nullptr;
static PFN_writeValue32 g_writeValue32 = nullptr;
static PFN_writeValue32 g_waitValue32 = nullptr;  // cuStreamWaitValue32 has the same signature
static std::once_flag g_drv_once;

static void load_driver_entry_points() {
  std::call_once(g_drv_once, [] {
    void *fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      g_getAddrRange = (PFN_getAddrRange)fn;
    fn = nullptr;
    if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &fn, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      g_writeValue32 = (PFN_writeValue32)fn;
    fn = nullptr;
    if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &fn, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      g_waitValue32 = (PFN_writeValue32)fn;
    cudaGetLastError();
  });
}

bool memops_available() {
  load_driver_entry_points();
  return g_writeValue32 != nullptr && !env_flag("PC_NO_MEMOPS");
}

int stream_write_u32(Comm *c, cudaStream_t s, uint32_t *addr, uint32_t value) {
  if (c->memops) {
    CUresult r = g_writeValue32((CUstream)s, (CUdeviceptr)addr, value, 0 /* with memory barrier */);
    if (r == CUDA_SUCCESS) return 0;
    logf("cuStreamWriteValue32 failed (%d); falling back to a 1-thread kernel", (int)r);
    c->memops = false;
  }
  return launch_set_word(addr, value, s);
}

// Stream-ordered "wait until *addr >= value" (wrap-unaware GEQ memop, or a
// 1-block bounded spin kernel when memops are unavailable).
int stream_wait_geq_u32(Comm *c, cudaStream_t s, const uint32_t *addr, uint32_t value, bool sys) {
  if (c->memops && g_waitValue32) {
    CUresult r = g_waitValue32((CUstream)s, (CUdeviceptr)addr, value, 0x0 /* CU_STREAM_WAIT_VALUE_GEQ */);
    if (r == CUDA_SUCCESS) return 0;
    logf("cuStreamWaitValue32 failed (%d); falling back to a wait kernel", (int)r);
  }
  return launch_wait_value(addr, value, s, sys, c->timeout_ms);
}

// ------------------------------------------------------------------ progression engine (PC_COPY_HOST)
// The paper's host Progression Engine as a
// comparison mode: device Pready stores the epoch into hready[t] (pinned host
// memory); this thread sees it and enqueues, on its own stream, (once per
// epoch) the wait for the receiver's ready-to-receive word, the copy of the
// transport partition, the receiver's arrival flag and the sender's sent[t].
static void progress_main(Comm *c) {
  cudaSetDevice(c->device);
  Progress &pe = c->pe;
  int idle = 0;
  while (!pe.stop.load(std::memory_order_acquire)) {
    bool any = false;
    {
      std::lock_guard<std::mutex> lk(pe.mu);
      for (Request *q : pe.reqs) {
        // one sweep over the ready flags; consecutive transport partitions
        // that became ready in the same epoch move as ONE copy and are
        // signalled by ONE small kernel (arrival flags + sent words)
        int t = 0;
        while (t < q->ntransport) {
          const uint32_t v = __atomic_load_n(q->hready + t, __ATOMIC_ACQUIRE);
          if (v == q->pe_done[t]) {
            ++t;
            continue;
          }
          int t1 = t + 1;
          while (t1 < q->ntransport && __atomic_load_n(q->hready + t1, __ATOMIC_ACQUIRE) == v &&
                 q->pe_done[t1] != v)
            ++t1;
          any = true;
          for (int k = t; k < t1; ++k) q->pe_done[k] = v;
          int rc = 0;
          if ((int32_t)(v - q->pe_rtr_epoch) > 0) {  // first partition of epoch v: receiver ready?
            rc = stream_wait_geq_u32(c, pe.stream, q->ctrl + q->L.rtr, v, q->sys_scope != 0);
            q->pe_rtr_epoch = v;
          }
          const uint64_t off = (uint64_t)t * q->agg * q->part_bytes;
          const uint64_t end = std::min<uint64_t>((uint64_t)t1 * q->agg, (uint64_t)q->partitions) * q->part_bytes;
          if (!rc && end > off)
            rc = cudaMemcpyAsync(q->peer_buf + off, (const uint8_t *)q->sbuf + off, end - off,
                                 cudaMemcpyDeviceToDevice, pe.stream) == cudaSuccess
                     ? 0
                     : PC_ERR_CUDA;
          if (!rc)
            rc = launch_pe_signal(q->peer_ctrl + q->peer_flags_off + t, q->ctrl + q->L.sent + t, t1 - t, v,
                                  q->sys_scope != 0, pe.stream);
          if (rc) pe.err.store(rc);
          t = t1;
        }
      }
    }
    if (any) {
      idle = 0;
    } else if (++idle > 1000) {
      std::this_thread::sleep_for(std::chrono::microseconds(20));
    } else {
      std::this_thread::yield();
    }
  }
}

static int progress_register(Request *q) {
  Comm *c = q->comm;
  Progress &pe = c->pe;
  if (!q->hready) {
    PC_CUDA(cudaHostAlloc((void **)&q->hready, (size_t)q->ntransport * 4, cudaHostAllocMapped | cudaHostAllocPortable));
    memset(q->hready, 0, (size_t)q->ntransport * 4);
    PC_CUDA(cudaHostGetDevicePointer((void **)&q->hready_dev, q->hready, 0));
    q->pe_done.assign((size_t)q->ntransport, 0u);
  }
  if (int rc = pe_kernels_preload()) return rc;  // lazy loading must not happen under spinning kernels
  std::lock_guard<std::mutex> lk(pe.mu);
  if (!pe.started) {
    int lo = 0, hi = 0;
    PC_CUDA(cudaDeviceGetStreamPriorityRange(&lo, &hi));
    PC_CUDA(cudaStreamCreateWithPriority(&pe.stream, cudaStreamNonBlocking, hi));
    pe.stop.store(false);
    pe.th = std::thread(progress_main, c);
    pe.started = true;
  }
  if (!q->pe_registered) {
    pe.reqs.push_back(q);
    q->pe_registered = true;
  }
  return 0;
}

static void progress_unregister(Request *q) {
  Progress &pe = q->comm->pe;
  if (q->pe_registered) {
    std::lock_guard<std::mutex> lk(pe.mu);
    for (size_t i = 0; i < pe.reqs.size(); ++i)
      if (pe.reqs[i] == q) {
        pe.reqs.erase(pe.reqs.begin() + (long)i);
        break;
      }
    q->pe_registered = false;
  }
  if (pe.stream) cudaStreamSynchronize(pe.stream);  // copies that read this request's buffers
  if (q->hready) cudaFreeHost(q->hready);
  q->hready = q->hready_dev = nullptr;
}

static void progress_stop(Comm *c) {
  Progress &pe = c->pe;
  if (!pe.started) return;
  pe.stop.store(true, std::memory_order_release);
  if (pe.th.joinable()) pe.th.join();
  if (pe.stream) {
    cudaStreamSynchronize(pe.stream);
    cudaStreamDestroy(pe.stream);
  }
  pe.stream = nullptr;
  pe.started = false;
}

// ------------------------------------------------------------------ local groups
static int local_allgather_impl(LocalGroup *g, int rank, const void *send, size_t nbytes, void *recv) {
  std::unique_lock<std::mutex> lk(g->mu);
  g->cv.wait(lk, [&] { return g->readers_left == 0; });  // previous round fully consumed
  if (g->arrived == 0) {
    g->nbytes = nbytes;
    g->buf.assign(nbytes * (size_t)g->size, 0);
  } else if (g->nbytes != nbytes) {
    return PC_ERR_ARG;
  }
  memcpy(g->buf.data() + (size_t)rank * nbytes, send, nbytes);
  const uint64_t gen = g->generation;
  if (++g->arrived == g->size) {
    g->generation++;
    g->arrived = 0;
    g->readers_left = g->size;
    g->cv.notify_all();
  } else {
    g->cv.wait(lk, [&] { return g->generation != gen; });
  }
  memcpy(recv, g->buf.data(), nbytes * (size_t)g->size);
  if (--g->readers_left == 0) g->cv.notify_all();
  return 0;
}

// ------------------------------------------------------------------ bootstrap helpers
int allgather(Comm *c, const void *send, size_t nbytes, void *recv) {
  if (c->size == 1) {
    memcpy(recv, send, nbytes);
    return 0;
  }
  int r = c->ag(send, nbytes, recv, c->ag_ctx);
  return r == 0 ? 0 : PC_ERR_ARG;
}

static bool need_ipc(Comm *c) {
  if (c->dry) return false;
  for (int q = 0; q < c->size; ++q)
    if (q != c->rank && !c->same_proc[q]) return true;
  return false;
}

int export_ptr(Comm *c, const void *p, uint64_t bytes, ShareRec *out) {
  memset(out, 0, sizeof(*out));
  out->raw = (uint64_t)(uintptr_t)p;
  out->bytes = bytes;
  if (!p || !need_ipc(c)) return 0;
  load_driver_entry_points();
  if (!g_getAddrRange) return PC_ERR_UNSUPPORTED;
  CUdeviceptr base = 0;
  size_t sz = 0;
  if (g_getAddrRange(&base, &sz, (CUdeviceptr)p) != CUDA_SUCCESS) {
    fprintf(stderr, "[pc] cuMemGetAddressRange failed for %p (not device memory?)\n", p);
    return PC_ERR_ARG;
  }
  out->off = (uint64_t)((uintptr_t)p - (uintptr_t)base);
  cudaError_t e = cudaIpcGetMemHandle(&out->h, (void *)base);
  if (e != cudaSuccess) {
    fprintf(stderr,
            "[pc] cudaIpcGetMemHandle failed (%s): buffers must come from cudaMalloc / the torch caching "
            "allocator without expandable segments\n",
            cudaGetErrorString(e));
    cudaGetLastError();
    return PC_ERR_ARG;
  }
  return 0;
}

int import_ptr(Comm *c, int owner, const ShareRec &s, void **out) {
  if (c->dry || s.raw == 0) {
    *out = (void *)(uintptr_t)s.raw;
    return 0;
  }
  if (owner == c->rank || c->same_proc[owner]) {
    *out = (void *)(uintptr_t)s.raw;
    return 0;
  }
  std::string key((const char *)&s.h, sizeof(s.h));
  auto it = c->ipc_open.find(key);
  void *base = nullptr;
  if (it != c->ipc_open.end()) {
    base = it->second;
  } else {
    PC_CUDA(cudaIpcOpenMemHandle(&base, s.h, cudaIpcMemLazyEnablePeerAccess));
    c->ipc_open[key] = base;
  }
  *out = (uint8_t *)base + s.off;
  return 0;
}

static uint64_t process_token() {
  static uint64_t tok = [] {
    std::random_device rd;
    uint64_t t = ((uint64_t)rd() << 32) ^ rd();
    t ^= (uint64_t)std::chrono::steady_clock::now().time_since_epoch().count();
    t ^= (uint64_t)(uintptr_t)&tok;
    return t ? t : 1;
  }();
  return tok;
}

// ------------------------------------------------------------------ schedules (host, pure)
static int mod(int a, int p) { return ((a % p) + p) % p; }

// Alg 1 with reading R1 (exclusive loop bound: 2(P-1) steps).
static int ring_rows(int P, int r, int32_t *out) {
  const int n = 2 * (P - 1);
  for (int i = 0; i < n; ++i) {
    int32_t *row = out + 5 * i;
    row[0] = mod(r - 1, P);
    row[1] = mod(r + 2 * P - i, P);
    row[2] = i < P - 1 ? 1 : 0;
    row[3] = mod(r + 1, P);
    row[4] = mod(r + 2 * P - i - 1, P);
  }
  return n;
}

static int log2_exact(int P) {
  int k = 0;
  while ((1 << k) < P) ++k;
  return (1 << k) == P ? k : -1;
}

static int rd_rows(int P, int r, int32_t *out) {
  const int n = log2_exact(P);
  if (n < 0) return PC_ERR_ARG;
  for (int k = 0; k < n; ++k) {
    int32_t *row = out + 5 * k;
    row[0] = r ^ (1 << k);
    row[1] = -1;
    row[2] = 1;
    row[3] = r ^ (1 << k);
    row[4] = -1;
  }
  return n;
}

// Reading R4: q = ceil(L / (4P)) * 4 elements per chunk (16-byte multiples);
// trailing chunks may be short or empty.
// epv: elements per 16-byte vector (4 for 32-bit types, 2 for fp64, 8 for bf16)
static int64_t chunk_q(int64_t L, int P, int64_t epv = 4) { return ((L + epv * P - 1) / (epv * P)) * epv; }

// Slicing policy (deterministic from arguments every rank shares): split a
// length of `len` elements into ns slices of qs elements (multiple of 4), with
// about `target_units / nparts` slices per part but none below min_elems.
static void choose_slices(int64_t len, int nparts, int target_units, int64_t min_elems, int *ns_out,
                          int64_t *qs_out, int64_t epv = 4) {
  long fixed = env_long("PC_SLICE_BYTES", 0);
  int64_t qs;
  if (fixed > 0) {
    qs = std::max<int64_t>(epv, (fixed / (16 / epv) + epv - 1) / epv * epv);
  } else {
    // Balance: with W = target_units warps taking units in turn, the engine
    // time is ~ ceil(nparts*ns / W) slices of len/ns elements each; pick the
    // ns (not below min_elems per slice) that minimises ceil(nparts*ns/W)/ns,
    // preferring fewer, larger slices unless 15% better (smaller units pay pipeline
    // fill and flag overhead the model ignores).
    const int64_t by_size = std::max<int64_t>(1, (len + min_elems - 1) / std::max<int64_t>(min_elems, 1));
    const int64_t W = std::max(target_units, 1), np = std::max(nparts, 1);
    const int64_t max_ns = std::min<int64_t>(by_size, std::max<int64_t>(1, (4 * W + np - 1) / np));
    int64_t best = 1;
    double best_cost = 1e300;
    for (int64_t ns = 1; ns <= max_ns; ++ns) {
      const double cost = (double)((np * ns + W - 1) / W) / (double)ns;
      if (cost < best_cost * 0.85) {
        best_cost = cost;
        best = ns;
      }
    }
    qs = (len + best - 1) / best;
    qs = std::max<int64_t>(epv, (qs + epv - 1) / epv * epv);
  }
  int64_t ns = len > 0 ? (len + qs - 1) / qs : 1;
  *ns_out = (int)std::max<int64_t>(1, ns);
  *qs_out = qs;
}

// ------------------------------------------------------------------ request helpers
static size_t dtype_size(int dt) { return dt == PC_BYTE ? 1 : dt == PC_FLOAT64 ? 8 : dt == PC_BF16 ? 2 : 4; }

// Device resources of a request are allocated lazily (first pc_start, or the
// exchange): MPI_P*_init stays non-blocking and cheap.
static int alloc_ctrl(Request *q) {
  Comm *c = q->comm;
  if (c->dry || q->ctrl) return 0;
  PC_CUDA(cudaSetDevice(c->device));
  int lo = 0, hi = 0;
  PC_CUDA(cudaDeviceGetStreamPriorityRange(&lo, &hi));
  PC_CUDA(cudaStreamCreateWithPriority(&q->side, cudaStreamNonBlocking, hi));
  PC_CUDA(cudaEventCreateWithFlags(&q->ev_fork, cudaEventDisableTiming));
  PC_CUDA(cudaEventCreateWithFlags(&q->ev_done, cudaEventDisableTiming));
  PC_CUDA(cudaEventCreateWithFlags(&q->gs.ev, cudaEventDisableTiming));
  PC_CUDA(cudaMalloc((void **)&q->ctrl, q->L.words * 4));
  PC_CUDA(cudaMemsetAsync(q->ctrl, 0, q->L.words * 4, q->side));
  if (q->staging_bytes) {
    PC_CUDA(cudaMalloc((void **)&q->staging, q->staging_bytes));
    // LL line areas start with epoch 0 in every line (never a valid epoch)
    if (q->direct_ll) PC_CUDA(cudaMemsetAsync(q->staging, 0, q->staging_bytes, q->side));
  }
  PC_CUDA(cudaStreamSynchronize(q->side));
  return 0;
}

static int check_buf(const void *p, uint64_t bytes) {
  if (bytes == 0) return 0;
  if (!p) return PC_ERR_ARG;
  if (((uintptr_t)p) & 15) return PC_ERR_ARG;
  return 0;
}

static void fill_prequest(Request *q, pc_prequest_t *o) {
  memset(o, 0, sizeof(*o));
  o->kind = (uint32_t)q->kind;
  o->copy = (uint32_t)q->copy;
  o->partitions = q->partitions;
  o->agg = q->agg;
  o->ntransport = q->ntransport;
  o->timeout_ms = q->comm->timeout_ms;
  o->part_bytes = q->part_bytes;
  o->rank = q->comm->rank;
  if (!q->ctrl) return;
  o->epoch = q->ctrl + q->L.epoch;
  o->cnt = q->ctrl + q->L.cnt;
  o->ready = q->ctrl + q->L.ready;
  o->sent = q->ctrl + q->L.sent;
  o->sbuf = (const uint8_t *)q->sbuf;
  o->rtr = q->ctrl + q->L.rtr;
  o->flags = q->ctrl + q->L.flags;
  o->layout = q->ctrl + q->L.layout;
  o->done = q->ctrl + q->L.donecnt;
  o->done_mul = (uint32_t)q->slices;
  o->sys_scope = (uint32_t)q->sys_scope;
  o->err = (int32_t *)(q->ctrl + q->L.err);
  o->ll_lines = q->xpart ? 0 : q->ll_lines;
  o->xpart = q->xpart ? 1u : 0u;
  o->hready = q->hready_dev;
  o->peer_part_bytes = q->peer_part_bytes;
  o->coll = (uint32_t)q->coll;
  o->nranks = q->comm->size;
  o->dtype = (uint32_t)q->dtype;
  o->op = (uint32_t)q->op;
  if (q->inline_ar) {  // R33: completion words are the INLINE done array (epoch e = final)
    o->ar_tab = (const pc_ar_tab_s *)q->ar_tab;
    o->done = q->ctrl + q->L.sent;
    o->done_mul = 1;
  }
  if (q->kind == PC_KIND_PALLREDUCE && q->coll == PC_COLL_ALLGATHER)
    o->srcflags = q->ctrl + q->L.flags + (size_t)q->partitions * 2 * q->slices;
  if (q->kind == PC_KIND_PSEND) {
    o->peer_rbuf = q->peer_buf;
    o->peer_flags = q->peer_ctrl ? q->peer_ctrl + q->peer_flags_off : nullptr;
    o->peer_ll = (q->peer_ctrl && q->ll_lines && !q->xpart) ? (uint8_t *)(q->peer_ctrl + q->peer_ll_off) : nullptr;
  } else if (q->kind == PC_KIND_PRECV) {
    o->ll = q->ll_lines ? (uint8_t *)(q->ctrl + q->L.ll) : nullptr;
    o->rbuf = (uint8_t *)q->rbuf;
  }
}

static int new_request(Comm *c, int kind, pc_request_t *out, Request **rq) {
  if (!c || !out) return PC_ERR_ARG;
  Request *q = new Request();
  q->comm = c;
  q->kind = kind;
  q->index = (int)c->reqs.size();
  c->reqs.push_back(q);
  *rq = q;
  *out = (pc_request_t)q;
  return 0;
}

static int p2p_init(int kind, const void *sbuf, void *rbuf, int partitions, size_t count, int dtype, int peer,
                    int tag, Comm *c, pc_request_t *out) {
  if (!c || !out || partitions < 1 || dtype < 0 || dtype > 4 || peer < 0 || peer >= c->size || tag < 0)
    return PC_ERR_ARG;
  const uint64_t bytes = (uint64_t)partitions * count * dtype_size(dtype);
  if (!c->dry && check_buf(kind == PC_KIND_PSEND ? sbuf : rbuf, bytes)) return PC_ERR_ARG;
  Request *q;
  int rc = new_request(c, kind, out, &q);
  if (rc) return rc;
  q->sbuf = sbuf;
  q->rbuf = rbuf;
  q->partitions = partitions;
  q->count = count;
  q->dtype = dtype;
  q->esize = dtype_size(dtype);
  q->peer = peer;
  q->tag = tag;
  q->part_bytes = count * q->esize;
  q->total_bytes = bytes;
  q->seq = c->post_seq[std::make_tuple(kind, peer, tag)]++;
  // LL line area (PC_COPY_LL): both sides derive it from (partitions, count,
  // dtype), which matching requires to be equal, so their layouts agree.
  if (q->part_bytes <= PC_LL_MAX_PART_BYTES && bytes <= PC_LL_MAX_TOTAL_BYTES)
    q->ll_lines = (uint32_t)std::max<uint64_t>(1, (q->part_bytes + 7) / 8);
  q->L.build((size_t)partitions, (size_t)partitions, (size_t)2 * partitions * q->ll_lines * 4);
  q->agg = 1;
  q->ntransport = partitions;
  return 0;
}

// ------------------------------------------------------------------ exchange (first pbuf_prepare)
static int make_rec(Request *q, ReqRec *r) {
  Comm *c = q->comm;
  memset(r, 0, sizeof(*r));
  r->kind = q->kind;
  r->peer = q->peer;
  r->tag = q->tag;
  r->partitions = q->partitions;
  r->count = (int64_t)q->count;
  r->dtype = q->dtype;
  r->op = q->op;
  r->algo = q->direct_ll ? PC_ALGO_LL : q->direct_push ? PC_ALGO_DIRECT_PUSH : q->algo;  // the same variant everywhere
  r->seq = q->seq;
  r->coll = q->coll;
  r->root = q->root;
  r->owner = c->rank;
  r->req_index = q->index;
  r->host_req = (uint64_t)(uintptr_t)q;
  r->flags_off = (int64_t)q->L.flags;
  r->ll_off = (int64_t)q->L.ll;
  int rc = 0;
  if (q->kind == PC_KIND_PRECV || q->kind == PC_KIND_PALLREDUCE)
    if ((rc = export_ptr(c, q->rbuf, q->total_bytes, &r->buf))) return rc;
  if ((rc = export_ptr(c, q->ctrl, q->L.words * 4, &r->ctrl))) return rc;
  if (q->staging && (rc = export_ptr(c, q->staging, q->staging_bytes, &r->stage))) return rc;
  // DIRECT (PULL): the peers' reduce steps read this rank's send buffer
  // (PUSH exports its staging above: the peers write into it)
  if (q->kind == PC_KIND_PALLREDUCE && q->algo == PC_ALGO_DIRECT && !q->direct_push && !q->direct_ll && c->size > 1 &&
      (q->coll == PC_COLL_ALLREDUCE || q->coll == PC_COLL_REDUCE_SCATTER) &&
      (rc = export_ptr(c, q->sbuf, q->send_bytes, &r->stage)))
    return rc;
  return 0;
}

static const ReqRec *find_rec(const std::vector<ReqRec> &all, int M, int owner, int kind, int peer, int tag,
                              int seq, const std::vector<int> &counts) {
  for (int k = 0; k < counts[owner]; ++k) {
    const ReqRec &r = all[(size_t)owner * M + k];
    if (r.kind == kind && r.peer == peer && r.tag == tag && r.seq == seq) return &r;
  }
  return nullptr;
}

static int exchange_round(Comm *c, Request *target) {
  std::vector<Request *> pending;
  for (Request *q : c->reqs)
    if (q && !q->exchanged) {
      int arc = alloc_ctrl(q);  // exported below
      if (arc) return arc;
      pending.push_back(q);
    }
  int32_t mine = (int32_t)pending.size();
  std::vector<int32_t> counts(c->size);
  int rc = allgather(c, &mine, sizeof(mine), counts.data());
  if (rc) return rc;
  int M = 0;
  for (int v : counts) M = std::max(M, v);
  if (M == 0) return PC_ERR_STATE;
  std::vector<ReqRec> my(M), all((size_t)M * c->size);
  for (size_t k = 0; k < pending.size(); ++k)
    if ((rc = make_rec(pending[k], &my[k]))) return rc;
  if ((rc = allgather(c, my.data(), sizeof(ReqRec) * M, all.data()))) return rc;
  std::vector<int> cnt(counts.begin(), counts.end());

  int target_rc = PC_ERR_MATCH;
  for (Request *q : pending) {
    int qrc = 0;
    if (q->kind == PC_KIND_PSEND || q->kind == PC_KIND_PRECV) {
      const int want = q->kind == PC_KIND_PSEND ? PC_KIND_PRECV : PC_KIND_PSEND;
      const ReqRec *m = find_rec(all, M, q->peer, want, c->rank, q->tag, q->seq, cnt);
      if (!m) {
        qrc = PC_ERR_MATCH;
      } else if (m->dtype != q->dtype ||
                 (uint64_t)m->partitions * (uint64_t)m->count != (uint64_t)q->partitions * q->count ||
                 ((m->partitions != q->partitions) && (uint64_t)q->partitions * q->count == 0)) {
        // MPI-4: the partition counts may differ (reading R30), the type
        // signature (dtype x total elements) may not; empty buffers need equal
        // partitionings (a flag-only partition has no bytes to overlap)
        fprintf(stderr, "[pc] rank %d: %s to/from %d tag %d: partitions/count/dtype disagree (%d/%lld/%d vs %d/%lld/%d)\n",
                c->rank, q->kind == PC_KIND_PSEND ? "psend" : "precv", q->peer, q->tag, q->partitions,
                (long long)q->count, q->dtype, m->partitions, (long long)m->count, m->dtype);
        qrc = PC_ERR_MATCH;
        q->exchanged = true;  // matched but incompatible: report, do not retry
        q->matched = false;
      } else {
        void *pctrl = nullptr, *pbuf = nullptr;
        q->xpart = m->partitions != q->partitions;
        q->peer_part_bytes = (uint64_t)m->count * q->esize;
        q->peer_flags_off = (size_t)m->flags_off;
        q->peer_ll_off = (size_t)m->ll_off;
        if ((qrc = import_ptr(c, m->owner, m->ctrl, &pctrl)) == 0) {
          q->peer_ctrl = (uint32_t *)pctrl;
          if (q->kind == PC_KIND_PSEND) {
            qrc = import_ptr(c, m->owner, m->buf, &pbuf);
            q->peer_buf = (uint8_t *)pbuf;
          } else {
            // the receiver is the consumer: it writes ready-to-receive into the sender's rtr[0]
            q->rtr_targets.push_back({q->peer_ctrl, 0});
          }
        }
        if (qrc == 0) {
          q->exchanged = true;
          q->matched = true;
          q->match_peer_index = m->req_index;
          // PC_FORCE_SYS_SCOPE=1: system-scope ordering even between ranks of one GPU
          // (runs the cross-GPU code paths on a one-GPU box; stronger, never weaker)
          q->sys_scope = c->dry || memcmp(c->ranks[q->peer].uuid, c->ranks[c->rank].uuid, 16) != 0 ||
                         env_long("PC_FORCE_SYS_SCOPE", 0) != 0;
        }
      }
    } else {  // PALLREDUCE: the seq-th allreduce of every rank
      std::vector<const ReqRec *> peers(c->size, nullptr);
      for (int r = 0; r < c->size && !qrc; ++r) {
        const ReqRec *m = find_rec(all, M, r, PC_KIND_PALLREDUCE, -1, 0, q->seq, cnt);
        if (!m || m->partitions != q->partitions || m->count != (int64_t)q->count || m->dtype != q->dtype ||
            m->op != q->op ||
            m->algo != (q->direct_ll ? PC_ALGO_LL : q->direct_push ? PC_ALGO_DIRECT_PUSH : q->algo) || m->coll != q->coll ||
            m->root != q->root) {
          fprintf(stderr, "[pc] rank %d: allreduce #%d disagrees with rank %d\n", c->rank, q->seq, r);
          qrc = PC_ERR_MATCH;
        }
        peers[r] = m;
      }
      if (!qrc) {
        const int P = c->size, r = c->rank;
        auto imp = [&](int who, int slot) -> int {
          void *b = nullptr, *ct = nullptr, *st = nullptr;
          int e;
          if ((e = import_ptr(c, who, peers[who]->buf, &b))) return e;
          if ((e = import_ptr(c, who, peers[who]->ctrl, &ct))) return e;
          if ((e = import_ptr(c, who, peers[who]->stage, &st))) return e;
          q->nb_buf[slot] = (uint8_t *)b;
          q->nb_ctrl[slot] = (uint32_t *)ct;
          q->nb_stage[slot] = (uint8_t *)st;
          return 0;
        };
        if (P > 1) {
          if (q->algo == PC_ALGO_RING) {
            qrc = imp(mod(r + 1, P), 0);  // O: where this rank's steps land
            if (!qrc) {
              // consumer-side RTR: this rank receives from I = r-1, so it
              // tells I (rtr slot 0 of I's control block) when it is ready
              void *ict = nullptr;
              qrc = import_ptr(c, mod(r - 1, P), peers[mod(r - 1, P)]->ctrl, &ict);
              if (!qrc) q->rtr_targets.push_back({(uint32_t *)ict, 0});
            }
          } else if (q->algo == PC_ALGO_DIRECT) {
            // peer j = rank (r+1+j) mod P; in peer p's control block the RTR
            // slot of rank r is (r - p - 1) mod P
            for (int j = 0; j < P - 1 && !qrc; ++j) {
              const int pj = mod(r + 1 + j, P);
              qrc = imp(pj, j);
              // (the LL variant needs no ready-to-receive: its line areas are
              //  double-buffered by epoch parity, engine.cuh ll_body)
              if (!qrc && !q->direct_ll) q->rtr_targets.push_back({q->nb_ctrl[j], mod(r - pj - 1, P)});
            }
          } else {
            for (int k = 0; k < q->nsteps && !qrc; ++k) {
              qrc = imp(r ^ (1 << k), k);
              if (!qrc) q->rtr_targets.push_back({q->nb_ctrl[k], k});
            }
          }
        }
        if (!qrc) {
          q->exchanged = true;
          q->matched = true;
          q->sys_scope = (c->dry || env_long("PC_FORCE_SYS_SCOPE", 0) != 0) ? 1 : 0;
          for (int k = 0; k < P; ++k)
            if (memcmp(c->ranks[k].uuid, c->ranks[c->rank].uuid, 16) != 0) q->sys_scope = 1;
          // ranks of this comm sharing this GPU inside this process run their
          // engines as one grouped launch
          std::vector<int> loc;
          for (int k = 0; k < P; ++k)
            if (c->same_proc[k] && c->ranks[k].device == c->device &&
                memcmp(c->ranks[k].uuid, c->ranks[c->rank].uuid, 16) == 0)
              loc.push_back(k);
          if (loc.size() > 1) {
            if ((int)loc.size() > kMaxLocal) {
              qrc = PC_ERR_UNSUPPORTED;
            } else {
              Request *ld = (Request *)(uintptr_t)peers[loc[0]]->host_req;
              q->leader = ld;
              std::lock_guard<std::mutex> lk(ld->gs.mu);
              ld->gs.members.push_back(q);
              std::sort(ld->gs.members.begin(), ld->gs.members.end(),
                        [](Request *a, Request *b) { return a->comm->rank < b->comm->rank; });
            }
          }
        }
      } else {
        q->exchanged = true;
      }
    }
    if (q == target) target_rc = qrc;
    if (qrc) logf("rank %d: request %d exchange rc=%d", c->rank, q->index, qrc);
  }
  if (!c->dry) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_err(e, "exchange");
  }
  return target_rc;
}

// ------------------------------------------------------------------ engine launch
// The engine is launched lazily, from pc_wait / pc_wait_on_stream / pc_test,
// i.e. AFTER the user enqueued the producer kernel of the epoch (Listing 2
// order: Start, Pbuf_prepare, kernel, Wait).  A spinning engine can therefore
// never sit in front of the producer it waits for in a shared hardware queue
// (streams beyond CUDA_DEVICE_MAX_CONNECTIONS share queues).
static RingArgs make_ring_args(Request *q) {
  Comm *c = q->comm;
  RingArgs a{};
  a.epoch = q->ctrl + q->L.epoch;
  a.P = c->size;
  a.r = c->rank;
  a.Np = q->partitions;
  a.ns = q->slices;
  a.nunits = q->partitions * q->slices;
  a.op = q->op;
  a.dtype = q->dtype;
  a.L = (int64_t)q->count;
  a.q = q->chunk_elems;
  a.qs = q->slice_elems;
  a.sendbuf = (const uint8_t *)q->sbuf;
  a.recvbuf = (uint8_t *)q->rbuf;
  a.staging = q->staging;
  a.flags = q->ctrl + q->L.flags;
  a.ready = q->ctrl + q->L.ready;
  a.rtr = q->ctrl + q->L.rtr;
  a.done = q->ctrl + q->L.donecnt;
  a.o_staging = q->nb_stage[0];
  a.o_recvbuf = q->nb_buf[0];
  a.o_flags = q->nb_ctrl[0] ? q->nb_ctrl[0] + q->L.flags : nullptr;
  a.err = (int32_t *)(q->ctrl + q->L.err);
  a.timeout_ms = c->timeout_ms;
  a.sys = q->sys_scope;
  return a;
}

static RdArgs make_rd_args(Request *q) {
  Comm *c = q->comm;
  RdArgs a{};
  a.epoch = q->ctrl + q->L.epoch;
  a.P = c->size;
  a.r = c->rank;
  a.Np = q->partitions;
  a.ns = q->slices;
  a.nunits = q->partitions * q->slices;
  a.op = q->op;
  a.dtype = q->dtype;
  a.nsteps = q->nsteps;
  a.L = (int64_t)q->count;
  a.qs = q->slice_elems;
  a.sendbuf = (const uint8_t *)q->sbuf;
  a.recvbuf = (uint8_t *)q->rbuf;
  a.staging = q->staging;
  a.flags = q->ctrl + q->L.flags;
  a.ready = q->ctrl + q->L.ready;
  a.rtr = q->ctrl + q->L.rtr;
  a.done = q->ctrl + q->L.donecnt;
  const int64_t slot_bytes = (int64_t)q->partitions * (int64_t)q->count * (int64_t)q->esize;
  for (int k = 0; k < q->nsteps; ++k) {
    a.p_staging[k] = q->nb_stage[k] + (int64_t)k * slot_bytes;
    a.p_flags[k] = q->nb_ctrl[k] + q->L.flags;
  }
  a.err = (int32_t *)(q->ctrl + q->L.err);
  a.timeout_ms = c->timeout_ms;
  a.sys = q->sys_scope;
  return a;
}

static DirectArgs make_direct_args(Request *q) {
  Comm *c = q->comm;
  DirectArgs a{};
  a.epoch = q->ctrl + q->L.epoch;
  a.P = c->size;
  a.r = c->rank;
  a.Np = q->partitions;
  a.ns = q->slices;
  a.nunits = q->partitions * q->slices;
  a.op = q->op;
  a.dtype = q->dtype;
  a.L = (int64_t)q->count;
  a.q = q->chunk_elems;
  a.qs = q->slice_elems;
  a.sendbuf = (const uint8_t *)q->sbuf;
  a.recvbuf = (uint8_t *)q->rbuf;
  a.cnt = q->ctrl + q->L.flags;
  a.ready = q->ctrl + q->L.ready;
  a.rtr = q->ctrl + q->L.rtr;
  a.done = q->ctrl + q->L.donecnt;
  for (int j = 0; j < c->size - 1; ++j) {
    a.p_sendbuf[j] = q->nb_stage[j];  // DIRECT exports its send buffer in the stage slot
    a.p_recvbuf[j] = q->nb_buf[j];
    a.p_cnt[j] = q->nb_ctrl[j] + q->L.flags;
  }
  a.err = (int32_t *)(q->ctrl + q->L.err);
  a.timeout_ms = c->timeout_ms;
  a.sys = q->sys_scope;
  a.push = q->direct_push ? 1 : 0;
  a.staging = q->staging;
  a.ll = q->direct_ll ? 1 : 0;
  a.ll_lines = (int64_t)std::max<uint64_t>(1, (q->part_bytes + 7) / 8);
  return a;
}

static CollArgs make_coll_args(Request *q) {
  Comm *c = q->comm;
  CollArgs a{};
  a.epoch = q->ctrl + q->L.epoch;
  a.coll = q->coll;
  a.P = c->size;
  a.r = c->rank;
  a.root = q->root;
  a.Np = q->partitions;
  a.ns = q->slices;
  a.nunits = q->partitions * q->slices;
  a.op = q->op;
  a.dtype = q->dtype;
  a.count = (int64_t)q->count;
  a.qs = q->slice_elems;
  a.es = (int64_t)q->esize;
  a.sendbuf = (const uint8_t *)q->sbuf;
  a.recvbuf = (uint8_t *)q->rbuf;
  a.cnt = q->ctrl + q->L.flags;
  a.ready = q->ctrl + q->L.ready;
  a.rtr = q->ctrl + q->L.rtr;
  a.done = q->ctrl + q->L.donecnt;
  const size_t sf = (size_t)q->partitions * 2 * q->slices;  // allgather source flags follow the counters
  a.srcflags = q->ctrl + q->L.flags + sf;
  for (int j = 0; j < c->size - 1; ++j) {
    a.p_sendbuf[j] = q->nb_stage[j];
    a.p_recvbuf[j] = q->nb_buf[j];
    a.p_cnt[j] = q->nb_ctrl[j] + q->L.flags;
    a.p_srcflags[j] = q->nb_ctrl[j] + q->L.flags + sf;
  }
  a.err = (int32_t *)(q->ctrl + q->L.err);
  a.timeout_ms = c->timeout_ms;
  a.sys = q->sys_scope;
  return a;
}

// joined_stream value: the previous epoch's completion was observed by the host
static const cudaStream_t kHostJoined = reinterpret_cast<cudaStream_t>(~uintptr_t(0));

static bool needs_engine(Request *q) {
  return (q->kind == PC_KIND_PALLREDUCE && !q->inline_ar) || (q->kind == PC_KIND_PSEND && q->has_preq && q->copy == 1);
}

// Optional CUDA-event timing around an engine launch (pc_request_set_timing).
static int timing_begin(TimingLog &T, cudaStream_t s, int *a) {
  *a = -1;
  if (!T.on || T.pending.size() >= 16384) return 0;
  cudaEvent_t e;
  if ((*a = T.get(&e)) < 0) return PC_ERR_CUDA;
  PC_CUDA(cudaEventRecord(e, s));
  return 0;
}
static int timing_end(TimingLog &T, cudaStream_t s, int a) {
  if (a < 0) return 0;
  cudaEvent_t e;
  int b = T.get(&e);
  if (b < 0) return PC_ERR_CUDA;
  PC_CUDA(cudaEventRecord(e, s));
  T.pending.push_back({(size_t)a, (size_t)b});
  return 0;
}

// ---------------------------------------------------------------- overlap
// Producer/engine overlap (§8(a) a6: "each partition forwarded and reduced as
// soon as it is ready").  The engine is still
// ENQUEUED at the wait (after the user's producer in host order, so no
// spinning kernel ever depends on work submitted behind it), but it is forked
// from ev_fork, which the epoch's control calls record: it starts as soon as
// the epoch word and the ready-to-receive words are written and reduces each
// partition while the producer is still running.
static int fork_point(Request *q, cudaStream_t s) {
  if (q->comm->dry || !q->ev_fork) return 0;
  PC_CUDA(cudaEventRecord(q->ev_fork, s));
  q->forked = true;
  q->fork_ev_ext = nullptr;
  return 0;
}
// The event the engine forks from: the request's own, or the one a batched
// control call recorded once for all its requests.
static cudaEvent_t fork_event(const Request *q) { return q->fork_ev_ext ? q->fork_ev_ext : q->ev_fork; }

// The engine's width.  When every partition was made ready by a host-side op
// before ev_fork (pc_epoch_all with Pready, pc_preadyall, pc_pready_range of
// all partitions) no user kernel can be running that the engine waits for:
// full width.  Otherwise a producer kernel may still have blocks to place, so
// the engine takes whole CTAs on at most PC_OVERLAP_FRAC of the SMs per GPU —
// at least one SM carries no engine CTA, so every producer block that fits an
// empty SM can always be placed (deadlock freedom).
static bool full_width(const Request *q) { return !q->overlap || q->host_ready_all; }
static int engine_width(const Request *q, bool full) {
  return full ? q->engine_warps : std::min(q->engine_warps, q->comm->overlap_warps);
}

// Start of an epoch (pc_start / pc_startall / pc_epoch_all): reset the
// per-epoch overlap state; a co-located group member may not start while the
// group's engine of its previous epoch is not launched (the engine reads the
// epoch word at entry); and when the previous epoch's completion was joined
// on another stream, this epoch's control op waits for it first.
static bool group_blocks_start(Request *q) {
  if (!q->leader) return false;
  GroupState &g = q->leader->gs;
  std::lock_guard<std::mutex> lk(g.mu);
  return g.epoch == q->epoch && q->engine_registered && !g.launched;
}
static int epoch_begin(Request *q, cudaStream_t s, bool capturing) {
  if (group_blocks_start(q)) return PC_ERR_STATE;
  if (!q->comm->dry && q->epoch > 0 && !capturing && q->joined_stream != s && q->joined_stream != kHostJoined &&
      needs_engine(q) && q->engine_launched && q->last_done)
    PC_CUDA(cudaStreamWaitEvent(s, q->last_done, 0));
  q->forked = false;
  q->batch_launched = false;
  q->host_ready_all = false;
  q->join_pending = false;
  return 0;
}

// Single-rank launch on the request's side stream, forked from ev_fork.
static int launch_single(Request *q) {
  if (!q->forked || !q->overlap) {
    PC_CUDA(cudaEventRecord(q->ev_fork, q->user_stream));
    q->fork_ev_ext = nullptr;
  }
  PC_CUDA(cudaStreamWaitEvent(q->side, fork_event(q), 0));
  const bool full = full_width(q);
  const int w = engine_width(q, full);
  int rc, tk;
  if ((rc = timing_begin(q->tlog, q->side, &tk))) return rc;
  if (q->kind == PC_KIND_PALLREDUCE && q->coll != PC_COLL_ALLREDUCE) {
    rc = launch_coll_engine(make_coll_args(q), w, q->side);
  } else if (q->kind == PC_KIND_PALLREDUCE) {
    rc = q->algo == PC_ALGO_RING     ? launch_ring_engine(make_ring_args(q), w, q->side)
         : q->algo == PC_ALGO_DIRECT ? launch_direct_engine(make_direct_args(q), w, q->side, !full && q->comm->overlap_thin)
                                     : launch_rd_engine(make_rd_args(q), w, q->side);
  } else {
    P2pEngineArgs a{};
    a.epoch = q->ctrl + q->L.epoch;
    a.nt = q->ntransport;
    a.agg = q->agg;
    a.ns = q->slices;
    a.nunits = q->ntransport * q->slices;
    a.part_bytes = q->part_bytes;
    a.slice_bytes = (uint64_t)q->slice_elems;
    a.partitions = q->partitions;
    a.sbuf = (const uint8_t *)q->sbuf;
    a.peer_rbuf = q->peer_buf;
    a.peer_flags = q->peer_ctrl + q->peer_flags_off;
    a.ready = q->ctrl + q->L.ready;
    a.rtr = q->ctrl + q->L.rtr;
    a.donecnt = q->ctrl + q->L.donecnt;
    a.sent = q->ctrl + q->L.sent;
    a.err = (int32_t *)(q->ctrl + q->L.err);
    a.timeout_ms = q->comm->timeout_ms;
    a.sys = q->sys_scope;
    a.xpart = q->xpart ? 1u : 0u;
    a.peer_part_bytes = q->peer_part_bytes;
    rc = launch_p2p_engine(a, w, q->side);
  }
  if (rc) return rc;
  if ((rc = timing_end(q->tlog, q->side, tk))) return rc;
  PC_CUDA(cudaEventRecord(q->ev_done, q->side));
  q->engine_launched = true;
  q->last_done = q->ev_done;
  return 0;
}

// Co-located ranks (same process, same GPU): register this rank's epoch; the
// last rank to register launches ONE kernel running every member's engine,
// ordered after every member's producer work (their ev_fork events).
// *launched tells whether that launch has happened (then q->ev_done of the
// group leader marks completion).  block: wait (host) until it has.
static int group_register(Request *q, bool block, cudaStream_t ws, bool *launched) {
  Request *ld = q->leader;
  GroupState &g = ld->gs;
  std::unique_lock<std::mutex> lk(g.mu);
  if (g.epoch != q->epoch) {
    if (g.pending > 0 && !g.launched) return PC_ERR_STATE;  // a member is still in the previous epoch
    g.epoch = q->epoch;
    g.pending = 0;
    g.launched = false;
  }
  if (!q->engine_registered) {
    if (!q->forked || !q->overlap) {
      PC_CUDA(cudaEventRecord(q->ev_fork, q->user_stream));
      q->fork_ev_ext = nullptr;
    }
    q->engine_registered = true;
    g.pending++;
  }
  if (!g.launched && g.pending == (int)g.members.size()) {
    bool full = true;
    cudaEvent_t waited = nullptr;
    for (Request *m : g.members) {
      if (fork_event(m) != waited) PC_CUDA(cudaStreamWaitEvent(q->side, fork_event(m), 0));
      waited = fork_event(m);  // members forked by one batched call share the event
      full = full && full_width(m);
    }
    const int w = engine_width(q, full);
    int rc, tk;
    if ((rc = timing_begin(g.tlog, q->side, &tk))) return rc;
    if (q->coll != PC_COLL_ALLREDUCE) {
      CollGroupArgs ga{};
      ga.n = (int)g.members.size();
      for (int k = 0; k < ga.n; ++k) ga.a[k] = make_coll_args(g.members[k]);
      rc = launch_coll_engine_group(ga, w, q->side);
    } else if (q->algo == PC_ALGO_RING) {
      RingGroupArgs ga{};
      ga.n = (int)g.members.size();
      for (int k = 0; k < ga.n; ++k) ga.a[k] = make_ring_args(g.members[k]);
      rc = launch_ring_engine_group(ga, w, q->side);
    } else if (q->algo == PC_ALGO_DIRECT) {
      DirectGroupArgs ga{};
      ga.n = (int)g.members.size();
      for (int k = 0; k < ga.n; ++k) ga.a[k] = make_direct_args(g.members[k]);
      rc = launch_direct_engine_group(ga, w, q->side, !full && q->comm->overlap_thin);
    } else {
      RdGroupArgs ga{};
      ga.n = (int)g.members.size();
      for (int k = 0; k < ga.n; ++k) ga.a[k] = make_rd_args(g.members[k]);
      rc = launch_rd_engine_group(ga, w, q->side);
    }
    if (rc) return rc;
    if ((rc = timing_end(g.tlog, q->side, tk))) return rc;
    PC_CUDA(cudaEventRecord(g.ev, q->side));
    for (Request *m : g.members) m->last_done = g.ev;
    // members that already waited on their own stream (before the group was
    // complete) get their completion ordered there now (pc.h "In-process
    // rank groups": work they enqueued between their wait and this launch is
    // not covered)
    for (Request *m : g.members)
      if (m != q && m->join_pending) {
        if (!ws || m->wait_stream != ws) PC_CUDA(cudaStreamWaitEvent(m->wait_stream, g.ev, 0));
        m->joined_stream = m->wait_stream;
        m->join_pending = false;
      }
    g.launched = true;
    g.cv.notify_all();
  }
  if (block && !g.cv.wait_for(lk, std::chrono::milliseconds(q->comm->timeout_ms ? q->comm->timeout_ms : 3600000),
                              [&] { return g.launched || g.epoch != q->epoch; })) {
    fprintf(stderr,
            "[pc] rank %d: pc_wait timed out waiting for the other co-located ranks' waits (every rank sharing this "
            "GPU in this process must call pc_wait/pc_wait_on_stream for the epoch; use one thread per rank or "
            "pc_wait_on_stream)\n",
            q->comm->rank);
    return PC_ERR_TIMEOUT;
  }
  *launched = g.launched && g.epoch == q->epoch;
  if (*launched) q->engine_launched = true;
  return 0;
}

static int read_error(Request *q, int *code, int *part) {
  *code = 0;
  *part = 0;
  if (q->comm->dry || !q->ctrl) return 0;
  int32_t h[2] = {0, 0};
  PC_CUDA(cudaMemcpyAsync(h, q->ctrl + q->L.err, sizeof(h), cudaMemcpyDeviceToHost, q->side));
  PC_CUDA(cudaStreamSynchronize(q->side));
  *code = h[0];
  *part = h[1];
  return 0;
}

static int error_rc(Request *q) {
  int code, part;
  int rc = read_error(q, &code, &part);
  if (rc) return rc;
  if (code == 0) return 0;
  fprintf(stderr, "[pc] rank %d request %d: device error %d (partition %d)\n", q->comm->rank, q->index, code, part);
  return code == PC_ERR_TIMEOUT ? PC_ERR_TIMEOUT : PC_ERR_DEVICE;
}

// ---------------------------------------------------------------- batch caches
// Device tables of batched calls over a fixed request list (BatchCache,
// pc_internal.h).  Built eagerly on first use (a synchronous copy: not while
// a stream captures), reused every epoch, dropped with any of its requests.
static std::mutex g_batch_mu;
static std::map<std::vector<Request *>, BatchCache *> g_epoch_batches, g_engine_batches;

static void batch_destroy(BatchCache *b) {
  for (Request *q : b->reqs) {
    if (q->fork_ev_ext == b->ev) {
      q->fork_ev_ext = nullptr;
      q->forked = false;
    }
    if (q->last_done == b->ev) q->last_done = nullptr;
  }
  // cudaFree waits for the device (the last eager launch that read the
  // tables); the event may have been recorded inside a graph capture, where
  // it cannot be waited on — so no event sync, and no error left behind for
  // the next launch's cudaGetLastError
  if (b->dev) cudaFree(b->dev);
  if (b->ev) cudaEventDestroy(b->ev);
  cudaGetLastError();
  delete b;
}

// Drop every cache that lists q (pc_request_free).
static void batch_drop(Request *q) {
  std::lock_guard<std::mutex> lk(g_batch_mu);
  for (auto *m : {&g_epoch_batches, &g_engine_batches})
    for (auto it = m->begin(); it != m->end();) {
      if (std::find(it->first.begin(), it->first.end(), q) != it->first.end()) {
        batch_destroy(it->second);
        it = m->erase(it);
      } else {
        ++it;
      }
    }
}

static int batch_upload(BatchCache *b, const void *host, size_t bytes, cudaStream_t s) {
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  PC_CUDA(cudaStreamIsCapturing(s, &cs));
  if (cs != cudaStreamCaptureStatusNone) return PC_ERR_STATE;  // first use of a request list: eagerly
  PC_CUDA(cudaMalloc(&b->dev, bytes));
  PC_CUDA(cudaMemcpy(b->dev, host, bytes, cudaMemcpyHostToDevice));
  b->dev_bytes = bytes;
  PC_CUDA(cudaEventCreateWithFlags(&b->ev, cudaEventDisableTiming));
  return 0;
}

// pc_epoch_all over more requests / RTR words than one kernel's parameters
// hold: one single-block kernel reading the lists from device memory, one
// fork event for all requests.
static int epoch_all_batched(const std::vector<Request *> &rq, int pready, cudaStream_t s) {
  BatchCache *b = nullptr;
  {
    std::lock_guard<std::mutex> lk(g_batch_mu);
    auto it = g_epoch_batches.find(rq);
    if (it != g_epoch_batches.end()) b = it->second;
  }
  if (!b) {
    b = new BatchCache();
    b->reqs = rq;
    std::vector<EpochEnt> ent(rq.size());
    std::vector<RtrEnt> rtr;
    for (size_t i = 0; i < rq.size(); ++i) {
      Request *q = rq[i];
      ent[i].epoch = q->ctrl + q->L.epoch;
      ent[i].ready = q->ctrl + q->L.ready;
      ent[i].partitions = q->partitions;
      for (auto &t : q->rtr_targets) rtr.push_back({t.first + q->L.rtr + t.second, (int)i, q->sys_scope});
    }
    std::vector<int> big;
    for (size_t i = 0; i < rq.size(); ++i)
      if (rq[i]->partitions > kEpochSmallParts) big.push_back((int)i);
    const size_t o_rtr = ent.size() * sizeof(EpochEnt), o_big = o_rtr + rtr.size() * sizeof(RtrEnt);
    std::vector<uint8_t> host(o_big + big.size() * sizeof(int));
    memcpy(host.data(), ent.data(), o_rtr);
    if (!rtr.empty()) memcpy(host.data() + o_rtr, rtr.data(), rtr.size() * sizeof(RtrEnt));
    if (!big.empty()) memcpy(host.data() + o_big, big.data(), big.size() * sizeof(int));
    b->n = (int)ent.size();
    b->nrtr = (int)rtr.size();
    b->nreq = (int)big.size();  // (epoch batch: the large-request list)
    if (int rc = batch_upload(b, host.data(), host.size(), s)) {
      batch_destroy(b);
      return rc;
    }
    std::lock_guard<std::mutex> lk(g_batch_mu);
    g_epoch_batches[rq] = b;
  }
  EpochBatchArgs a{};
  a.n = b->n;
  a.nrtr = b->nrtr;
  a.pready = pready ? 1 : 0;
  a.ent = (const EpochEnt *)b->dev;
  a.rtr = (const RtrEnt *)((const uint8_t *)b->dev + (size_t)b->n * sizeof(EpochEnt));
  a.nbig = b->nreq;
  a.big = (const int *)((const uint8_t *)a.rtr + (size_t)b->nrtr * sizeof(RtrEnt));
  if (int rc = launch_epoch_batch(a, s)) return rc;
  PC_CUDA(cudaEventRecord(b->ev, s));
  for (Request *q : rq) {
    q->host_ready_all = pready != 0;
    q->forked = true;
    q->fork_ev_ext = b->ev;
  }
  return 0;
}

// pc_waitall_on_stream over several DIRECT allreduces of one GPU: ONE
// batched engine launch (direct_engine_batch) instead of one per request.
// Eligible: engine-moved (not INLINE) DIRECT allreduces, one dtype / op,
// not yet launched this epoch, and either all single-rank (R = 1) or all
// members of co-located groups of the same size R whose members are all in
// the list.  Returns 1 if the batch was not applicable (caller falls back).
static int engine_batch(const std::vector<Request *> &rq, cudaStream_t s) {
  if (rq.size() < 2) return 1;
  Request *q0 = rq[0];
  const int R = q0->leader ? (int)q0->leader->gs.members.size() : 1;
  std::vector<Request *> leaders;
  for (Request *q : rq) {
    if (q->kind != PC_KIND_PALLREDUCE || q->coll != PC_COLL_ALLREDUCE || q->algo != PC_ALGO_DIRECT ||
        q->direct_push || q->direct_ll || q->inline_ar || !q->active || q->engine_registered || q->engine_launched ||
        q->batch_launched)
      return 1;
    if (q->dtype != q0->dtype || q->op != q0->op || q->comm->device != q0->comm->device) return 1;
    const int r = q->leader ? (int)q->leader->gs.members.size() : 1;
    if (r != R || (R > 1) != (q->leader != nullptr)) return 1;
    Request *ld = q->leader ? q->leader : q;
    if (std::find(leaders.begin(), leaders.end(), ld) == leaders.end()) leaders.push_back(ld);
  }
  if ((int)(leaders.size() * R) != (int)rq.size() || leaders.size() < 2) return 1;
  for (Request *ld : leaders)  // every group complete in the list
    if (R > 1)
      for (Request *m : ld->gs.members)
        if (std::find(rq.begin(), rq.end(), m) == rq.end()) return 1;
  BatchCache *b = nullptr;
  {
    std::lock_guard<std::mutex> lk(g_batch_mu);
    auto it = g_engine_batches.find(rq);
    if (it != g_engine_batches.end()) b = it->second;
  }
  if (!b) {
    b = new BatchCache();
    b->reqs = rq;
    b->nreq = (int)leaders.size();
    b->R = R;
    b->dtype = q0->dtype;
    b->op = q0->op;
    std::vector<DirectArgs> tab;
    std::vector<int> ubase(1, 0);
    for (Request *ld : leaders) {
      if (R > 1)
        for (Request *m : ld->gs.members) tab.push_back(make_direct_args(m));
      else
        tab.push_back(make_direct_args(ld));
      ubase.push_back(ubase.back() + ld->partitions * ld->slices * R);
    }
    b->units = ubase.back();
    std::vector<uint8_t> host(tab.size() * sizeof(DirectArgs) + ubase.size() * sizeof(int));
    memcpy(host.data(), tab.data(), tab.size() * sizeof(DirectArgs));
    memcpy(host.data() + tab.size() * sizeof(DirectArgs), ubase.data(), ubase.size() * sizeof(int));
    if (int rc = batch_upload(b, host.data(), host.size(), s)) {
      batch_destroy(b);
      return rc;
    }
    std::lock_guard<std::mutex> lk(g_batch_mu);
    g_engine_batches[rq] = b;
  }
  bool full = true;
  for (Request *q : rq) full = full && full_width(q);
  // width: the whole GPU's engine capacity (every local rank's share), or the
  // overlap bound while producers may still run (thin CTAs)
  const int per_rank = full ? q0->engine_warps : std::min(q0->engine_warps, q0->comm->overlap_warps);
  const int warps = std::max(1, std::min(per_rank * R, b->units));
  const int blocks = (warps * 32 + kEngineBlock - 1) / kEngineBlock;
  cudaStream_t side = q0->side;
  cudaEvent_t waited = nullptr;
  for (Request *q : rq) {
    if (!q->forked || !q->overlap) {
      PC_CUDA(cudaEventRecord(q->ev_fork, q->user_stream));
      q->fork_ev_ext = nullptr;
    }
    if (fork_event(q) != waited) PC_CUDA(cudaStreamWaitEvent(side, fork_event(q), 0));
    waited = fork_event(q);
  }
  DirectBatchArgs a{};
  a.tab = (const DirectArgs *)b->dev;
  a.ubase = (const int *)((const uint8_t *)b->dev + (size_t)b->nreq * R * sizeof(DirectArgs));
  a.nreq = b->nreq;
  a.R = R;
  a.err = (int32_t *)(q0->ctrl + q0->L.err);
  a.timeout_ms = q0->comm->timeout_ms;
  if (int rc = launch_direct_engine_batch(a, b->dtype, b->op, blocks, side, !full && q0->comm->overlap_thin))
    return rc;
  PC_CUDA(cudaEventRecord(b->ev, side));
  PC_CUDA(cudaStreamWaitEvent(s, b->ev, 0));
  for (Request *q : rq) {
    q->engine_launched = true;
    q->batch_launched = true;
    q->last_done = b->ev;
    q->joined_stream = s;
    q->active = false;
  }
  return 0;
}

}  // namespace pc

using namespace pc;

// ====================================================================== C ABI
extern "C" {

const char *pc_version(void) { return "libpc 0.1 (sm_100a)"; }

const char *pc_strerror(int err) {
  switch (err) {
    case PC_SUCCESS: return "success";
    case PC_ERR_ARG: return "invalid argument";
    case PC_ERR_CUDA: return "CUDA error";
    case PC_ERR_STATE: return "invalid request state";
    case PC_ERR_MATCH: return "send/recv or collective parameters do not match";
    case PC_ERR_TIMEOUT: return "device wait timed out";
    case PC_ERR_DEVICE: return "device-side error (bad partition / duplicate Pready)";
    case PC_ERR_NOMEM: return "out of memory";
    case PC_ERR_UNSUPPORTED: return "unsupported";
    default: return "unknown error";
  }
}

size_t pc_prequest_size(void) { return sizeof(pc_prequest_t); }

int pc_local_group_create(int size, pc_local_group_t *group) {
  if (size < 1 || !group) return PC_ERR_ARG;
  LocalGroup *g = new LocalGroup();
  g->size = size;
  g->ctxs.resize(size);
  for (int r = 0; r < size; ++r) g->ctxs[r] = {g, r};
  *group = (pc_local_group_t)g;
  return 0;
}

int pc_local_group_destroy(pc_local_group_t group) {
  delete (LocalGroup *)group;
  return 0;
}

void *pc_local_group_ctx(pc_local_group_t group, int rank) {
  LocalGroup *g = (LocalGroup *)group;
  if (!g || rank < 0 || rank >= g->size) return nullptr;
  return &g->ctxs[rank];
}

int pc_local_allgather(const void *send, size_t nbytes, void *recv, void *ctx) {
  auto *p = (std::pair<LocalGroup *, int> *)ctx;
  if (!p) return PC_ERR_ARG;
  return local_allgather_impl(p->first, p->second, send, nbytes, recv);
}

int pc_comm_create(int rank, int size, int cuda_device, pc_allgather_fn ag, void *ctx, pc_comm_t *comm) {
  if (!comm || size < 1 || size > kMaxRanks || rank < 0 || rank >= size || (size > 1 && !ag)) return PC_ERR_ARG;
  Comm *c = new Comm();
  c->rank = rank;
  c->size = size;
  c->device = cuda_device;
  c->dry = cuda_device < 0;
  c->ag = ag;
  c->ag_ctx = ctx;
  c->timeout_ms = (uint32_t)env_long("PC_TIMEOUT_MS", 20000);
  RankRec me{};
  me.magic = 0x50432431u;
  me.rank = rank;
  me.size = size;
  me.device = cuda_device;
  me.dry = c->dry;
  me.pid = (int64_t)getpid();
  me.proc_token = process_token();
  if (!c->dry) {
    cudaError_t e = cudaSetDevice(cuda_device);
    if (e != cudaSuccess) {
      delete c;
      return cuda_err(e, "cudaSetDevice");
    }
    cudaFree(nullptr);
    cudaDeviceProp prop;
    e = cudaGetDeviceProperties(&prop, cuda_device);
    if (e != cudaSuccess) {
      delete c;
      return cuda_err(e, "cudaGetDeviceProperties");
    }
    memcpy(me.uuid, &prop.uuid, 16);
    me.sms = prop.multiProcessorCount;
    int occ = 0;
    int rc = kernels_preload();  // no lazy load may later stall behind spinning kernels
    if (rc) {
      delete c;
      return rc;
    }
    rc = engine_occupancy_ctas_per_sm(&occ);
    if (rc) {
      delete c;
      return rc;
    }
    const int want = (int)env_long("PC_ENGINE_CTAS_PER_SM", 2);
    me.engine_warps = me.sms * std::max(1, std::min(occ, want)) * (kEngineBlock / 32);
    int docc = 0;
    if ((rc = direct_occupancy_ctas_per_sm(&docc))) {
      delete c;
      return rc;
    }
    me.direct_warps = me.sms * std::max(1, std::min(docc, (int)env_long("PC_DIRECT_CTAS_PER_SM", 1))) *
                      (kEngineBlock / 32);
    c->sms = me.sms;
    c->memops = memops_available();
  }
  std::vector<RankRec> all(size);
  int rc = allgather(c, &me, sizeof(me), all.data());
  if (rc) {
    delete c;
    return rc;
  }
  c->ranks = all;
  c->same_proc.assign(size, false);
  int ew = INT32_MAX, dw = INT32_MAX, ow = INT32_MAX;
  const double ofrac = std::min(1.0, std::max(0.0, env_double("PC_OVERLAP_FRAC", 0.5)));
  for (int q = 0; q < size; ++q) {
    const RankRec &r = all[q];
    if (r.magic != me.magic || r.size != size || r.rank != q || r.dry != me.dry) {
      fprintf(stderr, "[pc] comm_create: inconsistent bootstrap record from rank %d\n", q);
      delete c;
      return PC_ERR_ARG;
    }
    c->same_proc[q] = (r.pid == me.pid && r.proc_token == me.proc_token);
    if (!c->dry) {
      int on_dev = 0;
      for (int k = 0; k < size; ++k)
        if (memcmp(all[k].uuid, r.uuid, 16) == 0) ++on_dev;
      // whole CTAs per rank, so every co-located rank's engine CTAs fit at once
      const int wpb = kEngineBlock / 32;
      ew = std::min(ew, r.engine_warps / std::max(on_dev, 1) / wpb * wpb);
      dw = std::min(dw, r.direct_warps / std::max(on_dev, 1) / wpb * wpb);
      // overlap width: at most ofrac of the SMs carry an engine CTA in total,
      // so whole SMs stay free for the producer the engine waits on
      ow = std::min(ow, (int)(r.sms * ofrac) / std::max(on_dev, 1) * wpb);
    }
  }
  c->engine_warps = c->dry ? 1184 : std::max(8, (int)env_long("PC_ENGINE_WARPS", ew));
  c->direct_warps = c->dry ? 592 : std::max(8, (int)env_long("PC_DIRECT_WARPS", dw));
  c->overlap_warps = c->dry ? 592 : std::max(8, ow);
  c->overlap_thin = env_long("PC_OVERLAP_THIN", 1) != 0;
  if (!c->dry) {
    for (int q = 0; q < size; ++q) {
      if (q == rank || !c->same_proc[q] || all[q].device == cuda_device) continue;
      int can = 0;
      cudaDeviceCanAccessPeer(&can, cuda_device, all[q].device);
      if (can) {
        cudaError_t e = cudaDeviceEnablePeerAccess(all[q].device, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) {
          delete c;
          return cuda_err(e, "cudaDeviceEnablePeerAccess");
        }
        cudaGetLastError();
      }
    }
  }
  logf("comm rank %d/%d dev %d engine_warps %d memops %d", rank, size, cuda_device, c->engine_warps, (int)c->memops);
  *comm = (pc_comm_t)c;
  return 0;
}

int pc_comm_destroy(pc_comm_t comm) {
  Comm *c = (Comm *)comm;
  if (!c) return PC_ERR_ARG;
  for (Request *q : c->reqs)
    if (q) return PC_ERR_STATE;  // free requests first
  if (!c->dry) {
    cudaSetDevice(c->device);
    progress_stop(c);
    for (auto &kv : c->ipc_open) cudaIpcCloseMemHandle(kv.second);
  }
  delete c;
  return 0;
}

int pc_comm_rank(pc_comm_t comm, int *rank) {
  if (!comm || !rank) return PC_ERR_ARG;
  *rank = ((Comm *)comm)->rank;
  return 0;
}
int pc_comm_size(pc_comm_t comm, int *size) {
  if (!comm || !size) return PC_ERR_ARG;
  *size = ((Comm *)comm)->size;
  return 0;
}
int pc_comm_engine_warps(pc_comm_t comm, int *warps) {
  if (!comm || !warps) return PC_ERR_ARG;
  *warps = ((Comm *)comm)->engine_warps;
  return 0;
}

int pc_comm_overlap_warps(pc_comm_t comm, int *warps) {
  if (!comm || !warps) return PC_ERR_ARG;
  *warps = ((Comm *)comm)->overlap_warps;
  return 0;
}

int pc_psend_init(const void *buf, int partitions, size_t count, pc_dtype_t dtype, int dest, int tag,
                  pc_comm_t comm, pc_request_t *req) {
  return p2p_init(PC_KIND_PSEND, buf, nullptr, partitions, count, dtype, dest, tag, (Comm *)comm, req);
}

int pc_precv_init(void *buf, int partitions, size_t count, pc_dtype_t dtype, int source, int tag, pc_comm_t comm,
                  pc_request_t *req) {
  return p2p_init(PC_KIND_PRECV, nullptr, buf, partitions, count, dtype, source, tag, (Comm *)comm, req);
}

int pc_pallreduce_init(const void *sendbuf, void *recvbuf, int partitions, size_t count, pc_dtype_t dtype,
                       pc_op_t op, pc_algo_t algo, pc_comm_t comm, pc_request_t *req) {
  Comm *c = (Comm *)comm;
  if (!c || !req || partitions < 1 ||
      (dtype != PC_INT32 && dtype != PC_FLOAT32 && dtype != PC_FLOAT64 && dtype != PC_BF16) || op < 0 || op > 2 ||
      algo < 0 || algo > PC_ALGO_LL)
    return PC_ERR_ARG;
  const int P = c->size;
  const size_t esz = dtype_size(dtype);
  const int64_t epv = 16 / (int64_t)esz;
  const uint64_t bytes = (uint64_t)partitions * count * esz;
  if (!c->dry && (check_buf(sendbuf, bytes) || check_buf(recvbuf, bytes))) return PC_ERR_ARG;
  int a = algo;
  const bool pow2 = log2_exact(P) >= 0;
  if (a == PC_ALGO_AUTO) {
    // crossovers measured on one B200 with virtual ranks
    // (profiles/r01_sweep_allreduce_pull.jsonl): DIRECT with PULL reduce (2
    // steps, S read + S written per rank) is fastest at every size for
    // 3 <= P <= 8; at P = 2 recursive doubling (one exchange) wins up to a few
    // MiB; beyond DIRECT's peer limit: RD for small messages, ring above.
    const long rd_max = env_long("PC_RD_MAX_BYTES", 4 << 20);
    const long direct_max = env_long("PC_DIRECT_MAX_BYTES", -1);
    const bool direct_ok = P > 1 && P <= kMaxDirect && (direct_max < 0 || (long long)bytes <= direct_max);
    if (P > 1 && pow2 && (long long)bytes <= rd_max && (P == 2 || !direct_ok))
      a = PC_ALGO_RD;
    else if (direct_ok)
      a = PC_ALGO_DIRECT;
    else
      a = PC_ALGO_RING;
  }
  bool push = false, ll = false;
  // small messages: the one-shot LL variant (one hop, no fences).  Measured
  // on one B200 (virtual ranks, graph-replayed epochs, profiles/r02_ll_probe.txt)
  // it wins from ~32 KiB to 64 KiB per rank at P = 8 (256 KiB at P <= 4;
  // profiles/r02_sweep_small_graph.jsonl) — below, both are launch-bound
  // and DIRECT is ~1 us ahead; across GPUs it also saves DIRECT's two
  // system-scope fences and one NVLink hop, so it is taken from 1 byte there.
  bool spans_gpus = false;
  for (int k = 0; k < P && !c->dry; ++k)
    if (memcmp(c->ranks[k].uuid, c->ranks[c->rank].uuid, 16) != 0) spans_gpus = true;
  const long ll_min = env_long("PC_LL_AR_MIN_BYTES", spans_gpus ? 0 : 32 << 10);
  const long ll_max = env_long("PC_LL_AR_MAX_BYTES", P <= 4 ? 256 << 10 : 64 << 10);
  if (algo == PC_ALGO_AUTO && P > 1 && P <= kMaxDirect && (long long)bytes >= ll_min && (long long)bytes <= ll_max)
    a = PC_ALGO_LL;
  if (a == PC_ALGO_LL) {
    a = PC_ALGO_DIRECT;
    ll = P > 1;
  } else if (a == PC_ALGO_DIRECT_PUSH) {
    a = PC_ALGO_DIRECT;
    push = true;
  } else if (algo == PC_ALGO_AUTO && a == PC_ALGO_DIRECT) {
    const char *m = getenv("PC_DIRECT_MODE");
    push = m && strcmp(m, "push") == 0;
  }
  if (a == PC_ALGO_RD && !pow2) return PC_ERR_UNSUPPORTED;
  if (a == PC_ALGO_DIRECT && P > kMaxDirect) return PC_ERR_UNSUPPORTED;
  if (a < PC_ALGO_RING || a > PC_ALGO_DIRECT) return PC_ERR_ARG;
  Request *q;
  int rc = new_request(c, PC_KIND_PALLREDUCE, req, &q);
  if (rc) return rc;
  q->sbuf = sendbuf;
  q->rbuf = recvbuf;
  q->partitions = partitions;
  q->count = count;
  q->dtype = dtype;
  q->op = op;
  q->algo_req = algo;
  q->algo = a;
  q->direct_push = push && P > 1;
  q->direct_ll = ll;
  q->esize = esz;
  q->peer = -1;
  q->tag = 0;
  q->part_bytes = count * esz;
  q->total_bytes = bytes;
  q->send_bytes = bytes;
  q->seq = c->allreduce_seq++;
  q->agg = 1;
  q->ntransport = partitions;
  q->engine_warps = c->engine_warps;
  const int64_t L = (int64_t)count;
  const int64_t min_elems = env_long("PC_MIN_SLICE_BYTES", 8192) / (int64_t)esz;
  // units (partition slices) per engine warp: each warp sweeps its units
  // round-robin (Alg 2), so a few per warp absorb upstream skew
  const int upw = (int)std::max(1L, std::min(8L, env_long("PC_UNITS_PER_WARP", 1)));
  if (a == PC_ALGO_RING) {
    q->nsteps = 2 * (P - 1);
    q->chunk_elems = chunk_q(L, P, epv);
    choose_slices(q->chunk_elems, partitions, c->engine_warps * upw, min_elems, &q->slices, &q->slice_elems, epv);
    q->staging_bytes = P > 1 ? bytes : 0;
  } else if (a == PC_ALGO_DIRECT) {
    q->nsteps = 2;  // phase counters [u][0..1][slice]
    q->chunk_elems = chunk_q(L, P, epv);
    q->engine_warps = c->direct_warps;
    choose_slices(q->chunk_elems, partitions, c->direct_warps * upw, min_elems, &q->slices, &q->slice_elems, epv);
    // PULL: owners read the peers' send buffers directly; PUSH: staging
    // [u][source rank][q] receives every rank's copy of this rank's chunk
    q->staging_bytes = q->direct_push ? (size_t)partitions * P * (size_t)q->chunk_elems * esz : 0;
    if (q->direct_ll) {  // [2 epoch parities][P sources][N_p][lines] of 16-B LL lines, one unit per partition
      const size_t lines = std::max<size_t>(1, (q->part_bytes + 7) / 8);
      q->staging_bytes = 2 * (size_t)P * partitions * lines * 16;
      q->slices = (int)((lines + 63) / 64);  // units of 64 lines (engine.cuh kLLSlice)
      q->slice_elems = L;
    }
  } else {
    q->nsteps = log2_exact(P);
    q->chunk_elems = L;
    choose_slices(L, partitions, c->engine_warps * upw, min_elems, &q->slices, &q->slice_elems, epv);
    q->staging_bytes = bytes * (uint64_t)q->nsteps;
  }
  const size_t nflags = (size_t)partitions * (size_t)std::max(q->nsteps, 1) * (size_t)q->slices;
  q->L.build((size_t)partitions, nflags);
  return 0;
}

// Partitioned reduce-scatter / allgather / broadcast: one
// collective request on the DIRECT machinery (all peers mapped, per-peer RTR,
// co-located grouped launch), engine coll_body.  Collective over the comm:
// every rank calls it with identical arguments, in the same order as its other
// collective inits (they share the allreduce sequence numbers).
static int coll_init(int coll, const void *sendbuf, void *recvbuf, int partitions, size_t count, int dtype, int op,
                     int root, Comm *c, pc_request_t *req) {
  if (!c || !req || partitions < 1 || op < 0 || op > 2) return PC_ERR_ARG;
  const int P = c->size;
  if (coll == PC_COLL_REDUCE_SCATTER &&
      dtype != PC_INT32 && dtype != PC_FLOAT32 && dtype != PC_FLOAT64 && dtype != PC_BF16)
    return PC_ERR_ARG;
  if (dtype < 0 || dtype > 4) return PC_ERR_ARG;
  if (coll == PC_COLL_BCAST && (root < 0 || root >= P)) return PC_ERR_ARG;
  if (P > kMaxDirect) return PC_ERR_UNSUPPORTED;
  const size_t esz = dtype_size(dtype);
  const uint64_t blk = (uint64_t)partitions * count * esz;  // one rank's block set
  const uint64_t sbytes = coll == PC_COLL_REDUCE_SCATTER ? blk * P : blk;
  const uint64_t rbytes = coll == PC_COLL_ALLGATHER ? blk * P : blk;
  if (!c->dry && (check_buf(sendbuf, sbytes) || check_buf(recvbuf, rbytes))) return PC_ERR_ARG;
  Request *q;
  int rc = new_request(c, PC_KIND_PALLREDUCE, req, &q);
  if (rc) return rc;
  q->coll = coll;
  q->root = coll == PC_COLL_BCAST ? root : 0;
  q->sbuf = sendbuf;
  q->rbuf = recvbuf;
  q->partitions = partitions;
  q->count = count;
  q->dtype = dtype;
  q->op = coll == PC_COLL_REDUCE_SCATTER ? op : 0;
  q->algo_req = q->algo = PC_ALGO_DIRECT;
  q->esize = esz;
  q->peer = -1;
  q->part_bytes = count * esz;
  q->total_bytes = rbytes;
  q->send_bytes = sbytes;
  q->seq = c->allreduce_seq++;
  q->agg = 1;
  q->ntransport = partitions;
  q->engine_warps = c->direct_warps;  // fat CTAs, like the DIRECT allreduce
  q->nsteps = 2;
  q->chunk_elems = (int64_t)count;
  const int64_t epv = std::max<int64_t>(1, 16 / (int64_t)esz);
  const int64_t min_elems = std::max<int64_t>(1, env_long("PC_MIN_SLICE_BYTES", 8192) / (int64_t)esz);
  choose_slices((int64_t)count, partitions, c->direct_warps, min_elems, &q->slices, &q->slice_elems, epv);
  q->staging_bytes = 0;
  size_t nflags = (size_t)partitions * 2 * (size_t)q->slices;
  if (coll == PC_COLL_ALLGATHER) nflags += (size_t)P * partitions * (size_t)q->slices;
  q->L.build((size_t)partitions, nflags);
  return 0;
}

int pc_preduce_scatter_init(const void *sendbuf, void *recvbuf, int partitions, size_t count, pc_dtype_t dtype,
                            pc_op_t op, pc_comm_t comm, pc_request_t *req) {
  return coll_init(PC_COLL_REDUCE_SCATTER, sendbuf, recvbuf, partitions, count, dtype, op, 0, (Comm *)comm, req);
}

int pc_pallgather_init(const void *sendbuf, void *recvbuf, int partitions, size_t count, pc_dtype_t dtype,
                       pc_comm_t comm, pc_request_t *req) {
  return coll_init(PC_COLL_ALLGATHER, sendbuf, recvbuf, partitions, count, dtype, 0, 0, (Comm *)comm, req);
}

int pc_pbcast_init(void *buf, int partitions, size_t count, pc_dtype_t dtype, int root, pc_comm_t comm,
                   pc_request_t *req) {
  return coll_init(PC_COLL_BCAST, buf, buf, partitions, count, dtype, 0, root, (Comm *)comm, req);
}

int pc_start(pc_request_t req, pc_stream_t stream) {
  Request *q = (Request *)req;
  if (!q) return PC_ERR_ARG;
  if (q->active) return PC_ERR_STATE;
  Comm *c = q->comm;
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  if (!c->dry) {
    PC_CUDA(cudaSetDevice(c->device));
    PC_CUDA(cudaStreamIsCapturing((cudaStream_t)stream, &cs));
  }
  if (int rc = epoch_begin(q, (cudaStream_t)stream, cs != cudaStreamCaptureStatusNone)) return rc;
  q->epoch++;
  q->active = true;
  q->engine_launched = false;
  q->engine_registered = false;
  q->prepared_this_epoch = false;
  q->user_stream = (cudaStream_t)stream;
  if (c->dry) return 0;
  if (!q->ctrl) {
    int arc = alloc_ctrl(q);
    if (arc) return arc;
  }
  if (cs != cudaStreamCaptureStatusNone) q->graph_mode = true;
  // Eager requests write the epoch with a stream memop (cheapest); once a
  // request has been captured into a CUDA graph its epoch is advanced on the
  // device, so replays produce new epochs without the host.
  int rc;
  if (!q->graph_mode && c->memops) {
    rc = stream_write_u32(c, (cudaStream_t)stream, q->ctrl + q->L.epoch, q->epoch);
  } else {
    q->graph_mode = true;
    rc = launch_epoch_bump(q->ctrl + q->L.epoch, (cudaStream_t)stream);
  }
  return rc ? rc : fork_point(q, (cudaStream_t)stream);
}

int pc_pbuf_prepare(pc_request_t req, pc_stream_t stream) {
  Request *q = (Request *)req;
  if (!q) return PC_ERR_ARG;
  if (!q->active) return PC_ERR_STATE;
  Comm *c = q->comm;
  if (!c->dry) PC_CUDA(cudaSetDevice(c->device));
  if (!q->exchanged) {
    int rc = exchange_round(c, q);
    if (rc) return rc;
  }
  if (!q->matched) return PC_ERR_MATCH;
  if (c->dry) return 0;
  q->user_stream = (cudaStream_t)stream;
  if (!q->prepared_this_epoch) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    PC_CUDA(cudaStreamIsCapturing((cudaStream_t)stream, &cs));
    if (cs != cudaStreamCaptureStatusNone) q->graph_mode = true;
    if (!q->graph_mode && c->memops) {  // eager: host epoch == device epoch
      for (auto &t : q->rtr_targets) {
        int rc = stream_write_u32(c, (cudaStream_t)stream, t.first + q->L.rtr + t.second, q->epoch);
        if (rc) return rc;
      }
    } else if (!q->rtr_targets.empty()) {
      RtrArgs a{};
      a.epoch = q->ctrl + q->L.epoch;
      a.sys = q->sys_scope;
      for (auto &t : q->rtr_targets) {
        if (a.n == kMaxRdSteps + 2) return PC_ERR_UNSUPPORTED;
        a.dst[a.n++] = t.first + q->L.rtr + t.second;
      }
      int rc = launch_rtr(a, (cudaStream_t)stream);
      if (rc) return rc;
    }
    q->prepared_this_epoch = true;
    if (int rc = fork_point(q, (cudaStream_t)stream)) return rc;
  }
  return 0;
}

// Start + Pbuf_prepare (+ Pready of every partition) of n already-exchanged
// requests of one GPU in ONE kernel (the small-message epoch: one launch
// instead of three; CUDA-graph capturable).
int pc_epoch_all(int n, pc_request_t *reqs, int pready, pc_stream_t stream) {
  if (n < 1 || !reqs) return PC_ERR_ARG;
  // validate everything before any request is touched (no half-started batch)
  int nrtr = 0;
  for (int i = 0; i < n; ++i) {
    Request *q = (Request *)reqs[i];
    if (!q) return PC_ERR_ARG;
    for (int j = 0; j < i; ++j)
      if (reqs[j] == reqs[i]) return PC_ERR_ARG;  // one epoch per request per call
    if (q->active) return PC_ERR_STATE;
    if (!q->exchanged) return PC_ERR_STATE;
    if (!q->matched) return PC_ERR_MATCH;
    if (pready && (q->kind != PC_KIND_PALLREDUCE || q->inline_ar)) return PC_ERR_ARG;  // R33: Pready folds
    if (q->comm->device != ((Request *)reqs[0])->comm->device || q->comm->dry != ((Request *)reqs[0])->comm->dry)
      return PC_ERR_ARG;
    if (group_blocks_start(q)) return PC_ERR_STATE;
    nrtr += (int)q->rtr_targets.size();
  }
  const bool dry = ((Request *)reqs[0])->comm->dry;
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  if (!dry) {
    PC_CUDA(cudaSetDevice(((Request *)reqs[0])->comm->device));
    PC_CUDA(cudaStreamIsCapturing((cudaStream_t)stream, &cs));
  }
  if (!dry && (n > kMaxPreadyAll || nrtr > kMaxCtl)) {  // beyond one kernel's parameters: device tables
    std::vector<Request *> rq(n);
    for (int i = 0; i < n; ++i) rq[i] = (Request *)reqs[i];
    {
      std::lock_guard<std::mutex> lk(g_batch_mu);
      if (!g_epoch_batches.count(rq) && cs != cudaStreamCaptureStatusNone) return PC_ERR_STATE;
    }
    for (Request *q : rq) {
      if (int rc = epoch_begin(q, (cudaStream_t)stream, cs != cudaStreamCaptureStatusNone)) return rc;
      if (cs != cudaStreamCaptureStatusNone) q->graph_mode = true;
      q->epoch++;
      q->active = true;
      q->engine_launched = false;
      q->engine_registered = false;
      q->prepared_this_epoch = true;
      q->user_stream = (cudaStream_t)stream;
    }
    return epoch_all_batched(rq, pready, (cudaStream_t)stream);
  }
  EpochAllArgs a{};
  for (int i = 0; i < n; ++i) {
    Request *q = (Request *)reqs[i];
    if (int rc = epoch_begin(q, (cudaStream_t)stream, cs != cudaStreamCaptureStatusNone)) return rc;
    if (cs != cudaStreamCaptureStatusNone) q->graph_mode = true;
    q->epoch++;
    q->active = true;
    q->engine_launched = false;
    q->engine_registered = false;
    q->prepared_this_epoch = true;
    q->user_stream = (cudaStream_t)stream;
    if (dry) continue;
    const int k = a.n++;
    a.epoch[k] = q->ctrl + q->L.epoch;
    for (auto &t : q->rtr_targets) {
      a.rtr_dst[a.nrtr] = t.first + q->L.rtr + t.second;
      a.rtr_req[a.nrtr] = (uint8_t)k;
      if (q->sys_scope) a.rtr_sysmask |= 1ull << a.nrtr;
      ++a.nrtr;
    }
    if (pready) {
      a.ready[k] = q->ctrl + q->L.ready;
      a.partitions[k] = q->partitions;
    }
  }
  if (dry) return 0;
  a.pready = pready ? 1 : 0;
  if (int rc = launch_epoch_all(a, (cudaStream_t)stream)) return rc;
  for (int i = 0; i < n; ++i) {
    Request *q = (Request *)reqs[i];
    q->host_ready_all = pready != 0;
    if (int rc = fork_point(q, (cudaStream_t)stream)) return rc;
  }
  return 0;
}

// MPI_Startall: one device kernel advances the epochs of all n requests.
int pc_startall(int n, pc_request_t *reqs, pc_stream_t stream) {
  if (n < 0 || (n > 0 && !reqs)) return PC_ERR_ARG;
  for (int i = 0; i < n; ++i) {
    Request *q = (Request *)reqs[i];
    if (!q) return PC_ERR_ARG;
    for (int j = 0; j < i; ++j)
      if (reqs[j] == reqs[i]) return PC_ERR_ARG;  // one epoch per request per call
    if (q->active) return PC_ERR_STATE;
    if (q->comm->device != ((Request *)reqs[0])->comm->device || q->comm->dry != ((Request *)reqs[0])->comm->dry)
      return PC_ERR_ARG;
    if (group_blocks_start(q)) return PC_ERR_STATE;
  }
  const bool dry = n == 0 || ((Request *)reqs[0])->comm->dry;
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  if (!dry) {
    PC_CUDA(cudaSetDevice(((Request *)reqs[0])->comm->device));
    PC_CUDA(cudaStreamIsCapturing((cudaStream_t)stream, &cs));
    for (int i = 0; i < n; ++i)  // device resources first: nothing below can fail half-way on allocation
      if (int arc = alloc_ctrl((Request *)reqs[i])) return arc;
  }
  CtlArgs a{};
  int first = 0;  // requests [first, i] are in the pending kernel
  for (int i = 0; i < n; ++i) {
    Request *q = (Request *)reqs[i];
    if (int rc = epoch_begin(q, (cudaStream_t)stream, cs != cudaStreamCaptureStatusNone)) return rc;
    if (cs != cudaStreamCaptureStatusNone) q->graph_mode = true;
    q->epoch++;
    q->active = true;
    q->engine_launched = false;
    q->engine_registered = false;
    q->prepared_this_epoch = false;
    q->user_stream = (cudaStream_t)stream;
    if (dry) continue;
    a.epoch[a.n] = q->ctrl + q->L.epoch;
    a.dst[a.n] = nullptr;
    if (++a.n == kMaxCtl || i == n - 1) {
      if (int rc = launch_ctl(a, (cudaStream_t)stream)) return rc;
      for (int k = first; k <= i; ++k)
        if (int rc = fork_point((Request *)reqs[k], (cudaStream_t)stream)) return rc;
      a.n = 0;
      first = i + 1;
    }
  }
  return 0;
}

// Ready-to-receive for n already-exchanged requests in one kernel (the first
// pc_pbuf_prepare of each request, which exchanges and maps, must be a
// pc_pbuf_prepare call).
int pc_pbuf_prepare_all(int n, pc_request_t *reqs, pc_stream_t stream) {
  if (n < 0 || (n > 0 && !reqs)) return PC_ERR_ARG;
  for (int i = 0; i < n; ++i) {
    Request *q = (Request *)reqs[i];
    if (!q) return PC_ERR_ARG;
    if (!q->active) return PC_ERR_STATE;
    if (!q->exchanged) return PC_ERR_STATE;
    if (!q->matched) return PC_ERR_MATCH;
  }
  CtlArgs a{};
  std::vector<Request *> prepared;
  for (int i = 0; i < n; ++i) {
    Request *q = (Request *)reqs[i];
    q->user_stream = (cudaStream_t)stream;
    if (q->comm->dry || q->prepared_this_epoch) continue;
    for (auto &t : q->rtr_targets) {
      a.epoch[a.n] = q->ctrl + q->L.epoch;
      a.dst[a.n] = t.first + q->L.rtr + t.second;
      a.sys[a.n] = q->sys_scope;
      if (++a.n == kMaxCtl) {
        PC_CUDA(cudaSetDevice(q->comm->device));
        int rc = launch_ctl(a, (cudaStream_t)stream);
        if (rc) return rc;
        a.n = 0;
      }
    }
    q->prepared_this_epoch = true;
    prepared.push_back(q);
  }
  if (a.n) {
    PC_CUDA(cudaSetDevice(((Request *)reqs[0])->comm->device));
    if (int rc = launch_ctl(a, (cudaStream_t)stream)) return rc;
  }
  for (Request *q : prepared)
    if (int rc = fork_point(q, (cudaStream_t)stream)) return rc;
  return 0;
}

int pc_prequest_create(pc_request_t req, pc_gran_t gran, int aggregation, pc_copy_t copy, pc_prequest_t *out) {
  Request *q = (Request *)req;
  if (!q || !out || gran < 0 || gran > 2 || copy < 0 || copy > 3) return PC_ERR_ARG;
  Comm *c = q->comm;
  if (!q->exchanged || !q->matched) return PC_ERR_STATE;  // after the first pbuf_prepare (Listing 2)
  if (q->kind == PC_KIND_PALLREDUCE && aggregation != 1) return PC_ERR_ARG;
  if (q->kind == PC_KIND_PALLREDUCE && copy == PC_COPY_LL) return PC_ERR_UNSUPPORTED;
  if (q->kind == PC_KIND_PSEND && copy == PC_COPY_LL && (!q->ll_lines || q->xpart)) return PC_ERR_UNSUPPORTED;
  if (q->kind == PC_KIND_PALLREDUCE && copy == PC_COPY_HOST) return PC_ERR_UNSUPPORTED;
  // the progress thread signals with stream memops (stores), not the counters R30 needs
  if (q->kind == PC_KIND_PSEND && copy == PC_COPY_HOST && q->xpart) return PC_ERR_UNSUPPORTED;
  if (q->kind == PC_KIND_PSEND) {
    if (aggregation < 1 || aggregation > q->partitions) return PC_ERR_ARG;
    if (q->has_preq && (aggregation != q->agg)) return PC_ERR_STATE;  // the transport layout is fixed
    q->agg = aggregation;
    q->ntransport = (q->partitions + aggregation - 1) / aggregation;
    q->copy = copy;
    const uint64_t tb = (uint64_t)aggregation * q->part_bytes;
    const int64_t min_bytes = env_long("PC_MIN_SLICE_BYTES", 16384);
    int ns;
    int64_t sl;
    // slices in 4-byte "elements" of the transport partition's bytes
    choose_slices((int64_t)((tb + 3) / 4), q->ntransport, c->engine_warps, std::max<int64_t>(1, min_bytes / 4), &ns,
                  &sl);
    q->slices = ns;
    q->slice_elems = sl * 4;  // bytes per slice
    q->engine_warps = c->engine_warps;
    if (!c->dry) {
      PC_CUDA(cudaSetDevice(c->device));
      if (copy == PC_COPY_HOST) {
        int prc = progress_register(q);
        if (prc) return prc;
      }
      // publish the transport layout (g) in the receiver's control block
      uint32_t g = (uint32_t)aggregation | (copy == PC_COPY_LL ? PC_LAYOUT_LL : 0u) | (q->xpart ? PC_LAYOUT_XP : 0u);
      PC_CUDA(cudaMemcpyAsync(q->peer_ctrl + q->L.layout, &g, 4, cudaMemcpyHostToDevice, q->side));
      PC_CUDA(cudaStreamSynchronize(q->side));
    }
  } else if (q->kind == PC_KIND_PALLREDUCE) {
    if (copy == PC_COPY_INLINE) {  // R33: INLINE allreduce (DIRECT schedule bits, P <= 8)
      if (q->coll != PC_COLL_ALLREDUCE || q->algo != PC_ALGO_DIRECT || q->direct_push || q->direct_ll ||
          c->size > PC_AR_MAX)
        return PC_ERR_UNSUPPORTED;
      if (!c->dry && !q->ar_tab) {
        pc_ar_tab_s t{};
        const int P = c->size, r = c->rank;
        for (int k = 0; k < P; ++k) {
          if (k == r) {
            t.send[k] = (const uint8_t *)q->sbuf;
            t.recv[k] = (uint8_t *)q->rbuf;
            t.done[k] = q->ctrl + q->L.sent;
          } else {
            const int j = mod(k - r - 1, P);  // peer j = rank (r + 1 + j) mod P
            t.send[k] = q->nb_stage[j];        // DIRECT exports its send buffer in the stage slot
            t.recv[k] = q->nb_buf[j];
            t.done[k] = q->nb_ctrl[j] + q->L.sent;
          }
        }
        t.cnt = (r == 0 ? q->ctrl : q->nb_ctrl[mod(0 - r - 1, P)]) + q->L.cnt;
        t.rtr = q->ctrl + q->L.rtr;
        PC_CUDA(cudaSetDevice(c->device));
        PC_CUDA(cudaMalloc(&q->ar_tab, sizeof(t)));
        PC_CUDA(cudaMemcpy(q->ar_tab, &t, sizeof(t), cudaMemcpyHostToDevice));
      }
      q->inline_ar = true;
    } else {
      q->inline_ar = false;
    }
    q->copy = copy;
  } else {
    q->copy = copy;
  }
  q->has_preq = true;
  fill_prequest(q, out);
  return 0;
}

int pc_prequest_free(pc_prequest_t *preq) {
  if (!preq) return PC_ERR_ARG;
  memset(preq, 0, sizeof(*preq));
  return 0;
}

// Make sure this epoch's engine is (or will be) launched; *ev = the event that
// completes with it, or null when a co-located group is still incomplete.
static int ensure_engine(Request *q, bool block, cudaStream_t ws, cudaEvent_t *ev) {
  *ev = nullptr;
  if (!needs_engine(q)) return 0;
  if (q->batch_launched) {  // this epoch's engine ran in a batched waitall launch
    *ev = q->last_done;
    return 0;
  }
  if (q->leader) {
    bool launched = false;
    int rc = group_register(q, block, ws, &launched);
    if (launched) *ev = q->leader->gs.ev;
    return rc;
  }
  if (!q->engine_launched) {
    int rc = launch_single(q);
    if (rc) return rc;
  }
  *ev = q->ev_done;
  return 0;
}

static int wait_common(Request *q, cudaStream_t s, bool host) {
  Comm *c = q->comm;
  if (!q->active) return 0;
  if (c->dry) {
    q->active = false;
    return 0;
  }
  PC_CUDA(cudaSetDevice(c->device));
  if (!q->exchanged || !q->matched) return PC_ERR_STATE;
  int32_t *err = (int32_t *)(q->ctrl + q->L.err);
  const bool engine = (q->kind == PC_KIND_PALLREDUCE && !q->inline_ar) || (q->kind == PC_KIND_PSEND && q->copy == 1);
  int rc;
  if (q->inline_ar) {  // R33: every done[u] of this rank reached the epoch (written by the folding ranks)
    cudaStream_t ws = host ? q->side : s;
    if (host) {
      PC_CUDA(cudaEventRecord(q->ev_fork, q->user_stream));
      PC_CUDA(cudaStreamWaitEvent(q->side, q->ev_fork, 0));
    }
    if ((rc = launch_wait_words(q->ctrl + q->L.sent, q->partitions, q->ctrl + q->L.epoch, 1, nullptr, q->partitions,
                                err, c->timeout_ms, ws, q->sys_scope != 0)))
      return rc;
    if (host) PC_CUDA(cudaStreamSynchronize(q->side));
    q->joined_stream = host ? kHostJoined : s;
  } else if (engine) {
    if (q->kind == PC_KIND_PSEND && !q->has_preq) return PC_ERR_STATE;
    cudaEvent_t ev = nullptr;
    if ((rc = ensure_engine(q, host, host ? nullptr : s, &ev))) return rc;
    if (host) {
      if (!ev) return PC_ERR_STATE;
      PC_CUDA(cudaEventSynchronize(ev));
      q->joined_stream = kHostJoined;
    } else if (ev) {
      PC_CUDA(cudaStreamWaitEvent(s, ev, 0));
      q->joined_stream = s;
    } else {
      q->join_pending = true;  // the group's last wait joins it on s
      q->wait_stream = s;
    }
    // (co-located group not complete yet: the last local rank's wait launches
    //  the grouped engine on its stream; see pc.h "In-process rank groups")
  } else {
    cudaStream_t ws = host ? q->side : s;
    if (host) {
      // ordered after the work the user enqueued before pc_wait on the epoch's stream
      PC_CUDA(cudaEventRecord(q->ev_fork, q->user_stream));
      PC_CUDA(cudaStreamWaitEvent(q->side, q->ev_fork, 0));
    }
    if (q->kind == PC_KIND_PSEND) {
      if (!q->has_preq) return PC_ERR_STATE;
      rc = launch_wait_words(q->ctrl + q->L.sent, q->ntransport, q->ctrl + q->L.epoch, 1, nullptr, q->partitions, err,
                             c->timeout_ms, ws, false, q->copy == PC_COPY_LL ? q->ctrl + q->L.rtr : nullptr);
    } else {
      pc_prequest_t rq;
      fill_prequest(q, &rq);
      rc = launch_recv_wait(rq, nullptr, ws);
    }
    if (rc) return rc;
    if (host) PC_CUDA(cudaStreamSynchronize(q->side));
  }
  q->active = false;
  if (host) return error_rc(q);
  return 0;
}

int pc_wait(pc_request_t req) {
  Request *q = (Request *)req;
  if (!q) return PC_ERR_ARG;
  return wait_common(q, nullptr, true);
}

int pc_wait_on_stream(pc_request_t req, pc_stream_t stream) {
  Request *q = (Request *)req;
  if (!q) return PC_ERR_ARG;
  return wait_common(q, (cudaStream_t)stream, false);
}

int pc_waitall_on_stream(int n, pc_request_t *reqs, pc_stream_t stream) {
  if (n < 0 || (n > 0 && !reqs)) return PC_ERR_ARG;
  for (int i = 0; i < n; ++i)
    if (!reqs[i]) return PC_ERR_ARG;
  cudaStream_t s = (cudaStream_t)stream;
  // validate first (as wait_common), then enqueue
  std::vector<Request *> fused;
  for (int i = 0; i < n; ++i) {
    Request *q = (Request *)reqs[i];
    if (!q->active || q->comm->dry) continue;
    const bool engine = q->kind == PC_KIND_PALLREDUCE || (q->kind == PC_KIND_PSEND && q->copy == 1);
    if (engine) continue;
    if (!q->exchanged || !q->matched) return PC_ERR_STATE;
    if (q->kind == PC_KIND_PSEND && !q->has_preq) return PC_ERR_STATE;
    if (!fused.empty() && q->comm->device != fused[0]->comm->device) return PC_ERR_ARG;
    fused.push_back(q);
  }
  {  // several DIRECT allreduces: one batched engine launch
    std::vector<Request *> eng;
    for (int i = 0; i < n; ++i) {
      Request *q = (Request *)reqs[i];
      if (q->active && !q->comm->dry && needs_engine(q) && q->kind == PC_KIND_PALLREDUCE) eng.push_back(q);
    }
    if (eng.size() >= 2) {
      PC_CUDA(cudaSetDevice(eng[0]->comm->device));
      const int rc = engine_batch(eng, s);
      if (rc < 0) return rc;
    }
  }
  for (int i = 0; i < n; ++i) {  // engine-moved (not batched) and dry requests: their own path
    Request *q = (Request *)reqs[i];
    if (std::find(fused.begin(), fused.end(), q) != fused.end()) continue;
    if (int rc = wait_common(q, s, false)) return rc;
  }
  if (fused.empty()) return 0;
  PC_CUDA(cudaSetDevice(fused[0]->comm->device));
  // The fused grid stays within what is co-resident at once (4 spinning
  // 256-thread blocks per SM, as one recv_wait kernel): several LL receives
  // share that budget (their bodies are grid-stride over their block range).
  const int budget = 4 * std::max(fused[0]->comm->sms, 1) - kMaxWaitAll;
  for (size_t g0 = 0; g0 < fused.size(); g0 += kMaxWaitAll) {
    WaitAllArgs a{};
    a.block_start[0] = 0;
    int want[kMaxWaitAll], total = 0;
    for (size_t k = g0; k < fused.size() && a.n < kMaxWaitAll; ++k) {
      fill_prequest(fused[k], &a.q[a.n]);
      want[a.n] = fused[k]->kind == PC_KIND_PSEND ? wait_words_blocks(fused[k]->ntransport) : recv_wait_blocks(a.q[a.n]);
      total += want[a.n];
      ++a.n;
    }
    for (int k = 0; k < a.n; ++k) {
      const int nb = total <= budget ? want[k] : std::max(1, (int)((int64_t)want[k] * budget / total));
      a.block_start[k + 1] = a.block_start[k] + nb;
    }
    if (int rc = launch_wait_all(a, s)) return rc;
    for (size_t k = g0; k < g0 + (size_t)a.n; ++k) fused[k]->active = false;
  }
  return 0;
}

static int read_words(Request *q, size_t off, size_t n, uint32_t *h) {
  PC_CUDA(cudaMemcpyAsync(h, q->ctrl + off, n * 4, cudaMemcpyDeviceToHost, q->side));
  PC_CUDA(cudaStreamSynchronize(q->side));
  return 0;
}

static bool reached_h(uint32_t v, uint32_t t) { return (int32_t)(v - t) >= 0; }

// R30 (host copy of pc_detail::xp_need): send transport partitions of g
// partitions x peer_part_bytes overlapping receive partition p
static uint32_t xp_need_h(uint64_t p, uint64_t part_bytes, uint32_t g, uint64_t peer_part_bytes) {
  const uint64_t tb = (uint64_t)g * peer_part_bytes, lo = p * part_bytes, hi = lo + part_bytes;
  return (uint32_t)((hi - 1) / tb - lo / tb + 1);
}

// The epoch a host-side query compares against: the later of the host's count
// of pc_start calls and the device epoch word (which CUDA-graph replays of a
// captured Start advance without the host seeing it).
static int current_epoch(Request *q, uint32_t *e) {
  uint32_t d = 0;
  int rc = read_words(q, q->L.epoch, 1, &d);
  if (rc) return rc;
  if (reached_h(d, q->epoch)) q->epoch = d;
  *e = q->epoch;
  return 0;
}

int pc_parrived(pc_request_t req, int partition, int *flag) {
  Request *q = (Request *)req;
  const bool ag = q && q->kind == PC_KIND_PALLREDUCE && q->coll == PC_COLL_ALLGATHER;
  if (!q || !flag || partition < 0 || partition >= (ag ? q->comm->size : 1) * q->partitions) return PC_ERR_ARG;
  *flag = 0;
  if (q->comm->dry) return 0;
  PC_CUDA(cudaSetDevice(q->comm->device));
  uint32_t v = 0, e = 0;
  int rc;
  if ((rc = current_epoch(q, &e))) return rc;
  if (ag) {  // receive partition k * partitions + u: rank k's partition u, every slice
    std::vector<uint32_t> h((size_t)q->slices);
    const size_t off = q->L.flags + (size_t)q->partitions * 2 * q->slices + (size_t)partition * q->slices;
    if ((rc = read_words(q, off, h.size(), h.data()))) return rc;
    *flag = 1;
    for (uint32_t w : h) *flag = *flag && reached_h(w, e);
  } else if (q->kind == PC_KIND_PALLREDUCE) {
    if ((rc = read_words(q, (q->inline_ar ? q->L.sent : q->L.donecnt) + partition, 1, &v))) return rc;
    *flag = reached_h(v, e * (uint32_t)(q->inline_ar ? 1 : q->slices));
  } else if (q->kind == PC_KIND_PRECV) {
    uint32_t g = 0;
    if ((rc = read_words(q, q->L.layout, 1, &g))) return rc;
    if (g == 0) return 0;
    if (g & PC_LAYOUT_LL) {  // check the lines and unpack them on the device
      pc_prequest_t rq;
      fill_prequest(q, &rq);
      if ((rc = launch_parrived(rq, partition, (int32_t *)(q->ctrl + q->L.scratch), q->side))) return rc;
      if ((rc = read_words(q, q->L.scratch, 1, &v))) return rc;
      *flag = v != 0;
      return 0;
    }
    if (g & PC_LAYOUT_XP) {  // R30: counter of this receive partition, one bump per overlapping transport
      if ((rc = read_words(q, q->L.flags + partition, 1, &v))) return rc;
      *flag = reached_h(v, e * xp_need_h((uint64_t)partition, q->part_bytes, g & PC_LAYOUT_G, q->peer_part_bytes));
      return 0;
    }
    if ((rc = read_words(q, q->L.flags + partition / g, 1, &v))) return rc;
    *flag = reached_h(v, e);
  } else {
    if ((rc = read_words(q, q->L.sent + partition / q->agg, 1, &v))) return rc;
    *flag = reached_h(v, e);
  }
  return 0;
}

int pc_test(pc_request_t req, int *flag) {
  Request *q = (Request *)req;
  if (!q || !flag) return PC_ERR_ARG;
  *flag = 1;
  if (!q->active || q->comm->dry) {
    if (q->active) q->active = false;
    return 0;
  }
  PC_CUDA(cudaSetDevice(q->comm->device));
  int rc;
  const bool engine = (q->kind == PC_KIND_PALLREDUCE && !q->inline_ar) || (q->kind == PC_KIND_PSEND && q->copy == 1);
  bool done = false;
  if (q->inline_ar) {  // R33: every INLINE done word reached the epoch
    uint32_t e = 0;
    if ((rc = current_epoch(q, &e))) return rc;
    std::vector<uint32_t> h((size_t)q->partitions);
    if ((rc = read_words(q, q->L.sent, h.size(), h.data()))) return rc;
    done = true;
    for (uint32_t v : h) done = done && reached_h(v, e);
  } else if (engine) {
    cudaEvent_t ev = nullptr;
    if (q->kind == PC_KIND_PSEND && !q->has_preq) {
      *flag = 0;
      return 0;
    }
    if ((rc = ensure_engine(q, false, nullptr, &ev))) return rc;
    if (!ev) {
      *flag = 0;
      return 0;
    }
    cudaError_t e = cudaEventQuery(ev);
    if (e == cudaErrorNotReady) {
      cudaGetLastError();
      done = false;
    } else if (e == cudaSuccess) {
      done = true;
    } else {
      return cuda_err(e, "cudaEventQuery");
    }
  } else {
    int n = q->kind == PC_KIND_PSEND ? q->ntransport : 0;
    size_t off = q->kind == PC_KIND_PSEND ? q->L.sent : q->L.flags;
    bool ll = false;
    if (q->kind == PC_KIND_PRECV) {
      uint32_t g = 0;
      if ((rc = read_words(q, q->L.layout, 1, &g))) return rc;
      if (g & (PC_LAYOUT_LL | PC_LAYOUT_XP)) {  // LL: count lines not there yet (and unpack those that
                                                // are) on the device; XP (R30): per-partition targets
        pc_prequest_t rq;
        fill_prequest(q, &rq);
        int32_t *pend = (int32_t *)(q->ctrl + q->L.scratch);
        PC_CUDA(cudaMemsetAsync(pend, 0, 4, q->side));
        if ((rc = launch_recv_wait(rq, pend, q->side))) return rc;
        uint32_t np = 1;
        if ((rc = read_words(q, q->L.scratch, 1, &np))) return rc;
        ll = true;
        done = np == 0;
      } else {
        n = g ? (q->partitions + (int)g - 1) / (int)g : -1;
      }
    }
    if (!ll) done = n >= 0;
    if (!ll && n > 0) {
      uint32_t e = 0;
      if ((rc = current_epoch(q, &e))) return rc;
      std::vector<uint32_t> h((size_t)n);
      if ((rc = read_words(q, off, (size_t)n, h.data()))) return rc;
      for (uint32_t v : h) done = done && reached_h(v, e);
      if (done && q->kind == PC_KIND_PSEND && q->copy == PC_COPY_LL) {  // R29: receiver posted RTR(e)
        uint32_t r = 0;
        if ((rc = read_words(q, q->L.rtr, 1, &r))) return rc;
        done = reached_h(r, e);
      }
    }
  }
  int erc = error_rc(q);
  if (erc) {
    q->active = false;
    return erc;
  }
  *flag = done ? 1 : 0;
  if (done) {
    q->active = false;
    q->joined_stream = kHostJoined;
  }
  return 0;
}

int pc_preadyall(int n, pc_request_t *reqs, pc_stream_t stream) {
  if (n < 0 || (n > 0 && !reqs)) return PC_ERR_ARG;
  PreadyAllArgs a{};
  for (int i = 0; i < n; ++i) {
    Request *q = (Request *)reqs[i];
    if (!q) return PC_ERR_ARG;
    if (!q->active) return PC_ERR_STATE;
    if (q->kind == PC_KIND_PRECV) return PC_ERR_ARG;
    if (q->kind == PC_KIND_PSEND && !q->has_preq) return PC_ERR_STATE;
    if (q->comm->device != ((Request *)reqs[0])->comm->device) return PC_ERR_ARG;
    if (q->comm->dry) continue;
    fill_prequest(q, &a.q[a.n]);
    if (++a.n == kMaxPreadyAll) {
      PC_CUDA(cudaSetDevice(q->comm->device));
      int rc = launch_pready_all(a, (cudaStream_t)stream);
      if (rc) return rc;
      a.n = 0;
    }
  }
  if (a.n) {
    PC_CUDA(cudaSetDevice(((Request *)reqs[0])->comm->device));
    if (int rc = launch_pready_all(a, (cudaStream_t)stream)) return rc;
  }
  // every partition is ready once this kernel ran: the engine may start after
  // it at full width (no producer left to overlap)
  for (int i = 0; i < n; ++i) {
    Request *q = (Request *)reqs[i];
    if (q->comm->dry) continue;
    q->host_ready_all = true;
    if (int rc = fork_point(q, (cudaStream_t)stream)) return rc;
  }
  return 0;
}

int pc_pready_range(int lo, int hi, pc_request_t req, pc_stream_t stream) {
  Request *q = (Request *)req;
  if (!q || lo < 0 || hi < lo || hi >= q->partitions) return PC_ERR_ARG;
  if (!q->active) return PC_ERR_STATE;
  if (q->kind == PC_KIND_PRECV) return PC_ERR_ARG;
  if (q->comm->dry) return 0;
  if (q->kind == PC_KIND_PSEND && !q->has_preq) return PC_ERR_STATE;
  PC_CUDA(cudaSetDevice(q->comm->device));
  pc_prequest_t p;
  fill_prequest(q, &p);
  if (int rc = launch_pready_range(p, lo, hi, (cudaStream_t)stream)) return rc;
  if (lo == 0 && hi == q->partitions - 1) {  // every partition: as pc_preadyall
    q->host_ready_all = true;
    return fork_point(q, (cudaStream_t)stream);
  }
  return 0;
}

int pc_pready(int partition, pc_request_t req, pc_stream_t stream) {
  return pc_pready_range(partition, partition, req, stream);
}

int pc_request_free(pc_request_t *req) {
  if (!req || !*req) return PC_ERR_ARG;
  Request *q = (Request *)*req;
  if (q->active && q->matched) return PC_ERR_STATE;  // an unmatched request has nothing in flight
  Comm *c = q->comm;
  if (!c->dry) {
    cudaSetDevice(c->device);
    if (q->side) cudaStreamSynchronize(q->side);
    batch_drop(q);
    if (q->hready || q->pe_registered) progress_unregister(q);
    if (q->ctrl) cudaFree(q->ctrl);
    if (q->staging) cudaFree(q->staging);
    if (q->side) cudaStreamDestroy(q->side);
    if (q->ev_fork) cudaEventDestroy(q->ev_fork);
    if (q->ar_tab) cudaFree(q->ar_tab);
    if (q->ev_done) cudaEventDestroy(q->ev_done);
    if (q->gs.ev) cudaEventDestroy(q->gs.ev);
    for (cudaEvent_t e : q->gs.tlog.pool) cudaEventDestroy(e);
    for (cudaEvent_t e : q->tlog.pool) cudaEventDestroy(e);
  }
  c->reqs[q->index] = nullptr;
  delete q;
  *req = nullptr;
  return 0;
}

int pc_schedule_ring(int P, int r, int32_t *out_rows5) {
  if (P < 1 || P > kMaxRanks || r < 0 || r >= P || !out_rows5) return PC_ERR_ARG;
  return ring_rows(P, r, out_rows5);
}

int pc_schedule_rd(int P, int r, int32_t *out_rows5) {
  if (P < 1 || P > kMaxRanks || r < 0 || r >= P || !out_rows5) return PC_ERR_ARG;
  return rd_rows(P, r, out_rows5);
}

int pc_chunk_bounds(int64_t L, int P, int64_t *out) {
  if (L < 0 || P < 1 || !out) return PC_ERR_ARG;
  const int64_t q = chunk_q(L, P);
  for (int c = 0; c < P; ++c) out[c] = std::min<int64_t>((int64_t)c * q, L);
  out[P] = L;
  return 0;
}

int pc_request_info(pc_request_t req, int *algo, int *slices, int64_t *slice_elems, int *engine_warps) {
  Request *q = (Request *)req;
  if (!q) return PC_ERR_ARG;
  if (algo) *algo = q->direct_ll ? PC_ALGO_LL : q->direct_push ? PC_ALGO_DIRECT_PUSH : q->algo;
  if (slices) *slices = q->slices;
  if (slice_elems) *slice_elems = q->slice_elems;
  if (engine_warps) *engine_warps = q->engine_warps;
  return 0;
}

int pc_request_match(pc_request_t req, int *peer, int *peer_request_index) {
  Request *q = (Request *)req;
  if (!q || !peer || !peer_request_index) return PC_ERR_ARG;
  if (!q->exchanged || !q->matched) return PC_ERR_STATE;
  *peer = q->peer;
  *peer_request_index = q->match_peer_index;
  return 0;
}

int pc_request_peer_buffer(pc_request_t req, int j, void **ptr) {
  Request *q = (Request *)req;
  if (!q || !ptr) return PC_ERR_ARG;
  if (!q->exchanged || !q->matched) return PC_ERR_STATE;
  *ptr = nullptr;
  if (q->kind == PC_KIND_PSEND) {
    if (j != 0) return PC_ERR_ARG;
    *ptr = q->peer_buf;
  } else if (q->kind == PC_KIND_PALLREDUCE && q->algo == PC_ALGO_DIRECT && !q->direct_push && !q->direct_ll) {
    if (j < 0 || j >= q->comm->size - 1) return PC_ERR_ARG;
    *ptr = q->nb_buf[j];
  } else {
    return PC_ERR_UNSUPPORTED;
  }
  return 0;
}

uint64_t pc_launch_count(void) { return launch_count(); }

int pc_request_set_overlap(pc_request_t req, int on) {
  Request *q = (Request *)req;
  if (!q) return PC_ERR_ARG;
  if (q->active) return PC_ERR_STATE;
  q->overlap = on != 0;
  return 0;
}

int pc_request_set_timing(pc_request_t req, int on) {
  Request *q = (Request *)req;
  if (!q) return PC_ERR_ARG;
  TimingLog &T = q->leader ? q->leader->gs.tlog : q->tlog;
  T.on = on != 0;
  q->tlog.on = on != 0;
  return 0;
}

int pc_request_engine_times(pc_request_t req, float *ms, int max) {
  Request *q = (Request *)req;
  if (!q || (max > 0 && !ms)) return PC_ERR_ARG;
  if (q->comm->dry) return 0;
  PC_CUDA(cudaSetDevice(q->comm->device));
  TimingLog &T = q->leader ? q->leader->gs.tlog : q->tlog;
  int n = 0;
  for (auto &pr : T.pending) {
    PC_CUDA(cudaEventSynchronize(T.pool[pr.second]));
    float v = 0.f;
    PC_CUDA(cudaEventElapsedTime(&v, T.pool[pr.first], T.pool[pr.second]));
    if (n < max) ms[n] = v;
    ++n;
  }
  T.pending.clear();
  T.next = 0;
  return n < max ? n : max;
}

int pc_request_words(pc_request_t req, int which, int offset, int n, uint32_t *out) {
  Request *q = (Request *)req;
  if (!q || !out || which < 0 || which > 8 || offset < 0 || n < 0) return PC_ERR_ARG;
  if (q->comm->dry || !q->ctrl) return PC_ERR_STATE;
  const size_t base[9] = {q->L.flags, q->L.sent, q->L.cnt, q->L.ready, q->L.donecnt, q->L.rtr, q->L.epoch, q->L.layout, q->L.err};
  const size_t lim[9] = {q->L.words - q->L.flags, q->L.donecnt - q->L.sent, q->L.ready - q->L.cnt,
                         q->L.sent - q->L.ready, q->L.flags - q->L.donecnt, 8, 1, 1, 2};
  if ((size_t)offset + (size_t)n > lim[which]) return PC_ERR_ARG;
  PC_CUDA(cudaSetDevice(q->comm->device));
  uint32_t *tmp = nullptr;
  PC_CUDA(cudaMallocHost((void **)&tmp, (size_t)std::max(n, 1) * 4));
  int rc = 0;
  cudaError_t e = cudaMemcpyAsync(tmp, q->ctrl + base[which] + offset, (size_t)n * 4, cudaMemcpyDeviceToHost, q->side);
  if (e == cudaSuccess) e = cudaStreamSynchronize(q->side);
  if (e != cudaSuccess) rc = cuda_err(e, "pc_request_words");
  else memcpy(out, tmp, (size_t)n * 4);
  cudaFreeHost(tmp);
  return rc;
}

int pc_request_error(pc_request_t req, int *code, int *partition) {
  Request *q = (Request *)req;
  if (!q || !code || !partition) return PC_ERR_ARG;
  if (q->comm->dry) {
    *code = 0;
    *partition = 0;
    return 0;
  }
  PC_CUDA(cudaSetDevice(q->comm->device));
  return read_error(q, code, partition);
}

}  // extern "C"
