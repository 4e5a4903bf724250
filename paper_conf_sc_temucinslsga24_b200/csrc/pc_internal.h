// Internal host-side structures of libpc (not part of the ABI).
#pragma once

#include <cuda_runtime.h>

#include <atomic>
#include <condition_variable>
#include <cstdint>
#include <map>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "pc.h"
#include "pc_prequest.h"

namespace pc {

constexpr int kMaxRanks = 64;
constexpr int kMaxRdSteps = 6;        // log2(kMaxRanks)
constexpr int kEngineBlock = 256;     // threads per engine CTA (8 warps)

// ------------------------------------------------------------------ errors
int cuda_err(cudaError_t e, const char *what);
#define PC_CUDA(call)                                     \
  do {                                                    \
    cudaError_t _e = (call);                              \
    if (_e != cudaSuccess) return ::pc::cuda_err(_e, #call); \
  } while (0)
void logf(const char *fmt, ...);

// ------------------------------------------------------------------ bootstrap records
struct RankRec {
  uint32_t magic;
  int32_t rank, size, device, dry;
  int32_t sms, engine_warps;  // this rank's engine capacity (already divided by ranks on its device)
  int32_t direct_warps;  // capacity of the DIRECT engines (fewer, fatter CTAs), same division
  int64_t pid;
  uint64_t proc_token;
  uint8_t uuid[16];
};

struct ShareRec {  // one exported allocation
  cudaIpcMemHandle_t h;
  uint64_t off;    // offset of the pointer inside its allocation
  uint64_t raw;    // raw pointer (valid in the exporting process)
  uint64_t bytes;  // bytes meaningful from the pointer
};

struct ReqRec {
  int32_t kind, peer, tag, partitions;
  int64_t count;
  int32_t dtype, op, algo, seq;
  int32_t coll, root;  // collective kind (PC_COLL_*) and root (broadcast)
  int32_t owner;     // exporting rank
  int32_t req_index; // index in the owner's request list
  uint64_t host_req; // Request* in the owner's process (co-located grouping)
  ShareRec buf;      // p2p: user buffer; allreduce: recvbuf
  ShareRec ctrl;     // control block
  ShareRec stage;    // allreduce staging
  int64_t flags_off; // word offsets of the flags / LL areas in the owner's control block
  int64_t ll_off;    // (they depend on the owner's partition count, R30)
};

// ------------------------------------------------------------------ local group
struct LocalGroup {
  int size;
  std::mutex mu;
  std::condition_variable cv;
  uint64_t generation = 0;
  int arrived = 0;
  int readers_left = 0;
  std::vector<uint8_t> buf;
  size_t nbytes = 0;
  std::vector<std::pair<LocalGroup *, int>> ctxs;
};

// ------------------------------------------------------------------ control block layout
// One device allocation per request.  Words are u32.  Offsets in words.
struct CtrlLayout {
  size_t epoch = 0;        // [1]   (pc_device.cuh loads {epoch, rtr[0]} as one 8-byte word)
  size_t rtr = 1;          // [kMaxRdSteps + 2] ready-to-receive words (per incoming producer slot)
  size_t layout = 10;      // [1] g published by the sender (receive side)
  size_t err = 12;         // [2] sticky device error (int32 code, partition)
  size_t cnt = 16;         // [n1] aggregation counters
  size_t ready = 0;        // [n1]
  size_t sent = 0;         // [n1]
  size_t donecnt = 0;      // [n1] engine slice-completion counters / allreduce done[u]
  size_t flags = 0;        // [nflags] arrival flags
  size_t ll = 0;           // [ll_words] LL lines (p2p, PC_COPY_LL), 256-B aligned
  size_t scratch = 0;      // [4] host-query results (pc_parrived / pc_test on LL requests)
  size_t words = 0;
  void build(size_t n1, size_t nflags, size_t ll_words = 0) {
    ready = cnt + n1;
    sent = ready + n1;
    donecnt = sent + n1;
    flags = donecnt + n1;
    scratch = flags + nflags;
    ll = (scratch + 4 + 63) & ~size_t(63);
    words = ll + ll_words;
    words = (words + 63) & ~size_t(63);
  }
};

struct Comm;
struct Request;

// CUDA-event timing of engine launches (bench roofline: the dominant kernel's
// duration measured live on the stream it runs on).
struct TimingLog {
  bool on = false;
  std::vector<cudaEvent_t> pool;
  size_t next = 0;
  std::vector<std::pair<size_t, size_t>> pending;
  int get(cudaEvent_t *ev) {  // returns pool index or -1
    if (next == pool.size()) {
      cudaEvent_t e;
      if (cudaEventCreate(&e) != cudaSuccess) return -1;
      pool.push_back(e);
    }
    *ev = pool[next];
    return (int)next++;
  }
};

// Grouped engine launch state of co-located ranks (lives in the leader).
struct GroupState {
  std::mutex mu;
  std::condition_variable cv;
  uint32_t epoch = 0;
  int pending = 0;
  bool launched = false;
  cudaEvent_t ev = nullptr;
  std::vector<Request *> members;  // sorted by rank
  TimingLog tlog;
};

struct Request {
  Comm *comm = nullptr;
  int index = -1;  // position in comm->reqs
  int kind = 0;    // PC_KIND_*
  const void *sbuf = nullptr;
  void *rbuf = nullptr;
  int partitions = 0;
  size_t count = 0;
  int dtype = 0, op = 0, algo_req = 0, algo = 0;
  int peer = -1, tag = 0, seq = 0;
  size_t esize = 4;
  uint64_t part_bytes = 0, total_bytes = 0;  // total_bytes: recv buffer (exported to peers)
  uint64_t send_bytes = 0;                   // collectives: send buffer bytes (PULL export)
  int coll = 0, root = 0;                    // PC_COLL_* for collective requests; broadcast root

  // state
  uint32_t epoch = 0;
  bool active = false;
  bool exchanged = false;
  bool prepared_this_epoch = false;
  bool engine_launched = false;
  bool engine_registered = false;
  bool graph_mode = false;  // captured into a CUDA graph: epochs advance on the device only
  // Producer/engine overlap (§8(a) a6): ev_fork is recorded at the
  // epoch's control points (start / pbuf_prepare / epoch_all / host Pready of
  // every partition), so the engine — still ENQUEUED at the wait, after the
  // user's producer — starts as soon as the epoch is set up and reduces each
  // partition while the producer is still running.
  bool forked = false;          // ev_fork recorded at a control point of this epoch
  bool host_ready_all = false;  // every partition was made ready by a host-side op before ev_fork
  bool overlap = true;          // pc_request_set_overlap (0: fork at the wait, the round-1 order)
  // INLINE allreduce (reading R33): a DIRECT allreduce whose prequest was
  // created with PC_COPY_INLINE — the completing Pready folds, no engine
  bool direct_push = false;     // DIRECT schedule, PUSH variant (PC_ALGO_DIRECT_PUSH)
  bool direct_ll = false;       // DIRECT schedule, one-shot LL variant (PC_ALGO_LL)
  bool inline_ar = false;
  void *ar_tab = nullptr;       // device pc_ar_tab_s (library-owned)
  cudaEvent_t fork_ev_ext = nullptr;  // fork point recorded by a batched control call (else ev_fork)
  cudaEvent_t last_done = nullptr;    // completion of the last launched engine (single / group / batch)
  bool batch_launched = false;        // this epoch's engine ran in a batched waitall launch
  // stream on which the previous epoch's completion is ordered (null: host
  // observed it); a later epoch's control op on another stream first waits
  // for that completion (the engine reads the epoch word at entry)
  cudaStream_t joined_stream = nullptr;
  bool join_pending = false;    // group member waited on a stream before the group engine launched
  cudaStream_t wait_stream = nullptr;
  bool matched = false;
  Request *leader = nullptr;  // co-located group leader (allreduce), or null
  GroupState gs;
  TimingLog tlog;
  int match_peer_index = -1;

  // device resources
  uint32_t *ctrl = nullptr;  // device control block
  CtrlLayout L;
  uint8_t *staging = nullptr;
  size_t staging_bytes = 0;
  cudaStream_t side = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_done = nullptr;
  cudaStream_t user_stream = nullptr;

  // peer addresses (after exchange)
  uint8_t *peer_buf = nullptr;       // p2p send: receiver's recvbuf
  uint32_t *peer_ctrl = nullptr;     // p2p: partner ctrl; allreduce ring: ctrl of O
  uint8_t *peer_stage = nullptr;     // allreduce ring: staging of O
  // allreduce RD: per step partner addresses; ring uses index 0 (= O)
  uint8_t *nb_buf[kMaxRdSteps + 1] = {};
  uint32_t *nb_ctrl[kMaxRdSteps + 1] = {};
  uint8_t *nb_stage[kMaxRdSteps + 1] = {};
  // consumers of this rank (they get an RTR write from us): ctrl + rtr slot
  std::vector<std::pair<uint32_t *, int>> rtr_targets;

  // memory-model scope: 1 when a peer of this request is on another GPU
  int sys_scope = 1;
  // prequest (p2p)
  bool has_preq = false;
  int agg = 1, ntransport = 0, copy = 0;
  bool xpart = false;            // p2p: the two sides partition the buffer differently (R30)
  uint64_t peer_part_bytes = 0;  // p2p: the partner's bytes per partition (after matching)
  size_t peer_flags_off = 0, peer_ll_off = 0;  // p2p: word offsets in the partner's control block
  // PC_COPY_HOST (progression engine, NEXT-4): ready epochs in pinned host
  // memory written by device Pready, and the progress thread's per-transport
  // "last epoch moved" (touched only by that thread) and last RTR-checked epoch
  uint32_t *hready = nullptr, *hready_dev = nullptr;
  std::vector<uint32_t> pe_done;
  uint32_t pe_rtr_epoch = 0;
  bool pe_registered = false;
  uint32_t ll_lines = 0;  // p2p: LL lines per partition (0 = no LL area; pc.h PC_LL_MAX_*)
  // engine slicing
  int nsteps = 0;
  int slices = 1;          // ns: slices per chunk (allreduce) or per transport partition (p2p ENGINE)
  int64_t slice_elems = 0; // allreduce: elements per slice; p2p: bytes per slice
  int64_t chunk_elems = 0; // allreduce ring: q
  int engine_warps = 0;
};

// Host progression engine (PC_COPY_HOST): one thread per comm polls the
// pinned ready flags of its HOST-mode send requests and enqueues, per ready
// transport partition, the ready-to-receive wait, the copy and the arrival /
// completion signals on its own stream.
struct Progress {
  std::thread th;
  std::mutex mu;
  std::vector<Request *> reqs;
  std::atomic<bool> stop{false};
  std::atomic<int> err{0};
  cudaStream_t stream = nullptr;
  bool started = false;
};

// Device tables of a batched control / wait call over a fixed list of
// requests (pc_epoch_all with > 16 requests, pc_waitall_on_stream over many
// allreduces), built once per distinct request list and reused every epoch;
// dropped when one of its requests is freed.
struct BatchCache {
  std::vector<Request *> reqs;
  void *dev = nullptr;       // tables (layout per kind)
  size_t dev_bytes = 0;
  int n = 0, nrtr = 0;       // epoch batch: request / RTR entries
  int nreq = 0, R = 1;       // engine batch: logical requests x local ranks
  int units = 0;
  int dtype = 0, op = 0;
  cudaEvent_t ev = nullptr;  // fork point (epoch batch) / completion (engine batch)
};

struct Comm {
  int rank = 0, size = 1, device = -1;
  bool dry = false;
  pc_allgather_fn ag = nullptr;
  void *ag_ctx = nullptr;
  std::vector<RankRec> ranks;
  std::vector<bool> same_proc;
  int engine_warps = 0;  // agreed (min over ranks)
  int direct_warps = 0;  // the same for the DIRECT allreduce engines
  bool overlap_thin = true;  // PC_OVERLAP_THIN (measurement knob): thin DIRECT CTAs while overlapping
  int overlap_warps = 0; // per-rank engine width when the engine may overlap a producer:
                         // whole CTAs, <= PC_OVERLAP_FRAC of the SMs per GPU in total
  int sms = 0;
  std::vector<Request *> reqs;
  std::map<std::tuple<int, int, int>, int> post_seq;  // (kind, peer, tag) -> next seq
  int allreduce_seq = 0;
  // IPC mappings opened by this comm: key = handle bytes
  std::map<std::string, void *> ipc_open;
  uint32_t timeout_ms = 10000;
  bool memops = false;  // cuStreamWriteValue32 usable
  Progress pe;
};

// ------------------------------------------------------------------ helpers
int allgather(Comm *c, const void *send, size_t nbytes, void *recv);
int export_ptr(Comm *c, const void *p, uint64_t bytes, ShareRec *out);
int import_ptr(Comm *c, int owner, const ShareRec &s, void **out);
int stream_write_u32(Comm *c, cudaStream_t s, uint32_t *addr, uint32_t value);
int stream_wait_geq_u32(Comm *c, cudaStream_t s, const uint32_t *addr, uint32_t value, bool sys);
bool memops_available();

// ------------------------------------------------------------------ kernel launchers (kernels.cu)
struct RingArgs {
  const uint32_t *epoch;  // device epoch word (read at kernel start)
  int P, r, Np, ns, nunits, op, dtype;
  int64_t L, q, qs;
  const uint8_t *sendbuf;
  uint8_t *recvbuf;
  const uint8_t *staging;
  const uint32_t *flags, *ready, *rtr;
  uint32_t *done;
  uint8_t *o_staging, *o_recvbuf;
  uint32_t *o_flags;
  int32_t *err;
  uint32_t timeout_ms;
  int sys;  // 1: some peer is another GPU -> system-scope fences/acquires
};
struct RdArgs {
  const uint32_t *epoch;
  int P, r, Np, ns, nunits, op, dtype, nsteps;
  int64_t L, qs;
  const uint8_t *sendbuf;
  uint8_t *recvbuf;
  const uint8_t *staging;  // [nsteps][Np*L]
  const uint32_t *flags, *ready, *rtr;
  uint32_t *done;
  uint8_t *p_staging[kMaxRdSteps];
  uint32_t *p_flags[kMaxRdSteps];
  int32_t *err;
  uint32_t timeout_ms;
  int sys;
};
struct P2pEngineArgs {
  const uint32_t *epoch;
  int nt, agg, ns, nunits;
  uint64_t part_bytes, slice_bytes;
  int partitions;
  const uint8_t *sbuf;
  uint8_t *peer_rbuf;
  uint32_t *peer_flags;
  const uint32_t *ready, *rtr;
  uint32_t *donecnt, *sent;
  int32_t *err;
  uint32_t timeout_ms;
  int sys;
  uint32_t xpart;            // partitionings differ (R30): per-receive-partition counters
  uint64_t peer_part_bytes;  // receiver's bytes per partition
};

constexpr int kMaxLocal = 8;  // ranks of one comm sharing one GPU in one process
struct RingGroupArgs {
  int n;
  int block_start[kMaxLocal];
  RingArgs a[kMaxLocal];
};
// Direct two-step schedule (reduce-scatter to chunk owners, allgather of the
// owned chunks) for P <= kMaxDirect ranks; peer j is rank (r + 1 + j) mod P.
constexpr int kMaxDirect = 8;
struct DirectArgs {
  const uint32_t *epoch;
  int P, r, Np, ns, nunits, op, dtype;
  int64_t L, q, qs;
  const uint8_t *sendbuf;
  uint8_t *recvbuf;
  const uint32_t *cnt, *ready, *rtr;  // cnt: [u][phase][slice] arrival counters (written by peers)
  uint32_t *done;
  // peer j = rank (r+1+j) mod P: its send buffer (read by the PULL reduce) and recvbuf
  const uint8_t *p_sendbuf[kMaxDirect - 1];  // PUSH variant: peer j's STAGING (written by this rank)
  uint8_t *p_recvbuf[kMaxDirect - 1];
  uint32_t *p_cnt[kMaxDirect - 1];
  int32_t *err;
  uint32_t timeout_ms;
  int sys;
  int push;            // PUSH variant: step 0 stores chunk o into owner o's staging slot r
  uint8_t *staging;    // PUSH: own staging [u][source rank][q elements]; LL: own line area
  int ll;              // LL one-shot variant: p_sendbuf[j] = peer j's line area
  int64_t ll_lines;    // LL: 16-B lines per partition = ceil(part bytes / 8)
};
struct DirectGroupArgs {
  int n;
  int block_start[kMaxLocal];
  DirectArgs a[kMaxLocal];
};
// Batched DIRECT engine (pc_waitall_on_stream over many allreduces of one
// GPU): entries (request t, local rank j) = tab[t * R + j] in device memory,
// ubase[t] = first global unit of request t (units ordered [t][x][j]).
struct DirectBatchArgs {
  const DirectArgs *tab;
  const int *ubase;  // [nreq + 1]
  int nreq, R;
  int32_t *err;      // the first request's error word (idle timeouts)
  uint32_t timeout_ms;
};
int launch_direct_engine_batch(const DirectBatchArgs &b, int dtype, int op, int blocks, cudaStream_t s, bool thin);
// Partitioned reduce-scatter / allgather / broadcast on the
// DIRECT machinery (engine.cuh coll_body).  Unit (u, slice s) of a block of
// `count` elements.
enum { PC_COLL_ALLREDUCE = 0, PC_COLL_REDUCE_SCATTER = 1, PC_COLL_ALLGATHER = 2, PC_COLL_BCAST = 3 };
struct CollArgs {
  const uint32_t *epoch;
  int coll, P, r, root, Np, ns, nunits, op, dtype;
  int64_t count, qs, es;  // block elements, slice elements, element size (bytes)
  const uint8_t *sendbuf;
  uint8_t *recvbuf;
  const uint32_t *cnt, *ready, *rtr;  // cnt: [u][phase 0..1][slice] (written by peers)
  uint32_t *done;
  uint32_t *srcflags;                 // allgather: [source rank][u][slice] arrival epochs
  const uint8_t *p_sendbuf[kMaxDirect - 1];  // peer j = rank (r+1+j) mod P
  uint8_t *p_recvbuf[kMaxDirect - 1];
  uint32_t *p_cnt[kMaxDirect - 1], *p_srcflags[kMaxDirect - 1];
  int32_t *err;
  uint32_t timeout_ms;
  int sys;
};
struct CollGroupArgs {
  int n;
  int block_start[kMaxLocal];
  CollArgs a[kMaxLocal];
};
int launch_coll_engine(const CollArgs &a, int warps, cudaStream_t s);
int launch_coll_engine_group(const CollGroupArgs &g, int warps, cudaStream_t s);
// thin: the 2-CTA/SM variant used while the engine overlaps producer kernels
int launch_direct_engine(const DirectArgs &a, int warps, cudaStream_t s, bool thin = false);
int launch_direct_engine_group(const DirectGroupArgs &g, int warps, cudaStream_t s, bool thin = false);
struct RdGroupArgs {
  int n;
  int block_start[kMaxLocal];
  RdArgs a[kMaxLocal];
};
int launch_ring_engine(const RingArgs &a, int warps, cudaStream_t s);
int launch_ring_engine_group(const RingGroupArgs &g, int warps, cudaStream_t s);
int launch_rd_engine_group(const RdGroupArgs &g, int warps, cudaStream_t s);
int launch_rd_engine(const RdArgs &a, int warps, cudaStream_t s);
int launch_p2p_engine(const P2pEngineArgs &a, int warps, cudaStream_t s);
// wait until words[i*stride] reached target (i < n); layout!=null: n derived
// as ceil(partitions / *layout) (receiver side)
struct RtrArgs {
  const uint32_t *epoch;
  int n, sys;
  uint32_t *dst[kMaxRdSteps + 2];
};
// Batched control ops (pc_startall / pc_pbuf_prepare_all): entry i either
// bumps epoch[i] (dst == null) or stores *epoch[i] into dst[i] (RTR).
constexpr int kMaxCtl = 64;
struct CtlArgs {
  int n;
  const uint32_t *epoch[kMaxCtl];
  uint32_t *dst[kMaxCtl];
  int sys[kMaxCtl];
};
int launch_ctl(const CtlArgs &a, cudaStream_t s);
int launch_epoch_bump(uint32_t *epoch, cudaStream_t s);
int launch_rtr(const RtrArgs &a, cudaStream_t s);
// rtr != null: also acquire-wait until *rtr reached the epoch (LL sender)
int launch_wait_words(const uint32_t *words, int n, const uint32_t *epoch, uint32_t mul, const uint32_t *layout,
                      int partitions, int32_t *err, uint32_t timeout_ms, cudaStream_t s, bool sys,
                      const uint32_t *rtr = nullptr);
// receive-side wait (pending == null) or test (pending: device counter of
// lines / flags not yet arrived, zeroed by the caller); handles LL and flags
int launch_recv_wait(const pc_prequest_t &q, int32_t *pending, cudaStream_t s);
// out[0] = pc_parrived(q, partition) on the device (LL receive requests)
int launch_parrived(const pc_prequest_t &q, int partition, int32_t *out, cudaStream_t s);
int launch_set_word(uint32_t *addr, uint32_t value, cudaStream_t s);
int launch_pe_signal(uint32_t *peer_flags, uint32_t *sent, int n, uint32_t v, bool sys, cudaStream_t s);
int pe_kernels_preload();
int kernels_preload();
int launch_wait_value(const uint32_t *addr, uint32_t value, cudaStream_t s, bool sys, uint32_t tmo_ms);
int launch_pready_range(pc_prequest_t q, int lo, int hi, cudaStream_t s);
constexpr int kMaxPreadyAll = 16;
struct PreadyAllArgs {
  int n;
  pc_prequest_t q[kMaxPreadyAll];
};
int launch_pready_all(const PreadyAllArgs &a, cudaStream_t s);
// pc_epoch_all: Start + ready-to-receive (+ Pready of every partition of
// allreduce-kind requests) for n requests in ONE single-block kernel.
// Kept under 1 KB of kernel parameters (a launch's parameter bytes travel in
// the push buffer: the earlier layout, 16 whole pc_prequest_t, was 4.6 KB and
// made this one launch slower than pc_startall + pc_pbuf_prepare_all).
struct EpochAllArgs {
  int n, nrtr, pready;
  uint64_t rtr_sysmask;                 // bit k: RTR k is a system-scope release
  uint32_t *epoch[kMaxPreadyAll];
  uint32_t *rtr_dst[kMaxCtl];
  uint8_t rtr_req[kMaxCtl];             // RTR k carries the epoch of request rtr_req[k]
  uint32_t *ready[kMaxPreadyAll];       // pready: allreduce S_0 ready words [partitions]
  int partitions[kMaxPreadyAll];
};
static_assert(sizeof(EpochAllArgs) <= 1024, "EpochAllArgs: keep kernel parameters small");
int launch_epoch_all(const EpochAllArgs &a, cudaStream_t s);
// pc_epoch_all for any number of requests (many per-tensor allreduces): the
// same three phases in one block, the request and RTR lists in device memory.
struct EpochEnt {
  uint32_t *epoch;
  uint32_t *ready;  // null: no Pready
  int partitions;
  int pad;
};
struct RtrEnt {
  uint32_t *dst;
  int req;  // index into the EpochEnt list (the RTR carries its epoch)
  int sys;
};
struct EpochBatchArgs {
  int n, nrtr, pready, nbig;
  const EpochEnt *ent;
  const RtrEnt *rtr;
  const int *big;  // requests with more than kEpochSmallParts partitions (block-cooperative Pready)
};
constexpr int kEpochSmallParts = 64;
int launch_epoch_batch(const EpochBatchArgs &a, cudaStream_t s);
// pc_waitall_on_stream: the p2p waits of up to kMaxWaitAll requests in one
// kernel; request k owns blocks [block_start[k], block_start[k+1]).
constexpr int kMaxWaitAll = 4;
struct WaitAllArgs {
  int n;
  int block_start[kMaxWaitAll + 1];
  pc_prequest_t q[kMaxWaitAll];
};
int recv_wait_blocks(const pc_prequest_t &q);
int wait_words_blocks(int n);
int launch_wait_all(const WaitAllArgs &a, cudaStream_t s);
int engine_occupancy_ctas_per_sm(int *ctas);
int direct_occupancy_ctas_per_sm(int *ctas);
uint64_t launch_count();

}  // namespace pc
