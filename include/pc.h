/*
 * include/pc.h — host C ABI of libpc: GPU-initiated MPI-Partitioned-style
 * communication for B200 (NVLink 5 / NVSwitch), after Temuçin et al., SC'24
 * ("Design and Implementation of MPI-Native GPU-Initiated MPI Partitioned
 * Communication"; reference text PAPER.md, cited as P:Lnn §section).
 *
 * Plain C: pointers, sizes, ints.  No torch or C++ types cross this boundary.
 * Every host call returns PC_SUCCESS (0) or a negative PC_ERR_* code and never
 * throws.  Device-side bindings are in pc_device.cuh.
 *
 * Flow (Listing 2; Fig. 1; §IV-A):
 *     pc_psend_init / pc_precv_init / pc_pallreduce_init      once
 *     loop:  pc_start -> pc_pbuf_prepare -> [first: pc_prequest_create]
 *            -> user kernel calling pc_pready*(p, preq) -> pc_wait
 *
 * Buffers: caller-owned device memory (cudaMalloc or the torch caching
 * allocator WITHOUT expandable segments), 16-byte aligned, valid and unmoved
 * until pc_request_free.  The library owns flags, counters, staging and the
 * device request storage.  Host calls for one request come from one host
 * thread at a time.
 */
#ifndef PC_H_
#define PC_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* cudaStream_t without including cuda_runtime.h (ABI-identical pointer). */
typedef struct CUstream_st *pc_stream_t;

typedef struct pc_comm_s *pc_comm_t;            /* opaque: rank, size, device, peer mappings     */
typedef struct pc_request_s *pc_request_t;      /* opaque: one persistent partitioned request    */
typedef struct pc_local_group_s *pc_local_group_t; /* in-process rank group (virtual ranks)      */
typedef struct pc_prequest_s pc_prequest_t;     /* POD device request, passed BY VALUE to kernels
                                                   (MPIX_Prequest); layout in pc_device.cuh */

/* Element types.  BF16: bfloat16 bits (upper half of an fp32); every reduction
 * step is one correctly rounded bf16 op (R27).  FLOAT64/BF16 are
 * accepted by pc_pallreduce_init; p2p requests take any type (bytes moved). */
typedef enum { PC_INT32 = 0, PC_FLOAT32 = 1, PC_BYTE = 2, PC_FLOAT64 = 3, PC_BF16 = 4 } pc_dtype_t;
typedef enum { PC_OP_SUM = 0, PC_OP_MAX = 1, PC_OP_MIN = 2 } pc_op_t;
/* Granularity of the device Pready call: informational — the device
 * function chosen (pc_pready / _warp / _block) decides who participates. */
typedef enum { PC_GRAN_THREAD = 0, PC_GRAN_WARP = 1, PC_GRAN_BLOCK = 2 } pc_gran_t;
/* Copy mechanism: INLINE = "Kernel Copy" — every contributor
 * pushes its partition over NVLink from inside the user kernel and the one
 * that completes a transport partition stores its flag; ENGINE = persistent
 * library warps poll ready flags and push (the GPU-resident replacement of the
 * paper's host Progression Engine); LL = Kernel Copy in 16-B lines that carry
 * the epoch next to every 8 payload bytes (NCCL-LL-style), so a partition
 * needs no fence and no separate flag and Pready->Parrived is one store's
 * flight.  LL is available when part_bytes <= PC_LL_MAX_PART_BYTES and the
 * buffer <= PC_LL_MAX_TOTAL_BYTES (else pc_prequest_create returns
 * PC_ERR_UNSUPPORTED); aggregation then only batches the sender's completion
 * accounting (each partition's lines are self-validating). */
/* PC_COPY_HOST: the paper's host Progression Engine (
 * SURVEY NEXT-4), kept as a comparison mode: Pready marks the transport
 * partition in pinned host memory, a library host thread polls those flags
 * and issues the copy (cudaMemcpyAsync) and the arrival signal (stream
 * memop) on its own stream. */
typedef enum { PC_COPY_INLINE = 0, PC_COPY_ENGINE = 1, PC_COPY_LL = 2, PC_COPY_HOST = 3 } pc_copy_t;
#define PC_LL_MAX_PART_BYTES 1024
#define PC_LL_MAX_TOTAL_BYTES (16u << 20)
/* Allreduce schedule (§IV-B).  RING = Alg 1; RD = recursive
 * doubling (BASELINE north_star; not in the paper; P a power of two);
 * DIRECT = two steps over neighbour SETS (the generic schedule of P:L155 with
 * |I| = |O| = P-1; P <= 8; the NVSwitch-native schedule of SURVEY NEXT-1):
 * each chunk owner PULLS its chunk from every peer's send buffer with peer
 * loads, folds in rank order, and pushes the result to every peer.
 * AUTO = DIRECT for 3 <= P <= 8 (RD for P = 2 up to PC_RD_MAX_BYTES, default
 * 4 MiB; PC_DIRECT_MAX_BYTES caps DIRECT); for P > 8 RD up to
 * PC_RD_MAX_BYTES, ring above. */
/* PC_ALGO_DIRECT: two-step schedule, owners PULL their chunk from every
 * rank's send buffer with peer loads; PC_ALGO_DIRECT_PUSH: the same schedule
 * and bits (rank-order fold, R25), every rank PUSHES its chunk o into owner
 * o's staging with peer stores and the owner folds from local memory (all
 * NVLink traffic is stores; +S staging per rank).  PC_ALGO_LL: one-shot for
 * small messages — every rank stores each ready partition as 16-B LL lines
 * {4 B data, epoch, 4 B data, epoch} into every peer's line area (no fence,
 * no flag: a line is its own arrival flag) and every rank folds all P
 * contributions itself in rank order (the same bits); one hop; line areas
 * double-buffered by epoch parity (4·P·S bytes per rank).  AUTO picks LL up
 * to PC_LL_AR_MAX_BYTES (default 64 KiB) per rank, else DIRECT (PULL), or
 * PUSH with PC_DIRECT_MODE=push. */
typedef enum {
  PC_ALGO_AUTO = 0,
  PC_ALGO_RING = 1,
  PC_ALGO_RD = 2,
  PC_ALGO_DIRECT = 3,
  PC_ALGO_DIRECT_PUSH = 4,
  PC_ALGO_LL = 5
} pc_algo_t;

enum {
  PC_SUCCESS = 0,
  PC_ERR_ARG = -1,         /* bad argument (null, range, misaligned buffer)             */
  PC_ERR_CUDA = -2,        /* a CUDA runtime/driver call failed                         */
  PC_ERR_STATE = -3,       /* start on active / free of active / pready on inactive     */
  PC_ERR_MATCH = -4,       /* send/recv (or allreduce) parameters disagree across ranks */
  PC_ERR_TIMEOUT = -5,     /* a device spin exceeded PC_TIMEOUT_MS (sticky error word)   */
  PC_ERR_DEVICE = -6,      /* a device call reported an error (bad partition, dup)       */
  PC_ERR_NOMEM = -7,
  PC_ERR_UNSUPPORTED = -8
};

/* ---------------------------------------------------------------- bootstrap
 * All-gather callback supplied by the caller (a torch ProcessGroup, MPI, …):
 * gather `nbytes` from every rank into recv[rank*nbytes].  Returns 0 on success.
 * It is called only from pc_comm_create and from the FIRST pc_pbuf_prepare of
 * a batch of new requests (see pc_pbuf_prepare), never on the hot path. */
typedef int (*pc_allgather_fn)(const void *send, size_t nbytes, void *recv, void *ctx);

/* cuda_device = -1 creates a host-only ("dry") comm: requests, matching and
 * schedules work, nothing touches a GPU (used by CPU tests of the host logic). */
int pc_comm_create(int rank, int size, int cuda_device, pc_allgather_fn ag, void *ctx, pc_comm_t *comm);
int pc_comm_destroy(pc_comm_t comm);
int pc_comm_rank(pc_comm_t comm, int *rank);
int pc_comm_size(pc_comm_t comm, int *size);
/* Number of engine warps every rank uses (agreed at comm creation: identical
 * on all ranks so per-warp work orders match — the deadlock-freedom argument
 * of DESIGN.md §"Engine"). */
int pc_comm_engine_warps(pc_comm_t comm, int *warps);
/* Per-rank engine warps while the engine may run beside a producer kernel
 * (pc_start's overlap rule): whole 8-warp CTAs, the ranks of one GPU together
 * on at most PC_OVERLAP_FRAC of its SMs (min over the comm's ranks). */
int pc_comm_overlap_warps(pc_comm_t comm, int *warps);

/* In-process rank groups: several ranks of one comm living in ONE process
 * (e.g. P virtual ranks sharing one GPU, or one process driving several GPUs).
 * Peers in the same process are addressed directly, without CUDA IPC.  Each
 * rank must be driven by its own host thread during pc_comm_create and the
 * first pc_pbuf_prepare (the all-gather blocks until every rank arrived).
 * The engines of co-located ranks of one GPU (allreduce-kind requests) run as
 * ONE grouped kernel, enqueued by the LAST member's wait of the epoch (every
 * member's producer work is then already enqueued).  A member whose
 * pc_wait_on_stream came earlier gets the completion ordered on its stream at
 * that launch: work it enqueued on that stream BEFORE the group's last wait is
 * not ordered after the collective — enqueue dependent work after every
 * member's wait (or wait from one host thread per rank with pc_wait).  A
 * member cannot start its next epoch before the group's engine of the current
 * one is enqueued (PC_ERR_STATE). */
int pc_local_group_create(int size, pc_local_group_t *group);
int pc_local_group_destroy(pc_local_group_t group);
/* ctx to pass to pc_comm_create together with pc_local_allgather */
void *pc_local_group_ctx(pc_local_group_t group, int rank);
int pc_local_allgather(const void *send, size_t nbytes, void *recv, void *ctx);

/* ---------------------------------------------------------------- init (non-blocking)
 * MPI-4 partitioned semantics: `count` is elements PER PARTITION, the
 * buffer holds partitions*count elements.  Matching is by (comm, peer, tag,
 * posting order).  The two sides must agree on dtype and on the TOTAL number
 * of elements; their partition counts may differ (MPI-4; reading R30): a
 * receive partition is then reported arrived (pc_parrived / device
 * pc_parrived / pc_wait_arrived) once every send transport partition that
 * overlaps its bytes has been pushed.  PC_COPY_LL needs equal partitionings
 * (PC_ERR_UNSUPPORTED otherwise); empty buffers need equal partitionings.
 * Nothing is exchanged here; mismatches surface as PC_ERR_MATCH at the first
 * pc_pbuf_prepare. */
int pc_psend_init(const void *buf, int partitions, size_t count, pc_dtype_t dtype, int dest, int tag,
                  pc_comm_t comm, pc_request_t *req);
int pc_precv_init(void *buf, int partitions, size_t count, pc_dtype_t dtype, int source, int tag,
                  pc_comm_t comm, pc_request_t *req);
/* Partitioned allreduce (MPIX_Pallreduce_init; schedule S of
 * P:L153-L155).  Collective: every rank calls it with identical arguments in
 * the same order.  sendbuf == recvbuf (in place) is allowed.  dtype INT32,
 * FLOAT32, FLOAT64 or BF16; op SUM/MAX/MIN. */
int pc_pallreduce_init(const void *sendbuf, void *recvbuf, int partitions, size_t count, pc_dtype_t dtype,
                       pc_op_t op, pc_algo_t algo, pc_comm_t comm, pc_request_t *req);

/* Partitioned reduce-scatter / allgather / broadcast (the two
 * halves of the DIRECT allreduce schedule and its one-to-all case; the generic
 * schedule of P:L151-L155 with neighbour sets).  Collective, like
 * pc_pallreduce_init (shared posting order), P <= 8.  Schedule: reduce-scatter
 * PULLS (owners fold the peers' blocks with peer loads, rank order, reading
 * R25); allgather PUSHES each 16-B vector once to all P buffers; broadcast is PULLED by the receivers.
 *
 * reduce_scatter: sendbuf partitions x P x count elements (partition u = P
 *   blocks of count, block k for rank k); recvbuf partitions x count:
 *   recvbuf[u] = op-fold over ranks 0..P-1 (in rank order) of sendbuf_k[u][me]
 *   (MPI_Reduce_scatter_block per partition).  dtype INT32/FLOAT32/FLOAT64/BF16.
 *   pc_pready(u): sendbuf[u] final.  pc_parrived(u): recvbuf[u] final and every
 *   peer done reading sendbuf[u].
 * allgather: sendbuf partitions x count; recvbuf P x partitions x count (rank
 *   major, as MPI_Allgather of the whole buffer): recvbuf[k][u] = sendbuf_k[u].
 *   Any dtype (bytes move).  pc_pready(u): sendbuf[u] final.  Receive
 *   partitions are the P x partitions blocks: pc_parrived(k * partitions + u)
 *   = rank k's partition u is in recvbuf.
 * bcast: buf partitions x count on every rank; the root's pc_pready(u) delivers
 *   buf[u] to every rank (the receivers PULL it with peer loads); pc_parrived(u)
 *   = buf[u] holds the root's data (root: every rank has pulled it). */
int pc_preduce_scatter_init(const void *sendbuf, void *recvbuf, int partitions, size_t count, pc_dtype_t dtype,
                            pc_op_t op, pc_comm_t comm, pc_request_t *req);
int pc_pallgather_init(const void *sendbuf, void *recvbuf, int partitions, size_t count, pc_dtype_t dtype,
                       pc_comm_t comm, pc_request_t *req);
int pc_pbcast_init(void *buf, int partitions, size_t count, pc_dtype_t dtype, int root, pc_comm_t comm,
                   pc_request_t *req);

/* ---------------------------------------------------------------- epoch
 * MPI_Start: epoch e <- e+1, written stream-ordered to the device
 * epoch word.  PC_ERR_STATE if the request is active.  If the previous epoch's
 * completion was ordered on another stream, `stream` first waits for it.
 *
 * Engines (allreduce-kind requests, ENGINE-copy sends): the engine kernel is
 * ENQUEUED on a library stream at pc_wait / pc_wait_on_stream / pc_test —
 * after the user's producer kernels in host order (Listing 2) — but it is
 * FORKED from the epoch's last control call (pc_start, pc_pbuf_prepare,
 * pc_startall, pc_pbuf_prepare_all, pc_epoch_all): it starts as soon as the
 * epoch is set up and forwards / reduces each partition as soon as its Pready
 * arrives, while the producer still runs (§IV-B1).  While a
 * producer may run beside it the engine takes whole CTAs on at most
 * PC_OVERLAP_FRAC (default 0.5) of the SMs; after a host-side Pready of every
 * partition (pc_epoch_all with pready, pc_preadyall, pc_pready_range over all
 * partitions), which re-records the fork point, it takes the full width.  Producer
 * kernels whose blocks need a whole SM still always find one.
 * pc_request_set_overlap(req, 0) forks the engine at the wait instead (the
 * engine then starts after everything enqueued before the wait: no overlap,
 * full width).  Call it while the request is inactive; PC_ERR_STATE otherwise. */
int pc_request_set_overlap(pc_request_t req, int on);
int pc_start(pc_request_t req, pc_stream_t stream);
/* MPIX_Pbuf_prepare: guarantees the remote buffers are
 * ready.  FIRST call (per batch of new requests): host-blocking exchange of
 * request records + IPC handles through the comm's all-gather, matching,
 * mapping of peer buffers.  Every call: stream-ordered "ready-to-receive"
 * epoch write into each producer's RTR word (no host blocking); producers
 * check it on the device before their first push of the epoch. */
int pc_pbuf_prepare(pc_request_t req, pc_stream_t stream);
/* MPI_Startall analogue: pc_start for n requests of one GPU, with a single
 * device kernel advancing all n epochs (CUDA-graph capturable). */
int pc_startall(int n, pc_request_t *reqs, pc_stream_t stream);
/* The whole control part of an epoch in ONE kernel, for n (<= 16) requests of
 * one GPU whose first pc_pbuf_prepare (exchange + mapping) already happened:
 * pc_startall + pc_pbuf_prepare_all, and with pready != 0 also the user's
 * Pready of every partition of each request (allreduce-kind requests only;
 * PC_ERR_ARG otherwise) — the small-message path, where launches dominate.
 * PC_ERR_STATE if a request is active or not yet exchanged.  Capturable. */
/* Any n >= 1 (round 2): beyond 16 requests or 64 ready-to-receive words the
 * lists live in a library-owned device table built on the first call with
 * that exact request list (a synchronous upload: that first call must not be
 * captured into a CUDA graph, PC_ERR_STATE otherwise) and reused afterwards;
 * the table is dropped when one of its requests is freed.  The same request
 * twice in one call: PC_ERR_ARG, nothing started. */
int pc_epoch_all(int n, pc_request_t *reqs, int pready, pc_stream_t stream);
/* pc_pbuf_prepare for n requests whose first pc_pbuf_prepare (exchange +
 * mapping) already happened: all ready-to-receive writes in one kernel.
 * PC_ERR_STATE if a request is inactive or not yet exchanged. */
int pc_pbuf_prepare_all(int n, pc_request_t *reqs, pc_stream_t stream);
/* MPIX_Prequest_create: build the POD device request.  `aggregation`
 * = g user partitions per transport partition (P:L129 threshold; 1 = none);
 * allreduce requires g = 1.  Blocking.  Writes the transport layout into the
 * receiver's control block. */
int pc_prequest_create(pc_request_t req, pc_gran_t gran, int aggregation, pc_copy_t copy, pc_prequest_t *out);
int pc_prequest_free(pc_prequest_t *preq);
/* sizeof(pc_prequest_t) as compiled into the library (bindings check it). */
size_t pc_prequest_size(void);

/* ---------------------------------------------------------------- completion
 * pc_parrived: host, non-blocking, 1 iff partition complete this epoch (P:L48,
 * P:L143; allreduce: final result in recvbuf).
 * pc_test: host, non-blocking MPI_Test.  pc_wait: host-blocking MPI_Wait
 * (P:L50); returns PC_ERR_TIMEOUT / PC_ERR_DEVICE if the device
 * reported one.  pc_wait_on_stream: enqueue "wait for completion" on `stream`
 * without host blocking (the request becomes inactive for the host; later
 * work on `stream` is ordered after completion).  Wait on an inactive request
 * returns PC_SUCCESS. */
int pc_parrived(pc_request_t req, int partition, int *flag);
int pc_test(pc_request_t req, int *flag);
int pc_wait(pc_request_t req);
int pc_wait_on_stream(pc_request_t req, pc_stream_t stream);
/* MPI_Waitall (MPI-4 §3.7.5; Listing 2 waits on each request), stream
 * ordered: pc_wait_on_stream of n requests of one GPU, with the waits of the
 * point-to-point requests (engine-less sends and all receives) fused into ONE
 * kernel per group of 4 — one launch where n pc_wait_on_stream calls take n.
 * Requests moved by library engines (allreduce, ENGINE-copy sends) take
 * pc_wait_on_stream's path (the engine launch is the wait).  Inactive requests
 * are skipped.  PC_ERR_ARG for n < 0 or a null array / entry, PC_ERR_STATE as
 * pc_wait_on_stream; on an error no request of the call was marked complete
 * unless its own wait was already enqueued. */
/* Round 2: two or more engine-moved DIRECT allreduces in the list (all of one
 * dtype / op; co-located groups complete in the list) run as ONE batched
 * engine launch over a device table built on the first call with that exact
 * list (not capturable, like pc_epoch_all's); other requests take their own
 * path. */
int pc_waitall_on_stream(int n, pc_request_t *reqs, pc_stream_t stream);
/* Host Pready bindings (MPI_Pready / MPI_Pready_range): enqueue a tiny kernel
 * on `stream` that marks partitions [lo, hi] ready. */
int pc_pready(int partition, pc_request_t req, pc_stream_t stream);
/* Host Pready of EVERY partition of n requests (one GPU) in one kernel. */
int pc_preadyall(int n, pc_request_t *reqs, pc_stream_t stream);
int pc_pready_range(int lo, int hi, pc_request_t req, pc_stream_t stream);
int pc_request_free(pc_request_t *req);

/* ---------------------------------------------------------------- introspection
 * (host logic exported for tests; pure functions, no GPU) */
/* Ring schedule (Alg 1) of rank r: rows (I, R, op, O, A) for the 2(P-1)
 * communicating steps; returns the number of steps. */
int pc_schedule_ring(int P, int r, int32_t *out_rows5);
/* Recursive-doubling schedule: rows (I, R=-1, op=1, O, A=-1); log2 P steps. */
int pc_schedule_rd(int P, int r, int32_t *out_rows5);
/* Chunk bounds of a partition of L elements split in P chunks (reading R4):
 * out[c] = first element of chunk c, out[P] = L.  Quantum 4 elements, i.e.
 * 32-bit types; for fp64 / bf16 requests the quantum is 2 / 8 (R27). */
int pc_chunk_bounds(int64_t L, int P, int64_t *out);
/* Request facts after the first pbuf_prepare: algo actually used, slices per
 * chunk, slice elements, engine warps. */
int pc_request_info(pc_request_t req, int *algo, int *slices, int64_t *slice_elems, int *engine_warps);
/* Matched peer request id (debug; p2p) after the first pbuf_prepare. */
int pc_request_match(pc_request_t req, int *peer, int *peer_request_index);
/* Read n control words of a request (which: 0 arrival flags, 1 sent, 2
 * aggregation counters, 3 ready, 4 done/slice counters, 5 RTR words, 6 epoch)
 * starting at `offset` into host memory `out` (debug / tests; blocking). */
int pc_request_words(pc_request_t req, int which, int offset, int n, uint32_t *out);
/* Engine timing for benchmarks: when on, every engine launch of the request
 * (or of its co-located group) is bracketed by CUDA events on the stream it
 * runs on; pc_request_engine_times drains the durations (ms) of the launches
 * since the last call into ms[0..max) and returns how many it wrote. */
int pc_request_set_timing(pc_request_t req, int on);
int pc_request_engine_times(pc_request_t req, float *ms, int max);
/* Peer-mapped address (CUDA IPC or same-process pointer, valid in this
 * process) of a peer's receive buffer after the first pc_pbuf_prepare: a send
 * request's receiver buffer (j = 0), or for a DIRECT-schedule collective
 * (pc_pallgather_init, pc_pallreduce_init with PC_ALGO_DIRECT) the recvbuf of
 * peer j = rank (r + 1 + j) mod P, 0 <= j < P - 1.  For measurement kernels
 * outside the library (the bench's bare NVLink peer-copy and flag floors).
 * PC_ERR_STATE before the exchange, PC_ERR_UNSUPPORTED for other kinds. */
int pc_request_peer_buffer(pc_request_t req, int j, void **ptr);
/* Number of kernels libpc has launched in this process (for the bench's
 * gpu_launches claim). */
uint64_t pc_launch_count(void);
/* Device error word of a request: code and partition (0,0 if none). */
int pc_request_error(pc_request_t req, int *code, int *partition);
const char *pc_strerror(int err);
/* Library version string. */
const char *pc_version(void);

#ifdef __cplusplus
}
#endif
#endif /* PC_H_ */
