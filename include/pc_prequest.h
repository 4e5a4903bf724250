/*
 * include/pc_prequest.h — layout of the device request pc_prequest_t
 * (MPIX_Prequest: "a device specific request object ... containing only
 * the necessary information for a GPU to conduct its duties"; copy
 * mechanism, aggregation threshold, counters, remote address).
 *
 * Plain C, shared by the host library (which fills it) and device code (which
 * receives it BY VALUE as a kernel argument: no pointer chasing).
 * Every pointer is a device address valid in the owning rank's CUDA context;
 * peer_* pointers are peer-mapped (CUDA IPC or same-process) addresses of the
 * partner rank's memory.  The epoch is NOT baked in: pc_prequest_create is
 * called once (Listing 2) and `epoch` points to the device word
 * pc_start writes.
 */
#ifndef PC_PREQUEST_H_
#define PC_PREQUEST_H_

#include <stdint.h>

#define PC_KIND_PSEND 1
#define PC_KIND_PRECV 2
#define PC_KIND_PALLREDUCE 3

struct pc_prequest_s {
  uint32_t kind;        /* PC_KIND_*                                                    */
  uint32_t copy;        /* pc_copy_t: 0 INLINE ("Kernel Copy"), 1 ENGINE                 */
  int32_t partitions;   /* N_p user partitions                                           */
  int32_t agg;          /* g user partitions per transport partition (send side)         */
  int32_t ntransport;   /* ceil(N_p / g)                                                 */
  uint32_t timeout_ms;  /* device spin bound (0 = forever)                               */
  uint64_t part_bytes;  /* bytes per user partition (count * sizeof(dtype))              */
  const uint32_t *epoch;      /* local epoch word written by pc_start                    */
  uint32_t *cnt;              /* [ntransport] aggregation counters (send), never reset   */
  uint32_t *ready;            /* [ntransport] ENGINE ready flags / [N_p] allreduce ready */
  uint32_t *sent;             /* [ntransport] "pushed and flagged" (send-side wait)      */
  const uint8_t *sbuf;        /* local send buffer                                        */
  uint8_t *peer_rbuf;         /* receiver's recv buffer (peer-mapped)                     */
  uint32_t *peer_flags;       /* receiver's arrival flags (peer-mapped) [ntransport]     */
  const uint32_t *rtr;        /* local ready-to-receive word, written by the consumer    */
  const uint32_t *flags;      /* receive side: local arrival flags [N_p]                  */
  const uint32_t *layout;     /* receive side: g, written by the sender at prequest time */
  const uint32_t *done;       /* allreduce: [N_p] per-partition completion counters      */
  uint32_t done_mul;          /* allreduce: partition u is final when done[u] >= e*done_mul */
  int32_t rank;               /* owning rank                                              */
  uint32_t sys_scope;         /* 1: a peer is on another GPU -> system-scope fences /
                                 acquires; 0: every peer shares this GPU -> GPU scope
                                 (a system-scope fence costs ~1.5 us on B200)           */
  int32_t *err;               /* sticky device error word [2] = {code, partition}         */
  /* LL line protocol (PC_COPY_LL): every 8 payload bytes travel
   * with the epoch in one 16-B line {d0, e, d1, e} (two single-copy-atomic
   * 8-B halves), so a line is its own arrival flag: no fence, no flag store. */
  uint32_t ll_lines;          /* 16-B lines per user partition = max(1, ceil(part_bytes/8)),
                                 0 = the request has no LL area                            */
  uint32_t ll_pad;
  uint8_t *peer_ll;           /* send, PC_COPY_LL: receiver's LL area (peer-mapped)        */
  uint8_t *ll;                /* receive: own LL area [2 epoch parities][N_p][ll_lines]   */
  uint8_t *rbuf;              /* receive: own recv buffer (LL lines are unpacked into it) */
  /* partitioned collectives (pc_preduce_scatter_init / pc_pallgather_init /
   * pc_pbcast_init): kind PC_KIND_PALLREDUCE with coll != 0 */
  uint32_t coll;              /* 0 allreduce, 1 reduce-scatter, 2 allgather, 3 broadcast    */
  int32_t nranks;             /* P (allgather: receive partitions = P * partitions)        */
  const uint32_t *srcflags;   /* allgather: [source rank][u][slice] arrival epochs         */
  /* MPI-4 partitioned p2p with DIFFERENT partition counts on the two sides
   * (same dtype and total bytes, reading R30): the receiver's
   * flags are then per RECEIVE partition, counters that every completed send
   * transport partition overlapping it bumps once per epoch. */
  uint32_t xpart;             /* 1: send and receive partitionings differ                  */
  uint32_t xpad;
  uint64_t peer_part_bytes;   /* send: receiver's bytes per partition; receive: sender's   */
  uint32_t *hready;           /* send, PC_COPY_HOST: [ntransport] ready epochs in pinned
                                 host memory (device-mapped), polled by the progress thread */
  /* INLINE allreduce ("Kernel Copy" for the collective, reading R33): the
   * Pready that completes partition u on the LAST of the P ranks folds u over
   * every rank's send buffer in rank order and stores it into every rank's
   * recvbuf (DIRECT schedule bits, oracle O6).  NULL: the engine reduces. */
  const struct pc_ar_tab_s *ar_tab;
  uint32_t dtype;             /* pc_dtype_t of the collective                             */
  uint32_t op;                /* pc_op_t of the collective                                */
};

/* Device table of an INLINE allreduce request (library-owned device memory,
 * written once at pc_prequest_create).  Indexed by comm rank k < nranks <= 8;
 * every pointer is valid in the owning rank's context (peer-mapped). */
#define PC_AR_MAX 8
struct pc_ar_tab_s {
  const uint8_t *send[PC_AR_MAX];  /* rank k's send buffer                                      */
  uint8_t *recv[PC_AR_MAX];        /* rank k's recv buffer                                      */
  uint32_t *done[PC_AR_MAX];       /* rank k's INLINE completion words [N_p] (epoch e = final)  */
  uint32_t *cnt;                   /* arrival counters [N_p] in rank 0's control block (target e*P) */
  const uint32_t *rtr;             /* this rank's ready-to-receive words [P-1], written by the peers */
};

/* Receive side: bit 31 of the layout word = the sender pushes LL lines; bit
 * 30 = the partitionings differ (per-receive-partition counters); bits 0-29 =
 * g, the sender's user partitions per transport partition. */
#define PC_LAYOUT_LL 0x80000000u
#define PC_LAYOUT_XP 0x40000000u
#define PC_LAYOUT_G 0x3fffffffu

#endif /* PC_PREQUEST_H_ */
