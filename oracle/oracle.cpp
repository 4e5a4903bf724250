// oracle/oracle.cpp — CPU ORACLE.  TEST INFRASTRUCTURE ONLY.
//
// Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
// reference legs may load this library.  The product path (libpc.so and the
// Python binding) never links, imports or calls it, and it shares no code,
// header, table or constant generator with the CUDA path.
//
// What it is: a plain, slow, obviously-correct implementation of what
// Temuçin et al., SC'24 (reference PAPER.md, cited as P:Lnn §sec) computes:
//   O1  partitioned point-to-point with transport-partition aggregation and the
//       Pbuf_prepare ready-to-receive handshake            (P:L46-L50, P:L60-L62,
//                                                            P:L127-L145 §IV-A)
//   O2  allreduce, plain definition                        (P:L95, P:L155 MPI_Op)
//   O3  partitioned allreduce, Alg 1 schedule + Alg 2 progression, literally,
//       one progression thread and one "user" thread per rank
//                                                          (Alg 1 P:L159-L171,
//                                                           Alg 2)
//   O4  the same progression over a recursive-doubling schedule (not in the
//       paper; BASELINE north_star; generic tuple of P:L151-L155)
//   O5  Jacobi 5-point sweep, sequential and rank-decomposed with halo flags
//       (stencil per DESIGN.md reading R17)
// Ranks are std::threads; "remote" buffers are shared arrays; every flag is a
// std::atomic<uint32_t> holding an epoch value, written with release and read
// with acquire.  Every reading of a silent/garbled passage is named R<n> and
// listed in DESIGN.md §"Readings of the paper".
//
// Build: g++ -O2 -std=c++17 -fPIC -shared -pthread (no -ffast-math: the fp32
// arithmetic below must be IEEE round-to-nearest, no contraction, no
// reassociation).
#include <atomic>
#include <chrono>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <thread>
#include <vector>

extern "C" {

enum { ORC_OK = 0, ORC_ERR_ARG = -1, ORC_ERR_TIMEOUT = -5 };
enum { ORC_INT32 = 0, ORC_FLOAT32 = 1, ORC_FLOAT64 = 3, ORC_BF16 = 4 };
enum { ORC_SUM = 0, ORC_MAX = 1, ORC_MIN = 2 };

}  // extern "C"

namespace {

// Jitter for thread interleavings (test stimulus only — not the method's
// arithmetic): a splitmix64 step used to decide when a thread yields.
struct Jitter {
  uint64_t s;
  explicit Jitter(uint64_t seed) : s(seed) {}
  uint64_t next() {
    uint64_t z = (s += 0x9E3779B97F4A7C15ull);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
  }
  void maybe_yield() {
    uint64_t v = next();
    if ((v & 3) == 0) std::this_thread::yield();
    if ((v & 255) == 0) std::this_thread::sleep_for(std::chrono::microseconds(v >> 60));
  }
};

// Bounded spin (so a protocol bug fails a test instead of hanging it).
template <class Pred>
bool spin_until(Pred pred, double timeout_s = 60.0) {
  auto t0 = std::chrono::steady_clock::now();
  unsigned n = 0;
  while (!pred()) {
    if (++n % 64 == 0) {
      std::this_thread::yield();
      if (std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() > timeout_s)
        return false;
    }
  }
  return true;
}

// ---- the reduction operators ⊕ ("MPI_Op") -------------------------
// R5: acc = local ⊕ incoming; fp32 in fp32 with round-to-nearest-even.
inline int32_t op_i32(int op, int32_t local, int32_t incoming) {
  switch (op) {
    case ORC_SUM: return (int32_t)((uint32_t)local + (uint32_t)incoming);  // wraps mod 2^32
    case ORC_MAX: return local > incoming ? local : incoming;
    default:      return local < incoming ? local : incoming;
  }
}
inline float op_f32(int op, float local, float incoming) {
  switch (op) {
    case ORC_SUM: {
      volatile float r = local + incoming;  // one IEEE fp32 add, no contraction
      return r;
    }
    case ORC_MAX: return std::fmax(local, incoming);
    default:      return std::fmin(local, incoming);
  }
}

// fp64 (R27): one IEEE binary64 add, round-to-nearest-even.
inline double op_f64(int op, double local, double incoming) {
  switch (op) {
    case ORC_SUM: {
      volatile double r = local + incoming;
      return r;
    }
    case ORC_MAX: return std::fmax(local, incoming);
    default:      return std::fmin(local, incoming);
  }
}

// bf16 (R27): a bf16 value is the top 16 bits of an IEEE binary32 (1-8-7).
// local ⊕ incoming = the bf16 nearest (ties to even) to the EXACT result, i.e.
// the correctly rounded bf16 operation.  Written out here from the definition:
// decode both operands exactly, add in binary64, round the binary64 value to
// 8 significant bits.  (The binary64 add is itself exact or double-rounding-
// innocuous: 53 >= 2*8+2, Figueroa's theorem.)
inline double bf16_decode(uint16_t b) {
  uint32_t u = (uint32_t)b << 16;
  float f;
  std::memcpy(&f, &u, 4);
  return (double)f;
}
inline uint16_t bf16_round(double v) {
  if (std::isnan(v)) return (uint16_t)(std::signbit(v) ? 0xFFC0 : 0x7FC0);
  const uint16_t sign = std::signbit(v) ? 0x8000 : 0;
  double a = std::fabs(v);
  if (a == 0.0) return sign;
  if (std::isinf(a)) return (uint16_t)(sign | 0x7F80);
  int E;
  std::frexp(a, &E);                           // a = m 2^E, m in [0.5, 1): leading bit 2^(E-1)
  const int ulp_exp = std::max(E - 8, -133);   // 8 significant bits; bf16 subnormal quantum 2^-133
  double r = std::nearbyint(std::ldexp(a, -ulp_exp));  // FE_TONEAREST: ties to even
  r = std::ldexp(r, ulp_exp);
  if (r >= std::ldexp(1.0, 128)) return (uint16_t)(sign | 0x7F80);  // overflow -> inf
  float f = (float)r;                          // exact: r has <= 8 significant bits in range
  uint32_t u;
  std::memcpy(&u, &f, 4);
  return (uint16_t)(sign | (u >> 16));
}
inline uint16_t op_bf16(int op, uint16_t local, uint16_t incoming) {
  const double a = bf16_decode(local), b = bf16_decode(incoming);
  switch (op) {
    case ORC_SUM: return bf16_round(a + b);
    case ORC_MAX: return bf16_round(std::fmax(a, b));
    default:      return bf16_round(std::fmin(a, b));
  }
}

int64_t esize_of(int dtype) { return dtype == ORC_FLOAT64 ? 8 : dtype == ORC_BF16 ? 2 : 4; }

void reduce_into(int dtype, int op, void *dst, const void *local, const void *incoming, int64_t n) {
  if (dtype == ORC_INT32) {
    auto d = (int32_t *)dst;
    auto a = (const int32_t *)local;
    auto b = (const int32_t *)incoming;
    for (int64_t k = 0; k < n; ++k) d[k] = op_i32(op, a[k], b[k]);
  } else if (dtype == ORC_FLOAT64) {
    auto d = (double *)dst;
    auto a = (const double *)local;
    auto b = (const double *)incoming;
    for (int64_t k = 0; k < n; ++k) d[k] = op_f64(op, a[k], b[k]);
  } else if (dtype == ORC_BF16) {
    auto d = (uint16_t *)dst;
    auto a = (const uint16_t *)local;
    auto b = (const uint16_t *)incoming;
    for (int64_t k = 0; k < n; ++k) d[k] = op_bf16(op, a[k], b[k]);
  } else {
    auto d = (float *)dst;
    auto a = (const float *)local;
    auto b = (const float *)incoming;
    for (int64_t k = 0; k < n; ++k) d[k] = op_f32(op, a[k], b[k]);
  }
}

inline int mod(int a, int p) { return ((a % p) + p) % p; }

}  // namespace

extern "C" {

// ===========================================================================
// O1: partitioned point-to-point (2 ranks: sender 0, receiver 1)
// ===========================================================================
// Follows the flow of P:L46-L50 and Fig. 1 / Listing 2:
//   sender:   Start -> Pbuf_prepare (wait RTR) -> Pready(p) by W
//             worker threads in the given order -> Wait
//   receiver: Start -> Pbuf_prepare (post RTR = e) -> Wait (all flags == e)
//             -> [delay] -> consume recvbuf
// Aggregation (readings R10, R12): user partition p belongs to
// transport partition t = p / g; each Pready increments cnt[t]; counters are
// never reset, the contributor that brings cnt[t] to e*g_t performs the copy
// of transport partition t ("Kernel Copy") and release-stores
// flag[t] = e ("completion").
//
// send:      epochs x (partitions*part_bytes) bytes; epoch e uses row e-1
// consumed:  epochs x total; what the receiver read after each Wait
// orders:    epochs x partitions; the Pready order of each epoch (stimulus)
// arrivals:  epochs x ntransport; how many times t was published in epoch e
//            (must be exactly 1 — "exactly-once")
// use_rtr=0 reproduces the restart hazard of P:L60 (with recv_delay_us > 0).
int orc_p2p(const uint8_t *send, uint8_t *consumed, int partitions, int64_t part_bytes, int agg,
            int workers, int epochs, const int32_t *orders, int use_rtr, int recv_delay_us,
            uint64_t jitter_seed, uint32_t *arrivals) {
  if (partitions < 1 || part_bytes < 0 || agg < 1 || workers < 1 || epochs < 1) return ORC_ERR_ARG;
  const int64_t total = (int64_t)partitions * part_bytes;
  const int nt = (partitions + agg - 1) / agg;
  std::vector<uint8_t> recvbuf((size_t)total);
  std::vector<std::atomic<uint64_t>> cnt(nt);
  std::vector<std::atomic<uint32_t>> flag(nt);
  std::vector<std::atomic<uint32_t>> arr((size_t)epochs * nt);
  for (auto &c : cnt) c.store(0);
  for (auto &f : flag) f.store(0);
  for (auto &a : arr) a.store(0);
  std::atomic<uint32_t> rtr{0};
  std::atomic<int> failed{0};

  auto pready = [&](uint32_t e, int p) {  // MPIX_Pready(p) in Kernel Copy mode
    const int t = p / agg;
    const int64_t g_t = std::min<int64_t>(agg, partitions - (int64_t)t * agg);
    const uint64_t mine = cnt[t].fetch_add(1, std::memory_order_acq_rel) + 1;
    if (mine == (uint64_t)e * (uint64_t)g_t) {  // last contributor of t in epoch e
      const int64_t off = (int64_t)t * agg * part_bytes;
      std::memcpy(recvbuf.data() + off, send + (int64_t)(e - 1) * total + off, (size_t)(g_t * part_bytes));
      arr[(size_t)(e - 1) * nt + t].fetch_add(1);
      flag[t].store(e, std::memory_order_release);
    }
  };

  std::thread sender([&] {
    Jitter jit(jitter_seed ^ 0x51);
    for (uint32_t e = 1; e <= (uint32_t)epochs; ++e) {
      // MPI_Start: e.  MPIX_Pbuf_prepare: wait ready-to-receive.
      if (use_rtr && !spin_until([&] { return rtr.load(std::memory_order_acquire) >= e; })) {
        failed = 1;
        return;
      }
      const int32_t *ord = orders + (int64_t)(e - 1) * partitions;
      std::vector<std::thread> ws;
      for (int w = 0; w < workers; ++w)
        ws.emplace_back([&, w] {
          Jitter j2(jitter_seed + 1000 * e + w);
          for (int k = w; k < partitions; k += workers) {
            j2.maybe_yield();
            pready(e, ord[k]);
          }
        });
      for (auto &t : ws) t.join();  // MPI_Wait (sender): every partition readied and delivered
      jit.maybe_yield();
    }
  });
  std::thread receiver([&] {
    for (uint32_t e = 1; e <= (uint32_t)epochs; ++e) {
      if (use_rtr) rtr.store(e, std::memory_order_release);  // MPIX_Pbuf_prepare: RTR
      for (int t = 0; t < nt; ++t)                             // MPI_Wait (receiver)
        if (!spin_until([&] { return flag[t].load(std::memory_order_acquire) >= e; })) {
          failed = 1;
          return;
        }
      if (recv_delay_us > 0) std::this_thread::sleep_for(std::chrono::microseconds(recv_delay_us));
      std::memcpy(consumed + (int64_t)(e - 1) * total, recvbuf.data(), (size_t)total);
    }
  });
  sender.join();
  receiver.join();
  for (size_t k = 0; k < arr.size(); ++k) arrivals[k] = arr[k].load();
  return failed ? ORC_ERR_TIMEOUT : ORC_OK;
}

// ===========================================================================
// O2: allreduce, plain definition  y = ⊕_r x_r
// ===========================================================================
// int32: exact integer semantics (sum wraps mod 2^32, max, min), rank order.
int orc_allreduce_def_i32(int P, int64_t n, const int32_t *x, int op, int32_t *y) {
  if (P < 1 || n < 0) return ORC_ERR_ARG;
  for (int64_t k = 0; k < n; ++k) {
    int32_t acc = x[k];
    for (int r = 1; r < P; ++r) acc = op_i32(op, acc, x[(int64_t)r * n + k]);
    y[k] = acc;
  }
  return ORC_OK;
}
// fp32 SUM: the fp64 sum of the fp32 inputs in rank order (effectively exact,
// error <= (P-1) 2^-53 sum|x|); also returns sum|x| for the R16 tolerance.
int orc_allreduce_def_f64(int P, int64_t n, const float *x, double *y, double *sumabs) {
  if (P < 1 || n < 0) return ORC_ERR_ARG;
  for (int64_t k = 0; k < n; ++k) {
    double acc = 0.0, a = 0.0;
    for (int r = 0; r < P; ++r) {
      acc += (double)x[(int64_t)r * n + k];
      a += std::fabs((double)x[(int64_t)r * n + k]);
    }
    y[k] = acc;
    if (sumabs) sumabs[k] = a;
  }
  return ORC_OK;
}

// ===========================================================================
// O3 / O4: partitioned allreduce, Alg 1 (or RD) schedule + Alg 2 progression
// ===========================================================================
namespace {

constexpr uint32_t kTerminal = 0xFFFFFFFFu;

// One step S_i = (I, R, ⊕, O, A).  |I| = |O| = 1 for both schedules
// built here.  R and A are chunk ids (ring) or -1 = "whole partition" (RD).
struct Step {
  int I, R, op, O, A;  // op: 1 = MPI_Op, 0 = NOP
};

// Alg 1.  R1: the loop is "for i <- 0 to 2(P-1)"; read with an
// exclusive bound -> exactly 2(P-1) communicating steps i in [0, 2(P-1)),
// matching "MPI_Op for the first P-1 steps and then a NOP for the remaining
// P-1 steps".  S_k is a terminal sentinel (R2).
std::vector<Step> alg1_ring(int P, int rank) {
  std::vector<Step> S;
  for (int i = 0; i < 2 * (P - 1); ++i) {
    Step s;
    s.I = mod(rank - 1, P);                 // line 2
    s.O = mod(rank + 1, P);                 // line 3
    s.R = mod(rank + 2 * P - i, P);         // line 4
    s.A = mod(rank + 2 * P - i - 1, P);     // line 5
    s.op = (i < (P - 1)) ? 1 : 0;           // lines 6-7
    S.push_back(s);                         // lines 8-9
  }
  return S;
}

// Recursive doubling (north_star; not in the paper): step k exchanges the whole
// partition with r xor 2^k and reduces every step.
std::vector<Step> rd_schedule(int P, int rank) {
  std::vector<Step> S;
  for (int k = 0; (1 << k) < P; ++k) S.push_back(Step{rank ^ (1 << k), -1, 1, rank ^ (1 << k), -1});
  return S;
}

struct RankState {
  // per-(u) progression state of Alg 2
  std::vector<std::atomic<uint32_t>> step, parrived, pready;
  std::vector<std::atomic<uint32_t>> local_ready;   // R23: user has Preadied u
  std::vector<std::atomic<uint32_t>> flag;          // [u][i] arrival flags (R3), value = epoch
  std::vector<uint8_t> staging;                     // ring: [u][chunk]; RD: [u][k][L]
  std::vector<uint8_t> work;                        // RS partial sums / RD accumulator
  std::atomic<uint32_t> rtr{0};                     // ready-to-receive epoch (R13)
  uint8_t *sendbuf = nullptr, *recvbuf = nullptr;
  std::vector<Step> S;
};

}  // namespace

// algo: 1 = ring (O3), 2 = recursive doubling (O4, P a power of two)
// x:       epochs x P x (Np*L) inputs (rank r's sendbuf of epoch e is row (e-1)*P + r)
// y:       epochs x P x (Np*L) the recvbuf each rank holds after its Wait of epoch e
// orders:  epochs x P x Np user Pready orders (stimulus)
// reduces: P x Np x nsteps number of reduceData() executions per (rank, u, step)
//          in the LAST epoch (must be 1 on MPI_Op steps, 0 on NOP steps)
// arrivals:P x Np x nsteps number of observed arrivals per (rank, u, step) in the
//          last epoch (must be 1)
int orc_pallreduce(int algo, int P, int Np, int64_t L, int dtype, int op, int epochs, int inplace,
                   const void *x, void *y, const int32_t *orders, uint64_t jitter_seed,
                   uint32_t *reduces, uint32_t *arrivals) {
  if (P < 1 || Np < 1 || L < 0 || epochs < 1 || (algo != 1 && algo != 2)) return ORC_ERR_ARG;
  if (algo == 2 && (P & (P - 1))) return ORC_ERR_ARG;
  const int64_t esz = esize_of(dtype);
  const int64_t part_bytes = L * esz;
  const int64_t nbytes = (int64_t)Np * part_bytes;
  // R4: chunking of a partition of L elements into P chunks: q = ceil(L/(vP))*v
  // elements with v = 16/esz (q elements are a 16-byte multiple); chunk
  // c = [c q, min((c+1) q, L)), possibly empty.
  const int64_t v = 16 / esz;
  const int64_t q = ((L + v * P - 1) / (v * P)) * v;
  auto chunk_lo = [&](int c) { return std::min<int64_t>((int64_t)c * q, L); };
  auto chunk_n = [&](int c) { return std::min<int64_t>((int64_t)(c + 1) * q, L) - chunk_lo(c); };
  int nsteps_rd = 0;
  while ((1 << nsteps_rd) < P) ++nsteps_rd;
  const int NS = (algo == 1) ? 2 * (P - 1) : nsteps_rd;  // communicating steps

  std::vector<RankState> R(P);
  std::vector<std::vector<uint8_t>> own_send(P), own_recv(P);
  for (int r = 0; r < P; ++r) {
    auto &st = R[r];
    st.S = (algo == 1) ? alg1_ring(P, r) : rd_schedule(P, r);
    st.step = std::vector<std::atomic<uint32_t>>(Np);
    st.parrived = std::vector<std::atomic<uint32_t>>(Np);
    st.pready = std::vector<std::atomic<uint32_t>>(Np);
    st.local_ready = std::vector<std::atomic<uint32_t>>(Np);
    st.flag = std::vector<std::atomic<uint32_t>>((size_t)Np * std::max(NS, 1));
    for (auto &f : st.flag) f.store(0);
    for (auto &f : st.local_ready) f.store(0);
    st.staging.assign((size_t)(algo == 1 ? nbytes : nbytes * std::max(NS, 1)), 0);
    st.work.assign((size_t)nbytes, 0);
    own_recv[r].assign((size_t)nbytes, 0);
    own_send[r].assign((size_t)nbytes, 0);
    st.recvbuf = own_recv[r].data();
    st.sendbuf = inplace ? st.recvbuf : own_send[r].data();
  }
  std::vector<std::atomic<uint32_t>> red((size_t)P * Np * std::max(NS, 1)), arr((size_t)P * Np * std::max(NS, 1));
  std::atomic<int> failed{0};

  // Byte ranges of a "region" (chunk id, or -1 = whole partition) of partition u.
  auto region_off = [&](int u, int c) { return (int64_t)u * part_bytes + (c < 0 ? 0 : chunk_lo(c) * esz); };
  auto region_len = [&](int c) { return c < 0 ? part_bytes : chunk_n(c) * esz; };
  // Where a payload sent at step i lands at the receiver (R3): MPI_Op steps land
  // in staging (ring: indexed by chunk id; RD: by step), NOP steps in recvbuf.
  auto landing = [&](int dst, int u, int i, int c) -> uint8_t * {
    auto &d = R[dst];
    if (d.S.empty()) return nullptr;
    const Step &s = d.S[i];
    if (!s.op) return d.recvbuf + region_off(u, c);
    if (algo == 1) return d.staging.data() + region_off(u, c);
    return d.staging.data() + ((int64_t)i * nbytes) + region_off(u, c);
  };
  // MPI_Pready of transport partition (u, step i) towards O: copy, then
  // release the receiver's (u, i) flag — the two puts of P:L133.
  auto send = [&](int r, int u, int i, const uint8_t *src_base, uint32_t e) {
    const Step &s = R[r].S[i];
    const int c = s.R;
    uint8_t *dst = landing(s.O, u, i, c);
    std::memcpy(dst, src_base + region_off(u, c), (size_t)region_len(c));
    R[s.O].flag[(size_t)u * NS + i].store(e, std::memory_order_release);
  };

  for (uint32_t e = 1; e <= (uint32_t)epochs; ++e) {
    const bool last = (e == (uint32_t)epochs);
    std::vector<std::thread> th;
    for (int r = 0; r < P; ++r) {
      // ---- MPI_Start: reset per-partition state for this epoch
      auto &st = R[r];
      const uint8_t *xin = (const uint8_t *)x + ((int64_t)(e - 1) * P + r) * nbytes;
      std::memcpy(st.sendbuf, xin, (size_t)nbytes);  // the user's kernel producing sendbuf
      for (int u = 0; u < Np; ++u) {
        st.step[u] = 0;
        st.parrived[u] = 0;
        st.pready[u] = 0;
        st.local_ready[u] = 0;
      }
    }
    for (int r = 0; r < P; ++r) {
      // ---- MPIX_Pbuf_prepare: post ready-to-receive to every
      // rank that will write into r this epoch (R13).
      R[r].rtr.store(e, std::memory_order_release);
    }
    for (int r = 0; r < P; ++r) {
      // ---- user thread: the kernel's MPIX_Pready(u) calls (Listing 2)
      th.emplace_back([&, r] {
        auto &st = R[r];
        Jitter jit(jitter_seed + 7919u * e + r);
        const int32_t *ord = orders + ((int64_t)(e - 1) * P + r) * Np;
        for (int k = 0; k < Np; ++k) {
          const int u = ord[k];
          jit.maybe_yield();
          if (st.S.empty()) {  // R1 with P = 1: no steps; the allreduce is a copy
            std::memmove(st.recvbuf + region_off(u, -1), st.sendbuf + region_off(u, -1), (size_t)part_bytes);
            st.local_ready[u].store(1, std::memory_order_release);
            continue;
          }
          // the sender waits for the receiver's ready-to-receive before
          // its first put of this epoch
          for (auto &s0 : {st.S[0].O})
            if (!spin_until([&] { return R[s0].rtr.load(std::memory_order_acquire) >= e; })) failed = 1;
          st.local_ready[u].store(1, std::memory_order_release);
          // "the first MPI_Pready should be called by the application programmer"
          // (P:L213): the user's Pready is the step-0 Pready.
          send(r, u, 0, st.sendbuf, e);
          st.pready[u].store(1, std::memory_order_release);
        }
      });
      // ---- progression thread: MPI_Wait running Alg 2
      th.emplace_back([&, r] {
        auto &st = R[r];
        Jitter jit(jitter_seed * 31 + 104729u * e + r);
        const int k_term = (int)st.S.size();  // index of S_k (terminal)
        auto t0 = std::chrono::steady_clock::now();
        for (;;) {
          bool all_terminal = true;
          for (int u = 0; u < Np; ++u) {                                    // line 1
            const int i = (int)st.step[u].load();                           // lines 2-3
            if (i >= k_term) continue;                                      // line 4
            all_terminal = false;
            const Step &s = st.S[i];
            if (st.parrived[u].load() != 1 /* |I| */) {                     // line 5
              // lines 6-12 with |I| = 1.  R23: a reduce needs u locally ready.
              const uint32_t f = st.flag[(size_t)u * NS + i].load(std::memory_order_acquire);  // line 7
              if (f == e && st.local_ready[u].load(std::memory_order_acquire)) {               // line 8
                st.parrived[u].store(1);                                                        // line 9
                if (last) arr[((size_t)r * Np + u) * NS + i].fetch_add(1);
                if (s.op) {                                                                     // line 10
                  // reduceData(): acc = local ⊕ incoming, exactly once (R6)
                  const int c = s.A;
                  const int64_t off = region_off(u, c), len = region_len(c);
                  const uint8_t *incoming = landing(r, u, i, c);
                  const uint8_t *local = (algo == 1 || i == 0) ? st.sendbuf + off : st.work.data() + off;
                  reduce_into(dtype, op, st.work.data() + off, local, incoming, len / esz);
                  if (last) red[((size_t)r * Np + u) * NS + i].fetch_add(1);
                  // ring: after the (P-2)th reduce chunk r+1 is final at r (R3)
                  if (algo == 1 && i == P - 2) std::memcpy(st.recvbuf + off, st.work.data() + off, (size_t)len);
                  if (algo == 2 && i == k_term - 1) std::memcpy(st.recvbuf + off, st.work.data() + off, (size_t)len);
                }
              }
            }
            if (st.parrived[u].load() == 1 && st.pready[u].load(std::memory_order_acquire) == 1) {  // lines 14-15
              st.step[u].store(i + 1);                                       // line 17
              st.parrived[u].store(0);                                       // line 18
              st.pready[u].store(0);                                         // line 19
              const int j = i + 1;
              // line 21 (R2): not S_0 (the user's), not S_k (terminal)
              if (j != 0 && j < k_term && st.pready[u].load() == 0) {
                // lines 24-27: Pready to every O.  The payload of step j is the
                // region R_j; ring: R_j == A_{j-1}, taken from work after a
                // reduce step and from recvbuf after a NOP step; RD: work.
                const uint8_t *src = st.S[j - 1].op ? st.work.data() : st.recvbuf;
                send(r, u, j, src, e);
                st.pready[u].store(1);                                       // line 26
              }
            }
          }
          if (all_terminal) break;
          jit.maybe_yield();
          if (std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() > 120.0) {
            failed = 1;
            break;
          }
        }
      });
    }
    for (auto &t : th) t.join();
    // ---- consume: the recvbuf after MPI_Wait
    for (int r = 0; r < P; ++r)
      std::memcpy((uint8_t *)y + ((int64_t)(e - 1) * P + r) * nbytes, R[r].recvbuf, (size_t)nbytes);
    if (failed) break;
  }
  if (reduces)
    for (size_t k = 0; k < red.size(); ++k) reduces[k] = red[k].load();
  if (arrivals)
    for (size_t k = 0; k < arr.size(); ++k) arrivals[k] = arr[k].load();
  return failed ? ORC_ERR_TIMEOUT : ORC_OK;
}

// ===========================================================================
// O7: DL proxy producer (§VI-D2; the BCE kernel of [34] is
// external, reading R28): gradient of the mean binary cross-entropy
//   l = -(1/n) sum_i [ y_i ln p_i + (1 - y_i) ln(1 - p_i) ]
// with respect to p_i:  dl/dp_i = (p_i - y_i) / (p_i (1 - p_i) n),
// evaluated in fp32 as five IEEE operations in this order:
//   ((p - y) / ((p * (1 - p)) * n)).
// ===========================================================================
int orc_bce_grad(int64_t n, const float *p, const float *y, float nf, float *g) {
  for (int64_t i = 0; i < n; ++i) {
    volatile float d = p[i] - y[i];
    volatile float t = 1.0f - p[i];
    volatile float q = p[i] * t;
    volatile float qn = q * nf;
    volatile float r = d / qn;
    g[i] = r;
  }
  return ORC_OK;
}

// bf16 arithmetic of R27, exported so tests can pin it (round-to-nearest-even
// of binary64 values to bf16 bit patterns; the ⊕ of two bf16 operands).
int orc_bf16_round(int64_t n, const double *x, uint16_t *out) {
  for (int64_t k = 0; k < n; ++k) out[k] = bf16_round(x[k]);
  return ORC_OK;
}
int orc_bf16_op(int op, int64_t n, const uint16_t *a, const uint16_t *b, uint16_t *out) {
  for (int64_t k = 0; k < n; ++k) out[k] = op_bf16(op, a[k], b[k]);
  return ORC_OK;
}

// ===========================================================================
// O6: partitioned allreduce over the DIRECT two-step schedule (
// the generic schedule of P:L151-L155 with neighbour SETS, progressed by Alg 2
// with |I| = |O| = P-1):
//   S_0 = (I = all others, R = chunk o for each O_o, MPI_Op, O = all others,
//          A = my chunk r from every I)          -- reduce-scatter to owners
//   S_1 = (I = all others, R = my chunk r (final), NOP, O = all others,
//          A = chunk i from every I_i)           -- allgather of owned chunks
// Chunk c (reading R4) is owned by rank c.  Reading R25: with |I| > 1 the
// arrivals of a step are reduced in rank order (reduceData of contribution k
// only after 0..k-1), so the fp32 result is the left fold over ranks
// 0..P-1, independent of arrival order.
// ===========================================================================
int orc_pallreduce_direct(int P, int Np, int64_t L, int dtype, int op, int epochs, int inplace, const void *x,
                          void *y, const int32_t *orders, uint64_t jitter_seed, uint32_t *reduces,
                          uint32_t *arrivals) {
  if (P < 1 || Np < 1 || L < 0 || epochs < 1) return ORC_ERR_ARG;
  const int64_t esz = esize_of(dtype), part_bytes = L * esz, nbytes = (int64_t)Np * part_bytes;
  const int64_t v = 16 / esz;
  const int64_t q = ((L + v * P - 1) / (v * P)) * v;  // R4
  auto chunk_lo = [&](int c) { return std::min<int64_t>((int64_t)c * q, L); };
  auto chunk_n = [&](int c) { return std::min<int64_t>((int64_t)(c + 1) * q, L) - chunk_lo(c); };
  struct Rk {
    std::vector<uint8_t> send, recv, staging;  // staging[u][sender][chunk r]
    uint8_t *sendbuf = nullptr, *recvbuf = nullptr;
    std::vector<std::atomic<uint32_t>> flag;  // [u][step][sender], value = epoch
    std::vector<std::atomic<uint32_t>> local_ready;
    std::atomic<uint32_t> rtr{0};
  };
  std::vector<Rk> R(P);
  for (int r = 0; r < P; ++r) {
    R[r].send.assign((size_t)nbytes, 0);
    R[r].recv.assign((size_t)nbytes, 0);
    R[r].staging.assign((size_t)(Np * P * q * esz + 16), 0);
    R[r].recvbuf = R[r].recv.data();
    R[r].sendbuf = inplace ? R[r].recvbuf : R[r].send.data();
    R[r].flag = std::vector<std::atomic<uint32_t>>((size_t)Np * 2 * P);
    for (auto &f : R[r].flag) f.store(0);
    R[r].local_ready = std::vector<std::atomic<uint32_t>>(Np);
  }
  std::vector<std::atomic<uint32_t>> red((size_t)P * Np * 2), arr((size_t)P * Np * 2);
  std::atomic<int> failed{0};
  auto stage_ptr = [&](int owner, int u, int sender) {
    return R[owner].staging.data() + (((int64_t)u * P + sender) * q) * esz;
  };
  for (uint32_t e = 1; e <= (uint32_t)epochs; ++e) {
    const bool last = e == (uint32_t)epochs;
    for (int r = 0; r < P; ++r) {  // MPI_Start + the user's kernel producing sendbuf
      std::memcpy(R[r].sendbuf, (const uint8_t *)x + ((int64_t)(e - 1) * P + r) * nbytes, (size_t)nbytes);
      for (auto &f : R[r].local_ready) f.store(0);
    }
    for (int r = 0; r < P; ++r) R[r].rtr.store(e, std::memory_order_release);  // MPIX_Pbuf_prepare
    std::vector<std::thread> th;
    for (int r = 0; r < P; ++r) {
      th.emplace_back([&, r] {  // user: Pready(u) = the step-0 Pready to every O
        Jitter jit(jitter_seed + 7919u * e + r);
        const int32_t *ord = orders + ((int64_t)(e - 1) * P + r) * Np;
        for (int k = 0; k < Np; ++k) {
          const int u = ord[k];
          jit.maybe_yield();
          R[r].local_ready[u].store(1, std::memory_order_release);
          for (int o = 0; o < P; ++o) {
            if (o == r) continue;
            if (!spin_until([&] { return R[o].rtr.load(std::memory_order_acquire) >= e; })) failed = 1;
            std::memcpy(stage_ptr(o, u, r), R[r].sendbuf + (int64_t)u * part_bytes + chunk_lo(o) * esz,
                        (size_t)(chunk_n(o) * esz));
            R[o].flag[((size_t)u * 2 + 0) * P + r].store(e, std::memory_order_release);
          }
        }
      });
      th.emplace_back([&, r] {  // MPI_Wait: Alg 2 over the two steps
        auto &me = R[r];
        std::vector<int> step(Np, 0), next(Np, 0), seen(Np, 0);
        std::vector<std::vector<uint8_t>> work(Np, std::vector<uint8_t>((size_t)(q * esz + 16)));
        Jitter jit(jitter_seed * 31 + 104729u * e + r);
        auto t0 = std::chrono::steady_clock::now();
        const int64_t n = chunk_n(r), off = chunk_lo(r) * esz;
        for (;;) {
          bool all = true;
          for (int u = 0; u < Np; ++u) {
            if (step[u] >= 2 || P == 1) {
              if (P == 1 && step[u] == 0 && me.local_ready[u].load(std::memory_order_acquire)) {
                std::memmove(me.recvbuf + (int64_t)u * part_bytes, me.sendbuf + (int64_t)u * part_bytes,
                             (size_t)part_bytes);
                step[u] = 2;
              }
              if (step[u] < 2) all = false;
              continue;
            }
            all = false;
            if (!me.local_ready[u].load(std::memory_order_acquire)) continue;  // R23
            if (step[u] == 0) {
              // arrivals of S_0 reduced in rank order (R25), each exactly once
              while (next[u] < P) {
                const int k = next[u];
                const uint8_t *src;
                if (k == r) {
                  src = me.sendbuf + (int64_t)u * part_bytes + off;
                } else {
                  if (me.flag[((size_t)u * 2 + 0) * P + k].load(std::memory_order_acquire) != e) break;
                  if (last) arr[((size_t)r * Np + u) * 2 + 0]++;
                  src = stage_ptr(r, u, k);
                }
                if (k == 0) {
                  std::memcpy(work[u].data(), src, (size_t)(n * esz));
                } else {
                  reduce_into(dtype, op, work[u].data(), work[u].data(), src, n);
                  if (last) red[((size_t)r * Np + u) * 2 + 0]++;
                }
                next[u] = k + 1;
              }
              if (next[u] < P) continue;
              // parrived = |I|, pready(S_0) = |O| (the user's) -> S_1: Pready the final chunk to every O
              std::memcpy(me.recvbuf + (int64_t)u * part_bytes + off, work[u].data(), (size_t)(n * esz));
              for (int o = 0; o < P; ++o) {
                if (o == r) continue;
                std::memcpy(R[o].recvbuf + (int64_t)u * part_bytes + off, work[u].data(), (size_t)(n * esz));
                R[o].flag[((size_t)u * 2 + 1) * P + r].store(e, std::memory_order_release);
              }
              step[u] = 1;
            }
            if (step[u] == 1) {  // S_1 arrivals: chunk i from every I_i (NOP)
              int got = 0;
              for (int k = 0; k < P; ++k)
                if (k != r && me.flag[((size_t)u * 2 + 1) * P + k].load(std::memory_order_acquire) == e) ++got;
              if (got == P - 1) {
                if (last) arr[((size_t)r * Np + u) * 2 + 1] += (uint32_t)got;
                step[u] = 2;  // S_k: terminal
              }
            }
          }
          if (all) break;
          jit.maybe_yield();
          if (std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() > 120.0) {
            failed = 1;
            break;
          }
        }
      });
    }
    for (auto &t : th) t.join();
    for (int r = 0; r < P; ++r)
      std::memcpy((uint8_t *)y + ((int64_t)(e - 1) * P + r) * nbytes, R[r].recvbuf, (size_t)nbytes);
    if (failed) break;
  }
  if (reduces)
    for (size_t k = 0; k < red.size(); ++k) reduces[k] = red[k].load();
  if (arrivals)
    for (size_t k = 0; k < arr.size(); ++k) arrivals[k] = arr[k].load();
  return failed ? ORC_ERR_TIMEOUT : ORC_OK;
}

// Alg 1 table for (P, rank): out[i*5 + {0..4}] = I, R, op, O, A for i in [0, 2(P-1)).
int orc_alg1_table(int P, int rank, int32_t *out) {
  if (P < 1 || rank < 0 || rank >= P) return ORC_ERR_ARG;
  auto S = alg1_ring(P, rank);
  for (size_t i = 0; i < S.size(); ++i) {
    out[i * 5 + 0] = S[i].I;
    out[i * 5 + 1] = S[i].R;
    out[i * 5 + 2] = S[i].op;
    out[i * 5 + 3] = S[i].O;
    out[i * 5 + 4] = S[i].A;
  }
  return (int)S.size();
}

// Closed forms of O3/O4 for one element (c.1): the value every rank holds.
//   ring: left fold starting at rank `start` (= the chunk id) around the ring,
//         fl(...fl(fl(x_c + x_{c+1}) + x_{c+2}) ... + x_{c-1})
//   rd:   balanced tree in rank order
// x: P x n, start: n (chunk id of each element), out: n.  These are pinned
// against orc_pallreduce on small inputs (tests/test_oracle_allreduce.py).
int orc_ring_fold_f32(int P, int64_t n, const float *x, const int32_t *start, float *out) {
  for (int64_t k = 0; k < n; ++k) {
    const int c = start[k];
    float acc = x[(int64_t)c * n + k];
    for (int j = 1; j < P; ++j) acc = op_f32(ORC_SUM, x[(int64_t)mod(c + j, P) * n + k], acc);
    out[k] = acc;
  }
  return ORC_OK;
}
int orc_rd_tree_f32(int P, int64_t n, const float *x, float *out) {
  std::vector<float> v(P);
  for (int64_t k = 0; k < n; ++k) {
    for (int r = 0; r < P; ++r) v[r] = x[(int64_t)r * n + k];
    for (int w = 1; w < P; w <<= 1)
      for (int r = 0; r < P; r += 2 * w) v[r] = op_f32(ORC_SUM, v[r], v[r + w]);
    out[k] = v[0];
  }
  return ORC_OK;
}

// ===========================================================================
// O5: Jacobi (R17 stencil)
// ===========================================================================
// Grid ny x nx including the Dirichlet boundary (row 0, row ny-1, col 0,
// col nx-1 held fixed).  One iteration:
//   a_new[i][j] = 0.25f * ((a[i-1][j] + a[i+1][j]) + (a[i][j-1] + a[i][j+1]))
static inline float stencil(float up, float down, float left, float right) {
  volatile float s1 = up + down;
  volatile float s2 = left + right;
  volatile float s = s1 + s2;
  volatile float r = 0.25f * s;
  return r;
}

int orc_jacobi_seq(int ny, int nx, int iters, const float *a0, float *out) {
  if (ny < 2 || nx < 2 || iters < 0) return ORC_ERR_ARG;
  std::vector<float> a(a0, a0 + (size_t)ny * nx), b(a);
  for (int it = 0; it < iters; ++it) {
    for (int i = 1; i < ny - 1; ++i)
      for (int j = 1; j < nx - 1; ++j)
        b[(size_t)i * nx + j] = stencil(a[(size_t)(i - 1) * nx + j], a[(size_t)(i + 1) * nx + j],
                                        a[(size_t)i * nx + j - 1], a[(size_t)i * nx + j + 1]);
    std::swap(a, b);
  }
  std::memcpy(out, a.data(), sizeof(float) * (size_t)ny * nx);
  return ORC_OK;
}

// Rank-decomposed Jacobi: Py x Px ranks (threads), rank (py, px) owns rows
// [py*ny/Py, (py+1)*ny/Py) x cols [px*nx/Px, ...) of the global grid (R18:
// ny % Py == 0, nx % Px == 0).  Each rank keeps two local buffers with a
// one-cell halo ring.  Iteration k: wait for the halos of the buffer being
// read (neighbour flags >= k), update own cells (global-boundary cells stay
// fixed), put own edge rows/cols into the neighbours' halos of the buffer
// being written, release flag = k+1 (the partitioned halo exchange of P:L304;
// no RTR is needed, R18).  Result must equal orc_jacobi_seq
// bit for bit.
int orc_jacobi_decomp(int ny, int nx, int Py, int Px, int iters, const float *a0, float *out) {
  if (Py < 1 || Px < 1 || ny % Py || nx % Px || iters < 0) return ORC_ERR_ARG;
  const int ly = ny / Py, lx = nx / Px, W = lx + 2;
  const int P = Py * Px;
  struct Rank {
    std::vector<float> buf[2];
    // flag[dir] written by the neighbour in direction dir (0 up,1 down,2 left,3 right)
    std::atomic<uint32_t> flag[4];
  };
  std::vector<Rank> R(P);
  auto at = [&](std::vector<float> &b, int i, int j) -> float & { return b[(size_t)(i + 1) * W + (j + 1)]; };
  for (int py = 0; py < Py; ++py)
    for (int px = 0; px < Px; ++px) {
      auto &rk = R[py * Px + px];
      for (int s = 0; s < 2; ++s) rk.buf[s].assign((size_t)(ly + 2) * W, 0.0f);
      for (int d = 0; d < 4; ++d) rk.flag[d].store(0);
      // initial data including halos from the global grid (iteration 0 halos)
      for (int i = -1; i <= ly; ++i)
        for (int j = -1; j <= lx; ++j) {
          const int gi = py * ly + i, gj = px * lx + j;
          if (gi < 0 || gi >= ny || gj < 0 || gj >= nx) continue;
          at(rk.buf[0], i, j) = a0[(size_t)gi * nx + gj];
          at(rk.buf[1], i, j) = a0[(size_t)gi * nx + gj];
        }
    }
  std::atomic<int> failed{0};
  std::vector<std::thread> th;
  for (int py = 0; py < Py; ++py)
    for (int px = 0; px < Px; ++px)
      th.emplace_back([&, py, px] {
        auto &me = R[py * Px + px];
        const int nb[4] = {py > 0 ? (py - 1) * Px + px : -1, py < Py - 1 ? (py + 1) * Px + px : -1,
                           px > 0 ? py * Px + px - 1 : -1, px < Px - 1 ? py * Px + px + 1 : -1};
        const int opposite[4] = {1, 0, 3, 2};
        for (int it = 0; it < iters; ++it) {
          auto &a = me.buf[it & 1];
          auto &b = me.buf[(it + 1) & 1];
          // Parrived: halos of `a` written by neighbours in iteration it-1
          for (int d = 0; d < 4; ++d)
            if (nb[d] >= 0 && it > 0 &&
                !spin_until([&] { return me.flag[d].load(std::memory_order_acquire) >= (uint32_t)it; }))
              failed = 1;
          for (int i = 0; i < ly; ++i)
            for (int j = 0; j < lx; ++j) {
              const int gi = py * ly + i, gj = px * lx + j;
              if (gi == 0 || gi == ny - 1 || gj == 0 || gj == nx - 1) {
                at(b, i, j) = at(a, i, j);  // Dirichlet: fixed
                continue;
              }
              at(b, i, j) = stencil(at(a, i - 1, j), at(a, i + 1, j), at(a, i, j - 1), at(a, i, j + 1));
            }
          // Pready: put edges into the neighbours' halos of `b`, then release
          for (int d = 0; d < 4; ++d) {
            if (nb[d] < 0) continue;
            auto &nbb = R[nb[d]].buf[(it + 1) & 1];
            if (d == 0) for (int j = 0; j < lx; ++j) at(nbb, ly, j) = at(b, 0, j);        // my top row -> up's bottom halo
            if (d == 1) for (int j = 0; j < lx; ++j) at(nbb, -1, j) = at(b, ly - 1, j);   // my bottom row -> down's top halo
            if (d == 2) for (int i = 0; i < ly; ++i) at(nbb, i, lx) = at(b, i, 0);        // my left col -> left's right halo
            if (d == 3) for (int i = 0; i < ly; ++i) at(nbb, i, -1) = at(b, i, lx - 1);   // my right col -> right's left halo
            R[nb[d]].flag[opposite[d]].store((uint32_t)it + 1, std::memory_order_release);
          }
        }
      });
  for (auto &t : th) t.join();
  for (int py = 0; py < Py; ++py)
    for (int px = 0; px < Px; ++px) {
      auto &rk = R[py * Px + px];
      auto &fin = rk.buf[iters & 1];
      for (int i = 0; i < ly; ++i)
        for (int j = 0; j < lx; ++j) out[(size_t)(py * ly + i) * nx + px * lx + j] = at(fin, i, j);
    }
  return failed ? ORC_ERR_TIMEOUT : ORC_OK;
}

}  // extern "C"
