// executor.cu — persistent sm_100a executor of an irregular, deadline-bounded
// streaming pipeline under enforced waiting (Plano & Buhler, SRMPDS '21).
//
// One CTA = one independent stream = one "processor" of PAPER.md §2.2 (L67).
// Node i of the linear pipeline (§2.1) is a warp group of v threads (one
// SIMD lane per item, L69).  Edges are smem ring queues that spill to an HBM
// ring when full.  Firing rules:
//   FIXED_WAIT       — node i fires at m*(t_i+w_i), taking <= v ready entries (§4)
//   THRESHOLD_SLACK  — an idle node fires when >= theta_i entries are ready or
//                      when the head item's slack a+D-R_i is reached (north_star)
//   MONOLITHIC       — separate kernel below (§5)
// The schedule is computed in logical time by a conservative parallel
// discrete-event protocol: node i may commit a firing at time T only once node
// i-1's watermark W_{i-1} (a lower bound on the ready time of anything it has not
// yet published) exceeds T, or once v entries with ready <= T are already queued.
// In the physical clock mode the same decisions are additionally paced against
// %globaltimer, so the real-time run replays the logical schedule and measures
// lateness / overruns instead of silently changing it.
#include <cuda_runtime.h>
#include <stdint.h>
#include "pl_internal.h"

namespace {

constexpr uint32_t LOC_SMEM = 0, LOC_SPILL = 1;
constexpr uint32_t NO_ROOT = 0xffffffffu;

__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void bar_sync(int id, int n) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}
template <class T>
__device__ __forceinline__ T vld(const T* p) { return *(const volatile T*)p; }
template <class T>
__device__ __forceinline__ void vst(T* p, T v) { *(volatile T*)p = v; }

__device__ __forceinline__ int64_t ceil_div64(int64_t a, int64_t b) { return a <= 0 ? 0 : (a + b - 1) / b; }

// ------------------------------------------------------------- counter-based RNG
// SplitMix64 finaliser; h = mix(seed ^ stage*GAMMA ^ root*M1 ^ lineage)  (DESIGN.md R-RNG)
__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t gain_hash(uint64_t seed, uint32_t stage, uint32_t root, uint32_t lin) {
  return splitmix64(seed ^ ((uint64_t)stage * 0x9E3779B97F4A7C15ull) ^ ((uint64_t)root * 0xBF58476D1CE4E5B9ull) ^
                    (uint64_t)lin);
}

// ------------------------------------------------------------------ DNA access
struct Dna {
  const uint32_t* db;
  uint32_t nwords;
  uint64_t db_len;
  const uint32_t* qw;      // query words (smem)
  const uint16_t* qoff;    // smem
  const uint16_t* qpos;    // smem
  int k, q_len;
  __device__ __forceinline__ uint32_t dbw(uint32_t w) const { return w < nwords ? __ldg(db + w) : 0u; }
  __device__ __forceinline__ uint32_t dbase(uint32_t j) const { return (dbw(j >> 4) >> ((j & 15) * 2)) & 3u; }
  __device__ __forceinline__ uint32_t qbase(uint32_t j) const { return (qw[j >> 4] >> ((j & 15) * 2)) & 3u; }
  // key(db, p) = sum_{j<k} db[p+j] 4^(k-1-j)  (first base most significant; R-S0)
  __device__ __forceinline__ uint32_t key(uint32_t p) const {
    uint64_t x = (((uint64_t)dbw((p >> 4) + 1) << 32) | dbw(p >> 4)) >> ((p & 15) * 2);
    uint32_t key = 0;
#pragma unroll 7
    for (int j = 0; j < PL_MAX_K; ++j)
      if (j < k) key = (key << 2) | (uint32_t)((x >> (2 * j)) & 3u);
    return key;
  }
  // best extension to the right of the seed (db[p+k-1+d] vs query[q+k-1+d]), d <= W
  // or X-drop (W < 0).  Returns best score (>= 0) and smallest d attaining it.
  __device__ __forceinline__ int ext_right(uint32_t p, uint32_t q, int W, int X, int* dbest) const {
    int score = 0, best = 0, db_ = 0;
    uint64_t i = (uint64_t)p + k, j = (uint64_t)q + k;   // first position right of the seed
    for (int d = 1;; ++d, ++i, ++j) {
      if (W >= 0 && d > W) break;
      if (i >= db_len || j >= (uint64_t)q_len) break;
      score += (dbase((uint32_t)i) == qbase((uint32_t)j)) ? 1 : -3;
      if (score > best) { best = score; db_ = d; }
      if (X > 0 && score <= best - X) break;
    }
    *dbest = db_;
    return best;
  }
  __device__ __forceinline__ int ext_left(uint32_t p, uint32_t q, int W, int X, int* dbest) const {
    int score = 0, best = 0, db_ = 0;
    for (int d = 1;; ++d) {
      if (W >= 0 && d > W) break;
      if ((uint32_t)d > p || (uint32_t)d > q) break;
      score += (dbase(p - d) == qbase(q - d)) ? 1 : -3;
      if (score > best) { best = score; db_ = d; }
      if (X > 0 && score <= best - X) break;
    }
    *dbest = db_;
    return best;
  }
};

// --------------------------------------------------------------- shared state
struct EdgeCtl {            // queue INTO node i
  uint32_t head;            // consumer: next sequence number to consume
  uint32_t seg_head;        // consumer: first live segment
  uint32_t seg_tail;        // producer: segments published
  uint32_t tail;            // producer: one past last published entry
  int64_t  W;               // producer watermark
  uint32_t spill_end;       // producer: end seq of the last spilled segment
  uint32_t pad;
};
struct GroupCtl {           // broadcast from a node's leader to its lanes
  int64_t  T;
  uint64_t end_ns_prev;     // physical: end time of the previous firing
  uint32_t n, head, done, segh, st, log_idx;
  uint32_t in_spill_end;    // input edge: end seq of its last spilled segment
  uint32_t out_base, out_loc;
  uint32_t wtot[8];
};
struct Shared {
  EdgeCtl e[PL_MAX_STAGES];
  GroupCtl g[PL_MAX_STAGES];
  unsigned long long max_lat;
  unsigned long long max_lat_ns;
  unsigned long long miss_events;
  uint32_t errors;
  uint32_t log_count;       // firing-log records reserved by all nodes of this stream
  uint64_t T0;
};

struct Ctx {
  const DevParams* p;
  Shared* sh;
  uint2* ent[PL_MAX_STAGES];   // smem rings (edge into node i)
  Seg* seg[PL_MAX_STAGES];
  uint2* spill[PL_MAX_STAGES]; // this stream's HBM rings
  Dna dna;
  uint64_t lo, hi;             // roots [lo, hi)
  int64_t X, H;
};

__device__ __forceinline__ int64_t arrival(const Ctx& c, uint32_t root) { return (int64_t)(root - c.lo) * c.p->tau; }

// location of sequence number s of edge i: spilled iff it lies in a spilled segment
__device__ __forceinline__ uint2 load_entry(const Ctx& c, int i, uint32_t s, uint32_t segh, uint32_t st,
                                            uint32_t spill_end) {
  const DevParams& p = *c.p;
  if ((int32_t)(s - spill_end) >= 0) return c.ent[i][s & (p.cap_s[i] - 1)];
  // binary search the live segments [segh, st) for the first with end > s
  uint32_t lo = segh, hi = st;
  while (lo < hi) {
    uint32_t mid = lo + ((hi - lo) >> 1);
    if ((int32_t)(c.seg[i][mid & (p.segcap - 1)].end - s) > 0) hi = mid; else lo = mid + 1;
  }
  if (c.seg[i][lo & (p.segcap - 1)].loc == LOC_SPILL) return __ldcg(c.spill[i] + (s & (p.cap_g - 1)));
  return c.ent[i][s & (p.cap_s[i] - 1)];
}

// ------------------------------------------------------------ stage functions
// Phase A: number of outputs of one input entry (and per-lane state for phase B).
struct LaneOut {
  uint32_t c;       // outputs
  uint32_t a, b;    // kind-specific state (S1: off; S3: db_start|len ...)
  int32_t score;
  uint32_t q_start, len;
};

__device__ __forceinline__ LaneOut stage_count(const Ctx& c, int i, uint2 e) {
  const DevParams& p = *c.p;
  const DevStage& s = p.st[i];
  LaneOut o;
  o.c = 0; o.a = 0; o.b = 0; o.score = 0; o.q_start = 0; o.len = 0;
  switch (s.kind) {
    case PL_BERNOULLI: o.c = gain_hash(p.seed, i, e.x, e.y) < s.thr[0] ? 1u : 0u; break;
    case PL_FIXED_GAIN: o.c = s.cfix; break;
    case PL_POISSON_CAPPED: {
      uint64_t h = gain_hash(p.seed, i, e.x, e.y);
      uint32_t n = 0;
      for (uint32_t k = 0; k < s.max_out; ++k) n += (h >= s.thr[k]) ? 1u : 0u;
      o.c = n;
      break;
    }
    case PL_KEEP_EVERY: o.c = (e.x % s.cfix) == 0 ? 1u : 0u; break;
    case PL_SEED_LOOKUP: {
      uint32_t key = c.dna.key(e.x);
      o.c = c.dna.qoff[key + 1] > c.dna.qoff[key] ? 1u : 0u;
      break;
    }
    case PL_HIT_ENUM: {
      uint32_t key = c.dna.key(e.x);
      uint32_t off = c.dna.qoff[key], cnt = c.dna.qoff[key + 1] - off;
      o.a = off;
      o.c = cnt < s.max_out ? cnt : s.max_out;
      break;
    }
    case PL_UNGAPPED_WINDOW: {
      uint32_t q = e.y & 0xffffu;
      int d;
      int bl = c.dna.ext_left(e.x, q, s.ip[1], 0, &d);
      int br = c.dna.ext_right(e.x, q, s.ip[1], 0, &d);
      o.c = (c.dna.k + bl + br >= s.ip[2]) ? 1u : 0u;
      break;
    }
    case PL_UNGAPPED_XDROP: {
      uint32_t q = e.y & 0xffffu;
      int dl, dr;
      int bl = c.dna.ext_left(e.x, q, -1, s.ip[1], &dl);
      int br = c.dna.ext_right(e.x, q, -1, s.ip[1], &dr);
      int score = c.dna.k + bl + br;
      if (score >= s.ip[2]) {
        o.c = 1;
        o.score = score;
        o.a = e.x - dl;
        o.q_start = q - dl;
        o.len = c.dna.k + dl + dr;
      }
      break;
    }
  }
  return o;
}

// Phase B: output j of an entry (non-sink nodes).
__device__ __forceinline__ uint2 stage_output(const Ctx& c, int i, uint2 e, const LaneOut& o, uint32_t j) {
  const DevStage& s = c.p->st[i];
  switch (s.kind) {
    case PL_FIXED_GAIN: return make_uint2(e.x, e.y * s.cfix + j);
    case PL_POISSON_CAPPED: return make_uint2(e.x, e.y * s.max_out + j);
    case PL_HIT_ENUM: return make_uint2(e.x, (uint32_t)c.dna.qpos[o.a + j] | (j << 16));
    default: return e;
  }
}

// ---------------------------------------------------------------- leader logic
struct Decision {
  bool done;
  int64_t T;
  uint32_t n;
};

struct Leader {   // leader-private schedule state of one node
  int64_t m;      // FIXED_WAIT: index of the next firing
  int64_t B;      // THRESHOLD_SLACK: busy until
  uint64_t c0;    // node 0: roots consumed
  uint32_t head, segh;      // consumer side of the input edge
  uint32_t out_tail, out_segt;  // producer side of the output edge
  int64_t W_pub;
  uint64_t empties;
  uint64_t sched_cycles;
};

__device__ __forceinline__ void publish_W(Ctx& c, int i, Leader& L, int64_t w) {
  if (i + 1 >= c.p->N) return;
  if (w > L.W_pub) {
    L.W_pub = w;
    __threadfence_block();
    vst(&c.sh->e[i + 1].W, w);
  }
}

__device__ __forceinline__ void backoff(int& spins) {
  if (spins < 4) { ++spins; return; }
  __nanosleep(spins < 64 ? 32 : 256);
  ++spins;
}

// number of entries of edge i with ready <= T among the published ones (stops at v)
__device__ __forceinline__ uint32_t count_le(const Ctx& c, int i, const Leader& L, uint32_t st, int64_t T,
                                             uint32_t v) {
  uint32_t end = L.head;
  for (uint32_t k = L.segh; k != st; ++k) {
    const Seg& sg = c.seg[i][k & (c.p->segcap - 1)];
    if (sg.ready > T) break;
    end = sg.end;
    if (end - L.head >= v) break;
  }
  return end - L.head;
}

__device__ Decision decide(Ctx& c, int i, Leader& L) {
  const DevParams& p = *c.p;
  const uint32_t v = (uint32_t)p.v;
  const int64_t t_i = p.t[i];
  Decision d;
  d.done = false; d.T = 0; d.n = 0;
  int spins = 0;
  const bool fixed = p.policy == PL_FIXED_WAIT;
  for (;;) {
    if (i == 0) {
      // arrivals are fully known: root lo+r arrives at r*tau0 (L63)
      const int64_t X = c.X;
      if ((int64_t)L.c0 >= X) { d.done = true; return d; }
      if (fixed) {
        const int64_t P = p.P[0];
        int64_t T = L.m * P;
        int64_t arrived = T / p.tau + 1; if (arrived > X) arrived = X;
        int64_t avail = arrived - (int64_t)L.c0;
        if (avail <= 0) {   // empty firings until the next root has arrived
          int64_t m2 = ceil_div64((int64_t)L.c0 * p.tau, P);
          L.empties += (uint64_t)(m2 - L.m);
          L.m = m2;
          continue;
        }
        d.T = T; d.n = (uint32_t)(avail < (int64_t)v ? avail : v);
        return d;
      } else {
        int64_t Tth = ((int64_t)L.c0 + p.theta[0] - 1 < X) ? ((int64_t)L.c0 + p.theta[0] - 1) * p.tau : PL_INF64;
        int64_t ah = (int64_t)L.c0 * p.tau;
        int64_t Tf = ah + p.D - p.R[0]; if (Tf < ah) Tf = ah;
        int64_t T = Tth < Tf ? Tth : Tf; if (T < L.B) T = L.B;
        int64_t arrived = T / p.tau + 1; if (arrived > X) arrived = X;
        int64_t avail = arrived - (int64_t)L.c0;
        d.T = T; d.n = (uint32_t)(avail < (int64_t)v ? avail : v);
        return d;
      }
    }
    // node i >= 1: read the upstream watermark first, then the published segments
    EdgeCtl& E = c.sh->e[i];
    const int64_t Wup = vld(&E.W);
    __threadfence_block();
    const uint32_t st = vld(&E.seg_tail);
    const uint32_t tail_known = (st != L.segh) ? c.seg[i][(st - 1) & (p.segcap - 1)].end : L.head;
    const bool any = tail_known != L.head;
    if (fixed) {
      const int64_t P = p.P[i];
      const int64_t T = L.m * P;
      uint32_t cnt = count_le(c, i, L, st, T, v);
      if (cnt >= v || Wup > T) {
        if (cnt > 0) { d.T = T; d.n = cnt < v ? cnt : v; return d; }
        if (!any && Wup == PL_INF64) { d.done = true; return d; }
        int64_t r = any ? c.seg[i][L.segh & (p.segcap - 1)].ready : Wup;
        int64_t m2 = ceil_div64(r, P);
        if (m2 < L.m + 1) m2 = L.m + 1;
        L.empties += (uint64_t)(m2 - L.m);
        L.m = m2;
        publish_W(c, i, L, L.m * P + t_i);
        spins = 0;
        continue;
      }
      publish_W(c, i, L, T + t_i);
      backoff(spins);
      continue;
    }
    // THRESHOLD_SLACK
    if (!any) {
      if (Wup == PL_INF64) { d.done = true; return d; }
      int64_t lb = Wup > L.B ? Wup : L.B;
      publish_W(c, i, L, lb + t_i);
      backoff(spins);
      continue;
    }
    const Seg& hs = c.seg[i][L.segh & (p.segcap - 1)];
    __threadfence_block();
    uint2 he = load_entry(c, i, L.head, L.segh, st, vld(&E.spill_end));
    int64_t Tf = arrival(c, he.x) + p.D - p.R[i];
    if (Tf < hs.ready) Tf = hs.ready;
    const uint32_t kth = L.head + p.theta[i] - 1;
    const bool th_known = (int32_t)(tail_known - kth) > 0;
    int64_t Tth = PL_INF64;
    if (th_known) {
      for (uint32_t k = L.segh; k != st; ++k) {
        const Seg& sg = c.seg[i][k & (p.segcap - 1)];
        if ((int32_t)(sg.end - kth) > 0) { Tth = sg.ready; break; }
      }
    }
    int64_t Tk = Tth < Tf ? Tth : Tf;
    if (Tk < L.B) Tk = L.B;
    if (th_known || Tk < Wup) {
      uint32_t cnt = count_le(c, i, L, st, Tk, v);
      if (Wup > Tk || cnt >= v) { d.T = Tk; d.n = cnt < v ? cnt : v; return d; }
    }
    int64_t lb = Tk < Wup ? Tk : Wup;
    if (lb < L.B) lb = L.B;
    publish_W(c, i, L, lb + t_i);
    backoff(spins);
  }
}

// reserve `total` entries on the output edge of node i; returns location or ~0u on overflow
__device__ uint32_t reserve_out(Ctx& c, int i, Leader& L, uint32_t total) {
  const DevParams& p = *c.p;
  EdgeCtl& E = c.sh->e[i + 1];
  int spins = 0;
  for (;;) {
    const uint32_t h = vld(&E.head), sh = vld(&E.seg_head);
    const bool seg_ok = (L.out_segt - sh) < p.segcap;
    const uint32_t need = L.out_tail + total - h;
    if (seg_ok && need <= p.cap_s[i + 1]) return LOC_SMEM;
    if (seg_ok && need <= p.cap_g) return LOC_SPILL;
    if (p.clock == PL_CLOCK_GLOBALTIMER) {
      atomicOr(&c.sh->errors, seg_ok ? PL_ERR_QUEUE_OVERFLOW : PL_ERR_SEG_OVERFLOW);
      return ~0u;
    }
    backoff(spins);   // logical mode: back-pressure (deadlock-free)
  }
}

__device__ __forceinline__ void pace(Ctx& c, int64_t T, uint64_t* start_ns, int64_t* late) {
  const uint64_t target = c.sh->T0 + (uint64_t)((double)T * c.p->ns_per_unit);
  uint64_t now = gtimer();
  while (now < target) {
    uint64_t rem = target - now;
    __nanosleep(rem > 2048 ? 1024 : (rem > 256 ? 128 : 0));
    now = gtimer();
  }
  *start_ns = now;
  *late = (int64_t)(now - target);
}


// exclusive scan of per-lane output counts over the node's v lanes (warp shuffles
// + one named barrier); returns the lane's offset and the group total.
__device__ __forceinline__ uint32_t group_scan(GroupCtl& G, uint32_t x, uint32_t* total, int gtid, int v, int bid) {
  const int lane = gtid & 31, w = gtid >> 5;
  uint32_t inc = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += y;
  }
  if (lane == 31) G.wtot[w] = inc;
  bar_sync(bid, v);                                                    // B2
  uint32_t pre = 0, tot = 0;
  for (int k = 0; k < (v >> 5); ++k) {
    uint32_t t = G.wtot[k];
    pre += (k < w) ? t : 0u;
    tot += t;
  }
  *total = tot;
  return pre + inc - x;
}

__device__ __forceinline__ int64_t overlap(int64_t s, int64_t e, int64_t lo, int64_t hi) {
  int64_t a = s > lo ? s : lo, b = e < hi ? e : hi;
  return b > a ? b - a : 0;
}

// ------------------------------------------------------------------- node loop
__device__ void run_node(Ctx& c, int i, int gtid) {
  const DevParams& p = *c.p;
  const int v = p.v, N = p.N;
  const bool leader = gtid == 0;
  const bool sink = i == N - 1;
  const int bid = 1 + i;
  const bool phys = p.clock == PL_CLOCK_GLOBALTIMER;
  const int64_t t_i = p.t[i];
  GroupCtl& G = c.sh->g[i];
  const uint32_t stream = blockIdx.x;
  const uint32_t rec = p.flags;

  Leader L;
  L.m = 0; L.B = 0; L.c0 = 0; L.head = 0; L.segh = 0; L.out_tail = 0; L.out_segt = 0;
  L.W_pub = -1; L.empties = 0; L.sched_cycles = 0;
  uint64_t firings = 0, consumed = 0, produced = 0, spilled = 0, overruns = 0;
  int64_t active = 0, busy_ns = 0, lateness = 0, t_end = 0;
  uint32_t n_log = 0;
  uint64_t start_ns = 0, end_ns_prev = 0;
  uint32_t pend_root = NO_ROOT;          // lane: physical terminal event awaiting its end time
  uint32_t out_loc = LOC_SMEM;

  for (;;) {
    if (leader) {
      long long c0 = clock64();
      Decision d = decide(c, i, L);
      L.sched_cycles += (uint64_t)(clock64() - c0);
      G.done = d.done ? 1u : 0u;
      G.T = d.T;
      G.n = d.n;
      G.head = (i == 0) ? (uint32_t)L.c0 : L.head;
      G.segh = L.segh;
      if (i > 0) {
        G.st = vld(&c.sh->e[i].seg_tail);
        __threadfence_block();
        G.in_spill_end = vld(&c.sh->e[i].spill_end);
      }
      G.end_ns_prev = end_ns_prev;
      if (!d.done && (rec & PL_REC_FIRINGS)) G.log_idx = atomicAdd(&c.sh->log_count, 1u);
      if (d.done) {
        publish_W(c, i, L, PL_INF64);
      } else if (phys) {
        int64_t late;
        pace(c, d.T, &start_ns, &late);
        if (late > lateness) lateness = late;
      }
    }
    bar_sync(bid, v);                                                  // B1: decision
    if (pend_root != NO_ROOT) {          // deferred physical latency of the previous firing
      const uint64_t a_ns = c.sh->T0 + (uint64_t)((double)arrival(c, pend_root) * p.ns_per_unit);
      const int64_t l = (int64_t)G.end_ns_prev - (int64_t)a_ns;
      if (rec & PL_REC_LATENCY) atomicMax((long long*)&p.lat_ns[pend_root], (long long)l);
      atomicMax(&c.sh->max_lat_ns, (unsigned long long)(l > 0 ? l : 0));
      pend_root = NO_ROOT;
    }
    if (G.done) break;
    const int64_t T = G.T;
    const uint32_t n = G.n, head = G.head;
    const bool act = (uint32_t)gtid < n;
    uint2 e = make_uint2(0u, 0u);
    if (act) {
      if (i == 0) e = make_uint2((uint32_t)(c.lo + head + gtid), 0u);
      else e = load_entry(c, i, head + gtid, G.segh, G.st, G.in_spill_end);
    }
    LaneOut o;
    if (act) o = stage_count(c, i, e);
    else { o.c = 0; o.a = 0; o.b = 0; o.score = 0; o.q_start = 0; o.len = 0; }
    uint32_t total;
    const uint32_t off = group_scan(G, o.c, &total, gtid, v, bid);   // B2 inside
    // --- per-item records: trace, terminal events (reading R-DONE)
    if (act) {
      if (rec & PL_REC_TRACE) {
        atomicAdd(&p.trace[(uint64_t)e.x * (N + 1) + i], 1u);
        if (sink && o.c) atomicAdd(&p.trace[(uint64_t)e.x * (N + 1) + N], o.c);
      }
      if (sink || o.c == 0) {
        const int64_t l = T + t_i - arrival(c, e.x);
        if (rec & PL_REC_LATENCY) atomicMax((long long*)&p.lat[e.x], (long long)l);
        atomicMax(&c.sh->max_lat, (unsigned long long)l);
        if (l > p.D) atomicAdd(&c.sh->miss_events, 1ull);
        if (phys) pend_root = e.x;
      }
      if ((rec & PL_REC_FIRINGS) && (gtid == 0 || (uint32_t)gtid == n - 1)) {
        const uint32_t li = G.log_idx;
        if (li < p.log_cap) {
          pl_firing* f = p.flog + (uint64_t)stream * p.log_cap + li;
          if (gtid == 0) { f->start = T; f->node = i; f->n = n; f->first_root = e.x; f->stream = stream; f->pad = 0; }
          if ((uint32_t)gtid == n - 1) f->last_root = e.x;
        } else if (gtid == 0) {
          atomicOr(&c.sh->errors, PL_ERR_LOG_OVERFLOW);
        }
      }
      if (sink && o.c && p.st[i].kind == PL_UNGAPPED_XDROP) {
        unsigned long long mi = atomicAdd(p.match_count, 1ull);
        if (mi < p.match_cap) {
          pl_match mt;
          mt.p = e.x; mt.q = e.y & 0xffffu; mt.db_start = o.a; mt.q_start = o.q_start;
          mt.len = o.len; mt.score = o.score;
          p.matches[mi] = mt;
        } else {
          atomicOr(&c.sh->errors, PL_ERR_MATCH_OVERFLOW);
        }
      }
    }
    // --- release the input slots (every lane has loaded its entry: B2 passed)
    if (leader) {
      if (i == 0) {
        L.c0 += n;
      } else {
        L.head = head + n;
        const uint32_t st = G.st;
        while (L.segh != st && (int32_t)(c.seg[i][L.segh & (p.segcap - 1)].end - L.head) <= 0) ++L.segh;
        __threadfence_block();
        vst(&c.sh->e[i].head, L.head);
        vst(&c.sh->e[i].seg_head, L.segh);
      }
    }
    // --- compaction into the next queue (stable: lane order, then child order)
    if (!sink && total > 0) {
      if (leader) {
        G.out_loc = reserve_out(c, i, L, total);
        G.out_base = L.out_tail;
      }
      bar_sync(bid, v);                                                // B3: output slot
      out_loc = G.out_loc;
      const uint32_t base = G.out_base;
      if (act && out_loc != ~0u) {
        for (uint32_t j = 0; j < o.c; ++j) {
          const uint32_t s = base + off + j;
          const uint2 val = stage_output(c, i, e, o, j);
          if (out_loc == LOC_SMEM) c.ent[i + 1][s & (p.cap_s[i + 1] - 1)] = val;
          else __stcg(c.spill[i + 1] + (s & (p.cap_g - 1)), val);
        }
      }
    }
    bar_sync(bid, v);                                                  // B4: outputs written
    if (leader) {
      if (phys) {
        const uint64_t en = gtimer();
        busy_ns += (int64_t)(en - start_ns);
        if ((double)(en - start_ns) > (double)t_i * p.ns_per_unit) ++overruns;
        end_ns_prev = en;
      }
      ++firings;
      consumed += n;
      produced += total;
      active += overlap(T, T + t_i, 0, c.H);
      if (T + t_i > t_end) t_end = T + t_i;
      if (rec & PL_REC_FIRINGS) ++n_log;
      if (!sink && total > 0 && out_loc != ~0u) {
        EdgeCtl& E = c.sh->e[i + 1];
        Seg sg;
        sg.ready = T + t_i;
        sg.end = L.out_tail + total;
        sg.loc = out_loc;
        c.seg[i + 1][L.out_segt & (p.segcap - 1)] = sg;
        if (out_loc == LOC_SPILL) { vst(&E.spill_end, sg.end); spilled += total; }
        __threadfence_block();
        ++L.out_segt;
        L.out_tail += total;
        vst(&E.seg_tail, L.out_segt);
        vst(&E.tail, L.out_tail);
      }
      if (p.policy == PL_FIXED_WAIT) {
        ++L.m;
        publish_W(c, i, L, L.m * p.P[i] + t_i);
      } else {
        L.B = T + t_i;
        publish_W(c, i, L, L.B + t_i);
      }
    }
  }
  if (leader) {
    CtaStats& S = p.stats[stream];
    S.firings[i] = firings;
    S.empty[i] = L.empties;
    S.consumed[i] = consumed;
    S.produced[i] = produced;
    S.active_ne[i] = active;
    S.busy_ns[i] = busy_ns;
    S.spilled[i] = spilled;
    S.overruns[i] = overruns;
    S.lateness[i] = lateness;
    S.sched_cycles[i] = L.sched_cycles;
    (void)n_log;
    atomicMax((long long*)&S.t_end, (long long)t_end);
  }
}

__host__ __device__ inline uint32_t layout_enforced(const DevParams& p, SmemLayout* L) {
  uint32_t off = 0;
  for (int i = 0; i < PL_MAX_STAGES; ++i) { L->off_ent[i] = 0; L->off_seg[i] = 0; }
  for (int i = 1; i < p.N; ++i) {
    L->off_ent[i] = off;
    off += p.cap_s[i] * 8u;
    L->off_seg[i] = off;
    off += p.segcap * (uint32_t)sizeof(Seg);
  }
  L->off_qoff = off;
  const bool dna = p.k > 0;
  off += dna ? (((1u << (2 * p.k)) + 1u) * 2u + 15u) & ~15u : 0u;
  L->off_qpos = off;
  off += dna ? (((uint32_t)(p.q_len - p.k + 1) * 2u) + 15u) & ~15u : 0u;
  L->off_qw = off;
  off += dna ? (((uint32_t)(p.q_len + 15) / 16u) * 4u + 15u) & ~15u : 0u;
  L->total = off;
  return off;
}

__device__ void cta_setup(Ctx& c, Shared& sh, unsigned char* dsm, const DevParams& p) {
  SmemLayout Lo;
  layout_enforced(p, &Lo);
  const uint32_t s = blockIdx.x, tid = threadIdx.x, nt = blockDim.x;
  c.p = &p;
  c.sh = &sh;
  c.lo = (p.total_roots * s) / (uint64_t)p.n_streams;
  c.hi = (p.total_roots * (s + 1)) / (uint64_t)p.n_streams;
  c.X = (int64_t)(c.hi - c.lo);
  c.H = c.X * p.tau;
  for (int i = 0; i < PL_MAX_STAGES; ++i) {
    c.ent[i] = (uint2*)(dsm + Lo.off_ent[i]);
    c.seg[i] = (Seg*)(dsm + Lo.off_seg[i]);
    c.spill[i] = p.spill ? p.spill + ((uint64_t)s * p.N + i) * p.cap_g : nullptr;
  }
  c.dna.db = p.db;
  c.dna.nwords = p.db_words;
  c.dna.db_len = p.db_len;
  c.dna.k = p.k;
  c.dna.q_len = p.q_len;
  c.dna.qoff = (const uint16_t*)(dsm + Lo.off_qoff);
  c.dna.qpos = (const uint16_t*)(dsm + Lo.off_qpos);
  c.dna.qw = (const uint32_t*)(dsm + Lo.off_qw);
  if (p.k > 0) {   // query index -> smem
    uint16_t* qo = (uint16_t*)(dsm + Lo.off_qoff);
    uint16_t* qp = (uint16_t*)(dsm + Lo.off_qpos);
    uint32_t* qw = (uint32_t*)(dsm + Lo.off_qw);
    const uint32_t nko = (1u << (2 * p.k)) + 1u, nqp = (uint32_t)(p.q_len - p.k + 1), nqw = (uint32_t)(p.q_len + 15) / 16u;
    for (uint32_t j = tid; j < nko; j += nt) qo[j] = p.qoff[j];
    for (uint32_t j = tid; j < nqp; j += nt) qp[j] = p.qpos[j];
    for (uint32_t j = tid; j < nqw; j += nt) qw[j] = p.qwords[j];
  }
  if (tid < PL_MAX_STAGES) {
    EdgeCtl& E = sh.e[tid];
    E.head = 0; E.seg_head = 0; E.seg_tail = 0; E.tail = 0; E.W = -1; E.spill_end = 0; E.pad = 0;
  }
  if (tid == 0) { sh.max_lat = 0; sh.max_lat_ns = 0; sh.miss_events = 0; sh.errors = 0; sh.log_count = 0; }
  // per-root records of this stream
  if (p.flags & PL_REC_LATENCY)
    for (uint64_t r = c.lo + tid; r < c.hi; r += nt) { p.lat[r] = -1; if (p.lat_ns) p.lat_ns[r] = -1; }
  if (p.flags & PL_REC_TRACE)
    for (uint64_t r = c.lo * (p.N + 1) + tid; r < c.hi * (p.N + 1); r += nt) p.trace[r] = 0u;
  if (tid == 0) {
    CtaStats& S = p.stats[s];
    S.n_log = 0;
    S.t_end = 0;
  }
}

__device__ void cta_finish(Ctx& c, Shared& sh, const DevParams& p) {
  if (threadIdx.x == 0) {
    CtaStats& S = p.stats[blockIdx.x];
    S.miss_events = sh.miss_events;
    S.max_lat = (int64_t)sh.max_lat;
    S.max_lat_ns = (int64_t)sh.max_lat_ns;
    S.wall_ns = (int64_t)(gtimer() - sh.T0);
    S.n_roots = (uint64_t)c.X;
    S.n_log = sh.log_count < p.log_cap ? sh.log_count : p.log_cap;
    S.errors = sh.errors;
  }
}


// block-wide exclusive scan (all threads of the CTA), two __syncthreads
__device__ __forceinline__ uint32_t block_scan(uint32_t x, uint32_t* total, uint32_t* wt) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  uint32_t inc = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += y;
  }
  if (lane == 31) wt[w] = inc;
  __syncthreads();
  uint32_t pre = 0, tot = 0;
  for (int k = 0; k < nw; ++k) {
    uint32_t t = wt[k];
    pre += (k < w) ? t : 0u;
    tot += t;
  }
  *total = tot;
  __syncthreads();
  return pre + inc - x;
}

// MONOLITHIC (§5; reading R-MONO): blocks of M consecutive
// arrivals, ready at the arrival of their last item, served FIFO; for a block node
// i fires ceil(n_i/v) times back to back (logical accounting), the CTA's threads
// processing the block's vectors together (the no-internal-wait throughput form).
__device__ void run_monolithic(Ctx& c) {
  const DevParams& p = *c.p;
  const int N = p.N, v = p.v;
  const uint32_t tid = threadIdx.x, nt = blockDim.x, stream = blockIdx.x;
  const bool phys = p.clock == PL_CLOCK_GLOBALTIMER;
  const uint32_t rec = p.flags;
  __shared__ uint32_t wt[32];
  __shared__ uint64_t sh_start_ns;
  uint2* buf0 = p.mono_buf + (uint64_t)stream * 2u * p.mono_cap;
  uint2* buf1 = buf0 + p.mono_cap;
  uint64_t firings[PL_MAX_STAGES], consumed[PL_MAX_STAGES], produced[PL_MAX_STAGES];
  int64_t active[PL_MAX_STAGES];
  for (int i = 0; i < PL_MAX_STAGES; ++i) { firings[i] = consumed[i] = produced[i] = 0; active[i] = 0; }
  int64_t proc_free = 0, t_end = 0, busy_ns = 0, lateness = 0;
  const int64_t M = p.M;
  for (int64_t b0 = 0; b0 < c.X; b0 += M) {
    const int64_t b1 = (b0 + M < c.X) ? b0 + M : c.X;
    const int64_t ready = (b1 - 1) * p.tau;
    int64_t T = ready > proc_free ? ready : proc_free;
    if (phys) {
      if (tid == 0) {
        uint64_t s_ns; int64_t late;
        pace(c, ready, &s_ns, &late);      // the block is complete in real time
        sh_start_ns = s_ns;
      }
      __syncthreads();
    }
    uint2* cur = buf0;
    uint2* nxt = buf1;
    uint32_t ncur = (uint32_t)(b1 - b0);
    for (int i = 0; i < N && ncur > 0; ++i) {
      const bool sink = i == N - 1;
      const int64_t t_i = p.t[i];
      const uint32_t nf = (ncur + v - 1) / v;
      uint32_t nxt_count = 0;
      for (uint32_t base = 0; base < ncur; base += nt) {
        const uint32_t idx = base + tid;
        const bool act = idx < ncur;
        uint2 e = make_uint2(0u, 0u);
        if (act) e = (i == 0) ? make_uint2((uint32_t)(c.lo + b0 + idx), 0u) : cur[idx];
        LaneOut o;
        if (act) o = stage_count(c, i, e);
        else { o.c = 0; o.a = 0; o.b = 0; o.score = 0; o.q_start = 0; o.len = 0; }
        uint32_t total;
        const uint32_t off = block_scan(o.c, &total, wt);
        if (act) {
          const uint32_t f = idx / (uint32_t)v;
          const int64_t end = T + (int64_t)(f + 1) * t_i;
          if (rec & PL_REC_TRACE) {
            atomicAdd(&p.trace[(uint64_t)e.x * (N + 1) + i], 1u);
            if (sink && o.c) atomicAdd(&p.trace[(uint64_t)e.x * (N + 1) + N], o.c);
          }
          if (sink || o.c == 0) {
            const int64_t l = end - arrival(c, e.x);
            if (rec & PL_REC_LATENCY) atomicMax((long long*)&p.lat[e.x], (long long)l);
            atomicMax(&c.sh->max_lat, (unsigned long long)l);
            if (l > p.D) atomicAdd(&c.sh->miss_events, 1ull);
            if (phys) {
              const uint64_t a_ns = c.sh->T0 + (uint64_t)((double)arrival(c, e.x) * p.ns_per_unit);
              const int64_t ln = (int64_t)gtimer() - (int64_t)a_ns;
              if (rec & PL_REC_LATENCY) atomicMax((long long*)&p.lat_ns[e.x], (long long)ln);
              atomicMax(&c.sh->max_lat_ns, (unsigned long long)(ln > 0 ? ln : 0));
            }
          }
          if ((rec & PL_REC_FIRINGS) && (idx % (uint32_t)v == 0 || idx == ncur - 1 || idx % (uint32_t)v == (uint32_t)v - 1)) {
            // record of firing f: first lane writes the header, last lane the last root
            const uint32_t li = c.sh->log_count + f;
            if (li < p.log_cap) {
              pl_firing* fr = p.flog + (uint64_t)stream * p.log_cap + li;
              if (idx % (uint32_t)v == 0) {
                fr->start = T + (int64_t)f * t_i; fr->node = i;
                fr->n = (ncur - f * v) < (uint32_t)v ? (ncur - f * v) : (uint32_t)v;
                fr->first_root = e.x; fr->stream = stream; fr->pad = 0;
              }
              if (idx == ncur - 1 || idx % (uint32_t)v == (uint32_t)v - 1) fr->last_root = e.x;
            } else {
              atomicOr(&c.sh->errors, PL_ERR_LOG_OVERFLOW);
            }
          }
          if (sink && o.c && p.st[i].kind == PL_UNGAPPED_XDROP) {
            unsigned long long mi = atomicAdd(p.match_count, 1ull);
            if (mi < p.match_cap) {
              pl_match mt;
              mt.p = e.x; mt.q = e.y & 0xffffu; mt.db_start = o.a; mt.q_start = o.q_start;
              mt.len = o.len; mt.score = o.score;
              p.matches[mi] = mt;
            } else {
              atomicOr(&c.sh->errors, PL_ERR_MATCH_OVERFLOW);
            }
          }
          if (!sink) {
            for (uint32_t j = 0; j < o.c; ++j) {
              const uint32_t s = nxt_count + off + j;
              if (s < p.mono_cap) nxt[s] = stage_output(c, i, e, o, j);
              else atomicOr(&c.sh->errors, PL_ERR_QUEUE_OVERFLOW);
            }
          }
        }
        nxt_count += total;
        produced[i] += total;
      }
      __syncthreads();   // nxt complete; firing-log slots consumed
      if (tid == 0 && (rec & PL_REC_FIRINGS)) c.sh->log_count += nf;
      firings[i] += nf;
      consumed[i] += ncur;
      for (uint32_t f = 0; f < nf; ++f) active[i] += overlap(T + (int64_t)f * t_i, T + (int64_t)(f + 1) * t_i, 0, c.H);
      T += (int64_t)nf * t_i;
      t_end = T;
      uint2* tmp = cur; cur = nxt; nxt = tmp;
      ncur = nxt_count < p.mono_cap ? nxt_count : p.mono_cap;
      __syncthreads();
    }
    proc_free = T;
    if (phys && tid == 0) {
      const uint64_t en = gtimer();
      busy_ns += (int64_t)(en - sh_start_ns);
      (void)lateness;
    }
  }
  if (tid == 0) {
    CtaStats& S = p.stats[stream];
    for (int i = 0; i < PL_MAX_STAGES; ++i) {
      S.firings[i] = firings[i]; S.empty[i] = 0; S.consumed[i] = consumed[i]; S.produced[i] = produced[i];
      S.active_ne[i] = active[i]; S.busy_ns[i] = i == 0 ? busy_ns : 0; S.spilled[i] = 0; S.overruns[i] = 0;
      S.lateness[i] = 0; S.sched_cycles[i] = 0;
    }
    S.t_end = t_end;
  }
}

}  // namespace

// FIXED_WAIT / THRESHOLD_SLACK executor: grid = n_streams, block = N*v threads.
extern "C" __global__ void __launch_bounds__(1024, 1) pl_exec_enforced(const __grid_constant__ DevParams p) {
  extern __shared__ __align__(16) unsigned char dsm[];
  __shared__ Shared sh;
  Ctx c;
  cta_setup(c, sh, dsm, p);
  __syncthreads();
  if (threadIdx.x == 0) sh.T0 = gtimer();
  __syncthreads();
  const int gi = threadIdx.x / p.v;
  if (gi < p.N) run_node(c, gi, threadIdx.x % p.v);
  __syncthreads();
  cta_finish(c, sh, p);
}

uint32_t pl_layout_enforced_host(const DevParams& p) {
  SmemLayout L;
  return layout_enforced(p, &L);
}

// MONOLITHIC executor: grid = n_streams, block = any multiple of 32 (N*v by default).
extern "C" __global__ void __launch_bounds__(1024, 1) pl_exec_monolithic(const __grid_constant__ DevParams p) {
  extern __shared__ __align__(16) unsigned char dsm[];
  __shared__ Shared sh;
  Ctx c;
  cta_setup(c, sh, dsm, p);
  __syncthreads();
  if (threadIdx.x == 0) sh.T0 = gtimer();
  __syncthreads();
  run_monolithic(c);
  __syncthreads();
  cta_finish(c, sh, p);
}
