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
#include <stdio.h>
#include "pl_internal.h"

namespace {

constexpr uint32_t LOC_SMEM = 0, LOC_SPILL = 1;
constexpr uint32_t NO_ROOT = 0xffffffffu;

__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Named barriers (.aligned bar.sync: every warp reaches them converged -- the node loop
// reconverges its warps after the leader's and the accountant's single-lane work, __syncwarp).
// The non-.aligned barrier.sync was measured: node 1-3 firings 1.75x slower.
__device__ __forceinline__ void bar_sync(int id, int n) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}
template <class T>
__device__ __forceinline__ T vld(const T* p) { return *(const volatile T*)p; }
template <class T>
__device__ __forceinline__ void vst(T* p, T v) { *(volatile T*)p = v; }
// CTA-scope acquire-release fence between the data and the flag of the SPSC queues (pure
// message passing, so no sequentially consistent fence is needed): MEMBAR.ALL.CTA in SASS,
// where __threadfence_block() emits the costlier MEMBAR.SC.CTA.
__device__ __forceinline__ void fence_cta() { asm volatile("fence.acq_rel.cta;" ::: "memory"); }
// queue fences: CTA scope, or cluster scope when the nodes are the CTAs of a cluster (N4)
__device__ __forceinline__ void fence_q(bool cl) {
  if (cl) asm volatile("fence.acq_rel.cluster;" ::: "memory");
  else asm volatile("fence.acq_rel.cta;" ::: "memory");
}


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
// The DB is read through a per-stream smem window with an __ldg fallback outside it.  The
// window is a ring of win_cap words (word w at slot w & win_mask) refilled chunk by chunk by
// TMA bulk copies as the stream advances (win_step); [win_lo,
// win_lo + win_n) is this thread's snapshot of the words it holds.  Extensions compare 16
// bases per step: XOR of two 2-bit-packed 32-bit windows gives a mismatch mask.
// experiment switches (tools/build_variant.py -D...; defaults = the product build)
#ifndef PL_WINSTEP_NOINLINE
#define PL_WINSTEP_NOINLINE 0   // out of line, the call inside the accountant's divergent branch leaves its warp diverged at the next scan barrier (synccheck)
#endif
#ifndef PL_LIVE_GATE
#define PL_LIVE_GATE 1
#endif
#ifndef PL_WATCHDOG
#define PL_WATCHDOG 1
#endif
#ifndef PL_S3_PREFETCH
#define PL_S3_PREFETCH 0    // X-drop walks load the next step's words one step ahead (experiment)
#endif
#ifndef PL_SINK_SPREAD
#define PL_SINK_SPREAD 0    // the sink's items dealt round-robin over its warps: c4 node-3 mean firing -6 %, but c2's longest
                            // node-3 firing +30 % (every warp then iterates the longest walk): rejected
#endif
#ifndef PL_NAP_SHIFT
#define PL_NAP_SHIFT 1      // long naps sleep half the remaining time (__nanosleep: at most 2x): -9 % instructions on c4
#endif
#ifndef PL_NAP_HALF
#define PL_NAP_HALF 1       // every nap above the spin threshold sleeps half the remaining time (no 256 / 64 ns tiers):
                            // c3 THRESHOLD_SLACK -9 to -11 % warp instructions per root, c4 budgets and rate unchanged or better
#endif
#ifndef PL_S3_TAB
#define PL_S3_TAB 1         // S3 X-drop walks 8 steps per table lookup ([deficit][mismatch byte] transitions in smem):
                            // K-BENCH S3 2.54 -> 1.27 ms, c4 node-3 longest probe firing 16.4 -> 10.5 us, bit-exact
#endif
#ifndef PL_S3_TAB2
#define PL_S3_TAB2 0        // experiment: the left and right table walks advanced together (two chains per lane);
                            // bit-exact but node 3's longest c4 probe firing 10.6 -> 17.9 us, bench 4.9e7: rejected
#endif
#ifndef PL_PUB_WAIT
#define PL_PUB_WAIT 0       // physical clock: a waiting leader sleeps on its input edge's mbarrier (woken by the
                            // producer's publication or the nap's time limit) instead of a plain nap; parity-exact
                            // (110 physical/live/window tests) but no fewer instructions at the c3 points
                            // (37.2 vs 37.0 per root) and the c4 edge no faster: rejected (profiles/r02_ab/pub_wait.txt)
#endif
#ifndef PL_PHYS_SPINS
#define PL_PHYS_SPINS 2     // physical-clock polls before the first backoff nap
#endif
#ifndef PL_DBMASK
#define PL_DBMASK 1
#endif
#ifndef PL_INJECT
#define PL_INJECT 1
#endif
#ifndef PL_S3_COOP
#define PL_S3_COOP 0        // S3 X-drop: serial rounds, then a warp-cooperative finisher for the last long walks;
                            // bit-exact, but c4 node-3 longest firing x2 (17.5 -> 36 us) and nodes 0-2 +10-20 %: rejected
#endif
#ifndef PL_S3_SB
#define PL_S3_SB 8          // serial 16-base steps per round of the hybrid walk
#endif
#ifndef PL_S3_COOPMAX
#define PL_S3_COOPMAX 4     // unfinished lanes the cooperative finisher takes over
#endif
#ifndef PL_S3_MSB
#define PL_S3_MSB 1
#endif
#ifndef PL_S3_DEBUG
#define PL_S3_DEBUG 0
#endif

struct Dna {
  const uint32_t* db;      // packed DB (global); live ingest: this stream's device ring (word w at db[w & dbmask])
  uint32_t dbmask;         // ~0u, or the live ring's size - 1: then L2-only loads (__ldcg) -- the copy
                           // engine rewrites the ring's slots and L1 is not coherent with it
  uint32_t nwords;
  uint64_t db_len;
  const uint32_t* win;     // smem ring of DB words: word w at win[w & win_mask], valid for [win_lo, win_lo + win_n)
  int64_t win_lo;
  uint32_t win_lo32;        // (uint32_t)win_lo: window word index arithmetic in 32 bits
  uint32_t win_n;
  uint32_t win_mask;
  bool nofast;             // experiment switch (PL_VARIANT & 16): always the checked walk
  const uint8_t* s2tab;    // smem: max(0, max prefix score) of an 8-step walk by mismatch pattern
  const uint16_t* xtab;    // smem (PL_S3_TAB): 8-step X-drop transitions [deficit][mismatch byte] (xdrop_tab_entry)
  int xtab_X;              // the X the table was built for (0: no table)
  const uint32_t* qw;      // query words (smem), nqw valid words
  uint32_t nqw;
  const uint16_t* qoff;    // smem
  const uint16_t* qpos;    // smem
  int k, q_len;
  __device__ __forceinline__ uint32_t dbw(int64_t w) const {
    const uint64_t r = (uint64_t)(w - win_lo);
    if (r < win_n) return win[(uint32_t)w & win_mask];
    if (!(w >= 0 && w < (int64_t)nwords)) return 0u;
#if PL_DBMASK
    return dbmask == 0xffffffffu ? __ldg(db + w) : __ldcg(db + ((uint32_t)w & dbmask));
#else
    return __ldg(db + w);   // experiment: the live ring's mask compiled out
#endif
  }
  __device__ __forceinline__ uint32_t qww(int64_t w) const { return (w >= 0 && w < (int64_t)nqw) ? qw[w] : 0u; }
  // bases s..s+15 (base s in bits 0-1); s may be negative (out-of-range bases read as 0)
  __device__ __forceinline__ uint32_t db16(int64_t s) const {
    const int64_t w = s >> 4;
    return __funnelshift_r(dbw(w), dbw(w + 1), (uint32_t)(s & 15) * 2u);
  }
  __device__ __forceinline__ uint32_t q16(int64_t s) const {
    const int64_t w = s >> 4;
    return __funnelshift_r(qww(w), qww(w + 1), (uint32_t)(s & 15) * 2u);
  }
  // key(db, p) = sum_{j<k} db[p+j] 4^(k-1-j)  (first base most significant; R-S0):
  // reverse the order of the 2-bit fields of the window (bit-reverse, then swap each pair)
  __device__ __forceinline__ uint32_t kmer_of(uint32_t x) const {
    const uint32_t r = __brev(x);
    const uint32_t pr = ((r >> 1) & 0x55555555u) | ((r & 0x55555555u) << 1);
    return pr >> (32 - 2 * k);
  }
  __device__ __forceinline__ uint32_t key(uint32_t p) const { return kmer_of(db16(p)); }
  // Walk d = 1..limit away from the seed scoring +1/-3 (R-S2/R-S3); stop early on
  // X-drop (X > 0: score <= best - X).  Returns best (>= 0) and the smallest d
  // attaining it.  dir = +1: db[p+k-1+d] vs query[q+k-1+d]; dir = -1: db[p-d] vs query[q-d].
  __device__ __forceinline__ int extend(uint32_t p, uint32_t q, int dir, int64_t limit, int X, int* dbest) const {
    int score = 0, best = 0, db_ = 0;
    int64_t d = 0;
    while (d < limit) {
      const int64_t n = (limit - d) < 16 ? (limit - d) : 16;
      uint32_t mm;   // bit 2e set <=> mismatch at step d+1+e
      if (dir > 0) {
        const uint32_t x = db16((int64_t)p + k + d) ^ q16((int64_t)q + k + d);
        mm = (x | (x >> 1)) & 0x55555555u;
      } else {
        // window ending at p-d-1: step d+1+e is window position 15-e -> bit-reverse the pairs
        const uint32_t x = db16((int64_t)p - d - 16) ^ q16((int64_t)q - d - 16);
        mm = __brev((x | (x >> 1)) & 0x55555555u) >> 1;
      }
      // Between mismatches the score rises by 1 per step, so the running best can
      // only be set just before a mismatch (or at the chunk end) and an x-drop can
      // only happen just after one: visit the mismatch steps only.
      uint32_t mmv = mm & (n >= 16 ? 0xffffffffu : ((1u << (2 * n)) - 1u));
      int last = 0;                      // steps of this chunk already scored
      while (mmv) {
        const int e = (__ffs(mmv) - 1) >> 1;   // mismatch at step d+1+e
        mmv &= mmv - 1;
        score += e - last;               // matches at steps last+1 .. e (1-based within chunk)
        if (score > best) { best = score; db_ = (int)(d + e); }
        score -= 3;
        last = e + 1;
        if (X > 0 && score <= best - X) { *dbest = db_; return best; }
      }
      score += (int)n - last;
      if (score > best) { best = score; db_ = (int)(d + n); }
      d += n;
    }
    *dbest = db_;
    return best;
  }
  // Fast form of extend() for both walks of one seed whose DB words all lie in the smem
  // window (in_win): the left walk (ll steps), then the right walk (rl steps), in ONE loop,
  // so that a warp iterates max over lanes of (left + right) 16-base steps rather than
  // max(left) + max(right) (seeds on one planted diagonal split it at different points).
  // 32-bit indices, no per-word range checks, one new DB word and one new query word per
  // step (the shift is the same for every step of a walk).  The query copy in smem carries
  // zero pad words on both sides (layout_enforced), so reads past either end are in bounds;
  // bases past a walk's limit are masked as in extend().  Scoring and X-drop as extend().
  __device__ __forceinline__ void extend2_win(uint32_t p, uint32_t q, uint32_t ll, uint32_t rl, int X, int* bl,
                                              int* dl, int* br, int* dr) const {
    // left walk: step d+1+e compares db[p-d-1-e] with query[q-d-1-e]; its first 16-base
    // window is [p-16, p) = words (w, w+1), w = (p-16)>>4; later windows slide down a word
    int32_t sd = (int32_t)p - 16, sq = (int32_t)q - 16;
    uint32_t dw = (uint32_t)(sd >> 4);                                // next DB word to load (ring index)
    const uint32_t* qp = qw + (sq >> 4);
    uint32_t shd = (uint32_t)(sd & 15) * 2u, shq = (uint32_t)(sq & 15) * 2u;
    uint32_t dc = win[(dw + 1u) & win_mask], qc = qp[1];              // carried word
#if PL_S3_PREFETCH
    // the next step's words are loaded one step ahead, off the mismatch loop's dependency chain
    // (one word past a walk's end at most: the ring index is masked, the query is padded)
    uint32_t dnx = win[dw & win_mask], qnx = *qp;
#endif
    int step = -1;
    bool right = false;
    uint32_t limit = ll, d = 0;
    int score = 0, best = 0, db_ = 0;
    for (;;) {
      bool fin = d >= limit;
      if (!fin) {
#if PL_S3_PREFETCH
        const uint32_t dn = dnx, qn = qnx;
        dw += (uint32_t)step;
        qp += step;
        dnx = win[dw & win_mask];
        qnx = *qp;
#else
        const uint32_t dn = win[dw & win_mask], qn = *qp;
        dw += (uint32_t)step;
        qp += step;
#endif
        const uint32_t x = right ? (__funnelshift_r(dc, dn, shd) ^ __funnelshift_r(qc, qn, shq))
                                 : (__funnelshift_r(dn, dc, shd) ^ __funnelshift_r(qn, qc, shq));
        dc = dn;
        qc = qn;
        const uint32_t n = (limit - d) < 16u ? (limit - d) : 16u;
#if PL_S3_MSB
        // step-ordered from the most significant bit: step d+1+e owns bit 31-2e or 30-2e, so
        // the next mismatch is e = clz >> 1 (one FLO per mismatch, where __ffs is BREV + FLO
        // on the per-mismatch dependency chain) and it is cleared with everything above it.
        // Left: window position 15-e is step d+1+e, already MSB-first; right: one BREV per word.
        uint32_t mm = (x | (x >> 1)) & 0x55555555u;
        if (right) mm = __brev(mm);
        uint32_t mmv = mm & (0xffffffffu << (32u - 2u * n));   // n >= 1: steps e < n
        int last = 0;
        while (mmv) {
          const uint32_t c = __clz(mmv);
          const int e = (int)(c >> 1);
          mmv &= 0x7fffffffu >> c;
          score += e - last;
#else
        uint32_t mm = (x | (x >> 1)) & 0x55555555u;   // bit 2e set <=> mismatch at step d+1+e
        if (!right) mm = __brev(mm) >> 1;             // left: window position 15-e is step d+1+e
        uint32_t mmv = mm & (n >= 16u ? 0xffffffffu : ((1u << (2u * n)) - 1u));
        int last = 0;
        while (mmv) {
          const int e = (__ffs(mmv) - 1) >> 1;
          mmv &= mmv - 1;
          score += e - last;
#endif
          if (score > best) { best = score; db_ = (int)d + e; }
          score -= 3;
          last = e + 1;
          if (X > 0 && score <= best - X) { fin = true; break; }
        }
        if (!fin) {
          score += (int)n - last;
          if (score > best) { best = score; db_ = (int)(d + n); }
          d += n;
        }
      }
      if (fin) {
        if (right) break;
        *bl = best;
        *dl = db_;
        // right walk: step d+1+e compares db[p+k+d+e] with query[q+k+d+e]; first window
        // [p+k, p+k+16) = words (w, w+1), w = (p+k)>>4; later windows slide up a word
        right = true;
        step = 1;
        limit = rl;
        d = 0;
        score = best = db_ = 0;
        sd = (int32_t)(p + (uint32_t)k);
        sq = (int32_t)(q + (uint32_t)k);
        dw = (uint32_t)(sd >> 4);
        qp = qw + (sq >> 4);
        shd = (uint32_t)(sd & 15) * 2u;
        shq = (uint32_t)(sq & 15) * 2u;
        dc = win[dw++ & win_mask];
        qc = *qp++;
#if PL_S3_PREFETCH
        dnx = win[dw & win_mask];
        qnx = *qp;
#endif
      }
    }
    *br = best;
    *dr = db_;
  }
  // PL_S3_TAB: one 8-step chunk of an X-drop walk (+1 match / -3 mismatch, R-S3) entered with the
  // running best `def` above the score: bit e of m = mismatch at the chunk's step e + 1.  Entry:
  // bits 0-3 the best's rise (0..8), 4-7 the chunk step where the new best is first reached,
  // 8-13 the deficit after the chunk, bit 14 = the walk X-drops inside the chunk (score <= best - X
  // right after a mismatch; the best at that point is the walk's result).  Exactly extend()'s
  // arithmetic, 8 steps at a time.
  static __host__ __device__ __forceinline__ uint16_t xdrop_tab_entry(uint32_t def, uint32_t m, int X) {
    int s = -(int)def, b = 0, bpos = 0;
    for (int e = 0; e < 8; ++e) {
      if ((m >> e) & 1u) {
        s -= 3;
        if (s <= b - X) return (uint16_t)(b | (bpos << 4) | (1 << 14));
      } else {
        s += 1;
        if (s > b) { b = s; bpos = e + 1; }
      }
    }
    return (uint16_t)(b | (bpos << 4) | ((b - s) << 8));
  }
  // extend2_win with the mismatch loop replaced by two table steps per 16-base word: the word's
  // mismatch mask is compressed to 16 bits (bit j = step d+1+j), steps past the walk's limit are
  // marked as mismatches (they never raise the best, and a drop among them ends the walk where
  // the limit would), and each byte is one lookup.  Needs xtab_X == X (1..63) and in_win.
  __device__ __forceinline__ void extend2_tab(uint32_t p, uint32_t q, uint32_t ll, uint32_t rl, int* bl,
                                              int* dl, int* br, int* dr) const {
    int32_t sd = (int32_t)p - 16, sq = (int32_t)q - 16;
    uint32_t dw = (uint32_t)(sd >> 4);
    const uint32_t* qp = qw + (sq >> 4);
    uint32_t shd = (uint32_t)(sd & 15) * 2u, shq = (uint32_t)(sq & 15) * 2u;
    uint32_t dc = win[(dw + 1u) & win_mask], qc = qp[1];
    int step = -1;
    bool right = false;
    uint32_t limit = ll, d = 0, def = 0;
    int best = 0, db_ = 0;
    for (;;) {
      bool fin = d >= limit;
      if (!fin) {
        const uint32_t dn = win[dw & win_mask], qn = *qp;
        dw += (uint32_t)step;
        qp += step;
        const uint32_t x = right ? (__funnelshift_r(dc, dn, shd) ^ __funnelshift_r(qc, qn, shq))
                                 : (__funnelshift_r(dn, dc, shd) ^ __funnelshift_r(qn, qc, shq));
        dc = dn;
        qc = qn;
        uint32_t mm = (x | (x >> 1)) & 0x55555555u;   // bit 2e: mismatch at window position e
        if (!right) mm = __brev(mm) >> 1;             // left: window position 15-e is step d+1+e
        mm = (mm | (mm >> 1)) & 0x33333333u;
        mm = (mm | (mm >> 2)) & 0x0f0f0f0fu;
        mm = (mm | (mm >> 4)) & 0x00ff00ffu;
        mm = (mm | (mm >> 8)) & 0x0000ffffu;          // bit j: mismatch at step d+1+j
        const uint32_t n = (limit - d) < 16u ? (limit - d) : 16u;
        mm |= (0xffffu << n) & 0xffffu;
        uint32_t t = xtab[(def << 8) | (mm & 0xffu)];
        if (t & 15u) { best += (int)(t & 15u); db_ = (int)d + (int)((t >> 4) & 15u); }
        if (t & 0x4000u) fin = true;
        else {
          def = (t >> 8) & 63u;
          t = xtab[(def << 8) | (mm >> 8)];
          if (t & 15u) { best += (int)(t & 15u); db_ = (int)d + 8 + (int)((t >> 4) & 15u); }
          if (t & 0x4000u) fin = true;
          else { def = (t >> 8) & 63u; d += n; }
        }
      }
      if (fin) {
        if (right) break;
        *bl = best;
        *dl = db_;
        right = true;
        step = 1;
        limit = rl;
        d = 0;
        def = 0;
        best = db_ = 0;
        sd = (int32_t)(p + (uint32_t)k);
        sq = (int32_t)(q + (uint32_t)k);
        dw = (uint32_t)(sd >> 4);
        qp = qw + (sq >> 4);
        shd = (uint32_t)(sd & 15) * 2u;
        shq = (uint32_t)(sq & 15) * 2u;
        dc = win[dw++ & win_mask];
        qc = *qp++;
      }
    }
    *br = best;
    *dr = db_;
  }
#if PL_S3_TAB2
  // PL_S3_TAB2 (experiment): extend2_tab with the left and right walks advanced together, one word
  // of each per iteration -- two independent table chains per lane instead of one after the other
  struct TWalk {
    uint32_t dw, shd, shq, dc, qc, limit, d, def;
    const uint32_t* qp;
    int best, db_;
    bool fin;
  };
  __device__ __forceinline__ void tw_step(TWalk& w, bool right) const {
    const uint32_t dn = win[w.dw & win_mask], qn = *w.qp;
    w.dw += right ? 1u : 0xffffffffu;
    w.qp += right ? 1 : -1;
    const uint32_t x = right ? (__funnelshift_r(w.dc, dn, w.shd) ^ __funnelshift_r(w.qc, qn, w.shq))
                             : (__funnelshift_r(dn, w.dc, w.shd) ^ __funnelshift_r(qn, w.qc, w.shq));
    w.dc = dn;
    w.qc = qn;
    uint32_t mm = (x | (x >> 1)) & 0x55555555u;
    if (!right) mm = __brev(mm) >> 1;
    mm = (mm | (mm >> 1)) & 0x33333333u;
    mm = (mm | (mm >> 2)) & 0x0f0f0f0fu;
    mm = (mm | (mm >> 4)) & 0x00ff00ffu;
    mm = (mm | (mm >> 8)) & 0x0000ffffu;
    const uint32_t n = (w.limit - w.d) < 16u ? (w.limit - w.d) : 16u;
    mm |= (0xffffu << n) & 0xffffu;
    uint32_t t = xtab[(w.def << 8) | (mm & 0xffu)];
    if (t & 15u) { w.best += (int)(t & 15u); w.db_ = (int)w.d + (int)((t >> 4) & 15u); }
    if (t & 0x4000u) { w.fin = true; return; }
    w.def = (t >> 8) & 63u;
    t = xtab[(w.def << 8) | (mm >> 8)];
    if (t & 15u) { w.best += (int)(t & 15u); w.db_ = (int)w.d + 8 + (int)((t >> 4) & 15u); }
    if (t & 0x4000u) { w.fin = true; return; }
    w.def = (t >> 8) & 63u;
    w.d += n;
    if (w.d >= w.limit) w.fin = true;
  }
  __device__ __forceinline__ void extend2_tab2(uint32_t p, uint32_t q, uint32_t ll, uint32_t rl, int* bl,
                                               int* dl, int* br, int* dr) const {
    TWalk L, R;
    {
      const int32_t sd = (int32_t)p - 16, sq = (int32_t)q - 16;
      L.dw = (uint32_t)(sd >> 4);
      L.qp = qw + (sq >> 4);
      L.shd = (uint32_t)(sd & 15) * 2u;
      L.shq = (uint32_t)(sq & 15) * 2u;
      L.dc = win[(L.dw + 1u) & win_mask];
      L.qc = L.qp[1];
      L.limit = ll; L.d = 0; L.def = 0; L.best = 0; L.db_ = 0; L.fin = ll == 0;
    }
    {
      const int32_t sd = (int32_t)(p + (uint32_t)k), sq = (int32_t)(q + (uint32_t)k);
      R.dw = (uint32_t)(sd >> 4);
      R.qp = qw + (sq >> 4);
      R.shd = (uint32_t)(sd & 15) * 2u;
      R.shq = (uint32_t)(sq & 15) * 2u;
      R.dc = win[R.dw++ & win_mask];
      R.qc = *R.qp++;
      R.limit = rl; R.d = 0; R.def = 0; R.best = 0; R.db_ = 0; R.fin = rl == 0;
    }
    while (!(L.fin && R.fin)) {
      if (!L.fin) tw_step(L, false);
      if (!R.fin) tw_step(R, true);
    }
    *bl = L.best; *dl = L.db_; *br = R.best; *dr = R.db_;
  }
#endif
  // 16 bases starting at s (s >= win_lo * 16, in the window) / at query position s >= -16
  __device__ __forceinline__ uint32_t db16w(int32_t s) const {
    const uint32_t w = (uint32_t)(s >> 4);
    return __funnelshift_r(win[w & win_mask], win[(w + 1u) & win_mask], (uint32_t)(s & 15) * 2u);
  }
  __device__ __forceinline__ uint32_t q16w(int32_t s) const {
    const uint32_t* w = qw + (s >> 4);
    return __funnelshift_r(w[0], w[1], (uint32_t)(s & 15) * 2u);
  }
#if PL_S3_COOP
  // ---- S3 hybrid walk (PL_S3_COOP): extend2_win's loop made resumable, plus a warp-cooperative
  // finisher for the few lanes whose walks outlast the serial budget.  A warp of serial walks
  // iterates as long as its longest lane (repeat islands: one 1 kbp walk holds 31 idle lanes);
  // the finisher gives such a walk all 32 lanes, 16 steps each.  Scores, X-drop and the
  // smallest best position are exactly extend()'s (R-S3), so the outputs are unchanged.
  struct XWalk {
    uint32_t dw, dc, qc, shd, shq, limit, d;
    const uint32_t* qp;
    int step, score, best, db_, bl, dl;
    bool right, done;
  };
  __device__ __forceinline__ void xw_left(XWalk& w, uint32_t p, uint32_t q, uint32_t ll) const {
    const int32_t sd = (int32_t)p - 16, sq = (int32_t)q - 16;
    w.dw = (uint32_t)(sd >> 4);
    w.qp = qw + (sq >> 4);
    w.shd = (uint32_t)(sd & 15) * 2u;
    w.shq = (uint32_t)(sq & 15) * 2u;
    w.dc = win[(w.dw + 1u) & win_mask];
    w.qc = w.qp[1];
    w.step = -1;
    w.right = false;
    w.done = false;
    w.limit = ll;
    w.d = 0;
    w.score = w.best = w.db_ = 0;
    w.bl = w.dl = 0;
  }
  __device__ __forceinline__ void xw_right(XWalk& w, uint32_t p, uint32_t q, uint32_t rl) const {
    const int32_t sd = (int32_t)(p + (uint32_t)k), sq = (int32_t)(q + (uint32_t)k);
    w.dw = (uint32_t)(sd >> 4);
    w.qp = qw + (sq >> 4);
    w.shd = (uint32_t)(sd & 15) * 2u;
    w.shq = (uint32_t)(sq & 15) * 2u;
    w.dc = win[w.dw++ & win_mask];
    w.qc = *w.qp++;
    w.step = 1;
    w.right = true;
    w.limit = rl;
    w.d = 0;
    w.score = w.best = w.db_ = 0;
  }
  // up to `budget` 16-base steps of the left-then-right walk (extend2_win's loop, MSB-first)
  __device__ __forceinline__ void xw_run(XWalk& w, int budget, uint32_t p, uint32_t q, uint32_t rl, int X) const {
    for (; budget > 0; --budget) {
      bool fin = w.d >= w.limit;
      if (!fin) {
        const uint32_t dn = win[w.dw & win_mask], qn = *w.qp;
        w.dw += (uint32_t)w.step;
        w.qp += w.step;
        const uint32_t x = w.right ? (__funnelshift_r(w.dc, dn, w.shd) ^ __funnelshift_r(w.qc, qn, w.shq))
                                   : (__funnelshift_r(dn, w.dc, w.shd) ^ __funnelshift_r(qn, w.qc, w.shq));
        w.dc = dn;
        w.qc = qn;
        const uint32_t n = (w.limit - w.d) < 16u ? (w.limit - w.d) : 16u;
        uint32_t mm = (x | (x >> 1)) & 0x55555555u;
        if (w.right) mm = __brev(mm);
        uint32_t mmv = mm & (0xffffffffu << (32u - 2u * n));
        int last = 0;
        while (mmv) {
          const uint32_t c = __clz(mmv);
          const int e = (int)(c >> 1);
          mmv &= 0x7fffffffu >> c;
          w.score += e - last;
          if (w.score > w.best) { w.best = w.score; w.db_ = (int)w.d + e; }
          w.score -= 3;
          last = e + 1;
          if (X > 0 && w.score <= w.best - X) { fin = true; break; }
        }
        if (!fin) {
          w.score += (int)n - last;
          if (w.score > w.best) { w.best = w.score; w.db_ = (int)(w.d + n); }
          w.d += n;
        }
      }
      if (fin) {
        if (w.right) { w.done = true; return; }
        w.bl = w.best;
        w.dl = w.db_;
        xw_right(w, p, q, rl);
      }
    }
  }
  // Lane L's unfinished walk, finished by the whole (converged) warp.  Per round lane j scores
  // steps d+16j+1 .. d+16j+16 of the current direction: its chunk total, its peak (the
  // earliest), its lowest trough and its deepest fall below its own running peak.  A warp sum
  // scan gives each chunk its entering score S_j, a max scan its entering best B_j; chunk j
  // holds an X-drop iff S_j + trough - B_j <= -X or its own fall <= -X (a fall below the
  // running best happens only just after a mismatch, and is the larger of the two).  The
  // first such chunk is replayed serially by its lane from (S_j, B_j); without one the walk
  // moves on 512 steps.
  __device__ __forceinline__ void xw_coop(XWalk& w, int L, uint32_t p, uint32_t q, uint32_t rl, int X) const {
    const unsigned F = 0xffffffffu;
    const int lane = threadIdx.x & 31;
    bool right = __shfl_sync(F, (int)w.right, L) != 0;
    uint32_t d = __shfl_sync(F, w.d, L), limit = __shfl_sync(F, w.limit, L);
    int S = __shfl_sync(F, w.score, L), B = __shfl_sync(F, w.best, L), P = __shfl_sync(F, w.db_, L);
    int bl = __shfl_sync(F, w.bl, L), dl = __shfl_sync(F, w.dl, L);
    const uint32_t pL = __shfl_sync(F, p, L), qL = __shfl_sync(F, q, L), rlL = __shfl_sync(F, rl, L);
    for (;;) {
      bool end = d >= limit;   // warp-uniform
      if (!end) {
        const uint32_t d0 = d + 16u * (uint32_t)lane;
        const uint32_t n = d0 < limit ? ((limit - d0) < 16u ? (limit - d0) : 16u) : 0u;
        uint32_t mm = 0;         // bit 2e: mismatch at step d0 + 1 + e
        if (n) {
          if (right) {
            const uint32_t x = db16w((int32_t)(pL + (uint32_t)k + d0)) ^ q16w((int32_t)(qL + (uint32_t)k + d0));
            mm = (x | (x >> 1)) & 0x55555555u;
          } else {
            const uint32_t x = db16w((int32_t)pL - (int32_t)d0 - 16) ^ q16w((int32_t)qL - (int32_t)d0 - 16);
            mm = __brev((x | (x >> 1)) & 0x55555555u) >> 1;
          }
          mm &= n >= 16u ? 0xffffffffu : ((1u << (2u * n)) - 1u);
        }
        int pre = 0, mx = 0, am = 0, mn = 1 << 29, fall = 0, last = 0;
        for (uint32_t v = mm; v; v &= v - 1) {
          const int e = (__ffs(v) - 1) >> 1;
          pre += e - last;
          if (pre > mx) { mx = pre; am = e; }
          pre -= 3;
          last = e + 1;
          mn = min(mn, pre);
          fall = min(fall, pre - mx);
        }
        pre += (int)n - last;
        if (pre > mx) { mx = pre; am = (int)n; }
        int incl = pre;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int t = __shfl_up_sync(F, incl, o);
          if (lane >= o) incl += t;
        }
        const int Sin = S + incl - pre;
        const int cand = Sin + mx;
        int cm = cand;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int t = __shfl_up_sync(F, cm, o);
          if (lane >= o) cm = max(cm, t);
        }
        const int up = __shfl_up_sync(F, cm, 1);
        const int Bin = lane ? max(B, up) : B;
        const bool drop = X > 0 && n && (Sin + mn - Bin <= -X || fall <= -X);
        const uint32_t db = __ballot_sync(F, drop);
        const int top = db ? __ffs(db) - 1 : 31;
        const int V = db ? __shfl_sync(F, Bin, top) : max(B, __shfl_sync(F, cm, 31));
        int pos = P;
        if (V > B) {   // the earliest chunk (before the drop's) whose peak is V
          const uint32_t hit = __ballot_sync(F, cand == V && (!db || lane < top));
          pos = __shfl_sync(F, (int)d0 + am, __ffs(hit) - 1);
        }
        if (db) {
          int b = V, bp = pos;
          if (lane == top) {
            int s = Sin;
            last = 0;
            for (uint32_t v = mm; v; v &= v - 1) {
              const int e = (__ffs(v) - 1) >> 1;
              s += e - last;
              if (s > b) { b = s; bp = (int)d0 + e; }
              s -= 3;
              last = e + 1;
              if (s <= b - X) break;
            }
          }
          B = __shfl_sync(F, b, top);
          P = __shfl_sync(F, bp, top);
          end = true;
        } else {
          S += __shfl_sync(F, incl, 31);
          B = V;
          P = pos;
          d += 512u;
          end = d >= limit;
        }
      }
      if (end) {
        if (right) break;
        bl = B;
        dl = P;
        right = true;
        d = 0;
        limit = rlL;
        S = B = P = 0;
      }
    }
    if (lane == L) {
      w.bl = bl;
      w.dl = dl;
      w.best = B;
      w.db_ = P;
      w.right = true;
      w.done = true;
    }
  }
  // Both X-drop walks of every `on` lane (all 32 lanes call it, converged): serial rounds of
  // PL_S3_SB steps while more than PL_S3_COOPMAX lanes are unfinished, then the finisher.
  __device__ __forceinline__ void xdrop_hybrid(bool on, uint32_t p, uint32_t q, uint32_t ll, uint32_t rl, int X,
                                               int* bl, int* dl, int* br, int* dr) const {
    XWalk w;
    if (on) xw_left(w, p, q, ll);
    else w.done = true;
    for (;;) {
      if (!w.done) xw_run(w, PL_S3_SB, p, q, rl, X);
      uint32_t rem = __ballot_sync(0xffffffffu, !w.done);
      if (!rem) break;
      if (__popc(rem) <= PL_S3_COOPMAX) {
        while (rem) {
          const int L = __ffs(rem) - 1;
          rem &= rem - 1;
          xw_coop(w, L, p, q, rl, X);
        }
        break;
      }
    }
    if (on) {
      *bl = w.bl;
      *dl = w.dl;
      *br = w.best;
      *dr = w.db_;
    }
  }
#endif
  // bits 0, 2, .., 14 of x -> bits 0..7
  static __device__ __forceinline__ uint32_t even_bits8(uint32_t x) {
    x &= 0x5555u;
    x = (x | (x >> 1)) & 0x3333u;
    x = (x | (x >> 2)) & 0x0f0fu;
    return (x | (x >> 4)) & 0x00ffu;
  }
  // S2 for limits ll, rl <= 8 (R-S2): best_left + best_right of the two +1/-3 walks, each
  // looked up in the 256-entry table of max(0, max prefix score) over its 8-step mismatch
  // pattern (bit e: mismatch at step e+1).  Steps past a limit are marked as mismatches,
  // which never raise a prefix maximum, so the table value is the walk's best.  Needs in_win.
  __device__ __forceinline__ int s2_best8(uint32_t p, uint32_t q, uint32_t ll, uint32_t rl) const {
    const uint32_t xr = db16w((int32_t)(p + (uint32_t)k)) ^ q16w((int32_t)(q + (uint32_t)k));
    const uint32_t xl = db16w((int32_t)p - 16) ^ q16w((int32_t)q - 16);
    const uint32_t mr = even_bits8(xr | (xr >> 1)) | ((0xffu << rl) & 0xffu);
    const uint32_t ml = even_bits8(__brev((xl | (xl >> 1)) & 0x55555555u) >> 1) | ((0xffu << ll) & 0xffu);
    return (int)s2tab[ml] + (int)s2tab[mr];
  }
  // Every DB word a walk of ll bases left of p and rl bases right of the seed may read
  // (extend_win reads whole 16-base steps plus one word ahead) lies in the smem window.
  __device__ __forceinline__ bool in_win(uint32_t p, uint32_t ll, uint32_t rl) const {
    if (nofast) return false;
    const int32_t lo = ((int32_t)p - (int32_t)ll - 32) >> 4;
    const int32_t hi = (int32_t)((p + (uint32_t)k + rl + 32u) >> 4);
    return lo >= (int32_t)win_lo32 && hi < (int32_t)(win_lo32 + win_n);
  }
  __device__ __forceinline__ int64_t right_limit(uint32_t p, uint32_t q) const {
    const int64_t a = (int64_t)db_len - ((int64_t)p + k), b = (int64_t)q_len - ((int64_t)q + k);
    const int64_t m = a < b ? a : b;
    return m > 0 ? m : 0;
  }
  __device__ __forceinline__ int64_t left_limit(uint32_t p, uint32_t q) const { return p < q ? p : q; }
};

// --------------------------------------------------------------- shared state
struct EdgeCtl {            // queue INTO node i
  uint32_t head;            // consumer: next sequence number to consume
  uint32_t seg_head;        // consumer: first live segment
  uint32_t seg_tail;        // producer: segments published
  uint32_t tail;            // producer: one past last published entry
  int64_t  W;               // producer watermark
  uint32_t spill_end;       // producer: end seq of the last spilled segment
  uint32_t stalled;         // producer: waiting for room in this queue (reserve_out)
  alignas(8) uint64_t pub_bar;   // PL_PUB_WAIT: mbarrier (count 1) the producer arrives on at every publication
};
struct GroupCtl {           // broadcast from a node's leader to its lanes, double-buffered
  int64_t  T[2];            // by firing parity so that no barrier is needed between firings
  uint64_t end_ns[2];       // physical: publish time of the firing of that parity
  uint32_t n[2], head[2], done[2], segh[2], st[2], log_idx[2];
  uint32_t in_spill_end[2]; // input edge: end seq of its last spilled segment
  uint32_t out_base[2], out_loc[2];
  alignas(16) uint32_t wtot[2][8];
  alignas(16) uint32_t rmin[8];   // per warp: smallest terminal root of the current firing
  alignas(16) uint32_t rmax[8];   // per warp: largest terminal root + 1 (0: none; physical clock only)
};
// Leader-only per-node accumulators, in smem so that they take no registers in the node loop.
// 64-bit shared atomics compile to CAS spin loops (ATOMS.CAST.SPIN.64), so the single writer
// stores per-firing 32-bit deltas (d[]) as it goes and folds everything into the 64-bit sums
// with one vectorised read-modify-write per firing; maxima use native 32-bit ATOMS.MAX.
enum { C_FIRINGS, C_CONSUMED, C_PRODUCED, C_ACTIVE, C_BUSY, C_OVERRUNS, C_SPILLED, C_STALLS, C_ACTIVE_E, C_DRAINF, C_N };
enum { D_PH0, D_PH1, D_PH2, D_PH3, D_STALL, D_N = 8 };
struct NodeAcc {
  alignas(16) unsigned long long cnt[C_N];
  alignas(16) unsigned long long ph[6];
  alignas(16) uint32_t d[2][D_N];   // per-firing 32-bit deltas, double-buffered by firing parity
  long long t_end;
  uint32_t max_queue, lateness, max_fire, lmax, lmax_ns, nmiss, nmiss_ns;
  uint32_t max_loop;   // physical: longest firing-to-next-decision cycle (the node's real service time)
};
// Sliding DB window (a1): the ring holds chunks of 2^win_lg words at absolute chunk indices;
// chunk c lives at ring slots [c CH, (c+1) CH) & win_mask.  Owned by one thread at a time (node
// 0's accountant lane, or thread 0 of the monolithic kernel); readers see [cov_lo, cov_hi).
struct WinCtl {
  uint32_t cov_lo, cov_hi;  // words valid in the ring (absolute word indices), read as one 8-byte pair
  uint32_t wlo, whi;        // the stream's window range (words)
  uint32_t c_next, c_end;   // next chunk to load; one past the stream's last chunk
  uint32_t inflight, phase; // a refill is in flight on mbar_w; its completion parity
  uint32_t loaded_hi;       // cov_hi once the in-flight refill has landed
  uint32_t refills;         // chunks loaded after the initial staging
  uint32_t c_first;         // first chunk of the stream (chunks < c_first + K need no drop)
  uint32_t a_next;          // next word to load (a chunk loads in pieces as live ingest delivers it)
  uint32_t front;           // live: words [wlo, front) of the stream have been delivered (doorbell cache)
  uint32_t pub;             // live: the last consumed watermark published to the host
  uint32_t src_mask;        // source word index mask (~0u, or the live ring's size - 1)
  const uint32_t* src;      // refill source: the DB, or this stream's live ring
  const uint32_t* front_ptr;   // live: this stream's doorbell (device memory, written by the copy stream)
  uint32_t* consumed_ptr;      // live: this stream's consumed watermark (mapped pinned host memory)
};
struct Shared {
  EdgeCtl e[PL_MAX_STAGES];
  GroupCtl g[PL_MAX_STAGES];
  NodeAcc acc[PL_MAX_STAGES];
  uint32_t max_lat;         // per-stream aggregates: 32-bit so the smem atomics are native
  uint32_t max_lat_ns;      // (64-bit smem atomicMax compiles to a CAS loop)
  uint32_t miss_events;
  uint32_t miss_events_ns;  // physical: terminal items whose measured latency exceeded D
  uint32_t agr_bad;         // physical: terminal items outside the 5 % band of their logical latency
  uint32_t agr_ppm;         // physical: largest |measured - logical| / logical latency (ppm)
  uint32_t errors;
  uint32_t ingest_waits;    // live ingest: node-0 firings (or monolithic blocks) that waited for delivery
  uint32_t ingest_max_ns;   // live ingest: the longest such wait
  uint32_t log_count;       // firing-log records reserved by all nodes of this stream
  uint64_t T0;
  alignas(8) uint64_t mbar; // TMA completion barrier for the initial staging
  alignas(8) uint64_t mbar_w;   // TMA completion barrier of the window refills
  alignas(8) WinCtl win;
  // per node: a lower bound on every root the node will still read the DB for.  Queues are FIFO
  // and every stage emits in input order, so each node's input sequence is sorted by root: the
  // first root of its current firing bounds its whole future.  Monotone; an idle node with an
  // empty queue inherits its upstream's bound (decide).  The window may drop a chunk only below
  // (min_i bnd[i] - q_len - 48) / 16 words (win_step).
  uint32_t bnd[PL_MAX_STAGES];
};

struct Ctx {
  const DevParams* p;
  Shared* sh;
  unsigned char* dsm;          // dynamic smem base (rings, segments, index, DB window)
  Dna dna;
  uint64_t lo, hi;             // roots [lo, hi)
  int64_t X, H;
  bool sliding;                // the stream's DB range exceeds the window ring: refills (win_step)
  uint32_t stream;             // this CTA's stream (blockIdx.x, or the cluster's index: N4)
  int rank;                    // N4 (PL_CLUSTER_NODES): this CTA's rank in its cluster = its node; else -1
  Shared* agg;                 // the stream's aggregates: this CTA's Shared, or rank 0's (DSMEM)
};

__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ bool mbar_test(uint32_t bar, uint32_t parity) {
  uint32_t done;
  asm volatile("{ .reg .pred q; mbarrier.test_wait.parity.shared::cta.b64 q, [%1], %2; selp.u32 %0, 1, 0, q; }"
               : "=r"(done) : "r"(bar), "r"(parity) : "memory");
  return done != 0;
}
// one TMA bulk copy global -> smem completing on mbarrier `bar` (bytes: multiple of 16)
__device__ __forceinline__ void tma_load(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}

// Readers' snapshot of the window's valid range, taken before a firing's DB reads.
__device__ __forceinline__ void win_snap(Dna& dna, const Shared& sh) {
  uint32_t lo, hi;
  asm volatile("ld.volatile.shared.v2.u32 {%0, %1}, [%2];" : "=r"(lo), "=r"(hi) : "r"(smem_addr(&sh.win.cov_lo)));
  asm volatile("fence.acq_rel.cta;" ::: "memory");
  dna.win_lo = lo;
  dna.win_lo32 = lo;
  dna.win_n = hi - lo;
}

__device__ __forceinline__ uint32_t ld_acquire_gpu(const uint32_t* a) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(a) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(uint32_t* a, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(a), "r"(v) : "memory");
}
// Live ingest: the stream's delivered-word frontier, refreshed from its doorbell when `need`
// lies beyond the cached value.  The copy stream writes the doorbell (cuStreamWriteValue32,
// with its default system-scope fence) after the words' copy, so the acquire load orders every
// later read of those words -- generic (__ldcg) and, after the proxy fence, TMA -- behind it.
__device__ __forceinline__ uint32_t live_front(WinCtl& W, uint32_t need) {
  uint32_t f = vld(&W.front);
  if (f >= need) return f;
  const uint32_t g = ld_acquire_gpu(W.front_ptr);
  if (g > f) { atomicMax(&W.front, g); f = g; }
  asm volatile("fence.proxy.async.global;" ::: "memory");
  return f;
}

// One step of the sliding window, by its single owner thread: complete an in-flight refill
// (publish cov_hi), then start the next one if the chunk it overwrites is no longer needed.
// A root p reads DB words >= (p - q_len - 48) / 16 (extension walks reach q_len bases to the
// left, plus whole 16-base steps), so chunk c may replace chunk c - K once every node's bound
// is past that.  A reader's stale snapshot is harmless: it only reads words of its own roots,
// which are >= min bnd and so never in a dropped chunk.  wait = block until the refill lands.
// Live ingest: a chunk loads in 16-byte-aligned pieces as its words are delivered, and the
// consumed watermark min(floor, a_next) -- nothing below it is read or staged again -- goes to
// the host, which may then overwrite those ring slots.  Returns whether it made progress.
#if PL_WINSTEP_NOINLINE
__device__ __noinline__
#else
__device__
#endif
bool win_step(Shared& sh, const DevParams& p, unsigned char* ring, bool wait) {
  WinCtl& W = sh.win;
  const uint32_t bar = smem_addr(&sh.mbar_w);
  bool prog = false;
  if (W.inflight) {
    if (!mbar_test(bar, W.phase)) {
      if (!wait) return false;
      while (!mbar_test(bar, W.phase)) {}
    }
    W.phase ^= 1u;
    W.inflight = 0;
    asm volatile("fence.acq_rel.cta;" ::: "memory");
    *(volatile uint32_t*)&W.cov_hi = W.loaded_hi;
    prog = true;
  }
  if (W.c_next >= W.c_end) return prog;
  uint32_t m = 0xffffffffu;
  for (int i = 0; i < p.N; ++i) m = min(m, *(volatile uint32_t*)&sh.bnd[i]);
  const uint32_t need = (uint32_t)p.q_len + 48u;
  const uint32_t floor_w = m > need ? (m - need) >> 4 : 0u;
  const uint32_t c = W.c_next, K = p.win_cap >> p.win_lg;
  if (p.live) {
    const uint32_t fl = min(floor_w, W.a_next);
    if (fl >= W.pub + 64u) { W.pub = fl; st_release_sys(W.consumed_ptr, fl); }
  }
  const uint32_t b = min((c + 1u) << p.win_lg, W.whi);
  const bool drop = W.a_next == max(c << p.win_lg, W.wlo) && c >= W.c_first + K;   // first piece of chunk c
  const uint32_t lo_new = (c - K + 1u) << p.win_lg;
  if (drop && floor_w < lo_new) return prog;       // chunk c - K is still needed
  uint32_t e = b;
  if (p.live) {
    e = min(b, live_front(W, b) & ~3u);            // TMA moves whole 16-byte units
    if (e <= W.a_next) return prog;
  }
  if (drop) {
    *(volatile uint32_t*)&W.cov_lo = lo_new;  // drop chunk c - K (readers only narrow their snapshots)
    // the generic-proxy reads of the dropped chunk are ordered before the async-proxy refill
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  const uint32_t a = W.a_next;
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"((e - a) * 4u) : "memory");
  tma_load(smem_addr(ring + (a & (p.win_cap - 1u)) * 4u), W.src + (a & W.src_mask), (e - a) * 4u, bar);
  W.inflight = 1;
  W.loaded_hi = e;
  if (e == b) {
    W.c_next = c + 1u;
    W.a_next = (c + 1u) << p.win_lg;
    W.refills++;
  } else {
    W.a_next = e;
  }
  if (wait) {
    while (!mbar_test(bar, W.phase)) {}
    W.phase ^= 1u;
    W.inflight = 0;
    asm volatile("fence.acq_rel.cta;" ::: "memory");
    *(volatile uint32_t*)&W.cov_hi = e;
  }
  return true;
}

__device__ __forceinline__ int64_t arrival(const Ctx& c, uint32_t root) {
  return c.p->arr ? __ldg(c.p->arr + root) : (int64_t)(root - c.lo) * c.p->tau;
}

// floor(a / d) for 0 <= a < 2^63 by a host-precomputed reciprocal m = floor((2^64-1)/d):
// umulhi(a, m) is floor(a/d) or one less, fixed by one compare (no 64-bit division).
struct MDiv {
  uint64_t m;
  int64_t d;
};
__device__ __forceinline__ int64_t fdiv(int64_t a, const MDiv& D) {
  if (D.d == 1) return a;
  int64_t q = (int64_t)__umul64hi((uint64_t)a, D.m);
  if ((q + 1) * D.d <= a) ++q;
  return q;
}
__device__ __forceinline__ int64_t cdiv(int64_t a, const MDiv& D) { return a <= 0 ? 0 : fdiv(a - 1, D) + 1; }

// Per-node constants, built once per warp group and kept in registers.
struct Node {
  int i, N, v;
  bool sink, phys, fixed;
  int64_t t, P, R, D, tau, X, H;
  uint32_t theta;
  uint64_t lo;
  double nspu;
  bool ns1;                     // ns_per_unit == 1: unit -> ns conversions are the identity
  int64_t t_ns, D_ns;           // floor(t_i ns_per_unit), floor(D ns_per_unit): integer tests x > t_i nspu
  uint32_t segmask, capg;
  EdgeCtl* Ein;                 // input edge (i > 0)
  const uint2* in_ent;
  const Seg* in_seg;
  const uint2* in_spill;
  uint32_t in_mask;
  EdgeCtl* Eout;                // output edge (i < N-1)
  uint2* out_ent;
  Seg* out_seg;
  uint2* out_spill;
  uint32_t out_cap;
  uint32_t kind, max_out, cfix, umax;
  int32_t ip1, ip2;
  MDiv dtau, dP;
  int64_t Pq, Pr;               // floor(P / tau0), P mod tau0
  const int64_t* arr;           // per-root arrival times (NULL: fixed rate, L63)
  bool eager;                   // PL_EAGER_DRAIN (R-DRAIN): work-conserving at T >= A_last
  int64_t A_last;               // the stream's last arrival
  int64_t Mcap, B_per;          // FIXED_WAIT + eager: time-triggered slots m < Mcap (m P < A_last);
                                // the last of them ends at B_per
  uint32_t* troot;              // smem [v]: the current firing's terminal root per lane (or NO_ROOT)
  uint32_t* bnd_me;             // smem: this node's Shared::bnd entry (sliding window only)
  const uint32_t* bnd_up;       // the upstream node's entry (its CTA's smem under N4)
  bool cl;                      // N4: queues are in the consumer CTA's smem (cluster-scope fences)
  uint32_t nap_cap_ns;          // physical: longest poll nap of a waiting leader (t_i / 8, >= 256 ns)
  bool sliding;
  __device__ __forceinline__ int64_t arrival(uint32_t root) const {
    return arr ? __ldg(arr + root) : (int64_t)(root - lo) * tau;
  }
};

__host__ __device__ inline uint32_t layout_enforced(const DevParams& p, SmemLayout* L);
// PL_S3_TAB: the X of the DNA sink's X-drop when its transition table is built (1..63), else 0
__host__ __device__ inline int xtab_X(const DevParams& p) {
#if PL_S3_TAB
  if (p.k > 0 && p.N > 0 && p.st[p.N - 1].kind == PL_UNGAPPED_XDROP && p.st[p.N - 1].ip[1] >= 1 &&
      p.st[p.N - 1].ip[1] <= 63)
    return p.st[p.N - 1].ip[1];
#endif
  (void)p;
  return 0;
}

// logical time units -> ns of %globaltimer (physical clock)
__device__ __forceinline__ uint64_t units_ns(const Node& nd, int64_t t) {
  return nd.ns1 ? (uint64_t)t : (uint64_t)((double)t * nd.nspu);
}

template <bool CL = false>
__device__ __forceinline__ Node make_node(const Ctx& c, int i) {
  const DevParams& p = *c.p;
  SmemLayout Lo;
  layout_enforced(p, &Lo);
  Node n;
  n.i = i; n.N = p.N; n.v = p.v;
  n.sink = i == p.N - 1;
  n.phys = p.clock == PL_CLOCK_GLOBALTIMER;
  n.fixed = p.policy == PL_FIXED_WAIT;
  n.t = p.t[i]; n.P = p.P[i]; n.R = p.R[i]; n.D = p.D; n.tau = p.tau; n.X = c.X; n.H = c.H;
  n.theta = p.theta[i];
  n.lo = c.lo;
  n.nspu = p.ns_per_unit;
  n.ns1 = p.ns_per_unit == 1.0;
  n.t_ns = (int64_t)((double)p.t[i] * p.ns_per_unit);
  n.D_ns = (int64_t)((double)p.D * p.ns_per_unit);
  n.segmask = p.segcap - 1;
  n.capg = p.cap_g;
  n.Ein = &c.sh->e[i];
  const uint64_t sp = (uint64_t)c.stream * p.N;
  n.in_ent = (const uint2*)(c.dsm + Lo.off_ent[i]);
  n.in_seg = (const Seg*)(c.dsm + Lo.off_seg[i]);
  n.in_spill = p.spill ? p.spill + (sp + i) * p.cap_g : nullptr;
  n.in_mask = p.cap_s[i] ? p.cap_s[i] - 1 : 0;
  const int o = i + 1 < p.N ? i + 1 : i;
  n.cl = CL && c.rank >= 0;   // a compile-time false outside the cluster kernel
  if (n.cl && o != i) {   // N4: the edge into node i+1 lives in CTA i+1's shared memory (DSMEM)
    n.Eout = (EdgeCtl*)__cluster_map_shared_rank(&c.sh->e[o], (unsigned)o);
    n.out_ent = (uint2*)__cluster_map_shared_rank(c.dsm + Lo.off_ent[o], (unsigned)o);
    n.out_seg = (Seg*)__cluster_map_shared_rank(c.dsm + Lo.off_seg[o], (unsigned)o);
  } else {
    n.Eout = &c.sh->e[o];
    n.out_ent = (uint2*)(c.dsm + Lo.off_ent[o]);
    n.out_seg = (Seg*)(c.dsm + Lo.off_seg[o]);
  }
  n.out_spill = p.spill ? p.spill + (sp + o) * p.cap_g : nullptr;
  n.out_cap = p.cap_s[o];
  const DevStage& s = p.st[i];
  n.kind = s.kind; n.max_out = s.max_out; n.cfix = s.cfix;
  n.umax = s.kind == PL_FIXED_GAIN ? s.cfix : s.max_out;
  n.ip1 = s.ip[1]; n.ip2 = s.ip[2];
  n.dtau.m = p.tau_m; n.dtau.d = p.tau;
  n.dP.m = p.P_m[i]; n.dP.d = p.P[i];
  n.Pq = fdiv(p.P[i], n.dtau);
  n.Pr = p.P[i] - n.Pq * p.tau;
  n.arr = p.arr;
  n.eager = (p.flags & PL_EAGER_DRAIN) != 0u;
  n.A_last = c.X > 0 ? n.arrival((uint32_t)(c.hi - 1)) : 0;
  n.Mcap = (n.eager && n.fixed) ? cdiv(n.A_last, n.dP) : 0;
  n.B_per = n.Mcap > 0 ? (n.Mcap - 1) * n.P + n.t : 0;
  n.troot = (uint32_t*)(c.dsm + Lo.off_troot) + (uint32_t)i * (uint32_t)p.v;
  n.bnd_me = &c.sh->bnd[i];
  n.bnd_up = (n.cl && i > 0) ? (const uint32_t*)__cluster_map_shared_rank(&c.sh->bnd[i - 1], (unsigned)(i - 1))
                             : &c.sh->bnd[i > 0 ? i - 1 : 0];
  {
    const int64_t cap = n.t_ns / 8;
    n.nap_cap_ns = (uint32_t)(cap < 256 ? 256 : (cap > 8192 ? 8192 : cap));
  }
  n.sliding = c.sliding;
  return n;
}

// Entry with sequence number s of the node's input edge: spilled iff it lies in
// a spilled segment (binary search of the live segments [segh, st)).
__device__ __forceinline__ uint2 load_entry(const Node& nd, uint32_t s, uint32_t segh, uint32_t st,
                                            uint32_t spill_end) {
  if ((int32_t)(s - spill_end) >= 0) return nd.in_ent[s & nd.in_mask];
  uint32_t lo = segh, hi = st;
  while (lo < hi) {
    const uint32_t mid = lo + ((hi - lo) >> 1);
    if ((int32_t)(nd.in_seg[mid & nd.segmask].end - s) > 0) hi = mid; else lo = mid + 1;
  }
  if (nd.in_seg[lo & nd.segmask].loc == LOC_SPILL) return __ldcg(nd.in_spill + (s & (nd.capg - 1)));
  return nd.in_ent[s & nd.in_mask];
}

// ------------------------------------------------------------ stage functions
// Phase A: number of outputs of one input entry (and per-lane state for phase B).
struct LaneOut {
  uint32_t c;       // outputs
  uint32_t a;       // S1: offset into the query position list; S3: db_start
  int32_t score;    // S3
  uint32_t q_start, len;
};

// S2 / S3 for one entry.
__device__ __forceinline__ LaneOut stage_count_ext(const Node& nd, const Dna& dna, uint2 e) {
  LaneOut o;
  o.c = 0; o.a = 0; o.score = 0; o.q_start = 0; o.len = 0;
  const uint32_t q = e.y & 0xffffu;
  // both limits are <= q_len, so they fit 32 bits
  uint32_t ll = (uint32_t)dna.left_limit(e.x, q), rl = (uint32_t)dna.right_limit(e.x, q);
  if (nd.kind == PL_UNGAPPED_WINDOW) {
    const uint32_t W = (uint32_t)nd.ip1;
    ll = ll < W ? ll : W;
    rl = rl < W ? rl : W;
  }
  const int X = nd.kind == PL_UNGAPPED_WINDOW ? 0 : nd.ip1;
  int dl, dr, bl, br;
  if (nd.kind == PL_UNGAPPED_WINDOW && nd.ip1 <= 8 && dna.in_win(e.x, ll, rl)) {
    o.c = (dna.k + dna.s2_best8(e.x, q, ll, rl) >= nd.ip2) ? 1u : 0u;
    return o;
  }
  if (dna.in_win(e.x, ll, rl)) {
#if PL_S3_TAB
#if PL_S3_TAB2
    if (X > 0 && X == dna.xtab_X) dna.extend2_tab2(e.x, q, ll, rl, &bl, &dl, &br, &dr);
    else
#else
    if (X > 0 && X == dna.xtab_X) dna.extend2_tab(e.x, q, ll, rl, &bl, &dl, &br, &dr);
    else
#endif
#endif
    dna.extend2_win(e.x, q, ll, rl, X, &bl, &dl, &br, &dr);
  } else {
    bl = dna.extend(e.x, q, -1, ll, X, &dl);
    br = dna.extend(e.x, q, +1, rl, X, &dr);
  }
  if (nd.kind == PL_UNGAPPED_WINDOW) {
    o.c = (dna.k + bl + br >= nd.ip2) ? 1u : 0u;
  } else {
    const int score = dna.k + bl + br;
    if (score >= nd.ip2) {
      o.c = 1;
      o.score = score;
      o.a = e.x - dl;
      o.q_start = q - dl;
      o.len = dna.k + dl + dr;
    }
  }
  return o;
}

#if PL_S3_COOP
// S3 for one entry per lane, called by the whole converged warp: walks outside the smem window
// take the checked per-lane path, the others the hybrid walk (Dna::xdrop_hybrid).
__device__ __forceinline__ LaneOut stage_xdrop_warp(const Node& nd, const Dna& dna, uint2 e, bool act) {
  LaneOut o;
  o.c = 0; o.a = 0; o.score = 0; o.q_start = 0; o.len = 0;
  const uint32_t q = e.y & 0xffffu;
  const uint32_t ll = act ? (uint32_t)dna.left_limit(e.x, q) : 0u;
  const uint32_t rl = act ? (uint32_t)dna.right_limit(e.x, q) : 0u;
  const int X = nd.ip1;
  const bool fast = act && dna.in_win(e.x, ll, rl);
  int dl = 0, dr = 0, bl = 0, br = 0;
  if (act && !fast) {
    bl = dna.extend(e.x, q, -1, ll, X, &dl);
    br = dna.extend(e.x, q, +1, rl, X, &dr);
  }
  __syncwarp();
  dna.xdrop_hybrid(fast, e.x, q, ll, rl, X, &bl, &dl, &br, &dr);
  const int score = dna.k + bl + br;
  if (act && score >= nd.ip2) {
    o.c = 1;
    o.score = score;
    o.a = e.x - dl;
    o.q_start = q - dl;
    o.len = dna.k + dl + dr;
  }
  return o;
}
#endif

__device__ __forceinline__ LaneOut stage_count(const Node& nd, const Dna& dna, const DevParams& p, uint2 e) {
  LaneOut o;
  o.c = 0; o.a = 0; o.score = 0; o.q_start = 0; o.len = 0;
  switch (nd.kind) {
    case PL_BERNOULLI: o.c = gain_hash(p.seed, nd.i, e.x, e.y) < p.st[nd.i].thr[0] ? 1u : 0u; break;
    case PL_FIXED_GAIN: o.c = nd.cfix; break;
    case PL_POISSON_CAPPED: {
      const uint64_t h = gain_hash(p.seed, nd.i, e.x, e.y);
      uint32_t n = 0;
      for (uint32_t k = 0; k < nd.max_out; ++k) n += (h >= p.st[nd.i].thr[k]) ? 1u : 0u;
      o.c = n;
      break;
    }
    case PL_KEEP_EVERY: o.c = (e.x % nd.cfix) == 0 ? 1u : 0u; break;
    case PL_SEED_LOOKUP: {
      const uint32_t key = dna.key(e.x);
      o.c = dna.qoff[key + 1] > dna.qoff[key] ? 1u : 0u;
      break;
    }
    case PL_HIT_ENUM: {
      const uint32_t key = dna.key(e.x);
      const uint32_t off = dna.qoff[key], cnt = dna.qoff[key + 1] - off;
      o.a = off;
      o.c = cnt < nd.max_out ? cnt : nd.max_out;
      break;
    }
    case PL_UNGAPPED_WINDOW:
    case PL_UNGAPPED_XDROP: o = stage_count_ext(nd, dna, e); break;
  }
  return o;
}

// Phase B: output j of an entry (non-sink nodes).
__device__ __forceinline__ uint2 stage_output(const Node& nd, const Dna& dna, uint2 e, const LaneOut& o, uint32_t j) {
  switch (nd.kind) {
    case PL_FIXED_GAIN: return make_uint2(e.x, e.y * nd.cfix + j);
    case PL_POISSON_CAPPED: return make_uint2(e.x, e.y * nd.max_out + j);
    case PL_HIT_ENUM: return make_uint2(e.x, (uint32_t)dna.qpos[o.a + j] | (j << 16));
    default: return e;
  }
}

// ---------------------------------------------------------------- leader logic
struct Decision {
  bool done;
  int64_t T;
  uint32_t n;
  uint32_t qlen;    // input-queue length at the decision (all queued entries; L133's b_i v)
};

struct Leader {   // leader-private schedule state of one node
  int64_t m;      // FIXED_WAIT: index of the next firing
  int64_t B;      // THRESHOLD_SLACK: busy until
  uint64_t c0;    // node 0: roots consumed
  uint32_t head, segh;          // consumer side of the input edge
  uint32_t out_tail, out_segt;  // producer side of the output edge
  int64_t W_pub;
  uint64_t empties;
  uint32_t wd;                  // the watchdog fired (PL_ERR_WATCHDOG)
};

// Watchdog (SURVEY §5 failure detection): a node that keeps waiting -- for its upstream in
// decide(), or for room downstream in reserve_out() -- for PL_WATCHDOG_NS of %globaltimer gives
// up: error bit PL_ERR_WATCHDOG, the node ends (decide) or drops the firing's outputs
// (reserve_out), so a protocol fault or an abandoned live stream ends the run instead of hanging
// the GPU.  Checked every 256 spins of a wait, cold.
__device__ __noinline__ bool watchdog_expired(uint64_t& t0) {
  const uint64_t now = gtimer();
  if (t0 == 0) { t0 = now; return false; }
  return now - t0 > PL_WATCHDOG_NS;
}

// PL_PUB_WAIT: the producer's leader arrives on its output edge's mbarrier after every
// publication (a new watermark or segment); a waiting consumer leader sleeps in
// mbarrier.try_wait with the nap's length as the time limit, so it resumes at the publication
// instead of at the end of a nap.  A wake-up hint only: the consumer re-reads the edge with the
// usual fences either way.  Not under N4 (the edge lives in another CTA's smem).
__device__ __forceinline__ void pub_signal(const Node& nd) {
#if PL_PUB_WAIT
  if (nd.phys && !nd.cl)
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_addr(&nd.Eout->pub_bar)) : "memory");
#endif
}
// The input edge's current (incomplete) phase parity, read BEFORE the edge is polled: a
// publication after the poll then completes that phase and the sleep below returns at once
// (no lost wake-up).  Phase parity 0 is complete iff the current phase is odd.
__device__ __forceinline__ uint32_t pub_phase(const Node& nd) {
  uint32_t cur = 0;
#if PL_PUB_WAIT
  if (nd.phys && !nd.cl)
    asm volatile("{ .reg .pred q; mbarrier.test_wait.parity.shared::cta.b64 q, [%1], 0; selp.u32 %0, 1, 0, q; }"
                 : "=r"(cur) : "r"(smem_addr(&nd.Ein->pub_bar)) : "memory");
#endif
  return cur;
}

__device__ __forceinline__ void publish_W(const Node& nd, Leader& L, int64_t w) {
  if (nd.sink) return;
  if (w > L.W_pub) {
    L.W_pub = w;
    fence_q(nd.cl);
    vst(&nd.Eout->W, w);
    pub_signal(nd);
  }
}

// Poll backoff.  The logical clock polls hard (its schedule advances as fast as the nodes do).
// On the physical clock a poll costs issue slots that a waiting node is supposed to yield
// (PAPER.md L75/L85), so the nap doubles from 64 ns up to `cap_ns` -- an eighth of the node's
// service time (Node::nap_cap_ns): reacting that much later to an upstream publish delays a
// firing start by at most t_i / 8, which the time-triggered delivery (PL_FIXED_SERVICE) absorbs
// while the work itself takes well under t_i.  Measured on c4 (ncu source page): the fixed
// 256 ns nap made the waiting leaders' polls ~90 % of all instructions issued.
// The watchdog (above) is checked deep inside a wait only, every 4096 naps, off every firing's
// path; a waiter whose watchdog expired finds spins < 0.
__device__ __forceinline__ void backoff(int& spins, uint64_t& wd0, bool phys = false, uint32_t cap_ns = 256) {
  if (spins < (phys ? PL_PHYS_SPINS : 4)) { ++spins; return; }
  if (phys) {
    const int e = spins - PL_PHYS_SPINS < 16 ? spins - PL_PHYS_SPINS : 16;
    const uint32_t ns = 64u << e;
    __nanosleep(ns < cap_ns ? ns : cap_ns);
  } else {
    __nanosleep(spins < 64 ? 32 : 256);
  }
  ++spins;
  if (PL_WATCHDOG && (spins & 4095) == 0 && watchdog_expired(wd0)) spins = -(1 << 30);
}

// A waiting leader in decide(): every condition it waits for (upstream watermark past T, enough
// entries) changes only at an upstream publication, so under PL_PUB_WAIT it sleeps on the edge's
// mbarrier until the phase `ph` (read before its poll) completes, with t_i as a safety limit;
// otherwise the backoff naps above.
__device__ __forceinline__ void wait_up(const Node& nd, uint32_t ph, int& spins, uint64_t& wd0) {
#if PL_PUB_WAIT
  if (nd.phys && !nd.cl) {
    const uint32_t ns = min(nd.nap_cap_ns << 3, 1u << 20);
    uint32_t done;
    asm volatile("{ .reg .pred q; mbarrier.try_wait.parity.shared::cta.b64 q, [%1], %2, %3; selp.u32 %0, 1, 0, q; }"
                 : "=r"(done) : "r"(smem_addr(&nd.Ein->pub_bar)), "r"(ph), "r"(ns) : "memory");
    (void)done;
    ++spins;
    if (PL_WATCHDOG && (spins & 4095) == 0 && watchdog_expired(wd0)) spins = -(1 << 30);
    return;
  }
#endif
  (void)ph;
  backoff(spins, wd0, nd.phys, nd.nap_cap_ns);
}

// number of entries of the input edge with ready <= T among the published ones (stops at v)
__device__ __forceinline__ uint32_t count_le(const Node& nd, const Leader& L, uint32_t st, int64_t T) {
  uint32_t end = L.head;
  for (uint32_t k = L.segh; k != st; ++k) {
    const Seg& sg = nd.in_seg[k & nd.segmask];
    if (sg.ready > T) break;
    end = sg.end;
    if (end - L.head >= (uint32_t)nd.v) break;
  }
  return end - L.head;
}

// number of PUBLISHED entries of the input edge with ready <= T, uncapped: the queue length
// |Q_i| at a firing decision at T (PAPER.md L133's "maximum size b_i v").  Segments are
// published in firing order, so their ready times are non-decreasing: binary search.
__device__ __forceinline__ uint32_t count_all_le(const Node& nd, const Leader& L, uint32_t st, int64_t T) {
  uint32_t lo = L.segh, hi = st;          // first segment with ready > T
  while (lo != hi) {
    const uint32_t mid = lo + ((hi - lo) >> 1);
    if (nd.in_seg[mid & nd.segmask].ready <= T) lo = mid + 1; else hi = mid;
  }
  return lo == L.segh ? 0u : nd.in_seg[(lo - 1) & nd.segmask].end - L.head;
}

// Node 0: arrivals are fully known (root lo+r arrives at r*tau0), so every
// lane evaluates the firing decision itself from replicated state (no broadcast barrier).
struct Rep {
  int64_t m;        // FIXED_WAIT: next firing index
  int64_t B;        // THRESHOLD_SLACK: busy until
  int64_t c0;       // roots consumed
  uint64_t empties;
  int64_t qT, rT;   // FIXED_WAIT: floor(m P / tau0) and remainder, advanced without division
  bool qvalid;
};
__device__ __forceinline__ Decision decide0(const Node& nd, Rep& r) {
  Decision d;
  d.done = r.c0 >= nd.X;
  d.T = 0;
  d.n = 0;
  d.qlen = 0;
  if (d.done) return d;
  if (nd.arr) {   // arrival times given as data: the lanes test their own item (sorted -> a prefix)
    const int64_t* A = nd.arr + nd.lo;
    const int64_t ah = __ldg(A + r.c0);
    int64_t T;
    if (nd.fixed) {
      T = r.m * nd.P;
      if (T < ah) {
        const int64_t m2 = cdiv(ah, nd.dP);
        const int64_t me = nd.eager ? min(m2, nd.Mcap) : m2;   // R-DRAIN: no slots at or after A_last
        if (me > r.m) r.empties += (uint64_t)(me - r.m);
        r.m = m2;
        T = r.m * nd.P;
      }
      if (nd.eager && r.m >= nd.Mcap) T = max(max(nd.B_per, r.B), nd.A_last);
    } else {
      const int64_t Tth = (r.c0 + nd.theta - 1 < nd.X) ? __ldg(A + r.c0 + nd.theta - 1) : PL_INF64;
      int64_t Tf = ah + nd.D - nd.R;
      if (Tf < ah) Tf = ah;
      T = Tth < Tf ? Tth : Tf;
      if (T < r.B) T = r.B;
      if (nd.eager) T = min(T, max(r.B, nd.A_last));
    }
    d.T = T;
    d.n = (uint32_t)nd.v;                // upper bound; the exact count comes out of the scan
    return d;
  }
  int64_t T, q;
  if (nd.fixed) {
    T = r.m * nd.P;
    if (T < r.c0 * nd.tau) {             // empty firings until the next root has arrived
      const int64_t m2 = cdiv(r.c0 * nd.tau, nd.dP);
      const int64_t me = nd.eager ? min(m2, nd.Mcap) : m2;   // R-DRAIN: no slots at or after A_last
      if (me > r.m) r.empties += (uint64_t)(me - r.m);
      r.m = m2;
      T = r.m * nd.P;
      r.qvalid = false;
    }
    if (nd.eager && r.m >= nd.Mcap) {    // R-DRAIN: every root has arrived; fire when idle
      T = max(max(nd.B_per, r.B), nd.A_last);
      q = nd.X - 1;
    } else {
      if (!r.qvalid) {                   // floor(T / tau0), then advanced by P per firing
        r.qT = fdiv(T, nd.dtau);
        r.rT = T - r.qT * nd.tau;
        r.qvalid = true;
      }
      q = r.qT;
    }
  } else {
    const int64_t ah = r.c0 * nd.tau;
    const int64_t Tth = (r.c0 + nd.theta - 1 < nd.X) ? ah + (int64_t)(nd.theta - 1) * nd.tau : PL_INF64;
    int64_t Tf = ah + nd.D - nd.R;
    if (Tf < ah) Tf = ah;
    T = Tth < Tf ? Tth : Tf;
    if (T < r.B) T = r.B;
    if (nd.eager) T = min(T, max(r.B, nd.A_last));
    q = fdiv(T, nd.dtau);
  }
  int64_t arrived = q + 1;
  if (arrived > nd.X) arrived = nd.X;
  const int64_t avail = arrived - r.c0;
  d.T = T;
  d.n = (uint32_t)(avail < (int64_t)nd.v ? avail : nd.v);
  d.qlen = (uint32_t)(avail < 0xffffffffll ? avail : 0xffffffffll);
  return d;
}

// FIXED_WAIT node 0 after a firing: T += P, so floor(T/tau0) += floor(P/tau0) (+1 on carry)
__device__ __forceinline__ void advance0(const Node& nd, Rep& r) {
  ++r.m;
  if (r.qvalid) {
    r.qT += nd.Pq;
    r.rT += nd.Pr;
    if (r.rT >= nd.tau) { r.rT -= nd.tau; ++r.qT; }
  }
}

// Nodes i >= 1: the leader decides from the published queue state and watermark.
// Sleep until %globaltimer reaches `target` (chunks of at most a quarter of the remaining
// time, __nanosleep rounds up); returns whether it slept at all.
__device__ __forceinline__ bool nap_until(uint64_t target) {
  uint64_t now = gtimer();
  if (now >= target) return false;
  while (now < target) {   // __nanosleep sleeps at most 2x its argument: nap rem >> PL_NAP_SHIFT
    const uint64_t rem = target - now;
#if PL_NAP_HALF
    __nanosleep(rem > 128 ? (uint32_t)min(rem >> 1, (uint64_t)(1u << 20)) : 64u);
#else
    __nanosleep(rem > 4096 ? (uint32_t)min(rem >> PL_NAP_SHIFT, (uint64_t)(1u << 20)) : (rem > 1024 ? 256u : 64u));
#endif
    now = gtimer();
  }
  return true;
}

// A FIXED_WAIT node cannot start firing m before T = m P_i, so on the physical clock it sleeps
// until this far ahead of T before it polls its upstream (a waiting node then costs issue slots
// only for the poll that decides the firing; yielded time is usable).
#ifndef PL_NAP_LEAD
#define PL_NAP_LEAD 768     // 256: c3 THRESHOLD_SLACK -4 % instructions per root, but firings start late: busy/model
                            // 0.961 on the c4 bench, 0.930 on a FIXED_WAIT c2 replay (test_physical_replays_logical_schedule): rejected
#endif
constexpr uint64_t PL_NAP_LEAD_NS = PL_NAP_LEAD;

// THRESHOLD_SLACK on the physical clock: a node whose next firing cannot start before logical
// time lb = max(B, min(Tk, W_up)) -- nothing it has queued can fire earlier, and anything its
// upstream has not yet published is ready at >= W_up -- sleeps until PL_NAP_LEAD_NS before
// T0 + lb instead of polling every t_i / 8: its upstream's commit publishes W_up one firing
// ahead, so an idle node behind node 0 sleeps a whole node-0 period at a time (PAPER.md L75/L85:
// the waiting node's time is yielded).  At most one nap per distinct lb (`napped`); a node that
// is behind its schedule (T0 + lb already past) polls as before.
__device__ __forceinline__ bool nap_to(const Node& nd, uint64_t T0, int64_t lb, int64_t& napped) {
  if (!nd.phys || lb == napped || lb == PL_INF64) return false;
  napped = lb;
  const uint64_t due = T0 + units_ns(nd, lb);
  return due > T0 + PL_NAP_LEAD_NS && nap_until(due - PL_NAP_LEAD_NS);
}

// A node may commit a firing at T before its upstream watermark passes T once v entries with
// ready <= T are queued (the firing is full whatever else arrives).  On the logical clock it
// does so only when the producer is stalled on this queue -- needed for deadlock freedom,
// so that every other decision sees the complete queue at T and the
// recorded queue peak is the DES's |Q_i| exactly; the physical clock always may.
__device__ __forceinline__ bool early_ok(const Node& nd) { return nd.phys || vld(&nd.Ein->stalled) != 0u; }

__device__ __forceinline__ Decision decide(const Node& nd, Leader& L, bool& waited, uint64_t T0) {
  const uint32_t v = (uint32_t)nd.v;
  Decision d;
  d.done = false; d.T = 0; d.n = 0; d.qlen = 0;
  int spins = 0;
  int64_t napped = -1;
  uint64_t wd0 = 0;
  for (;;) {
    if (spins < 0) { L.wd = 1u; publish_W(nd, L, PL_INF64); d.done = true; return d; }   // watchdog
    if (nd.phys && nd.fixed && !(nd.eager && L.m >= nd.Mcap)) {
      const int64_t Tn = L.m * nd.P;
      if (Tn != napped) {
        napped = Tn;
        const uint64_t due = T0 + units_ns(nd, Tn);
        if (due > T0 + PL_NAP_LEAD_NS && nap_until(due - PL_NAP_LEAD_NS)) waited = true;
      }
    }
    // node i >= 1: read the upstream watermark (and window bound) first, then the published segments
    const uint32_t ph = pub_phase(nd);
    const int64_t Wup = vld(&nd.Ein->W);
    const uint32_t bup = nd.sliding ? vld(nd.bnd_up) : 0u;
    fence_q(nd.cl);
    const uint32_t st = vld(&nd.Ein->seg_tail);
    const uint32_t tail_known = (st != L.segh) ? nd.in_seg[(st - 1) & nd.segmask].end : L.head;
    const bool any = tail_known != L.head;
    // an empty queue: everything this node will still read comes from upstream's future
    if (nd.sliding && !any && bup > vld(nd.bnd_me)) vst(nd.bnd_me, bup);
    if (nd.fixed) {
      if (nd.eager && L.m >= nd.Mcap) {  // R-DRAIN: work-conserving from A_last on
        const int64_t B = max(max(nd.B_per, L.B), nd.A_last);
        if (!any) {
          if (Wup == PL_INF64) { d.done = true; return d; }
          publish_W(nd, L, max(B, Wup) + nd.t);
          wait_up(nd, ph, spins, wd0); waited = true;
          continue;
        }
        const int64_t Te = max(B, nd.in_seg[L.segh & nd.segmask].ready);
        const uint32_t cnt = count_le(nd, L, st, Te);
        publish_W(nd, L, Te + nd.t);     // the firing starts at Te; only its size is pending
        if (Wup > Te || (cnt >= v && early_ok(nd))) {
          d.T = Te; d.n = cnt < v ? cnt : v; d.qlen = count_all_le(nd, L, st, Te); return d;
        }
        wait_up(nd, ph, spins, wd0); waited = true;
        continue;
      }
      const int64_t T = L.m * nd.P;
      const uint32_t cnt = count_le(nd, L, st, T);
      if (Wup > T || (cnt >= v && early_ok(nd))) {
        if (cnt > 0) { d.T = T; d.n = cnt < v ? cnt : v; d.qlen = count_all_le(nd, L, st, T); return d; }
        if (!any && Wup == PL_INF64) { d.done = true; return d; }
        const int64_t r = any ? nd.in_seg[L.segh & nd.segmask].ready : Wup;
        int64_t m2 = cdiv(r, nd.dP);
        if (m2 < L.m + 1) m2 = L.m + 1;
        const int64_t me = nd.eager ? min(m2, nd.Mcap) : m2;   // R-DRAIN: no slots at or after A_last
        if (me > L.m) L.empties += (uint64_t)(me - L.m);
        L.m = m2;
        publish_W(nd, L, (nd.eager && L.m >= nd.Mcap ? max(max(nd.B_per, L.B), nd.A_last) : L.m * nd.P) + nd.t);
        spins = 0;
        continue;
      }
      publish_W(nd, L, T + nd.t);
      wait_up(nd, ph, spins, wd0); waited = true;
      continue;
    }
    // THRESHOLD_SLACK
    if (!any) {
      if (Wup == PL_INF64) { d.done = true; return d; }
      const int64_t lb = Wup > L.B ? Wup : L.B;
      publish_W(nd, L, lb + nd.t);
      if (nap_to(nd, T0, lb, napped)) { waited = true; spins = 0; continue; }
      wait_up(nd, ph, spins, wd0); waited = true;
      continue;
    }
    const Seg& hs = nd.in_seg[L.segh & nd.segmask];
    fence_q(nd.cl);
    const uint2 he = load_entry(nd, L.head, L.segh, st, vld(&nd.Ein->spill_end));
    int64_t Tf = nd.arrival(he.x) + nd.D - nd.R;
    if (Tf < hs.ready) Tf = hs.ready;
    const uint32_t kth = L.head + nd.theta - 1;
    const bool th_known = (int32_t)(tail_known - kth) > 0;
    int64_t Tth = PL_INF64;
    if (th_known) {
      for (uint32_t k = L.segh; k != st; ++k) {
        const Seg& sg = nd.in_seg[k & nd.segmask];
        if ((int32_t)(sg.end - kth) > 0) { Tth = sg.ready; break; }
      }
    }
    int64_t Tk = Tth < Tf ? Tth : Tf;
    if (Tk < L.B) Tk = L.B;
    if (nd.eager) Tk = min(Tk, max(max(L.B, nd.A_last), hs.ready));   // R-DRAIN
    if (th_known || Tk < Wup) {
      const uint32_t cnt = count_le(nd, L, st, Tk);
      if (Wup > Tk || (cnt >= v && early_ok(nd))) {
        d.T = Tk; d.n = cnt < v ? cnt : v; d.qlen = count_all_le(nd, L, st, Tk);
        // committed: nothing leaves this node before Tk + t_i.  Publish it now -- a physical
        // firing may be paced far into the future (slack) and downstream must not wait for it.
        publish_W(nd, L, Tk + nd.t);
        return d;
      }
    }
    int64_t lb = Tk < Wup ? Tk : Wup;
    if (lb < L.B) lb = L.B;
    publish_W(nd, L, lb + nd.t);
    if (nap_to(nd, T0, lb, napped)) { waited = true; spins = 0; continue; }
    wait_up(nd, ph, spins, wd0); waited = true;
  }
}

// Reserve room for `worst` outputs on the output edge (worst case n*u, decided before the
// stage runs so that no extra barrier is needed).  Returns the location.  A full queue
// back-pressures the producer in both clock modes (deadlock-free):
// in physical mode the wait shows up as lateness and, if it matters, as deadline misses.
__device__ __forceinline__ uint32_t reserve_out(const Node& nd, Leader& L, uint32_t worst, uint32_t* stalled) {
  int spins = 0;
  uint64_t wd0 = 0;
  for (;;) {
    if (spins < 0) { L.wd = 2u; return ~0u; }   // watchdog: outputs dropped
    const uint32_t h = vld(&nd.Eout->head), sh = vld(&nd.Eout->seg_head);
    const bool seg_ok = (L.out_segt - sh) <= nd.segmask;
    const uint32_t need = L.out_tail + worst - h;
    if (seg_ok && need <= nd.out_cap) { if (*stalled) vst(&nd.Eout->stalled, 0u); return LOC_SMEM; }
    if (seg_ok && need <= nd.capg) { if (*stalled) vst(&nd.Eout->stalled, 0u); return LOC_SPILL; }
    if (!*stalled) vst(&nd.Eout->stalled, 1u);
    *stalled = 1u;
    backoff(spins, wd0);
  }
}

__device__ __forceinline__ void pace(uint64_t target, uint64_t* start_ns, int64_t* late, uint64_t* entry_ns = nullptr) {
  uint64_t now = gtimer();
  if (entry_ns) *entry_ns = now;
  while (now < target) {   // __nanosleep sleeps at most 2x its argument: nap rem >> PL_NAP_SHIFT
    const uint64_t rem = target - now;
#if PL_NAP_HALF
    __nanosleep(rem > 256 ? (uint32_t)min(rem >> 1, (uint64_t)(1u << 20)) : 0u);
#else
    __nanosleep(rem > 4096 ? (uint32_t)min(rem >> PL_NAP_SHIFT, (uint64_t)(1u << 20)) : (rem > 1024 ? 256u : (rem > 256 ? 64u : 0u)));
#endif
    now = gtimer();
  }
  *start_ns = now;
  *late = (int64_t)(now - target);
}

// Stall injection (pl_pipeline_inject_stalls; SURVEY §5 fault injection, DESIGN.md R-STALL): the
// platform stops every SM for ~1.6 ms every few seconds (profiles/r02_pause_control.txt).  With
// p.inj_len_ns > 0 a node reaching a firing start inside [T0 + j P, T0 + j P + len), j >= 1,
// sleeps to the window's end -- every node of every stream stops over the same windows, as in
// the platform's stalls, only more often -- so a rate search can demand zero misses across them.
__device__ __noinline__ void inject_stall(const DevParams& p, uint64_t T0) {
  const uint64_t now = gtimer();
  const uint64_t j = (now - T0) / p.inj_period_ns;
  if (j == 0) return;
  const uint64_t we = T0 + j * p.inj_period_ns + p.inj_len_ns;
  if (now < we) nap_until(we);
}
__device__ __forceinline__ void pace_p(const DevParams& p, uint64_t T0, uint64_t target, uint64_t* start_ns,
                                       int64_t* late, uint64_t* entry_ns = nullptr) {
  if (PL_INJECT && p.inj_len_ns) inject_stall(p, T0);
  pace(target, start_ns, late, entry_ns);
}

// exclusive scan of per-lane output counts over the node's v lanes (warp shuffles
// + one named barrier); returns the lane's offset and the group total.
__device__ __forceinline__ uint32_t group_scan(uint32_t* wtot, uint32_t x, uint32_t* total, int gtid, int v, int bid,
                                               bool binary) {
  const int lane = gtid & 31, w = gtid >> 5;
  uint32_t inc;
  if (binary) {   // 0/1 outputs per lane: one ballot instead of five shuffles
    inc = __popc(__ballot_sync(0xffffffffu, x != 0u) & (0xffffffffu >> (31 - lane)));
  } else {
    inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += y;
    }
  }
  if (lane == 31) wtot[w] = inc;
  bar_sync(bid, v);                                                    // B2
  // warp totals: one or two 16-byte shared loads (wtot is 16-byte aligned, 8 slots; the
  // slots of absent warps stay zero from run_node's initialisation)
  const uint4 a = *reinterpret_cast<const uint4*>(wtot);
  uint32_t tot = (a.x + a.y) + (a.z + a.w);
  uint32_t pre = (w > 0 ? a.x : 0u) + (w > 1 ? a.y : 0u) + (w > 2 ? a.z : 0u);
  if (v > 128) {
    const uint4 b = *reinterpret_cast<const uint4*>(wtot + 4);
    tot += (b.x + b.y) + (b.z + b.w);
    pre += (w > 3 ? a.w : 0u) + (w > 4 ? b.x : 0u) + (w > 5 ? b.y : 0u) + (w > 6 ? b.z : 0u);
  }
  *total = tot;
  return pre + inc - x;
}

__device__ __forceinline__ int64_t overlap(int64_t s, int64_t e, int64_t lo, int64_t hi) {
  const int64_t a = s > lo ? s : lo, b = e < hi ? e : hi;
  return b > a ? b - a : 0;
}

__device__ __forceinline__ void bar_arrive(int id, int n) {
  asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory");
}


// K items of one lane through stage KIND (compile-time), written so that the K
// independent items interleave: S0/S1 read their k-mer words from the smem DB window
// with no per-item branch when the whole warp is inside it.
template <int K, int KIND>
__device__ __forceinline__ void stage_batch(const Node& nd, const Dna& dna, const DevParams& p, const uint2 (&e)[K],
                                            const bool (&act)[K], LaneOut (&o)[K]) {
#pragma unroll
  for (int j = 0; j < K; ++j) { o[j].c = 0; o[j].a = 0; o[j].score = 0; o[j].q_start = 0; o[j].len = 0; }
  if constexpr (KIND == PL_SEED_LOOKUP || KIND == PL_HIT_ENUM) {
    uint32_t r[K];
    bool inwin = true;
#pragma unroll
    for (int j = 0; j < K; ++j) {
      r[j] = (e[j].x >> 4) - dna.win_lo32;
      inwin &= r[j] + 1u < dna.win_n;
    }
    uint32_t key[K];
    if (__all_sync(0xffffffffu, inwin)) {
#pragma unroll
      for (int j = 0; j < K; ++j) {
        const uint32_t w = e[j].x >> 4;
        const uint32_t x = __funnelshift_r(dna.win[w & dna.win_mask], dna.win[(w + 1u) & dna.win_mask],
                                           (e[j].x & 15u) * 2u);
        key[j] = dna.kmer_of(x);
      }
    } else {
#pragma unroll
      for (int j = 0; j < K; ++j) key[j] = dna.key(e[j].x);
    }
#pragma unroll
    for (int j = 0; j < K; ++j) {
      const uint32_t lo = dna.qoff[key[j]], hi = dna.qoff[key[j] + 1];
      if (KIND == PL_SEED_LOOKUP) {
        o[j].c = (act[j] && hi > lo) ? 1u : 0u;
      } else {
        const uint32_t cnt = hi - lo;
        o[j].a = lo;
        o[j].c = act[j] ? (cnt < nd.max_out ? cnt : nd.max_out) : 0u;
      }
    }
  } else if constexpr (KIND == PL_BERNOULLI) {
#pragma unroll
    for (int j = 0; j < K; ++j) o[j].c = (act[j] && gain_hash(p.seed, nd.i, e[j].x, e[j].y) < p.st[nd.i].thr[0]) ? 1u : 0u;
  } else if constexpr (KIND == PL_FIXED_GAIN) {
#pragma unroll
    for (int j = 0; j < K; ++j) o[j].c = act[j] ? nd.cfix : 0u;
  } else if constexpr (KIND == PL_KEEP_EVERY) {
#pragma unroll
    for (int j = 0; j < K; ++j) o[j].c = (act[j] && (e[j].x % nd.cfix) == 0) ? 1u : 0u;
  } else if constexpr (KIND == PL_POISSON_CAPPED) {
#pragma unroll
    for (int j = 0; j < K; ++j) {
      const uint64_t h = gain_hash(p.seed, nd.i, e[j].x, e[j].y);
      uint32_t n = 0;
      for (uint32_t q = 0; q < nd.max_out; ++q) n += (h >= p.st[nd.i].thr[q]) ? 1u : 0u;
      o[j].c = act[j] ? n : 0u;
    }
  } else {   // S2 window filter / S3 x-drop: per item, one shared copy of the code
#if PL_S3_COOP
    if (nd.kind == PL_UNGAPPED_XDROP) {   // warp-uniform: the hybrid walk is warp-collective
#pragma unroll
      for (int j = 0; j < K; ++j) o[j] = stage_xdrop_warp(nd, dna, e[j], act[j]);
      return;
    }
#endif
#pragma unroll
    for (int j = 0; j < K; ++j) {
#if PL_S3_DEBUG
      const long long t0 = clock64();
      const bool inw = act[j] && dna.in_win(e[j].x, 1000, 1000);
#endif
      if (act[j]) o[j] = stage_count_ext(nd, dna, e[j]);
#if PL_S3_DEBUG
      const unsigned dt = (unsigned)(clock64() - t0);
      const unsigned mx = __reduce_max_sync(0xffffffffu, dt);
      const unsigned nin = __popc(__ballot_sync(0xffffffffu, inw));
      const unsigned nact = __popc(__ballot_sync(0xffffffffu, act[j]));
      if (nd.kind == PL_UNGAPPED_XDROP && blockIdx.x == 3 && (threadIdx.x & 31) == 0)
        printf("S3 warp %d: max %u cycles, lane0 %u, active %u, in_win %u\n", threadIdx.x >> 5, mx, dt, nact, nin);
#endif
    }
  }
}

template <int KIND>
__device__ __forceinline__ uint2 stage_output_k(const Node& nd, const Dna& dna, uint2 e, const LaneOut& o, uint32_t j) {
  if constexpr (KIND == PL_FIXED_GAIN) return make_uint2(e.x, e.y * nd.cfix + j);
  else if constexpr (KIND == PL_POISSON_CAPPED) return make_uint2(e.x, e.y * nd.max_out + j);
  else if constexpr (KIND == PL_HIT_ENUM) return make_uint2(e.x, (uint32_t)dna.qpos[o.a + j] | (j << 16));
  else return e;
}

// Physical-clock latency of a terminal item of the previous firing (its end time is that
// firing's publish time), per root: parity runs (PL_REC_LATENCY) only.  The per-stream
// maximum and the deadline misses are evaluated by the leader (run_node, "bookkeeping").
__device__ __forceinline__ void record_lat_ns(const Node& nd, const Ctx& c, uint64_t T0, uint64_t end_ns,
                                              uint32_t& pend_root) {
  const uint64_t a_ns = T0 + units_ns(nd, nd.arrival(pend_root));
  atomicMax((long long*)&c.p->lat_ns[pend_root], (long long)((int64_t)end_ns - (int64_t)a_ns));
  pend_root = NO_ROOT;
}

// Live ingest (pl_pipeline_live_start; a1): node 0 takes a root only once every
// DB word that its descendants can read has been delivered -- up to word (p + k + halo) / 16,
// the extension walks' reach (R-S3) -- so the logical schedule (arrivals a(r) = r tau0) is the
// oracle's and a late delivery shows up as lateness and measured latency, not as a different
// schedule.  Slow path only (the caller checks the cached frontier first); the accountant keeps
// the window sliding while it waits.  A stream that gets no delivery for 20 s proceeds on
// whatever its ring holds and flags PL_ERR_INGEST_TIMEOUT (the run must end).
__device__ __noinline__ void live_gate_slow(Shared& sh, const DevParams& p, unsigned char* win, uint32_t need,
                                            bool acct, bool leader) {
  WinCtl& W = sh.win;
  const uint64_t t0 = gtimer();
  int spins = 0;
  while (live_front(W, need) < need) {
    if (acct) win_step(sh, p, win, false);
    const uint64_t now = gtimer();
    if (now - t0 > PL_INGEST_TIMEOUT_NS) {
      atomicOr(&sh.errors, PL_ERR_INGEST_TIMEOUT);
      atomicMax(&W.front, W.whi);
      break;
    }
    if (++spins > 2) __nanosleep(spins < 16 ? 64 : 256);
  }
  if (leader) {
    sh.ingest_waits++;
    atomicMax(&sh.ingest_max_ns, (uint32_t)min(gtimer() - t0, (uint64_t)0xffffffffu));
  }
}
__device__ __forceinline__ uint32_t live_need(const Shared& sh, const DevParams& p, uint32_t p_last) {
  return min(sh.win.whi, (uint32_t)(((uint64_t)p_last + (uint32_t)p.k + p.win_halo) >> 4) + 1u);
}

// ------------------------------------------------------------------- node loop
// One warp group of v threads per node, one item per lane.  Measured faster on B200 than
// one warp with v/32 items per lane: the group's warps run the per-item latency chains in
// parallel (tools/node_scaling.py; profiles/r01_phase_cycles_*).
// Per firing of node i >= 1: leader decides (+ reserves output room, + paces) -> B1 ->
// lanes load / run the stage / scan (B2) -> leader releases the input slots -> lanes
// compact their outputs -> B4 (arrive; the leader's warp syncs) -> leader publishes the
// segment and its watermark.  Node 0 skips B1: its arrivals are fully known, so every lane
// evaluates the decision itself and the leader's reservation reaches the lanes through
// B2.  Broadcast slots are double-buffered by firing parity.
// REC: per-item records compiled in (parity / tracing runs); the bench kernel has none.
// (A separate node-0 instantiation was measured: faster alone, 1.33x slower with all nodes
// running -- the SM's instruction cache holds one ~76 KB node loop, not two.)
// LIVE: the live-ingest instantiation (node 0 gates its firings on delivered words); the other
// kernels do not carry that code (the node loop is instruction-cache bound: tools/bisect_fire.py)
template <bool REC, bool CL, bool LIVE = false>
__device__ void run_node(Ctx& c, Dna dna, int i, int gtid) {
  const DevParams& p = *c.p;
  const Node nd = make_node<CL>(c, i);
  const int v = nd.v, N = nd.N;
  const bool n0 = i == 0;
  const bool leader = gtid == 0;
  const int bidA = 1 + i;
  const int bidB = (i < 7) ? 9 + i : bidA;       // barrier ids 9..15 for the output barrier
  GroupCtl& G = c.sh->g[i];
  const uint32_t stream = c.stream;
  Shared& AG = CL ? *c.agg : *c.sh;      // the stream's aggregates (N4: rank 0's, over DSMEM)
  const uint32_t rec = REC ? p.flags : (p.flags & PL_FIXED_SERVICE);
  const uint64_t T0 = c.sh->T0;
  NodeAcc& A = c.sh->acc[i];
  const uint32_t lt_mask = (1u << (gtid & 31)) - 1u;

  Leader L;
  L.m = 0; L.B = 0; L.c0 = 0; L.head = 0; L.segh = 0; L.out_tail = 0; L.out_segt = 0;
  L.W_pub = -1; L.empties = 0; L.wd = 0;
  Rep R;
  R.m = 0; R.B = 0; R.c0 = 0; R.empties = 0; R.qT = 0; R.rT = 0; R.qvalid = false;
  auto clamp32 = [](int64_t x) { return (uint32_t)(x > 0 ? (x < 0xffffffffll ? x : 0xffffffffll) : 0); };
  uint64_t start_ns = 0;
  uint32_t pend_root = NO_ROOT;          // lane: physical terminal event awaiting its end time (REC)
  long long tc = 0;
  int par = 0;
  if (leader) {
    G.end_ns[0] = 0; G.end_ns[1] = 0;
    for (int k = 0; k < 8; ++k) { G.wtot[0][k] = 0; G.wtot[1][k] = 0; }
    for (int k = 0; k < C_N; ++k) A.cnt[k] = 0;
    for (int k = 0; k < 6; ++k) A.ph[k] = 0;
    for (int k = 0; k < D_N; ++k) { A.d[0][k] = 0; A.d[1][k] = 0; }
    for (int k = 0; k < 8; ++k) { G.rmin[k] = NO_ROOT; G.rmax[k] = 0u; }   // absent warps keep these
    A.t_end = 0;
    A.max_queue = A.lateness = A.max_fire = A.lmax = A.lmax_ns = A.nmiss = A.nmiss_ns = A.max_loop = 0;
  }

  for (;;) {
    int64_t T;
    uint32_t n, head;                    // n: items consumed (node 0 with arrival data: from the scan)
    if (n0) {
      const long long c0 = leader ? clock64() : 0;
      const Decision d = decide0(nd, R);
      if (d.done) break;
      T = d.T; n = d.n; head = (uint32_t)R.c0;
      if (LIVE && PL_LIVE_GATE && n) {   // live ingest: the firing's DB words must have been delivered
        const uint32_t last = (uint32_t)min((int64_t)head + n, nd.X) - 1u;
        const uint32_t need = live_need(*c.sh, p, (uint32_t)(nd.lo + last));
        if (vld(&c.sh->win.front) < need)
          live_gate_slow(*c.sh, p, (unsigned char*)dna.win, need, v > 32 ? gtid == 32 : leader, leader);
      }
      if (leader) {
        uint32_t ql = d.qlen;
        if (nd.arr) {                    // arrival data: roots arrived by T (binary search), not yet consumed
          int64_t a = R.c0, b = nd.X;    // first local root with arrival > T
          while (a < b) {
            const int64_t mid = (a + b) >> 1;
            if (__ldg(nd.arr + nd.lo + mid) <= T) a = mid + 1; else b = mid;
          }
          ql = (uint32_t)(a - R.c0);
        }
        atomicMax(&A.max_queue, ql);
        publish_W(nd, L, T + nd.t);      // committed: nothing leaves node 0 before T + t_0
        if (rec & PL_REC_FIRINGS) G.log_idx[par] = atomicAdd(&AG.log_count, 1u);
        A.d[par][D_STALL] = 0;
        G.out_loc[par] = nd.sink ? LOC_SMEM : reserve_out(nd, L, n * nd.umax, &A.d[par][D_STALL]);
        G.out_base[par] = L.out_tail;
        tc = clock64();
        A.d[par][D_PH0] = (uint32_t)(tc - c0);
      }
      if (nd.phys && (p.variant & 1u)) {  // the leader paces, one barrier releases the lanes
        if (leader) {
          int64_t late;
          uint64_t entry;
          const uint64_t prev = start_ns;
          pace_p(p, T0, T0 + units_ns(nd, T), &start_ns, &late, &entry);
          atomicMax(&A.lateness, clamp32(late));
          if (prev) atomicMax(&A.max_loop, clamp32((int64_t)(entry - prev)));
        }
        bar_sync(bidA, v);
        if (leader) tc = clock64();
      } else if (nd.phys && (gtid & 31) == 0) {   // every warp paces itself against %globaltimer
        uint64_t s_ns, entry; int64_t late;
        pace_p(p, T0, T0 + units_ns(nd, T), &s_ns, &late, &entry);
        if (leader) {
          if (start_ns) atomicMax(&A.max_loop, clamp32((int64_t)(entry - start_ns)));
          start_ns = s_ns; atomicMax(&A.lateness, clamp32(late)); tc = clock64();
        }
      }
      __syncwarp();
    } else {
      if (leader) {
        const long long c0 = clock64();
        bool waited = false;             // the decision waited for upstream (no service-time sample)
        const Decision d = decide(nd, L, waited, T0);
        atomicMax(&A.max_queue, d.qlen);
        G.done[par] = d.done ? 1u : 0u;
        G.T[par] = d.T;
        G.n[par] = d.n;
        G.head[par] = L.head;
        G.segh[par] = L.segh;
        G.st[par] = vld(&nd.Ein->seg_tail);
        fence_q(nd.cl);
        G.in_spill_end[par] = vld(&nd.Ein->spill_end);
        if (!d.done) {
          if (rec & PL_REC_FIRINGS) G.log_idx[par] = atomicAdd(&AG.log_count, 1u);
          A.d[par][D_STALL] = 0;
          G.out_loc[par] = nd.sink ? LOC_SMEM : reserve_out(nd, L, d.n * nd.umax, &A.d[par][D_STALL]);
          G.out_base[par] = L.out_tail;
        } else {
          publish_W(nd, L, PL_INF64);
        }
        tc = clock64();
        A.d[par][D_PH0] = (uint32_t)(tc - c0);
        if (!d.done && nd.phys) {
          int64_t late;
          uint64_t entry;
          const uint64_t prev = start_ns;
          pace_p(p, T0, T0 + units_ns(nd, d.T), &start_ns, &late, &entry);
          atomicMax(&A.lateness, clamp32(late));
          if (prev && !waited) atomicMax(&A.max_loop, clamp32((int64_t)(entry - prev)));
          tc = clock64();
        }
      }
      bar_sync(bidA, v);                                               // B1: decision
      if (leader) { const long long t2 = clock64(); A.d[par][D_PH1] = (uint32_t)(t2 - tc); tc = t2; }
      if (REC && pend_root != NO_ROOT)   // deferred physical latency of the previous firing
        record_lat_ns(nd, c, T0, G.end_ns[par ^ 1], pend_root);
      if (G.done[par]) break;
      T = G.T[par]; n = G.n[par]; head = G.head[par];
    }
    const bool arrmode = n0 && nd.arr != nullptr;
    // the item this lane serves: lane order, or -- the sink, whose outputs carry no order (matches,
    // terminal latencies) -- dealt round-robin over its warps, so that a partial vector's long
    // extension walks spread over every SMSP instead of filling the first warps (PL_SINK_SPREAD)
    const uint32_t jt = (PL_SINK_SPREAD && nd.sink && !n0 && v > 32)
                            ? (uint32_t)((gtid & 31) * (v >> 5) + (gtid >> 5)) : (uint32_t)gtid;
    const bool act = arrmode ? ((uint32_t)gtid < n && R.c0 + gtid < nd.X &&
                                __ldg(nd.arr + nd.lo + R.c0 + gtid) <= T)
                             : jt < n;
    uint2 e[1];
    const bool acts[1] = {act};
    LaneOut o[1];
    {
      const uint32_t ld = act ? jt : 0u;   // inactive lanes repeat a valid entry
      if (n0) e[0] = make_uint2((uint32_t)(nd.lo + head + ld), 0u);
      else e[0] = load_entry(nd, head + ld, G.segh[par], G.st[par], G.in_spill_end[par]);
    }
    if (nd.sliding) {                    // the window's current range, and this node's bound
      win_snap(dna, *c.sh);
      if (leader && act && !n0) vst(nd.bnd_me, e[0].x);   // the firing's first (smallest) root
    }
    {   // warp-uniform dispatch to the stage body: direct compare-and-branch chain (a switch
        // compiles to an indirect BRX, measured ~200 cycles per dispatch)
      const uint32_t kd = nd.kind;
      if (kd == PL_SEED_LOOKUP) stage_batch<1, PL_SEED_LOOKUP>(nd, dna, p, e, acts, o);
      else if (kd == PL_HIT_ENUM) stage_batch<1, PL_HIT_ENUM>(nd, dna, p, e, acts, o);
      else if (kd == PL_UNGAPPED_WINDOW || kd == PL_UNGAPPED_XDROP)
        stage_batch<1, PL_UNGAPPED_WINDOW>(nd, dna, p, e, acts, o);   // S2 / S3
      else if (kd == PL_BERNOULLI) stage_batch<1, PL_BERNOULLI>(nd, dna, p, e, acts, o);
      else if (kd == PL_FIXED_GAIN) stage_batch<1, PL_FIXED_GAIN>(nd, dna, p, e, acts, o);
      else if (kd == PL_KEEP_EVERY) stage_batch<1, PL_KEEP_EVERY>(nd, dna, p, e, acts, o);
      else stage_batch<1, PL_POISSON_CAPPED>(nd, dna, p, e, acts, o);
    }
    uint32_t total;
    uint32_t off;
    if (arrmode) {   // count the arrived items in the same scan: (items << 16) | outputs
      uint32_t packed;
      const uint32_t ex = group_scan(G.wtot[par], ((act ? 1u : 0u) << 16) | o[0].c, &packed, gtid, v, bidA, false);
      off = ex & 0xffffu;
      total = packed & 0xffffu;
      n = packed >> 16;
    } else {
      off = group_scan(G.wtot[par], o[0].c, &total, gtid, v, bidA, nd.umax <= 1);                 // B2
    }
    const uint32_t out_loc = G.out_loc[par], out_base = G.out_base[par];   // leader's reservation (B2)
    if (nd.sliding && n0 && leader) vst(nd.bnd_me, (uint32_t)(nd.lo + head));   // every lane is past the last firing
    if (leader) { const long long t2 = clock64(); A.d[par][D_PH2] = (uint32_t)(t2 - tc); tc = t2; }
    if (REC && n0 && pend_root != NO_ROOT)   // node 0: the previous publish time came through B2
      record_lat_ns(nd, c, T0, G.end_ns[par ^ 1], pend_root);
    // --- release the input slots (every lane has loaded its entry: B2 passed)
    if (leader && !n0) {
      L.head = head + n;
      const uint32_t st = G.st[par];
      while (L.segh != st && (int32_t)(nd.in_seg[L.segh & nd.segmask].end - L.head) <= 0) ++L.segh;
      fence_q(nd.cl);
      vst(&nd.Ein->head, L.head);
      vst(&nd.Ein->seg_head, L.segh);
    }
    // --- per-item records: terminal events (reading R-DONE), trace, log
    const uint2 ei = e[0];
    const LaneOut oi = o[0];
    const bool term = act && (nd.sink || oi.c == 0);
    if (REC && (rec & 7u)) {              // optional per-item records (parity / tracing runs)
      if (act && (rec & PL_REC_TRACE)) {
        atomicAdd(&p.trace[(uint64_t)ei.x * (N + 1) + i], 1u);
        if (nd.sink && oi.c) atomicAdd(&p.trace[(uint64_t)ei.x * (N + 1) + N], oi.c);
      }
      if (term && (rec & PL_REC_LATENCY)) {
        atomicMax((long long*)&p.lat[ei.x], (long long)(T + nd.t - nd.arrival(ei.x)));
        if (nd.phys) pend_root = ei.x;
      }
      if (act && (rec & PL_REC_FIRINGS) && (jt == 0 || jt == n - 1)) {
        const uint32_t li = G.log_idx[par];
        if (li < p.log_cap) {
          pl_firing* f = p.flog + (uint64_t)stream * p.log_cap + li;
          if (jt == 0) { f->start = T; f->node = i; f->n = n; f->first_root = ei.x; f->stream = stream; f->pad = 0; }
          if (jt == n - 1) f->last_root = ei.x;
        } else if (jt == 0) {
          atomicOr(&AG.errors, PL_ERR_LOG_OVERFLOW);
        }
      }
    }
    {   // latency bookkeeping, off the firing's path: arrivals are non-decreasing in root order
        // (L63, or sorted arrival data), so the firing's largest latency is that of its smallest
        // terminal root.  The lanes leave their terminal roots in smem; the leader evaluates
        // them after the publish (and counts misses root by root only when one exceeds D).
      const uint32_t tr = term ? ei.x : NO_ROOT;
      nd.troot[gtid] = tr;
      const uint32_t wmin = __reduce_min_sync(0xffffffffu, tr);
      if ((gtid & 31) == 0) G.rmin[gtid >> 5] = wmin;
      if (nd.phys) {                     // the latest-arriving terminal root: smallest logical latency
        const uint32_t wmax = __reduce_max_sync(0xffffffffu, term ? ei.x + 1u : 0u);
        if ((gtid & 31) == 0) G.rmax[gtid >> 5] = wmax;
      }
    }
    if (nd.sink && nd.kind == PL_UNGAPPED_XDROP) {   // matches: one global atomic per warp
      const bool hit = act && oi.c;
      const uint32_t mb = __ballot_sync(0xffffffffu, hit);
      if (mb) {
        unsigned long long base = 0;
        if ((gtid & 31) == 0) base = atomicAdd(p.match_count, (unsigned long long)__popc(mb));
        base = __shfl_sync(0xffffffffu, base, 0);
        if (hit) {
          const unsigned long long mi = base + __popc(mb & lt_mask);
          if (mi < p.match_cap) {
            pl_match mt;
            mt.p = ei.x; mt.q = ei.y & 0xffffu; mt.db_start = oi.a; mt.q_start = oi.q_start;
            mt.len = oi.len; mt.score = oi.score;
            p.matches[mi] = mt;
          } else {
            atomicOr(&AG.errors, PL_ERR_MATCH_OVERFLOW);
          }
        }
      }
    }
    if (leader) { const long long t2 = clock64(); A.d[par][D_PH3] = (uint32_t)(t2 - tc); tc = t2; }
    // --- compaction into the next queue (stable: lane order, then child order)
    if (!nd.sink && act && oi.c && out_loc != ~0u) {
      const uint32_t base = out_base + off;
      if (nd.umax <= 1 && nd.kind != PL_HIT_ENUM) {   // one output, the entry itself (S0, S2, Bernoulli, ...)
        if (out_loc == LOC_SMEM) nd.out_ent[base & (nd.out_cap - 1)] = ei;
        else __stcg(nd.out_spill + (base & (nd.capg - 1)), ei);
      } else for (uint32_t j = 0; j < oi.c; ++j) {
        const uint32_t s = base + j;
        const uint32_t kd = nd.kind;
        const uint2 val = kd == PL_HIT_ENUM ? stage_output_k<PL_HIT_ENUM>(nd, dna, ei, oi, j)
                        : kd == PL_FIXED_GAIN ? stage_output_k<PL_FIXED_GAIN>(nd, dna, ei, oi, j)
                        : kd == PL_POISSON_CAPPED ? stage_output_k<PL_POISSON_CAPPED>(nd, dna, ei, oi, j) : ei;
        if (out_loc == LOC_SMEM) nd.out_ent[s & (nd.out_cap - 1)] = val;
        else __stcg(nd.out_spill + (s & (nd.capg - 1)), val);
      }
    }
    // B4: outputs written.  The leader's warp and the accountant's warp sync, the others only
    // arrive; node 7 (no spare barrier id) syncs fully, since arrivals for B4 and the next B1
    // must not meet on one barrier instance.
    if (gtid < 64 || bidB == bidA) bar_sync(bidB, v);
    else bar_arrive(bidB, v);
    if (leader) {   // publish (the critical path to the next firing), then the leader's own sums
      long long t4 = clock64();
      const uint32_t ph4 = (uint32_t)(t4 - tc);
      // the leader's sums are loaded first and the statistics stored after the publish's
      // fences: a fence waits for the thread's outstanding shared-memory operations, so an
      // atomic or a read-modify-write ahead of it would sit on the critical path
      ulonglong2* Cp = reinterpret_cast<ulonglong2*>(A.cnt);
      ulonglong2* Pp = reinterpret_cast<ulonglong2*>(A.ph);
      ulonglong2 c2 = Cp[2], p2 = Pp[2];
      uint64_t en = 0, fire = 0;
      if (nd.phys) {
        en = gtimer();
        fire = en - start_ns;
        // PL_FIXED_SERVICE: time-triggered delivery -- the firing holds its processor and delivers
        // its terminal items at start + t_i (L69), or when done if later.  Its outputs are
        // published now: downstream consumes them at logical times >= T + t_i anyway (the
        // segment's ready time), and an early publish only lets its scheduler decide sooner.
        if (rec & PL_FIXED_SERVICE) en = max(en, T0 + units_ns(nd, T + nd.t));
      }
      // publish: the segment (outputs ready at T + t_i), then the watermark
      if (!nd.sink && total > 0 && out_loc != ~0u) {
        Seg sg;
        sg.ready = T + nd.t;
        sg.end = L.out_tail + total;
        sg.loc = out_loc;
        nd.out_seg[L.out_segt & nd.segmask] = sg;
        if (out_loc == LOC_SPILL) vst(&nd.Eout->spill_end, sg.end);
        fence_q(nd.cl);
        ++L.out_segt;
        L.out_tail += total;
        vst(&nd.Eout->seg_tail, L.out_segt);
        vst(&nd.Eout->tail, L.out_tail);
        pub_signal(nd);
      }
      if (nd.fixed) {
        ++L.m;
        const bool ef = nd.eager && T >= nd.A_last;   // an R-DRAIN firing: busy until T + t_i
        if (ef) L.B = T + nd.t;
        const int64_t mn = n0 ? R.m + 1 : L.m;
        const int64_t Bn = ef ? T + nd.t : (n0 ? R.B : L.B);
        publish_W(nd, L, (nd.eager && mn >= nd.Mcap ? max(max(nd.B_per, Bn), nd.A_last) : mn * nd.P) + nd.t);
      } else {
        L.B = T + nd.t;
        publish_W(nd, L, L.B + nd.t);
      }
      if (nd.phys) {
        G.end_ns[par] = en;
        atomicMax(&A.max_fire, clamp32((int64_t)fire));
      }
      // measured busy time, overruns, publish-phase cycles (the leader's slots of the sums)
      c2.x += nd.phys ? (en - start_ns) : 0ull;
      c2.y += (nd.phys && (int64_t)fire > nd.t_ns) ? 1ull : 0ull;   // work outlasted t_i
      p2.x += ph4;
      p2.y += (uint64_t)(clock64() - t4);
      Cp[2] = c2; Pp[2] = p2;
    }
    // The accountant (lane 0 of the node's second warp; the leader when v = 32) books the
    // firing off the leader's path: the lanes' troot / rmin stores and the leader's phase
    // deltas A.d[par] were ordered before B4, and the next writes of each come after this
    // warp has reached the next firing's scan barrier (A.d is double-buffered by parity).
    if (v > 32 ? gtid == 32 : leader) {
      uint64_t en = nd.phys ? gtimer() : 0ull;   // completion time of the terminal items
      if (nd.phys && (rec & PL_FIXED_SERVICE)) en = max(en, T0 + units_ns(nd, T + nd.t));   // delivery at start + t_i
      A.t_end = T + nd.t;                // firing starts increase: the last one ends last
      // the smallest terminal root has the largest latency
      uint32_t rmin;
      {
        const uint4 a = *reinterpret_cast<const uint4*>(G.rmin);
        rmin = min(min(a.x, a.y), min(a.z, a.w));
        if (v > 128) {
          const uint4 b = *reinterpret_cast<const uint4*>(G.rmin + 4);
          rmin = min(rmin, min(min(b.x, b.y), min(b.z, b.w)));
        }
      }
      if (rmin != NO_ROOT) {
        const int64_t ar = nd.arrival(rmin);
        const int64_t lat = T + nd.t - ar;
        atomicMax(&A.lmax, clamp32(lat));
        if (lat > nd.D) {                // a miss in this firing: count the late items exactly
          uint32_t m = 0;
          for (int k = 0; k < v; ++k) {
            const uint32_t r = nd.troot[k];
            if (r != NO_ROOT && T + nd.t - nd.arrival(r) > nd.D) ++m;
          }
          atomicAdd(&A.nmiss, m);
        }
        if (nd.phys) {
          const int64_t l = (int64_t)en - (int64_t)(T0 + units_ns(nd, ar));
          atomicMax(&A.lmax_ns, clamp32(l));
          if (l > nd.D_ns) {
            uint32_t m = 0;
            for (int k = 0; k < v; ++k) {
              const uint32_t r = nd.troot[k];
              if (r != NO_ROOT && (int64_t)en - (int64_t)(T0 + units_ns(nd, nd.arrival(r))) > nd.D_ns) ++m;
            }
            atomicAdd(&A.nmiss_ns, m);
          }
          // north_star: every item's measured latency within 5 % of the logical-clock prediction
          // T + t_i - a(r) (floor PL_AGREE_FLOOR_NS, DESIGN.md R-AGREE).  A firing's terminal items
          // complete together, so the error is common to them -- with PL_FIXED_SERVICE they are
          // delivered at max(done, start + t_i), the paper's fixed service time (L69) -- and its
          // relative size is largest for the latest-arriving terminal root.
          uint32_t rx;
          {
            const uint4 a = *reinterpret_cast<const uint4*>(G.rmax);
            rx = max(max(a.x, a.y), max(a.z, a.w));
            if (v > 128) {
              const uint4 b = *reinterpret_cast<const uint4*>(G.rmax + 4);
              rx = max(rx, max(max(b.x, b.y), max(b.z, b.w)));
            }
          }
          const int64_t due = (int64_t)(T0 + units_ns(nd, T + nd.t));
          const int64_t err = (int64_t)en > due ? (int64_t)en - due : due - (int64_t)en;
          const int64_t lsmall = (int64_t)units_ns(nd, T + nd.t - nd.arrival(rx - 1u));
          atomicMax(&AG.agr_ppm, clamp32((int64_t)((float)err * 1e6f / (float)(lsmall > 0 ? lsmall : 1))));
          // count the items outside the band exactly -- with PL_FIXED_SERVICE only, where the model's
          // completion time is realised and outliers are rare (in publish mode a firing completes
          // early by design and the count would cost a pass over the lanes on every firing)
          if ((rec & PL_FIXED_SERVICE) && err * 20 > lsmall + 20 * PL_AGREE_FLOOR_NS) {
            uint32_t m = 0;
            for (int k = 0; k < v; ++k) {
              const uint32_t r = nd.troot[k];
              if (r != NO_ROOT && err * 20 > (int64_t)units_ns(nd, T + nd.t - nd.arrival(r)) + 20 * PL_AGREE_FLOOR_NS) ++m;
            }
            atomicAdd(&AG.agr_bad, m);
          }
        }
      }
      {   // fold this firing into the 64-bit sums: one vectorised read-modify-write
        ulonglong2* Cp = reinterpret_cast<ulonglong2*>(A.cnt);
        ulonglong2* Pp = reinterpret_cast<ulonglong2*>(A.ph);
        ulonglong2 c0 = Cp[0], c1 = Cp[1], c3 = Cp[3], c4 = Cp[4], p0 = Pp[0], p1 = Pp[1];
        const uint4 dd = *reinterpret_cast<const uint4*>(A.d[par]);
        const uint32_t stl = A.d[par][D_STALL];
        c0.x += 1ull;
        c0.y += n;
        c1.x += total;
        const unsigned long long ov = (unsigned long long)overlap(T, T + nd.t, 0, nd.H);
        c1.y += ov;
        c4.x += (nd.eager && T >= nd.A_last) ? ov : 0ull;   // R-DRAIN firings (FIXED_WAIT window)
        c4.y += (nd.eager && T >= nd.A_last) ? 1ull : 0ull;
        c3.x += (!nd.sink && out_loc == LOC_SPILL) ? (unsigned long long)total : 0ull;
        c3.y += stl;
        p0.x += dd.x; p0.y += dd.y; p1.x += dd.z; p1.y += dd.w;
        Cp[0] = c0; Cp[1] = c1; Cp[3] = c3; Cp[4] = c4; Pp[0] = p0; Pp[1] = p1;
      }
      if ((CL || n0) && nd.sliding) win_step(*c.sh, p, (unsigned char*)dna.win, false);   // slide the DB window
    }
    __syncwarp();                        // the leader's and the accountant's warps reconverge (bar.sync is .aligned)
    if (n0) {                            // replicated node-0 state, identical in every lane
      R.c0 += n;
      if (nd.fixed) {
        advance0(nd, R);
        if (nd.eager && T >= nd.A_last) R.B = T + nd.t;   // R-DRAIN: busy until
      } else {
        R.B = T + nd.t;
      }
    }
    par ^= 1;
  }
  if (nd.sliding && leader) vst(nd.bnd_me, 0xffffffffu);   // reads nothing more
  if (leader && L.wd) atomicOr(&AG.errors, PL_ERR_WATCHDOG);
  if (n0) {
    if (leader) publish_W(nd, L, PL_INF64);   // after the last segment was published
    bar_sync(bidA, v);                   // the last publish time is visible to every lane
    if (REC && pend_root != NO_ROOT) record_lat_ns(nd, c, T0, G.end_ns[par ^ 1], pend_root);
  }
  if (leader) {
    if (A.lmax) atomicMax(&AG.max_lat, A.lmax);
    if (A.lmax_ns) atomicMax(&AG.max_lat_ns, A.lmax_ns);
    if (A.nmiss) atomicAdd(&AG.miss_events, A.nmiss);
    if (A.nmiss_ns) atomicAdd(&AG.miss_events_ns, A.nmiss_ns);
    CtaStats& S = p.stats[stream];
    S.firings[i] = A.cnt[C_FIRINGS];
    S.empty[i] = n0 ? R.empties : L.empties;
    S.consumed[i] = A.cnt[C_CONSUMED];
    S.produced[i] = A.cnt[C_PRODUCED];
    S.active_ne[i] = (int64_t)A.cnt[C_ACTIVE];
    if (nd.fixed) {   // every time-triggered firing m P_i < H is charged, empty or not (L97, R-WINDOW);
                      // with R-DRAIN only the slots m P_i < A_last, plus the drain firings
      const int64_t H = nd.H, P = nd.P, t = nd.t;
      const int64_t K = nd.eager ? min(H / P, nd.Mcap - 1) : H / P;
      S.active_win[i] = K < 0 ? 0 : K * t + min(t, H - K * P);
      if (nd.eager) S.active_win[i] += (int64_t)A.cnt[C_ACTIVE_E];
    } else {
      S.active_win[i] = (int64_t)A.cnt[C_ACTIVE];
    }
    S.busy_ns[i] = (int64_t)A.cnt[C_BUSY];
    S.spilled[i] = A.cnt[C_SPILLED];
    S.overruns[i] = A.cnt[C_OVERRUNS];
    S.stalls[i] = A.cnt[C_STALLS];
    S.drain_firings[i] = A.cnt[C_DRAINF];
    S.max_queue[i] = A.max_queue;
    S.lateness[i] = (int64_t)A.lateness;
    S.sched_cycles[i] = A.ph[0];
    S.max_fire_ns[i] = (int64_t)A.max_fire;
    S.max_loop_ns[i] = (int64_t)A.max_loop;
    for (int k = 0; k < 6; ++k) S.phase_cycles[i][k] = A.ph[k];
    atomicMax((long long*)&S.t_end, (long long)A.t_end);
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
  L->off_troot = off;
  off += (uint32_t)p.N * (uint32_t)p.v * 4u;
  L->off_qoff = off;
  const bool dna = p.k > 0;
  off += dna ? (((1u << (2 * p.k)) + 1u) * 2u + 15u) & ~15u : 0u;
  L->off_qpos = off;
  off += dna ? (((uint32_t)(p.q_len - p.k + 1) * 2u) + 15u) & ~15u : 0u;
  // packed query with one 16-byte pad on each side (Dna::extend_win reads one word past an end)
  L->off_qw = off + (dna ? 16u : 0u);
  off += dna ? 32u + ((((uint32_t)(p.q_len + 15) / 16u) * 4u + 15u) & ~15u) : 0u;
  L->off_win = off;
  off += p.win_cap * 4u;
  L->off_s2 = off;                // S2 table (Dna::s2_best8): 256 bytes
  off += dna ? 256u : 0u;
  L->off_xt = off;                // S3 transition table (PL_S3_TAB): 256 x X entries of 2 bytes
  off += (uint32_t)xtab_X(p) * 512u;
  L->total = off;
  return off;
}

// rank >= 0: N4 (PL_CLUSTER_NODES) -- this CTA is node `rank` of the stream given by its cluster
__device__ void cta_setup(Ctx& c, Shared& sh, unsigned char* dsm, const DevParams& p, int rank = -1) {
  SmemLayout Lo;
  layout_enforced(p, &Lo);
  const uint32_t s = rank >= 0 ? blockIdx.x / (uint32_t)p.N : blockIdx.x, tid = threadIdx.x, nt = blockDim.x;
  c.p = &p;
  c.sh = &sh;
  c.stream = s;
  c.rank = rank;
  c.agg = rank > 0 ? (Shared*)__cluster_map_shared_rank(&sh, 0u) : &sh;
  c.lo = (p.total_roots * s) / (uint64_t)p.n_streams;
  c.hi = (p.total_roots * (s + 1)) / (uint64_t)p.n_streams;
  c.X = (int64_t)(c.hi - c.lo);
  c.H = c.X * p.tau;
  c.dsm = dsm;
  c.dna.db = p.live ? p.ring + (size_t)s * (p.ring_mask + 1u) : p.db;
  c.dna.dbmask = p.live ? p.ring_mask : 0xffffffffu;
  c.dna.nwords = p.db_words;
  c.dna.db_len = p.db_len;
  c.dna.k = p.k;
  c.dna.q_len = p.q_len;
  c.dna.qoff = (const uint16_t*)(dsm + Lo.off_qoff);
  c.dna.qpos = (const uint16_t*)(dsm + Lo.off_qpos);
  c.dna.qw = (const uint32_t*)(dsm + Lo.off_qw);
  c.dna.nqw = (uint32_t)(p.q_len + 15) / 16u;
  c.dna.win = (const uint32_t*)(dsm + Lo.off_win);
  c.dna.win_lo = 0;
  c.dna.win_lo32 = 0;
  c.dna.win_n = 0;
  c.dna.win_mask = p.win_cap ? p.win_cap - 1u : 0u;
  c.sliding = false;
  if (s == 0 && tid < 8 && p.summary_next) p.summary_next[tid] = 0ull;   // the next launch's summary slot
  c.dna.nofast = (p.variant & 16u) != 0;
  c.dna.s2tab = dsm + Lo.off_s2;
  {
    const int XT = xtab_X(p);
    c.dna.xtab = (const uint16_t*)(dsm + Lo.off_xt);
    c.dna.xtab_X = XT;
    for (uint32_t m = tid; m < 256u * (uint32_t)XT; m += nt)
      ((uint16_t*)(dsm + Lo.off_xt))[m] = Dna::xdrop_tab_entry(m >> 8, m & 255u, XT);
  }
  if (p.k > 0)   // S2 table: max(0, max prefix) of the 8-step +1/-3 walk, bit e = mismatch at step e+1
    for (uint32_t m = tid; m < 256u; m += nt) {
      int sc = 0, best = 0;
      for (int e = 0; e < 8; ++e) {
        sc += ((m >> e) & 1u) ? -3 : 1;
        best = sc > best ? sc : best;
      }
      (dsm + Lo.off_s2)[m] = (unsigned char)best;
    }
  // DNA: the query index (offsets, positions, packed query) and the first chunks of this
  // stream's DB window (its roots plus the k-1 overlap and a halo for the extensions) are
  // staged into smem by TMA bulk copies (cp.async.bulk, one mbarrier), falling back to plain
  // loads for an unaligned caller-owned DB.  A stream longer than the ring slides it (win_step).
  if (p.k > 0) {
    const uint32_t nko = (1u << (2 * p.k)) + 1u, nqp = (uint32_t)(p.q_len - p.k + 1);
    const uint32_t nqw = (uint32_t)(p.q_len + 15) / 16u;
    const uint32_t b_qo = (nko * 2u + 15u) & ~15u, b_qp = (nqp * 2u + 15u) & ~15u, b_qw = (nqw * 4u + 15u) & ~15u;
    int64_t wlo = 0, whi = 0;
    if (p.win_cap > 0 && c.hi > c.lo) {
      wlo = ((int64_t)c.lo - (int64_t)p.win_halo) >> 4;
      whi = (((int64_t)c.hi + p.k + (int64_t)p.win_halo) >> 4) + 1;
      wlo = wlo < 0 ? 0 : (wlo & ~3ll);
      whi = (whi + 3) & ~3ll;
      if (whi > (int64_t)p.db_alloc_words) whi = (int64_t)p.db_alloc_words & ~3ll;
      if (whi < wlo) whi = wlo;
    }
    const uint32_t lg = p.win_lg, K = p.win_cap >> lg;
    const uint32_t c0 = (uint32_t)wlo >> lg;
    const uint32_t c_end = whi > wlo ? (uint32_t)((whi - 1) >> lg) + 1u : c0;
    // without TMA (unaligned DB) the window holds the first K chunks and never slides; live
    // ingest stages nothing up front -- win_step loads every chunk as it is delivered
    const uint32_t c_init = p.live ? c0 : min(c_end, c0 + K);
    const uint32_t hi0 = whi > wlo ? max((uint32_t)wlo, min((uint32_t)whi, c_init << lg)) : (uint32_t)wlo;
    c.sliding = p.db_tma && (c_end > c_init || p.live);
    c.dna.win_lo = wlo;
    c.dna.win_lo32 = (uint32_t)wlo;
    c.dna.win_n = hi0 - (uint32_t)wlo;
    uint32_t* win = (uint32_t*)(dsm + Lo.off_win);
    const bool win_tma = p.db_tma && c.dna.win_n;
    if (tid == 0) {
      WinCtl& W = sh.win;
      W.cov_lo = (uint32_t)wlo;
      W.cov_hi = hi0;
      W.wlo = (uint32_t)wlo;
      W.whi = (uint32_t)whi;
      W.c_next = c.sliding ? c_init : c_end;
      W.c_end = c_end;
      W.inflight = 0;
      W.phase = 0;
      W.loaded_hi = hi0;
      W.refills = 0;
      W.c_first = c0;
      W.a_next = max(c_init << lg, (uint32_t)wlo);
      W.front = (uint32_t)wlo;
      W.pub = (uint32_t)wlo;
      W.src = c.dna.db;
      W.src_mask = c.dna.dbmask;
      W.front_ptr = p.live ? p.front + s : nullptr;
      W.consumed_ptr = p.live ? p.consumed + s : nullptr;
      const uint32_t bar = smem_addr(&sh.mbar);
      const uint32_t bytes = b_qo + b_qp + b_qw + (win_tma ? c.dna.win_n * 4u : 0u);
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(&sh.mbar_w)));
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
      const void* src[3] = {p.qoff, p.qpos, p.qwords};
      const uint32_t off[3] = {Lo.off_qoff, Lo.off_qpos, Lo.off_qw};
      const uint32_t len[3] = {b_qo, b_qp, b_qw};
      for (int j = 0; j < 3; ++j) tma_load(smem_addr(dsm + off[j]), src[j], len[j], bar);
      if (win_tma)   // one copy per chunk: chunk c sits at ring slots (c CH) & mask, contiguous
        for (uint32_t ch = c0; ch < c_init; ++ch) {
          const uint32_t a = max(ch << lg, (uint32_t)wlo), b = min((ch + 1u) << lg, (uint32_t)whi);
          tma_load(smem_addr(dsm + Lo.off_win + (a & (p.win_cap - 1u)) * 4u), p.db + a, (b - a) * 4u, bar);
        }
      uint32_t done = 0;
      while (!done)
        asm volatile("{ .reg .pred q; mbarrier.try_wait.parity.shared::cta.b64 q, [%1], 0; selp.u32 %0, 1, 0, q; }"
                     : "=r"(done) : "r"(bar) : "memory");
    }
    if (tid < 8) {   // the query's pad words (outside the TMA destination)
      uint32_t* qwp = (uint32_t*)(dsm + Lo.off_qw);
      qwp[tid < 4 ? (int)tid - 4 : (int)(b_qw / 4u + tid - 4u)] = 0u;
    }
    if (!win_tma)
      for (uint32_t j = tid; j < c.dna.win_n; j += nt) {
        const int64_t w = wlo + j;
        win[(uint32_t)w & (p.win_cap - 1u)] = w < (int64_t)p.db_words ? p.db[w] : 0u;
      }
  }
  // no node reads below its stream's first root; under N4 this CTA's window serves its own node only
  if (tid < PL_MAX_STAGES) sh.bnd[tid] = (rank < 0 || (int)tid == rank) ? (uint32_t)c.lo : 0xffffffffu;
  if (tid < PL_MAX_STAGES) {
    EdgeCtl& E = sh.e[tid];
    E.head = 0; E.seg_head = 0; E.seg_tail = 0; E.tail = 0; E.W = -1; E.spill_end = 0; E.stalled = 0;
#if PL_PUB_WAIT
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(&E.pub_bar)) : "memory");
#endif
  }
  if (tid == 0) {
    sh.max_lat = 0; sh.max_lat_ns = 0; sh.miss_events = 0; sh.miss_events_ns = 0; sh.errors = 0; sh.log_count = 0;
    sh.agr_bad = 0; sh.agr_ppm = 0; sh.ingest_waits = 0; sh.ingest_max_ns = 0;
  }
  if (rank <= 0) {   // the stream's records and per-stream stats: one CTA of the cluster (N4)
    if (p.flags & PL_REC_LATENCY)
      for (uint64_t r = c.lo + tid; r < c.hi; r += nt) { p.lat[r] = -1; if (p.lat_ns) p.lat_ns[r] = -1; }
    if (p.flags & PL_REC_TRACE)
      for (uint64_t r = c.lo * (p.N + 1) + tid; r < c.hi * (p.N + 1); r += nt) p.trace[r] = 0u;
    if (tid == 0) {
      CtaStats& S = p.stats[s];
      S.n_log = 0;
      S.t_end = 0;
      S.win_refills = 0;
    }
  }
}

__device__ void cta_finish(Ctx& c, Shared& sh, const DevParams& p) {
  if (threadIdx.x == 0 && c.rank >= 0 && p.k > 0)   // N4: every CTA's window refills
    atomicAdd(&p.stats[c.stream].win_refills, sh.win.refills);
  if (threadIdx.x == 0 && c.rank <= 0) {
    CtaStats& S = p.stats[c.stream];
    S.miss_events = sh.miss_events;
    S.miss_events_ns = sh.miss_events_ns;
    S.max_lat = (int64_t)sh.max_lat;
    S.max_lat_ns = (int64_t)sh.max_lat_ns;
    S.wall_ns = (int64_t)(gtimer() - sh.T0);
    S.n_roots = (uint64_t)c.X;
    S.n_log = sh.log_count < p.log_cap ? sh.log_count : p.log_cap;
    S.errors = sh.errors;
    if (c.rank < 0) S.win_refills = p.k > 0 ? sh.win.refills : 0u;
    S.agr_bad = sh.agr_bad;
    S.agr_ppm = sh.agr_ppm;
    S.ingest_waits = sh.ingest_waits;
    S.ingest_max_ns = sh.ingest_max_ns;
    if (p.summary) {                     // device-side reduction for pl_pipeline_summary
      atomicAdd(p.summary + 0, (unsigned long long)c.X);
      atomicAdd(p.summary + 1, (unsigned long long)sh.miss_events);
      atomicMax(p.summary + 2, (unsigned long long)sh.max_lat);
      atomicMax(p.summary + 3, (unsigned long long)sh.max_lat_ns);
      atomicOr(p.summary + 4, (unsigned long long)sh.errors);
      atomicAdd(p.summary + 5, (unsigned long long)sh.miss_events_ns);
      if (sh.agr_bad) atomicAdd(p.summary + 7, (unsigned long long)sh.agr_bad);
    }
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
  int64_t proc_free = 0, t_end = 0, busy_ns = 0;
  const int64_t M = p.M;
  if (c.sliding && tid == 0)             // one processor: only node 0's bound (the block) matters
    for (int i = 1; i < N; ++i) c.sh->bnd[i] = 0xffffffffu;
  for (int64_t b0 = 0; b0 < c.X; b0 += M) {
    const int64_t b1 = (b0 + M < c.X) ? b0 + M : c.X;
    if (c.sliding) {                     // slide the DB window over the block (blocking refills)
      if (tid == 0) {
        vst(&c.sh->bnd[0], (uint32_t)(c.lo + b0));
        const uint32_t need_hi = min(c.sh->win.whi, (uint32_t)(((c.lo + b1 + p.k + p.win_halo) >> 4) + 1));
        if (p.live && vld(&c.sh->win.front) < need_hi)   // live ingest: the block's words must be delivered
          live_gate_slow(*c.sh, p, (unsigned char*)c.dna.win, need_hi, true, true);
        while (vld(&c.sh->win.cov_hi) < need_hi && win_step(*c.sh, p, (unsigned char*)c.dna.win, true)) {}
      }
      __syncthreads();
      win_snap(c.dna, *c.sh);
    }
    const int64_t ready = arrival(c, (uint32_t)(c.lo + b1 - 1));
    int64_t T = ready > proc_free ? ready : proc_free;
    if (phys) {
      if (tid == 0) {
        uint64_t s_ns; int64_t late;
        pace_p(p, c.sh->T0, c.sh->T0 + (uint64_t)((double)ready * p.ns_per_unit), &s_ns, &late);   // the block is complete in real time
        sh_start_ns = s_ns;
      }
      __syncthreads();
    }
    uint2* cur = buf0;
    uint2* nxt = buf1;
    uint32_t ncur = (uint32_t)(b1 - b0);
    for (int i = 0; i < N && ncur > 0; ++i) {
      const bool sink = i == N - 1;
      const Node nd = make_node(c, i);
      const int64_t t_i = p.t[i];
      const uint32_t nf = (ncur + v - 1) / v;
      uint32_t nxt_count = 0;
      for (uint32_t base = 0; base < ncur; base += nt) {
        const uint32_t idx = base + tid;
        const bool act = idx < ncur;
        uint2 e = make_uint2(0u, 0u);
        if (act) e = (i == 0) ? make_uint2((uint32_t)(c.lo + b0 + idx), 0u) : cur[idx];
        LaneOut o;
        if (act) o = stage_count(nd, c.dna, p, e);
        else { o.c = 0; o.a = 0; o.score = 0; o.q_start = 0; o.len = 0; }
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
            atomicMax(&c.sh->max_lat, (uint32_t)(l > 0 ? (l < 0xffffffffll ? l : 0xffffffffll) : 0));
            if (l > p.D) atomicAdd(&c.sh->miss_events, 1u);
            if (phys) {
              const uint64_t a_ns = c.sh->T0 + (uint64_t)((double)arrival(c, e.x) * p.ns_per_unit);
              const int64_t ln = (int64_t)gtimer() - (int64_t)a_ns;
              if (rec & PL_REC_LATENCY) atomicMax((long long*)&p.lat_ns[e.x], (long long)ln);
              atomicMax(&c.sh->max_lat_ns, (uint32_t)(ln > 0 ? (ln < 0xffffffffll ? ln : 0xffffffffll) : 0));
              if ((double)ln > (double)p.D * p.ns_per_unit) atomicAdd(&c.sh->miss_events_ns, 1u);
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
              if (s < p.mono_cap) nxt[s] = stage_output(nd, c.dna, e, o, j);
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
    }
  }
  if (tid == 0) {
    CtaStats& S = p.stats[stream];
    for (int i = 0; i < PL_MAX_STAGES; ++i) {
      S.firings[i] = firings[i]; S.empty[i] = 0; S.consumed[i] = consumed[i]; S.produced[i] = produced[i];
      S.active_ne[i] = active[i]; S.active_win[i] = active[i]; S.busy_ns[i] = i == 0 ? busy_ns : 0;
      S.spilled[i] = 0; S.overruns[i] = 0;
      S.stalls[i] = 0; S.max_queue[i] = 0; S.drain_firings[i] = 0;
      S.lateness[i] = 0; S.sched_cycles[i] = 0; S.max_fire_ns[i] = 0; S.max_loop_ns[i] = 0;
      for (int k = 0; k < 6; ++k) S.phase_cycles[i][k] = 0;
    }
    S.t_end = t_end;
  }
}

}  // namespace

// FIXED_WAIT / THRESHOLD_SLACK executor: grid = n_streams, block = N*32 threads (one warp
// per node); up to 4 CTAs (streams) per SM when N <= 4.
template <int MAXT, int MINB, bool REC, bool LIVE = false>
__global__ void __launch_bounds__(MAXT, MINB) pl_exec_enforced(const __grid_constant__ DevParams p) {
  extern __shared__ __align__(16) unsigned char dsm[];
  __shared__ Shared sh;
  Ctx c;
  cta_setup(c, sh, dsm, p);
  __syncthreads();
  if (threadIdx.x == 0) sh.T0 = gtimer() + (p.clock == PL_CLOCK_GLOBALTIMER ? p.t0_offset_ns : 0u);
  __syncthreads();
  // node i owns warps [i v/32, (i+1) v/32) (contiguous): with v = 128 each node has one warp
  // on every SM sub-partition, so a node's heavy firing (S3's worst vectors) issues from all four
  // SMSPs and node 0's loop shares each SMSP with one warp of every other node.  Measured at the
  // bench point against the interleaved mapping (warp w -> node w % N, one node per SMSP, one
  // code path per SMSP instruction cache; PL_VARIANT bit 4): node-0 lateness at tau0 = 15 ns
  // 2.8 vs 5.4 us, longest node-0 / node-3 firings 1248 / 10656 vs 1376 / 11296 ns.
  const int w = threadIdx.x >> 5;
  const bool contig = !(p.variant & 4u);
  const int gi = contig ? w / (p.v >> 5) : w % p.N;
  const int gt = (contig ? w % (p.v >> 5) : w / p.N) * 32 + (threadIdx.x & 31);
  if (w < p.N * (p.v >> 5)) run_node<REC, false, LIVE>(c, c.dna, gi, gt);
  __syncthreads();
  cta_finish(c, sh, p);
}

// N4 (PL_CLUSTER_NODES, "a fixed 1/N fraction of processor time",
// L265): one stream per cluster of N CTAs, node i = CTA rank i on an SM of its own.  The edge
// into node i (its smem ring, segment records and control words) lives in CTA i's shared memory;
// node i-1 writes its outputs and publishes them there over DSMEM, with cluster-scope fences;
// the stream's aggregates live in rank 0.  Every CTA stages the query index and slides its own
// DB window behind its own node's bound.  grid = n_streams x N CTAs of v threads.
template <bool REC>
__global__ void __launch_bounds__(256, 1) pl_exec_cluster(const __grid_constant__ DevParams p) {
  extern __shared__ __align__(16) unsigned char dsm[];
  __shared__ Shared sh;
  Ctx c;
  const int rank = (int)__clusterRelativeBlockRank();
  cta_setup(c, sh, dsm, p, rank);
  __syncthreads();
  __cluster_barrier_arrive();            // every CTA's queues are initialised before any remote access
  __cluster_barrier_wait();
  if (threadIdx.x == 0 && rank == 0) sh.T0 = gtimer() + (p.clock == PL_CLOCK_GLOBALTIMER ? p.t0_offset_ns : 0u);
  __cluster_barrier_arrive();
  __cluster_barrier_wait();
  if (threadIdx.x == 0 && rank > 0) sh.T0 = vld(&c.agg->T0);   // one time origin per stream
  __syncthreads();
  if ((int)threadIdx.x < p.v) run_node<REC, true>(c, c.dna, rank, (int)threadIdx.x);
  __syncthreads();
  __cluster_barrier_arrive();            // every node is done: rank 0's aggregates are final, and no
  __cluster_barrier_wait();              // CTA leaves while another may still access its smem
  cta_finish(c, sh, p);
}

uint32_t pl_layout_enforced_host(const DevParams& p) {
  SmemLayout L;
  return layout_enforced(p, &L);
}

// MONOLITHIC executor: grid = n_streams, block = any multiple of 32 (N*v by default).
template <int MAXT>
__global__ void __launch_bounds__(MAXT, 1) pl_exec_monolithic(const __grid_constant__ DevParams p) {
  extern __shared__ __align__(16) unsigned char dsm[];
  __shared__ Shared sh;
  Ctx c;
  cta_setup(c, sh, dsm, p);
  __syncthreads();
  if (threadIdx.x == 0) sh.T0 = gtimer() + (p.clock == PL_CLOCK_GLOBALTIMER ? p.t0_offset_ns : 0u);
  __syncthreads();
  run_monolithic(c);
  __syncthreads();
  cta_finish(c, sh, p);
}

// host-side launchers (the kernels are templates on the block-size bound)
cudaError_t pl_launch(const DevParams& p, unsigned grid, unsigned block, unsigned smem, cudaStream_t st) {
  const bool mono = p.policy == PL_MONOLITHIC;
  if (mono) {
    if (block <= 512) pl_exec_monolithic<512><<<grid, block, smem, st>>>(p);
    else pl_exec_monolithic<1024><<<grid, block, smem, st>>>(p);
  } else if (p.flags & PL_CLUSTER_NODES) {   // N4: grid = streams x N CTAs, clusters of N
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = (unsigned)p.N;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.gridDim = dim3(grid * (unsigned)p.N);
    cfg.blockDim = dim3((unsigned)p.v);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    const bool rec = (p.flags & (PL_REC_LATENCY | PL_REC_TRACE | PL_REC_FIRINGS)) != 0;
    cudaError_t e = rec ? cudaLaunchKernelEx(&cfg, pl_exec_cluster<true>, p) : cudaLaunchKernelEx(&cfg, pl_exec_cluster<false>, p);
    if (e != cudaSuccess) return e;
  } else {
    // two CTAs (streams) per SM when the grid asks for more streams than there are SMs and
    // the CTA fits twice (<= 512 threads, 64 registers, smem)
    // per-item records (parity / tracing) select the REC instantiation; the bench runs without
    const bool rec = (p.flags & (PL_REC_LATENCY | PL_REC_TRACE | PL_REC_FIRINGS)) != 0;
    if (p.live) {                        // live ingest: the instantiation with node 0's delivery gate
      if (block <= 512) {
        if (rec) pl_exec_enforced<512, 1, true, true><<<grid, block, smem, st>>>(p);
        else pl_exec_enforced<512, 1, false, true><<<grid, block, smem, st>>>(p);
      } else {
        if (rec) pl_exec_enforced<1024, 1, true, true><<<grid, block, smem, st>>>(p);
        else pl_exec_enforced<1024, 1, false, true><<<grid, block, smem, st>>>(p);
      }
    } else if (block <= 512 && p.ctas_per_sm >= 2) {
      if (rec) pl_exec_enforced<512, 2, true><<<grid, block, smem, st>>>(p);
      else pl_exec_enforced<512, 2, false><<<grid, block, smem, st>>>(p);
    } else if (block <= 512) {
      if (rec) pl_exec_enforced<512, 1, true><<<grid, block, smem, st>>>(p);
      else pl_exec_enforced<512, 1, false><<<grid, block, smem, st>>>(p);
    } else {
      if (rec) pl_exec_enforced<1024, 1, true><<<grid, block, smem, st>>>(p);
      else pl_exec_enforced<1024, 1, false><<<grid, block, smem, st>>>(p);
    }
  }
  return cudaGetLastError();
}

cudaError_t pl_kernel_attributes(unsigned max_smem) {
  cudaError_t e;
  if ((e = cudaFuncSetAttribute(pl_exec_enforced<512, 2, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  if ((e = cudaFuncSetAttribute(pl_exec_enforced<512, 2, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  if ((e = cudaFuncSetAttribute(pl_exec_enforced<512, 1, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  if ((e = cudaFuncSetAttribute(pl_exec_enforced<512, 1, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  if ((e = cudaFuncSetAttribute(pl_exec_enforced<1024, 1, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  if ((e = cudaFuncSetAttribute(pl_exec_enforced<1024, 1, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  if ((e = cudaFuncSetAttribute(pl_exec_enforced<512, 1, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  if ((e = cudaFuncSetAttribute(pl_exec_enforced<512, 1, true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  if ((e = cudaFuncSetAttribute(pl_exec_enforced<1024, 1, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  if ((e = cudaFuncSetAttribute(pl_exec_enforced<1024, 1, true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  if ((e = cudaFuncSetAttribute(pl_exec_cluster<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  if ((e = cudaFuncSetAttribute(pl_exec_cluster<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  if ((e = cudaFuncSetAttribute(pl_exec_monolithic<512>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem))) return e;
  return cudaFuncSetAttribute(pl_exec_monolithic<1024>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem);
}

// ------------------------------------------------------------- stage batch kernels
// K-BENCH (SURVEY K-BENCH; north_star "achieved HBM GB/s of each stage kernel"): one stage over
// a large device-resident batch at full occupancy, with the executor's own stage bodies
// (stage_batch<J, KIND>: J = 4 consecutive items per lane, their latency chains interleaved).
// Each warp takes chunks of 128 consecutive inputs (two coalesced 16-byte loads per lane), scans
// its lanes' output counts with shuffles and reserves its output range with ONE atomic per chunk;
// outputs stay in input order within a chunk.  The DB is the extension's "window" in global
// memory (the whole DB, read-only), so S2 / S3 take the executor's fast in-window walks; only
// seeds within a walk's reach of the DB ends take the checked ones.  Shared memory holds only
// the query index, so several CTAs share an SM.
struct KbLayout { uint32_t qpos, qw, s2, hit, xt, total; };
__host__ __device__ inline KbLayout layout_kbench(const DevParams& p) {
  KbLayout L;
  uint32_t off = 0;
  const bool dna = p.k > 0;
  off += dna ? (((1u << (2 * p.k)) + 1u) * 2u + 15u) & ~15u : 0u;   // qoff at 0
  L.qpos = off;
  off += dna ? (((uint32_t)(p.q_len - p.k + 1) * 2u) + 15u) & ~15u : 0u;
  L.qw = off + (dna ? 16u : 0u);                                     // one 16-byte pad on each side
  off += dna ? 32u + ((((uint32_t)(p.q_len + 15) / 16u) * 4u + 15u) & ~15u) : 0u;
  L.s2 = off;
  off += dna ? 256u : 0u;
  L.hit = off;                                                       // S0: one bit per k-mer (has hits)
  off += dna ? ((((1u << (2 * p.k)) + 31u) / 32u) * 4u + 15u) & ~15u : 0u;
  L.xt = off;                                                        // S3 transitions (PL_S3_TAB)
  off += (uint32_t)xtab_X(p) * 512u;
  L.total = off > 16u ? off : 16u;
  return L;
}
constexpr int KB_THREADS = 256;
constexpr int KB_J = 4;
constexpr int KB_KMAX = 8;
constexpr uint32_t KB_S1_U = 16;   // S1 staging: outputs per input a warp slice holds

// S0 over consecutive roots (K-BENCH fast path; north_star "coalesced 128-bit loads"): a lane
// takes 64 consecutive roots, i.e. 4 DB words loaded as one 16-byte vector plus the next lane's
// first word (a shuffle), rolls the k-mer key base by base (key = (key << 2 | base) mod 4^k,
// the first base most significant as in R-S0) and tests it in a smem bitmap of the k-mers that
// occur in the query (bit set iff qoff[key + 1] > qoff[key]).  Hits become a 64-bit lane mask,
// a shuffle scan and one atomic per warp place them, in root order within the warp's 2048 roots.
// k is a template parameter (4..8; the root index of each base is then a constant) and only a
// lane holding the batch's end checks the root bound.  Requires first_root % 64 == 0 and a
// 16-byte-aligned DB (else the per-item path).
template <int K, bool TAIL>
__device__ __forceinline__ uint64_t s0_roll64(const uint32_t (&wd)[5], const uint32_t* hitbm, uint64_t lim) {
  constexpr uint32_t kmask = (1u << (2 * K)) - 1u;
  uint32_t lo = 0, hi = 0, key = 0;
#pragma unroll
  for (int b = 0; b < 64 + K - 1; ++b) {
    key = ((key << 2) | ((wd[b >> 4] >> ((b & 15) * 2)) & 3u)) & kmask;
    const int j = b - K + 1;                                           // the root whose k-mer ends at base b
    if (j >= 0) {
      const uint32_t bit = (hitbm[key >> 5] >> (key & 31u)) & 1u;
      const uint32_t ok = TAIL ? (bit & ((uint64_t)j < lim ? 1u : 0u)) : bit;
      if (j < 32) lo |= ok << j; else hi |= ok << (j - 32);
    }
  }
  return ((uint64_t)hi << 32) | lo;
}
template <int K>
__device__ __forceinline__ uint64_t s0_roll(const uint32_t (&wd)[5], const uint32_t* hitbm, uint64_t lim) {
  return lim >= 64 ? s0_roll64<K, false>(wd, hitbm, lim) : s0_roll64<K, true>(wd, hitbm, lim);
}

__device__ __forceinline__ void kbench_s0_rolling(const DevParams& p, const uint32_t* hitbm, uint64_t n,
                                                  uint64_t first_root, uint2* out, uint64_t cap,
                                                  unsigned long long* cnt) {
  const int lane = (int)(threadIdx.x & 31u);
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  uint32_t maxc = 0;
  for (uint64_t ch = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; ch * 2048u < n; ch += nw) {
    const long long c0 = clock64();
    const uint64_t j0 = ch * 2048u + (uint64_t)lane * 64u;            // local index of the lane's first root
    const uint64_t r0 = first_root + j0;
    const uint64_t w0 = r0 >> 4;
    uint4 W = make_uint4(0u, 0u, 0u, 0u);
    if (w0 + 3 < p.db_words) W = __ldg(reinterpret_cast<const uint4*>(p.db + w0));
    else {
      if (w0 < p.db_words) W.x = __ldg(p.db + w0);
      if (w0 + 1 < p.db_words) W.y = __ldg(p.db + w0 + 1);
      if (w0 + 2 < p.db_words) W.z = __ldg(p.db + w0 + 2);
    }
    uint32_t nx = __shfl_down_sync(0xffffffffu, W.x, 1);
    if (lane == 31) nx = (w0 + 4 < p.db_words) ? __ldg(p.db + w0 + 4) : 0u;
    const uint32_t wd[5] = {W.x, W.y, W.z, W.w, nx};
    const uint64_t lim = n > j0 ? n - j0 : 0;                          // valid roots of this lane
    uint64_t hits = 0;
    switch (p.k) {
      case 4: hits = s0_roll<4>(wd, hitbm, lim); break;
      case 5: hits = s0_roll<5>(wd, hitbm, lim); break;
      case 6: hits = s0_roll<6>(wd, hitbm, lim); break;
      case 7: hits = s0_roll<7>(wd, hitbm, lim); break;
      default: hits = s0_roll<8>(wd, hitbm, lim); break;
    }
    const uint32_t mine = (uint32_t)__popcll(hits);
    uint32_t incl = mine;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, incl, d);
      if (lane >= d) incl += t;
    }
    const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
    unsigned long long base = 0;
    if (lane == 0 && total) base = atomicAdd(cnt, (unsigned long long)total);
    base = __shfl_sync(0xffffffffu, base, 0) + (incl - mine);
    for (uint64_t m = hits; m; m &= m - 1, ++base)
      if (base < cap) out[base] = make_uint2((uint32_t)(r0 + (uint64_t)(__ffsll((long long)m) - 1)), 0u);
    maxc = max(maxc, (uint32_t)(clock64() - c0));
  }
  maxc = __reduce_max_sync(0xffffffffu, maxc);
  if (lane == 0 && maxc) atomicMax(cnt + 1, (unsigned long long)maxc);
}

template <int KIND>
__global__ void __launch_bounds__(KB_THREADS, 4) pl_kbench_kernel(const __grid_constant__ DevParams p, int stage,
                                                                  const uint2* in, uint64_t n, uint64_t first_root,
                                                                  uint2* out, uint64_t cap, unsigned long long* cnt) {
  extern __shared__ __align__(16) unsigned char dsm[];
  const KbLayout Lo = layout_kbench(p);
  const uint32_t tid = threadIdx.x, nt = blockDim.x;
  Dna dna;
  dna.db = p.db; dna.dbmask = 0xffffffffu; dna.nwords = p.db_words; dna.db_len = p.db_len;
  dna.k = p.k; dna.q_len = p.q_len;
  dna.win = p.db; dna.win_lo = 0; dna.win_lo32 = 0; dna.win_n = p.db_words; dna.win_mask = 0xffffffffu;
  dna.nofast = false;
  dna.qoff = (const uint16_t*)dsm;
  dna.qpos = (const uint16_t*)(dsm + Lo.qpos);
  dna.qw = (const uint32_t*)(dsm + Lo.qw);
  dna.nqw = (uint32_t)(p.q_len + 15) / 16u;
  dna.s2tab = dsm + Lo.s2;
  dna.xtab = (const uint16_t*)(dsm + Lo.xt);
  dna.xtab_X = xtab_X(p);
  for (uint32_t m = tid; m < 256u * (uint32_t)dna.xtab_X; m += nt)
    ((uint16_t*)(dsm + Lo.xt))[m] = Dna::xdrop_tab_entry(m >> 8, m & 255u, dna.xtab_X);
  if (p.k > 0) {
    const uint32_t nko = (1u << (2 * p.k)) + 1u, nqp = (uint32_t)(p.q_len - p.k + 1);
    uint16_t* qo = (uint16_t*)dsm;
    uint16_t* qp = (uint16_t*)(dsm + Lo.qpos);
    uint32_t* qw = (uint32_t*)(dsm + Lo.qw);
    for (uint32_t j = tid; j < nko; j += nt) qo[j] = p.qoff[j];
    for (uint32_t j = tid; j < nqp; j += nt) qp[j] = p.qpos[j];
    for (uint32_t j = tid; j < dna.nqw; j += nt) qw[j] = p.qwords[j];
    if (tid < 8) qw[tid < 4 ? (int)tid - 4 : (int)(dna.nqw + tid - 4u)] = 0u;   // pad words
    uint32_t* hb = (uint32_t*)(dsm + Lo.hit);      // S0 bitmap: k-mers that occur in the query
    for (uint32_t w = tid; w < (nko - 1u + 31u) / 32u; w += nt) {
      uint32_t bits = 0;
      for (uint32_t b = 0; b < 32u && w * 32u + b < nko - 1u; ++b)
        bits |= (p.qoff[w * 32u + b + 1u] > p.qoff[w * 32u + b] ? 1u : 0u) << b;
      hb[w] = bits;
    }
    for (uint32_t m = tid; m < 256u; m += nt) {   // S2 table (as the executor's)
      int sc = 0, best = 0;
      for (int e = 0; e < 8; ++e) {
        sc += ((m >> e) & 1u) ? -3 : 1;
        best = sc > best ? sc : best;
      }
      (dsm + Lo.s2)[m] = (unsigned char)best;
    }
  }
  __syncthreads();
  if constexpr (KIND == PL_SEED_LOOKUP) {
    if (p.k >= 4 && p.k <= KB_KMAX && (first_root & 63u) == 0 && (reinterpret_cast<uintptr_t>(p.db) & 15u) == 0) {
      kbench_s0_rolling(p, (const uint32_t*)(dsm + Lo.hit), n, first_root, out, cap, cnt);
      return;
    }
  }
  Node nd;
  nd.i = stage; nd.N = p.N; nd.v = p.v;
  nd.sink = stage == p.N - 1;
  const DevStage& sd = p.st[stage];
  nd.kind = sd.kind; nd.max_out = sd.max_out; nd.cfix = sd.cfix;
  nd.umax = sd.kind == PL_FIXED_GAIN ? sd.cfix : sd.max_out;
  nd.ip1 = sd.ip[1]; nd.ip2 = sd.ip[2];
  const bool xdrop_sink = nd.sink && nd.kind == PL_UNGAPPED_XDROP;
  const int lane = (int)(tid & 31u);
  if constexpr (KIND == PL_HIT_ENUM) {
    // S1 amplifies (up to u outputs per input): one input per lane, the warp's outputs staged in its
    // own smem slice in output order, then written as contiguous 8-byte runs (scattered per-lane
    // runs cost ~4 partial-sector L2 writes per output)
    if (!nd.sink && nd.umax <= KB_S1_U) {
      uint2* wbuf = reinterpret_cast<uint2*>(dsm + Lo.total) + (tid >> 5) * (32u * KB_S1_U);
      const uint64_t nw1 = ((uint64_t)gridDim.x * nt) >> 5;
      uint32_t maxc1 = 0;
      for (uint64_t ch = ((uint64_t)blockIdx.x * nt + tid) >> 5; ch * 32u < n; ch += nw1) {
        const long long c0 = clock64();
        const uint64_t idx = ch * 32u + (uint64_t)lane;
        uint2 ea[1];
        bool aa[1] = {idx < n};
        ea[0] = aa[0] ? __ldg(in + idx) : __ldg(in);
        LaneOut oa[1];
        stage_batch<1, PL_HIT_ENUM>(nd, dna, p, ea, aa, oa);
        const uint32_t mine = oa[0].c;
        uint32_t incl = mine;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const uint32_t t = __shfl_up_sync(0xffffffffu, incl, d);
          if (lane >= d) incl += t;
        }
        const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
        unsigned long long base = 0;
        if (lane == 0 && total) base = atomicAdd(cnt, (unsigned long long)total);
        base = __shfl_sync(0xffffffffu, base, 0);
        for (uint32_t k = 0; k < mine; ++k) wbuf[incl - mine + k] = stage_output_k<PL_HIT_ENUM>(nd, dna, ea[0], oa[0], k);
        __syncwarp();
        for (uint32_t t = (uint32_t)lane; t < total; t += 32u)
          if (base + t < cap) out[base + t] = wbuf[t];
        __syncwarp();
        maxc1 = max(maxc1, (uint32_t)(clock64() - c0));
      }
      maxc1 = __reduce_max_sync(0xffffffffu, maxc1);
      if (lane == 0 && maxc1) atomicMax(cnt + 1, (unsigned long long)maxc1);
      return;
    }
  }
  constexpr uint32_t CH = 32u * KB_J;
  const uint64_t nw = ((uint64_t)gridDim.x * nt) >> 5;
  uint32_t maxc = 0;
  for (uint64_t ch = ((uint64_t)blockIdx.x * nt + tid) >> 5; ch * CH < n; ch += nw) {
    const long long c0 = clock64();
    const uint64_t b = ch * CH + (uint64_t)lane * KB_J;
    uint2 e[KB_J];
    bool act[KB_J];
#pragma unroll
    for (int j = 0; j < KB_J; ++j) act[j] = b + j < n;
    if (stage == 0) {
#pragma unroll
      for (int j = 0; j < KB_J; ++j) e[j] = make_uint2((uint32_t)(first_root + (act[j] ? b + j : 0)), 0u);
    } else if (b + KB_J <= n && ((reinterpret_cast<uintptr_t>(in) & 15u) == 0)) {
      const uint4 x = __ldg(reinterpret_cast<const uint4*>(in + b));
      const uint4 y = __ldg(reinterpret_cast<const uint4*>(in + b) + 1);
      e[0] = make_uint2(x.x, x.y); e[1] = make_uint2(x.z, x.w);
      e[2] = make_uint2(y.x, y.y); e[3] = make_uint2(y.z, y.w);
    } else {
#pragma unroll
      for (int j = 0; j < KB_J; ++j) e[j] = act[j] ? __ldg(in + b + j) : __ldg(in);
    }
    LaneOut o[KB_J];
    stage_batch<KB_J, KIND>(nd, dna, p, e, act, o);
    uint32_t mine = 0;
#pragma unroll
    for (int j = 0; j < KB_J; ++j) mine += o[j].c;
    uint32_t incl = mine;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, incl, d);
      if (lane >= d) incl += t;
    }
    const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
    unsigned long long base = 0;
    if (lane == 0 && total) base = atomicAdd(cnt, (unsigned long long)total);
    base = __shfl_sync(0xffffffffu, base, 0) + (incl - mine);
#pragma unroll
    for (int j = 0; j < KB_J; ++j) {
      if (!o[j].c) continue;
      if (xdrop_sink) {
        if (base < p.match_cap) {
          pl_match mt;
          mt.p = e[j].x; mt.q = e[j].y & 0xffffu; mt.db_start = o[j].a; mt.q_start = o[j].q_start;
          mt.len = o[j].len; mt.score = o[j].score;
          p.matches[base] = mt;
        }
        ++base;
      } else if (!nd.sink) {
        for (uint32_t k = 0; k < o[j].c; ++k, ++base)
          if (base < cap) out[base] = stage_output_k<KIND>(nd, dna, e[j], o[j], k);
      }
    }
    maxc = max(maxc, (uint32_t)(clock64() - c0));
  }
  maxc = __reduce_max_sync(0xffffffffu, maxc);
  if (lane == 0 && maxc) atomicMax(cnt + 1, (unsigned long long)maxc);
}

template <int KIND>
static cudaError_t kbench_launch(const DevParams& p, int stage, const void* in, uint64_t n, uint64_t first_root,
                                 void* out, uint64_t cap, unsigned long long* cnt, cudaStream_t st) {
  const uint32_t smem = layout_kbench(p).total +
                        (KIND == PL_HIT_ENUM ? (uint32_t)(KB_THREADS / 32) * 32u * KB_S1_U * 8u : 0u);
  cudaError_t e = cudaFuncSetAttribute(pl_kbench_kernel<KIND>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem);
  if (e) return e;
  int per_sm = 0, sms = 0, dev = 0;
  if ((e = cudaGetDevice(&dev))) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev))) return e;
  if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, pl_kbench_kernel<KIND>, KB_THREADS, smem))) return e;
  const uint64_t chunks = (n + 32u * KB_J - 1) / (32u * KB_J);
  const uint64_t need = (chunks + KB_THREADS / 32 - 1) / (KB_THREADS / 32);
  const uint64_t full = (uint64_t)sms * (uint64_t)(per_sm > 0 ? per_sm : 1);
  const unsigned grid = (unsigned)(need < full ? (need ? need : 1) : full);
  pl_kbench_kernel<KIND><<<grid, KB_THREADS, smem, st>>>(p, stage, (const uint2*)in, n, first_root, (uint2*)out,
                                                         cap, cnt);
  return cudaGetLastError();
}

cudaError_t pl_launch_stage_batch(const DevParams& p, int stage, const void* in, uint64_t n, uint64_t first_root,
                                  void* out, uint64_t cap, unsigned long long* cnt, unsigned /*smem*/, cudaStream_t st) {
  switch (p.st[stage].kind) {
    case PL_SEED_LOOKUP: return kbench_launch<PL_SEED_LOOKUP>(p, stage, in, n, first_root, out, cap, cnt, st);
    case PL_HIT_ENUM: return kbench_launch<PL_HIT_ENUM>(p, stage, in, n, first_root, out, cap, cnt, st);
    case PL_UNGAPPED_WINDOW:
    case PL_UNGAPPED_XDROP: return kbench_launch<PL_UNGAPPED_WINDOW>(p, stage, in, n, first_root, out, cap, cnt, st);
    case PL_BERNOULLI: return kbench_launch<PL_BERNOULLI>(p, stage, in, n, first_root, out, cap, cnt, st);
    case PL_FIXED_GAIN: return kbench_launch<PL_FIXED_GAIN>(p, stage, in, n, first_root, out, cap, cnt, st);
    case PL_KEEP_EVERY: return kbench_launch<PL_KEEP_EVERY>(p, stage, in, n, first_root, out, cap, cnt, st);
    default: return kbench_launch<PL_POISSON_CAPPED>(p, stage, in, n, first_root, out, cap, cnt, st);
  }
}
