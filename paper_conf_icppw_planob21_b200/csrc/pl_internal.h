// pl_internal.h — structures shared by the host runtime (runtime.cu) and the
// persistent executor kernels (executor.cu).  Not part of the public ABI.
#pragma once
#include <stdint.h>
#include <vector_types.h>
#include "../../include/pl.h"

#define PL_INF64 0x7fffffffffffffffLL
#define PL_MAX_K 7                      // query index 4^k u16 entries must fit in smem
#define PL_AGREE_FLOOR_NS 64            // R-AGREE: |measured - logical latency| <= 5 % + this (2 timer ticks)

// Error bits written by the device (pl_stats.errors).
#define PL_ERR_QUEUE_OVERFLOW   1u      // spill ring full in physical mode
#define PL_ERR_MATCH_OVERFLOW   2u
#define PL_ERR_LOG_OVERFLOW     4u
#define PL_ERR_SEG_OVERFLOW     8u
#define PL_ERR_INGEST_TIMEOUT  16u      // live ingest: no delivery for PL_INGEST_TIMEOUT_NS (proceeds on stale data)
#define PL_INGEST_TIMEOUT_NS   20000000000ull
#define PL_ERR_WATCHDOG        32u      // a node waited PL_WATCHDOG_NS without progress and gave up
#define PL_WATCHDOG_NS         30000000000ull

struct DevStage {
  uint32_t kind, max_out;
  int32_t  ip[4];                       // k, W/X/u, T2/T3
  uint32_t cfix;                        // FIXED_GAIN c, KEEP_EVERY modulus
  uint32_t pad;
  uint64_t thr[PL_MAX_U];               // Bernoulli thr[0]; Poisson thr[0..u-1]
};

// One segment = the outputs of one non-empty producer firing, contiguous in
// sequence space, all with the same ready time.
struct Seg {
  int64_t  ready;                       // producer firing start + t_i
  uint32_t end;                         // one past the last sequence number
  uint32_t loc;                         // 0 = smem ring, 1 = HBM spill ring
};

// Per-stream (per-CTA) results written once at the end of a run.
struct CtaStats {
  uint64_t firings[PL_MAX_STAGES];
  uint64_t empty[PL_MAX_STAGES];
  uint64_t consumed[PL_MAX_STAGES];
  uint64_t produced[PL_MAX_STAGES];
  int64_t  active_ne[PL_MAX_STAGES];    // sum |[s,s+t_i) ∩ [0,H)| over non-empty firings
  int64_t  active_win[PL_MAX_STAGES];   // the charged active time over [0,H) (R-WINDOW; R-DRAIN)
  int64_t  busy_ns[PL_MAX_STAGES];
  uint64_t spilled[PL_MAX_STAGES];
  uint64_t overruns[PL_MAX_STAGES];
  uint64_t stalls[PL_MAX_STAGES];
  uint64_t drain_firings[PL_MAX_STAGES]; // R-DRAIN firings (at T >= A_last)
  uint32_t max_queue[PL_MAX_STAGES];
  int64_t  lateness[PL_MAX_STAGES];
  uint64_t sched_cycles[PL_MAX_STAGES];
  int64_t  max_fire_ns[PL_MAX_STAGES];
  int64_t  max_loop_ns[PL_MAX_STAGES];
  uint64_t phase_cycles[PL_MAX_STAGES][6];
  uint64_t miss_events;
  uint64_t miss_events_ns;              // physical: measured latency > D
  int64_t  max_lat;                     // model units
  int64_t  max_lat_ns;
  int64_t  t_end;                       // drain end (model units)
  int64_t  wall_ns;
  uint64_t n_roots;
  uint32_t n_log;                       // firing-log records written
  uint32_t errors;
  uint32_t win_refills;                 // DB-window chunks loaded after the initial staging
  uint32_t agr_bad;                     // physical: terminal items outside the 5 % latency band (R-AGREE)
  uint32_t agr_ppm;                     // physical: largest relative latency error (ppm)
  uint32_t ingest_waits;                // live ingest: node-0 firings / blocks that waited for delivery
  uint32_t ingest_max_ns;               // live ingest: the longest such wait
  uint32_t pad_;
};

struct DevParams {
  int32_t  N, v, policy, clock;
  int64_t  t[PL_MAX_STAGES];            // service times
  int64_t  P[PL_MAX_STAGES];            // FIXED_WAIT periods t_i + w_i
  uint32_t theta[PL_MAX_STAGES];        // THRESHOLD_SLACK thresholds
  int64_t  R[PL_MAX_STAGES];            // THRESHOLD_SLACK reserves (incl. guard)
  int64_t  D, tau;
  uint64_t tau_m, P_m[PL_MAX_STAGES];    // reciprocals floor((2^64-1)/x) for division-free fdiv
  int64_t  M;                           // MONOLITHIC block size
  double   ns_per_unit;
  uint64_t seed;
  uint64_t total_roots;                 // roots over all streams
  int32_t  n_streams;
  uint32_t flags;
  int32_t  ctas_per_sm;                 // launch variant: 2 -> 64-register kernel, two streams per SM
  uint32_t variant;                     // experiment bits (PL_VARIANT): 1 leader-paced node 0, 4 interleaved warps (node = warp % N)
  // DNA workload
  const uint32_t* db;                   // packed DB (device)
  uint64_t db_len;
  uint32_t db_words;
  int32_t  k, q_len;
  const uint16_t* qoff;                 // [4^k + 1]
  const uint16_t* qpos;                 // [q_len - k + 1]
  const uint32_t* qwords;               // [ceil(q_len/16)]
  uint32_t win_cap;                     // smem DB window: a ring of win_cap words (power of 2; 0 = off)
  uint32_t win_lg;                      // log2 of the ring's chunk (words): the unit of a TMA refill
  uint32_t win_halo;                    // bases staged beyond the stream's roots on each side
  uint64_t db_alloc_words;              // readable words at db (>= db_words)
  uint32_t db_tma;                      // db is 16-byte aligned and padded: stage with cp.async.bulk
  // queues
  uint32_t cap_s[PL_MAX_STAGES];        // smem entries of the edge INTO node i (pow2), i >= 1
  uint32_t cap_g;                       // spill entries per edge per stream (pow2)
  uint32_t segcap;                      // segments per edge (pow2, >= v+1)
  uint2*   spill;                       // [n_streams][N][cap_g]
  uint2*   mono_buf;                    // MONOLITHIC ping-pong buffers [n_streams][2][mono_cap]
  uint32_t mono_cap;
  // outputs
  int64_t* lat;                         // [total_roots] model units (PL_REC_LATENCY)
  int64_t* lat_ns;                      // [total_roots] physical ns
  uint32_t* trace;                      // [total_roots][N+1]
  pl_match* matches;
  unsigned long long* match_count;
  uint64_t match_cap;
  pl_firing* flog;                      // [n_streams][log_cap]
  uint32_t log_cap;
  CtaStats* stats;                      // [n_streams]
  unsigned long long* summary;          // [8]: roots, miss_events, max_lat, max_lat_ns, errors, miss_ns,
                                        //      match count (= match_count), latency outliers (R-AGREE)
  uint32_t t0_offset_ns;                // physical clock: stream time origin = CTA start + this
  unsigned long long* summary_next;     // the other slot of the double buffer: zeroed by this launch
                                        // (stream order: the previous launch that used it is done)
  const int64_t* arr;                   // per-root arrival times (NULL: r * tau0)
  uint64_t inj_period_ns, inj_len_ns;   // stall injection (pl_pipeline_inject_stalls; 0 = off)
  // live ingest (pl_pipeline_live_start): the DB is delivered while the run executes
  uint32_t live;                        // 1: stream s reads DB word w from ring[s R + (w & ring_mask)]
  uint32_t ring_mask;                   // R - 1 (R = ring words per stream, a power of 2)
  const uint32_t* ring;                 // [n_streams][R] device rings, filled by the copy stream
  const uint32_t* front;                // [n_streams] doorbells: stream s holds words [wlo_s, front[s])
  uint32_t* consumed;                   // [n_streams] mapped host: slots below consumed[s] may be reused
  DevStage st[PL_MAX_STAGES];
};

// smem layout of the enforced-policy kernel (computed identically on host and device)
struct SmemLayout {
  uint32_t off_ent[PL_MAX_STAGES];      // uint2 rings, edge into node i (i >= 1)
  uint32_t off_seg[PL_MAX_STAGES];
  uint32_t off_troot;                   // [N][v] u32: terminal root per lane of the current firing
  uint32_t off_qoff, off_qpos, off_qw, off_win, off_s2, off_xt;
  uint32_t total;
};

#ifdef __cplusplus
static inline uint32_t pl_align16(uint32_t x) { return (x + 15u) & ~15u; }
#endif
