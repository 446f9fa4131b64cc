/*
 * pl.h — C-ABI of the B200 enforced-waiting streaming-pipeline executor.
 *
 * Implements the data-parallel hot path of Plano & Buhler, "Enabling Real-Time
 * Irregular Data-Flow Pipelines on SIMD Devices" (SRMPDS '21; PAPER.md):
 *   - a linear pipeline of N nodes with per-edge queues, average gains g_i and a
 *     stream of items arriving every tau0 = 1/rho0 time units     (§2.1)
 *   - each node fires a SIMD vector of up to v items taking a fixed service time t_i
 *                                                                  (§2.2)
 *   - a per-item deadline D and the active-fraction objective      (§2.3)
 *   - enforced waiting: node i waits w_i after every firing        (§4)
 *   - the monolithic block-of-M baseline                           (§5)
 *   - the optimisation problems of Fig. 1 (L139–L151) and Fig. 2 (L165–L180)
 * plus the north_star's threshold/deadline-slack firing rule (DESIGN.md R-THRESH).
 *
 * Every call is synchronous on the host unless stated; no C++ exception crosses
 * this boundary.  Every function returns PL_OK (0) or a negative pl_status and, on
 * failure, sets a thread-local message readable with pl_last_error().
 *
 * Ownership: every array in pl_config / pl_workload is COPIED at create; the
 * caller may free it afterwards.  The pipeline handle owns all device memory it
 * allocates (cudaMalloc on cfg->device) and frees it in pl_pipeline_destroy.
 * Result buffers are caller-allocated; pass buf == NULL to query the count.
 *
 * Time: all times are int64 "units".  With PL_CLOCK_LOGICAL the executor runs a
 * conservative parallel discrete-event schedule as fast as the GPU allows; with
 * PL_CLOCK_GLOBALTIMER one unit is cfg->ns_per_unit nanoseconds of %globaltimer
 * (32 ns resolution on B200, measured) and firings are paced in real time.
 */
#ifndef PL_H
#define PL_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PL_MAX_STAGES 8
#define PL_MAX_U 16            /* cap on outputs per input of any stage (u = 16) */

typedef int32_t pl_status;
#define PL_OK           0
#define PL_EINVAL      -1      /* bad argument / unsupported configuration          */
#define PL_ENOMEM      -2      /* device or pinned-host allocation failed           */
#define PL_EDEVICE     -3      /* CUDA error (launch, copy, device fault)           */
#define PL_EINFEASIBLE -4      /* solver: Fig. 1 / Fig. 2 has no feasible point     */
#define PL_ESTATE      -5      /* call out of order (e.g. push after drain)         */
#define PL_EAGAIN      -6      /* (reserved) non-blocking push would block          */
#define PL_EOVERFLOW   -7      /* a queue or output buffer overflowed during a run  */

/* Stage kinds.  DNA stages follow classic BLAST [1] (§6.1; readings
 * R-S0..R-S3 in DESIGN.md); random-gain stages follow PAPER.md L210.            */
enum pl_stage_kind {
  PL_BERNOULLI = 0,        /* 1 output with prob. param (=g), else 0; hash-driven    */
  PL_FIXED_GAIN = 1,       /* exactly (int)param outputs (<= max_out)               */
  PL_POISSON_CAPPED = 2,   /* min(Poisson(param), max_out) outputs (L210, u=max_out) */
  PL_SEED_LOOKUP = 3,      /* S0: keep DB position p iff its k-mer occurs in query   */
  PL_HIT_ENUM = 4,         /* S1: p -> (p,q_j), j < min(count, max_out)             */
  PL_UNGAPPED_WINDOW = 5,  /* S2: keep (p,q) iff k+best_left(W)+best_right(W) >= T2  */
  PL_UNGAPPED_XDROP = 6,   /* S3: X-drop ungapped extension, emit pl_match if >= T3  */
  PL_KEEP_EVERY = 7        /* deterministic filter: keep iff root % (int)param == 0  */
};

enum pl_policy {
  PL_FIXED_WAIT = 0,       /* paper §4: fire every t_i + w_i, even when empty (L97)  */
  PL_THRESHOLD_SLACK = 1,  /* north_star: fire when |Q| >= theta_i or slack forces it */
  PL_MONOLITHIC = 2        /* paper §5: blocks of M, whole pipeline per block        */
};

enum pl_clock { PL_CLOCK_LOGICAL = 0, PL_CLOCK_GLOBALTIMER = 1 };

/* pl_config.flags: optional per-root / per-firing records (parity & tracing).    */
#define PL_REC_LATENCY  1u     /* lat[r]: per-root latency (model units; + ns if physical) */
#define PL_REC_TRACE    2u     /* cnt[r][0..N]: per-root surviving-stage trace           */
#define PL_REC_FIRINGS  4u     /* per-stream log of non-empty firings                    */
#define PL_FIXED_SERVICE 8u    /* physical clock, time-triggered delivery: a firing occupies its
                                  node until start + t_i, the paper's fixed service time (L69),
                                  and its terminal items complete then (or when the work is done,
                                  if later: an overrun); without it they complete when done.  The
                                  schedule is the same either way (a segment's items are ready at
                                  start + t_i and consumed at logical times >= that).           */
#define PL_EAGER_DRAIN  16u    /* end of stream (reading R-DRAIN): at times T >= A_last, the
                                  stream's last arrival, every node fires whenever it is idle
                                  and its queue is non-empty (FIXED_WAIT's time-triggered
                                  starts at T >= A_last are dropped).  The paper models an
                                  unbounded stream (L63) and is silent on its end; without
                                  this flag the periodic / threshold rules run to the drain. */
#define PL_CLUSTER_NODES 32u   /* N4 ("a fixed 1/N fraction of processor
                                  time", L265): every stream runs on a cluster of N CTAs, node i on
                                  CTA rank i (an SM of its own), its input queue in that CTA's
                                  shared memory, written by node i-1 over DSMEM.  FIXED_WAIT and
                                  THRESHOLD_SLACK, N <= 8, v <= 256; not with live ingest.  Same
                                  schedule and results as the one-CTA-per-stream executor.      */

typedef struct {
  uint32_t kind;           /* enum pl_stage_kind                                        */
  uint32_t max_out;        /* u: cap on outputs per input (1..PL_MAX_U)                 */
  double   param;          /* g (Bernoulli), c (fixed gain), lambda (Poisson), modulus  */
  int32_t  iparam[4];      /* DNA: S0 {k}, S1 {k,u}, S2 {k,W,T2}, S3 {k,X,T3}           */
} pl_stage;

typedef struct {
  uint32_t n_stages;               /* N, 1..PL_MAX_STAGES; linear chain only (L61)      */
  const pl_stage* stages;          /* [N]                                               */
  const int64_t* service_time;     /* t_i [N] > 0                                       */
  const double*  gain;             /* g_i [N-1] for the solvers; NULL -> measured       */
  const uint32_t* b;               /* b_i [N] queue multipliers (L133); NULL -> all 1   */
  uint32_t vector_width;           /* v: 32, 64, 128 or 256; N*v <= 992                 */
  const int64_t*  wait_time;       /* w_i [N] (FIXED_WAIT) or NULL -> solve Fig. 1      */
  const uint32_t* wait_threshold;  /* theta_i [N] (THRESHOLD_SLACK) or NULL -> derived  */
  int64_t deadline;                /* D (L73)                                           */
  int64_t interarrival;            /* tau0 = 1/rho0 (L63), >= 1                          */
  int64_t slack_guard;             /* THRESHOLD_SLACK: extra reserve added to R_i        */
  uint32_t policy;                 /* enum pl_policy                                    */
  uint32_t clock;                  /* enum pl_clock                                     */
  uint32_t block_size;             /* M (MONOLITHIC); 0 -> solve Fig. 2                 */
  uint32_t mono_b;                 /* b of Fig. 2 (0 -> 1)                              */
  double   mono_S;                 /* S of Fig. 2 (0 -> 1)                              */
  uint32_t n_streams;              /* independent pipeline instances = CTAs (>= 1)      */
  uint64_t n_roots;                /* random-gain stages: roots per stream;             */
                                   /* DNA: 0 (roots are the DB positions [0, Ldb-k])    */
  uint64_t seed;                   /* counter-based RNG seed of random-gain stages      */
  int32_t  device;                 /* CUDA device ordinal                               */
  double   ns_per_unit;            /* physical clock: ns per time unit (> 0)            */
  uint32_t flags;                  /* PL_REC_* bits                                     */
  uint32_t queue_capacity;         /* smem entries per edge (power of 2; 0 -> default)  */
  uint32_t spill_capacity;         /* HBM overflow entries per edge per stream (2^k; 0->dflt) */
  uint32_t firing_log_capacity;    /* records per stream when PL_REC_FIRINGS (0 -> dflt) */
  uint64_t match_capacity;         /* pl_match records (0 -> default)                   */
  const int64_t* arrivals;         /* NULL: root r of a stream arrives at r*tau0 (L63).  Else
                                      arrival time (units, from its stream's start) of every
                                      root, non-decreasing within a stream, e.g. Poisson (L263);
                                      copied at create; n_arrivals must equal the root count */
  uint64_t n_arrivals;
  uint32_t window_words;           /* per-stream smem DB window: a ring of this many 32-bit words
                                      (power of 2, >= 2 chunks; 0 -> default: the whole stream range
                                      when it fits, else 16 chunks = 64 KB), refilled by TMA as the
                                      stream advances (a1); reads outside it go to the bound DB     */
  uint32_t window_chunk_words;     /* refill unit in words (power of 2, >= 4; 0 -> default 1024)    */
} pl_config;

/* Workload of the DNA pipeline: the query is known up front; the database is the
 * stream and arrives through pl_pipeline_push / pl_pipeline_bind_device.
 * Both sequences are 2-bit packed: base j at bits 2*(j mod 16) of uint32 word j/16,
 * A=0 C=1 G=2 T=3.  Ignored (may be NULL) for random-gain pipelines.            */
typedef struct {
  const uint32_t* query;           /* host pointer, ceil(q_len/16) words             */
  uint64_t q_len;                  /* <= 65535                                       */
  uint64_t db_len;                 /* total DB bases the stream will carry           */
} pl_workload;

/* One HSP emitted by the last DNA stage (reading R-S3).                          */
typedef struct {
  uint32_t p, q;                   /* seed position in DB / query (root = p)          */
  uint32_t db_start, q_start;      /* left end of the extension                       */
  uint32_t len;                    /* extension length                                */
  int32_t  score;
} pl_match;

/* One non-empty firing (PL_REC_FIRINGS).                                         */
typedef struct {
  int64_t  start;                  /* logical start time (units)                      */
  uint32_t node, n;                /* node index, inputs consumed (1..v)              */
  uint32_t first_root, last_root;  /* roots of the first and last consumed entry      */
  uint32_t stream, pad;
} pl_firing;

typedef struct {
  uint32_t n_stages, n_streams;
  uint64_t roots;                          /* roots processed (all streams)           */
  uint64_t firings[PL_MAX_STAGES];         /* non-empty firings                       */
  uint64_t empty_firings[PL_MAX_STAGES];   /* FIXED_WAIT firings skipped as empty     */
  uint64_t consumed[PL_MAX_STAGES];
  uint64_t produced[PL_MAX_STAGES];
  int64_t  active_window[PL_MAX_STAGES];   /* sum |[s,s+t_i) ∩ [0,H)| over ALL firings */
  int64_t  busy_ns[PL_MAX_STAGES];         /* physical: measured firing time (ns)     */
  uint64_t spilled[PL_MAX_STAGES];         /* entries written to the HBM overflow ring */
  uint64_t overruns[PL_MAX_STAGES];        /* physical: firings longer than t_i        */
  uint64_t stalls[PL_MAX_STAGES];          /* firings that waited for room in the next queue */
  uint32_t max_queue[PL_MAX_STAGES];       /* longest input queue seen at a firing decision (entries;
                                              PAPER.md L133: "maximum size b_i v"), max over streams */
  int64_t  max_lateness_ns[PL_MAX_STAGES]; /* physical: max(actual - scheduled start)  */
  uint64_t sched_cycles[PL_MAX_STAGES];    /* clock64 cycles spent deciding firings    */
  int64_t  max_fire_ns[PL_MAX_STAGES];     /* physical: longest firing (start->publish) */
  int64_t  max_loop_ns[PL_MAX_STAGES];     /* physical: longest cycle from a firing's start to the
                                              node's next decision (not counting waits for upstream):
                                              the real per-firing service time, incl. bookkeeping */
  /* leader-lane clock64 cycles per phase of a firing, summed over firings:
   * [0] decide (scheduler), [1] release barrier, [2] load+stage+scan,
   * [3] records+reserve, [4] output writes, [5] publish                        */
  uint64_t phase_cycles[PL_MAX_STAGES][6];
  uint64_t matches;
  uint64_t miss_events;                    /* terminal events with latency > D (schedule) */
  uint64_t miss_events_ns;                 /* physical clock: terminal events whose MEASURED
                                              latency exceeded D (always counted)          */
  uint64_t misses;                         /* distinct roots (needs PL_REC_LATENCY)    */
  int64_t  max_latency;                    /* model units (logical schedule)          */
  int64_t  max_latency_ns;                 /* physical: measured                       */
  int64_t  window;                         /* sum over streams of H = X*tau0           */
  int64_t  t_end;                          /* sum over streams of the drain end time   */
  double   active_fraction;                /* PAPER.md L75 over [0,H)                  */
  double   active_fraction_nonempty;       /* same, charging non-empty firings only    */
  double   active_fraction_drain;          /* the same ratio over [0, T_end], the drain included
                                              (SURVEY §8(c) C-D "Outputs"): every firing started
                                              before the stream's last completion, clipped to it */
  double   hw_busy_fraction;               /* physical: busy_ns / (N * wall)           */
  int64_t  wall_ns;                        /* max over streams of kernel-side runtime  */
  uint32_t errors;                         /* device error bits (PL_EOVERFLOW at drain): 1 spill ring
                                              full (physical clock), 2 match buffer full, 4 firing
                                              log full, 8 segment ring full, 16 live ingest: no
                                              delivery for 20 s, 32 watchdog: a node waited 30 s
                                              without progress and gave up                 */
  uint32_t launches;                       /* executor launches so far                 */
  uint64_t h2d_bytes;                      /* host->device bytes copied by this handle (cumulative) */
  uint64_t d2h_bytes;                      /* device->host bytes copied by this handle (cumulative) */
  uint64_t window_refills;                 /* DB-window chunks TMA-loaded as the streams advanced (a1) */
  /* physical clock: agreement of every terminal item's MEASURED latency with the logical-clock
   * prediction T + t_i - a(r) (north_star "within 5 % relative"; DESIGN.md R-AGREE: a floor of
   * 64 ns = two %globaltimer ticks; with PL_FIXED_SERVICE a firing completes at start + t_i)   */
  uint64_t latency_outliers;               /* terminal items with |err| > 5 % of their latency + 64 ns
                                              (counted with PL_FIXED_SERVICE only)                    */
  double   latency_rel_err_max;            /* largest |err| / logical latency over terminal items      */
  uint64_t ingest_waits;                   /* live ingest: node-0 firings / blocks that waited for words */
  int64_t  max_ingest_wait_ns;             /* live ingest: the longest such wait                        */
} pl_stats;

typedef struct pl_pipeline pl_pipeline;

/* Create a pipeline.  Validates cfg (PL_EINVAL), solves Fig. 1 / Fig. 2 when
 * w / M are missing and gains are given (PL_EINFEASIBLE), allocates device memory
 * (PL_ENOMEM) and uploads the query index.  *out is NULL on failure.            */
pl_status pl_pipeline_create(const pl_config* cfg, const pl_workload* wl, pl_pipeline** out);

/* Bind the CUDA stream (cudaStream_t passed as void*) every later launch and copy
 * uses.  NULL = the legacy default stream.                                      */
pl_status pl_pipeline_set_stream(pl_pipeline* pl, void* stream);

/* Append n items from HOST memory: for DNA pipelines `items` holds n bases, 2-bit
 * packed, and the running total must stay <= wl->db_len (every push but the last
 * must be a multiple of 16 bases); the copy to HBM is enqueued on the bound stream
 * and `items` may be reused as soon as the call returns (from page-locked memory the
 * call waits for the copy -- and so for the work queued before it on the stream).
 * This is the pre-staged path (one run over a finished stream); live ingest during
 * a run is pl_pipeline_push_stream / push_all (below).  For random-gain
 * pipelines items must be NULL and n counts roots per stream (<= cfg->n_roots).
 * After pl_pipeline_drain: PL_ESTATE until pl_pipeline_rewind.                  */
pl_status pl_pipeline_push(pl_pipeline* pl, const void* items, uint64_t n);

/* Use a caller-owned DEVICE buffer of n packed bases as the whole DB (no copy).
 * The buffer must stay alive until the last launch using it has completed.      */
pl_status pl_pipeline_bind_device(pl_pipeline* pl, const void* dev_items, uint64_t n);

/* Use a caller-owned PINNED HOST buffer (cudaHostAlloc'd, or cudaHostRegister'ed with
 * cudaHostRegisterMapped) of n packed bases as the whole DB, with no device copy: every CTA
 * stages its DB window straight from host memory with TMA bulk copies (cp.async.bulk over
 * PCIe/C2C) when the executor starts; reads outside the window go to host memory.
 * PL_EINVAL if the buffer is not mapped.  It must stay valid until the run completes.    */
pl_status pl_pipeline_bind_host(pl_pipeline* pl, const void* host_items, uint64_t n);

/* Direct the match records (pl_match, the last DNA stage's output) of later runs into a
 * caller-owned buffer of `cap` records: device memory, or PINNED+MAPPED host memory
 * (cudaHostAlloc(..., cudaHostAllocMapped) / cudaHostRegisterMapped), into which the executor
 * writes them over the host link as they are produced -- so a run's result needs no separate
 * device->host copy.  The buffer must stay valid until the last run using it has completed;
 * records beyond cap set PL_EOVERFLOW.  buf == NULL restores the handle's own device buffer.
 * pl_pipeline_results reads whichever buffer the last run used.                             */
pl_status pl_pipeline_bind_results(pl_pipeline* pl, void* buf, uint64_t cap);

/* Per-stream input-queue peaks of the last run: buf[s*N + i] = longest queue (entries) node i
 * of stream s saw at a firing decision.  The data of the paper's b_i calibration (L133,
 * L227-L230).  buf == NULL: *n = n_streams * N.                                          */
pl_status pl_pipeline_queue_peaks(pl_pipeline* pl, uint32_t* buf, uint64_t cap, uint64_t* n);

/* Compact result of the last run, reduced on the device (one small D->H copy).         */
typedef struct {
  uint64_t roots, matches, miss_events, miss_events_ns;
  int64_t  max_latency, max_latency_ns;
  uint32_t errors, launches;
  uint64_t latency_outliers;       /* physical: items outside the 5 % latency band (pl_stats) */
} pl_summary;
pl_status pl_pipeline_summary(pl_pipeline* pl, pl_summary* out);

/* ---- Live ingest (§2.1: "a stream of items, of unbounded length", arriving at
 * rate rho0; SURVEY §8(b) push(stream, items, n); a1).  The DB is delivered WHILE one persistent
 * run executes, through per-stream rings in device memory:
 *   pl_pipeline_live_start(pl, R)   launches the run (on the bound stream) with a ring of R words
 *                                   per stream (power of 2; 0 -> max(4 x the smem window, 64 K));
 *   pl_pipeline_stream_words(pl,s)  the DB words stream s needs: [word_lo, word_hi) -- its roots
 *                                   plus the k-1 overlap and a q_len halo on each side (the reach
 *                                   of an extension walk, reading R-S3), 2-bit packed as in pl.h;
 *   pl_pipeline_push_stream(pl, s, words, n, nonblocking)
 *   pl_pipeline_push_all(pl, words[S], n[S], nonblocking)
 *                                   append the next n words of stream s (of every stream), in
 *                                   order; the library zero-pads each stream's last word;
 *   pl_pipeline_drain(pl)           after the last words of every stream: waits for the run.
 * Each push copies its words into a pinned host mirror of the ring (so `words` may be reused as
 * soon as the call returns), enqueues their copy to the device ring on a handle-owned
 * non-blocking copy stream, and then the stream's doorbell (its delivered-word count, in device
 * memory) behind them in the same copy stream.  On the device, node 0 takes a root only once every word its descendants can
 * read has been delivered, and the window slides by TMA from the ring as words arrive: the
 * logical schedule stays the oracle's (root r arrives at r tau0 from the run's start, L63), and
 * a late delivery appears as node-0 lateness, measured latency and pl_stats.ingest_waits.  Ring
 * slots are reused once the device publishes (to mapped host memory) that no node reads below
 * them: memory stays bounded however long the stream.  A push that finds its ring full blocks
 * until room appears (PL_EAGAIN after 10 s without room), or with nonblocking != 0 returns
 * PL_EAGAIN at once, having taken nothing.  Errors: PL_EINVAL (not DNA, arrival array given,
 * n_streams above the resident-CTA count, bad ring size, a push past the stream's range),
 * PL_ESTATE (push without a live run; launch / pl_pipeline_push during one; drain before every
 * word was pushed), PL_ENOMEM, PL_EDEVICE.  A stream without delivery for 20 s proceeds on
 * stale ring contents and sets error bit 16 (PL_EOVERFLOW at drain).                         */
pl_status pl_pipeline_live_start(pl_pipeline* pl, uint32_t ring_words);
pl_status pl_pipeline_stream_words(const pl_pipeline* pl, uint32_t stream, uint64_t* word_lo, uint64_t* word_hi);
pl_status pl_pipeline_push_stream(pl_pipeline* pl, uint32_t stream, const uint32_t* words, uint64_t n,
                                  int nonblocking);
pl_status pl_pipeline_push_all(pl_pipeline* pl, const uint32_t* const* words, const uint64_t* n, int nonblocking);

/* Fault injection for measurement (DESIGN.md R-STALL).  The B200 platform stops
 * every SM for ~1.6 ms every few seconds (profiles/r02_pause_control.txt); with len_ns > 0 every
 * node of every stream of later physical-clock runs stops at its next firing start inside the
 * windows [T0 + j period_ns, T0 + j period_ns + len_ns), j >= 1, until the window ends -- the
 * same event on demand, so that a rate search can require zero deadline misses across it.  The
 * logical schedule (and so every parity output) is unchanged; only lateness and measured
 * latencies move.  len_ns = 0 turns it off.  PL_EINVAL: len_ns < 0, period_ns <= len_ns, or a
 * logical-clock pipeline.                                                                    */
pl_status pl_pipeline_inject_stalls(pl_pipeline* pl, int64_t period_ns, int64_t len_ns);

/* Enqueue one executor run over every item pushed so far on the bound stream and
 * return immediately (asynchronous).  Resets per-run outputs first.             */
pl_status pl_pipeline_launch(pl_pipeline* pl);

/* Pipelined stepping (a stream of runs, as a real-time deployment issues them): enqueue one
 * run (as pl_pipeline_launch) followed by an asynchronous D->H copy of its pl_summary words
 * into pinned host memory owned by the handle, then -- if an earlier pl_pipeline_step run
 * exists -- block until THAT run has completed and return its summary in *prev
 * (*has_prev = 1; prev->launches = its launch index).  The device executes run k while the
 * host reads run k-1.  The first call returns *has_prev = 0.  The copy is ordered before the
 * next launch on the stream, which reuses the run's device summary slot.  Errors: PL_EINVAL
 * (NULL argument), PL_ENOMEM (pinned buffer), PL_EDEVICE (CUDA error).                    */
pl_status pl_pipeline_step(pl_pipeline* pl, pl_summary* prev, int* has_prev);

/* Block until the last pl_pipeline_step run has completed and return its summary in *last
 * (*has_last = 0 if no step is outstanding); ends the step sequence.                      */
pl_status pl_pipeline_step_finish(pl_pipeline* pl, pl_summary* last, int* has_last);

/* Block until the last launched run has completed -- launching one first if nothing was
 * launched since the last push / bind / rewind -- and check its device-side error flags
 * (PL_EOVERFLOW) and CUDA errors (PL_EDEVICE).  pl_pipeline_summary / step_finish do not
 * consume the run: launch -> summary -> drain checks that same run.                      */
pl_status pl_pipeline_drain(pl_pipeline* pl);

/* Allow another push/launch cycle with the same pipeline (rewinds the stream).   */
pl_status pl_pipeline_rewind(pl_pipeline* pl);

/* Statistics of the last completed run (copies counters device->host).          */
pl_status pl_pipeline_stats(pl_pipeline* pl, pl_stats* out);

/* Matches of the last run, unsorted.  buf==NULL: *n = count.  Otherwise copies
 * min(cap, count) records and sets *n to the number copied.                     */
pl_status pl_pipeline_results(pl_pipeline* pl, pl_match* buf, uint64_t cap, uint64_t* n);

/* Per-root latencies (needs PL_REC_LATENCY): lat_units[r] (logical schedule) and,
 * if lat_ns != NULL and the clock is physical, measured ns.  -1 = no terminal event.
 * Arrays have *n = total roots entries (query with lat_units == NULL).          */
pl_status pl_pipeline_latency(pl_pipeline* pl, int64_t* lat_units, int64_t* lat_ns, uint64_t cap, uint64_t* n);

/* Per-root trace (needs PL_REC_TRACE): cnt[r*(N+1)+i] = descendants of root r
 * consumed by node i (i < N); cnt[r*(N+1)+N] = outputs emitted by node N-1.     */
pl_status pl_pipeline_trace(pl_pipeline* pl, uint32_t* cnt, uint64_t cap, uint64_t* n);

/* Non-empty firings of the last run (needs PL_REC_FIRINGS), grouped by stream.  */
pl_status pl_pipeline_firings(pl_pipeline* pl, pl_firing* buf, uint64_t cap, uint64_t* n);

/* The effective parameters in use (after solving): w_i, theta_i, M.            */
pl_status pl_pipeline_params(const pl_pipeline* pl, int64_t* w_out, uint32_t* theta_out, uint32_t* M_out);

void pl_pipeline_destroy(pl_pipeline* pl);

/* Thread-local message for the last non-OK status of this thread ("" if none).  */
const char* pl_last_error(void);

/* Fig. 1: minimise (1/N) sum t_i/(t_i+w_i) s.t. stability
 * (L125, L131) and sum b_i (t_i+w_i) <= D (L135), w_i >= 0 integer.  Needs
 * cfg->gain.  Writes w_out[N], theta_out[N] (THRESHOLD mapping, may be NULL),
 * *T_out (objective at the integer optimum) and T_cont (continuous optimum, may be NULL). */
pl_status pl_solve_enforced_waits(const pl_config* cfg, int64_t* w_out, uint32_t* theta_out,
                                  double* T_out, double* T_cont);

/* Fig. 2: best block size M by exhaustive search.          */
pl_status pl_solve_monolithic(const pl_config* cfg, uint32_t* M_out, double* T_out);

/* Standalone batch run of one stage (per-stage profiling kernels, SURVEY K-BENCH).
 * Consumes n device-resident entries {root, aux} (uint2: aux = q | j<<16 for DNA hits,
 * lineage for random gains); for stage 0 `in_dev` is ignored and the roots are
 * first_root .. first_root+n-1.  Outputs of non-sink stages are appended to out_dev
 * (device, capacity cap entries): in input order within each warp's chunk of consecutive
 * inputs, chunks in any order.  The last DNA stage writes pl_match records to
 * the pipeline's match buffer (read with pl_pipeline_results).  *n_out = outputs produced;
 * *max_vec_cycles (may be NULL) = longest per-chunk clock64 duration.  The kernel runs at
 * full occupancy (256-thread CTAs, the query index in smem): S0 rolls k-mers over 16-byte DB
 * loads (first_root a multiple of 64, 4 <= k <= 8; else per item), S1 writes its outputs
 * through smem as contiguous runs, the other stages run the executor's stage bodies.
 * Needs a pushed or bound DB for DNA; PL_EINVAL if stage 0's roots first_root .. first_root+n-1
 * reach past the DB's last k-mer.  PL_EOVERFLOW: more outputs than cap (the first cap
 * are written).                                                                        */
pl_status pl_stage_batch(pl_pipeline* pl, uint32_t stage, const void* in_dev, uint64_t n, uint64_t first_root,
                         void* out_dev, uint64_t cap, uint64_t* n_out, uint64_t* max_vec_cycles);

/* Library build identity (for logs): "plgpu <version> sm_100a".                  */
const char* pl_version(void);

#ifdef __cplusplus
}
#endif
#endif /* PL_H */
