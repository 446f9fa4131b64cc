// runtime.cu — host implementation of the C-ABI in include/pl.h.
//
// Owns device memory, validates configurations, derives the schedule parameters
// (periods P_i = t_i + w_i, thresholds theta_i, reserves R_i, block size M) —
// solving Fig. 1 / Fig. 2 when they are not given — builds the query index
// (direct-address k-mer table, reading R-S1), and launches the persistent
// executor kernels in executor.cu.  No exceptions cross the ABI.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <thread>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "pl_internal.h"

cudaError_t pl_launch(const DevParams& p, unsigned grid, unsigned block, unsigned smem, cudaStream_t st);
cudaError_t pl_kernel_attributes(unsigned max_smem);
cudaError_t pl_launch_stage_batch(const DevParams& p, int stage, const void* in, uint64_t n, uint64_t first_root,
                                  void* out, uint64_t cap, unsigned long long* cnt, unsigned smem, cudaStream_t st);
uint32_t pl_layout_enforced_host(const DevParams& p);

namespace plsolve {
int solve_fig1(int N, const int64_t* t, const double* g, const uint32_t* b, uint32_t v, int64_t tau, int64_t D,
               double* Pc, double* Tc, int64_t* Pi, double* Ti);
void thresholds(int N, const double* g, const int64_t* P, int64_t tau, uint32_t v, uint32_t* theta);
int solve_fig2(int N, const int64_t* t, const double* g, uint32_t v, int64_t tau, int64_t D, double bb, double S,
               uint32_t* M_out, double* T_out);
}  // namespace plsolve

namespace {

thread_local std::string g_err;

pl_status fail(pl_status st, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return st;
}

#define CUDA_TRY(x)                                                                              \
  do {                                                                                           \
    cudaError_t _e = (x);                                                                        \
    if (_e != cudaSuccess) return fail(PL_EDEVICE, "%s: %s", #x, cudaGetErrorString(_e));        \
  } while (0)

uint32_t next_pow2(uint32_t x) {
  uint32_t p = 1;
  while (p < x) p <<= 1;
  return p;
}
bool is_pow2(uint32_t x) { return x && !(x & (x - 1)); }

bool is_dna(uint32_t kind) {
  return kind == PL_SEED_LOOKUP || kind == PL_HIT_ENUM || kind == PL_UNGAPPED_WINDOW || kind == PL_UNGAPPED_XDROP;
}

// exact floor(p * 2^64) for p in [0,1], saturated at 2^64-1 (same rule as plgen.gaintab)
uint64_t prob_to_u64(double p) {
  if (!(p > 0)) return 0;
  if (p >= 1.0) return ~0ull;
  int e;
  double m = std::frexp(p, &e);             // p = m 2^e, m in [0.5, 1)
  uint64_t mant = (uint64_t)std::ldexp(m, 53);   // exact 53-bit integer
  int sh = 64 + e - 53;                     // p 2^64 = mant 2^(64+e-53)
  if (sh >= 0) return sh >= 11 + 53 ? ~0ull : (mant << sh);
  if (-sh >= 64) return 0;                  // p < 2^-64 (a shift >= 64 would be undefined)
  return mant >> (-sh);
}

double poisson_cdf(double lam, int k) {
  double term = std::exp(-lam), acc = term;
  for (int j = 1; j <= k; ++j) {
    term *= lam / j;
    acc += term;
  }
  return acc < 1.0 ? acc : 1.0;
}

}  // namespace

struct pl_pipeline {
  pl_config cfg;
  pl_stage stages[PL_MAX_STAGES];
  int64_t t[PL_MAX_STAGES], w[PL_MAX_STAGES];
  double g[PL_MAX_STAGES];
  bool have_g = false;
  uint32_t b[PL_MAX_STAGES], theta[PL_MAX_STAGES];
  uint32_t M = 0;
  bool dna = false;
  int k = 0;
  uint64_t q_len = 0, db_len = 0;
  std::vector<uint32_t> query;
  DevParams dp;
  uint32_t smem = 0, block = 0;
  cudaStream_t stream = nullptr;
  // device buffers
  uint32_t* d_db = nullptr;
  const uint32_t* d_db_bound = nullptr;   // caller-owned
  uint16_t *d_qoff = nullptr, *d_qpos = nullptr;
  uint32_t* d_qw = nullptr;
  uint2* d_spill = nullptr;
  uint2* d_mono = nullptr;
  int64_t *d_lat = nullptr, *d_lat_ns = nullptr;
  uint32_t* d_trace = nullptr;
  pl_match* d_matches = nullptr;
  uint64_t own_match_cap = 0;
  unsigned long long* d_match_count = nullptr;   // match count of the last launch (inside d_summary)
  uint32_t slot = 0;                             // d_summary slot of the next launch
  pl_firing* d_flog = nullptr;
  CtaStats* d_stats = nullptr;
  uint64_t roots_cap = 0;   // per-root arrays sized for this many roots
  uint64_t db_alloc_words = 0;
  // host state
  uint64_t pushed = 0;      // DNA: bases; gain: roots per stream
  bool launched = false;    // a run was launched since create / the last rewind (drain does not relaunch it)
  bool drained = false;
  uint32_t launches = 0;
  int device = 0;
  uint64_t h2d = 0, d2h = 0;  // bytes moved across the host boundary (cumulative)
  unsigned long long* d_scratch = nullptr;   // stage-batch counters
  unsigned long long* d_summary = nullptr;   // device-reduced run summary
  int64_t* d_arr = nullptr;                  // per-root arrival times (optional)
  std::vector<int64_t> h_arr;                // host copy (drain-window accounting)
  bool bound_host = false;
  // pl_pipeline_step: two pinned summary buffers + completion events, by step parity
  unsigned long long* h_step = nullptr;      // 2 x 7 words (cudaHostAlloc)
  cudaEvent_t step_ev[2] = {nullptr, nullptr};
  uint32_t step_launch[2] = {0, 0};          // launch index of the run in each buffer
  uint64_t steps = 0;                        // pl_pipeline_step calls since the last finish
  // live ingest (pl_pipeline_live_start / push_stream / push_all)
  bool live = false;                         // a live run is executing: pushes go to its rings
  uint32_t ring_words = 0;                   // R: ring words per stream
  uint32_t* d_ring = nullptr;                // [S][R] device rings
  uint32_t* d_front = nullptr;               // [S] doorbells (device)
  uint32_t* h_consumed = nullptr;            // [S] consumed watermarks (mapped pinned; written by the device)
  uint32_t* h_stage = nullptr;               // [S][R] pinned mirror of the rings (the copies' sources)
  uint32_t* h_bell = nullptr;                // [kBells][S] pinned doorbell slots
  cudaEvent_t bell_ev[16] = {};              // slot j's copy completed
  uint64_t bell_next = 0;
  cudaStream_t copy_stream = nullptr;        // non-blocking: copies run beside the executor
  std::vector<uint32_t> lw_lo, lw_end, lw_hi, lw_front;   // per stream: words [lo, end) pushed by the
                                             // caller, zero-padded to hi; front = next word to deliver
};

namespace {

void free_all(pl_pipeline* pl) {
  void* ptrs[] = {pl->d_db, pl->d_qoff, pl->d_qpos, pl->d_qw, pl->d_spill, pl->d_mono, pl->d_lat, pl->d_lat_ns,
                  pl->d_trace, pl->d_matches, pl->d_flog, pl->d_stats, pl->d_scratch,
                  pl->d_summary, pl->d_arr};
  for (void* p : ptrs)
    if (p) cudaFree(p);
  if (pl->h_step) cudaFreeHost(pl->h_step);
  if (pl->d_ring) cudaFree(pl->d_ring);
  if (pl->d_front) cudaFree(pl->d_front);
  if (pl->h_consumed) cudaFreeHost(pl->h_consumed);
  if (pl->h_stage) cudaFreeHost(pl->h_stage);
  if (pl->h_bell) cudaFreeHost(pl->h_bell);
  for (cudaEvent_t& e : pl->bell_ev)
    if (e) cudaEventDestroy(e);
  if (pl->copy_stream) cudaStreamDestroy(pl->copy_stream);
  for (cudaEvent_t& e : pl->step_ev)
    if (e) cudaEventDestroy(e);
}

bool v_too_big(const pl_pipeline* pl) { return pl->cfg.vector_width > 256; }

pl_status validate(const pl_config* c, const pl_workload* wl) {
  if (!c) return fail(PL_EINVAL, "cfg is NULL");
  const uint32_t N = c->n_stages;
  if (N < 1 || N > PL_MAX_STAGES) return fail(PL_EINVAL, "n_stages %u not in [1, %d]", N, PL_MAX_STAGES);
  if (!c->stages || !c->service_time) return fail(PL_EINVAL, "stages / service_time missing");
  const uint32_t v = c->vector_width;
  if (v != 32 && v != 64 && v != 128 && v != 256) return fail(PL_EINVAL, "vector_width %u not in {32,64,128,256}", v);
  if (N * v > 1024) return fail(PL_EINVAL, "N*v = %u exceeds 1024 threads", N * v);
  if (c->interarrival < 1) return fail(PL_EINVAL, "interarrival must be >= 1");
  if (c->deadline < 1) return fail(PL_EINVAL, "deadline must be >= 1");
  if (c->policy > PL_MONOLITHIC) return fail(PL_EINVAL, "bad policy %u", c->policy);
  if (c->clock > PL_CLOCK_GLOBALTIMER) return fail(PL_EINVAL, "bad clock %u", c->clock);
  if (c->clock == PL_CLOCK_GLOBALTIMER && !(c->ns_per_unit > 0)) return fail(PL_EINVAL, "ns_per_unit must be > 0");
  if (c->n_streams < 1 || c->n_streams > (1u << 20)) return fail(PL_EINVAL, "n_streams %u", c->n_streams);
  if (c->flags & PL_CLUSTER_NODES) {   // N4: one node per CTA of an N-CTA cluster
    if (c->policy == PL_MONOLITHIC) return fail(PL_EINVAL, "PL_CLUSTER_NODES: enforced policies only (one processor per node)");
    if (N > 8) return fail(PL_EINVAL, "PL_CLUSTER_NODES: N = %u exceeds the portable cluster size 8", N);
    if (v > 256) return fail(PL_EINVAL, "PL_CLUSTER_NODES: v must be <= 256");
  }
  bool dna = is_dna(c->stages[0].kind);
  for (uint32_t i = 0; i < N; ++i) {
    const pl_stage& s = c->stages[i];
    if (c->service_time[i] < 1) return fail(PL_EINVAL, "service_time[%u] must be >= 1", i);
    if (s.kind > PL_KEEP_EVERY) return fail(PL_EINVAL, "stage %u: bad kind %u", i, s.kind);
    if (is_dna(s.kind) != dna) return fail(PL_EINVAL, "stage %u mixes DNA and random-gain kinds", i);
    if (s.max_out < 1 || s.max_out > PL_MAX_U) return fail(PL_EINVAL, "stage %u: max_out %u", i, s.max_out);
    if (s.kind == PL_FIXED_GAIN && ((int)s.param < 0 || (uint32_t)s.param > s.max_out))
      return fail(PL_EINVAL, "stage %u: fixed gain %g exceeds max_out", i, s.param);
    if (s.kind == PL_KEEP_EVERY && (int)s.param < 1) return fail(PL_EINVAL, "stage %u: modulus < 1", i);
    if (s.kind == PL_BERNOULLI && !(s.param >= 0 && s.param <= 1)) return fail(PL_EINVAL, "stage %u: g not in [0,1]", i);
    if (s.kind == PL_POISSON_CAPPED && !(s.param >= 0)) return fail(PL_EINVAL, "stage %u: lambda < 0", i);
    if (s.kind != PL_FIXED_GAIN && s.kind != PL_POISSON_CAPPED && s.kind != PL_HIT_ENUM && s.max_out != 1)
      return fail(PL_EINVAL, "stage %u: filter stages have max_out 1", i);
  }
  if (c->wait_time)
    for (uint32_t i = 0; i < N; ++i)
      if (c->wait_time[i] < 0) return fail(PL_EINVAL, "wait_time[%u] < 0", i);
  if (c->wait_threshold)
    for (uint32_t i = 0; i < N; ++i)
      if (c->wait_threshold[i] < 1 || c->wait_threshold[i] > v) return fail(PL_EINVAL, "wait_threshold[%u] not in [1,v]", i);
  if (dna) {
    if (!wl || !wl->query) return fail(PL_EINVAL, "DNA pipeline needs a workload with a query");
    int k = c->stages[0].iparam[0];
    if (k < 1 || k > PL_MAX_K) return fail(PL_EINVAL, "k = %d not in [1, %d]", k, PL_MAX_K);
    for (uint32_t i = 0; i < N; ++i)
      if (c->stages[i].iparam[0] != k) return fail(PL_EINVAL, "stage %u: k differs", i);
    if (wl->q_len < (uint64_t)k || wl->q_len > 65535) return fail(PL_EINVAL, "q_len %llu", (unsigned long long)wl->q_len);
    if (wl->db_len >= (1ull << 32)) return fail(PL_EINVAL, "db_len must be < 2^32");
  } else {
    if (c->n_roots >= (1ull << 32) / c->n_streams) return fail(PL_EINVAL, "n_roots * n_streams must be < 2^32");
  }
  return PL_OK;
}

}  // namespace

extern "C" {

const char* pl_last_error(void) { return g_err.c_str(); }
const char* pl_version(void) { return "plgpu 0.1 sm_100a"; }

pl_status pl_solve_enforced_waits(const pl_config* cfg, int64_t* w_out, uint32_t* theta_out, double* T_out,
                                  double* T_cont) {
  if (!cfg || !cfg->service_time || !w_out) return fail(PL_EINVAL, "NULL argument");
  if (!cfg->gain && cfg->n_stages > 1) return fail(PL_EINVAL, "solver needs gains");
  const int N = (int)cfg->n_stages;
  if (N < 1 || N > PL_MAX_STAGES) return fail(PL_EINVAL, "n_stages");
  uint32_t b[PL_MAX_STAGES];
  for (int i = 0; i < N; ++i) b[i] = cfg->b ? cfg->b[i] : 1u;
  double g[PL_MAX_STAGES] = {0};
  for (int i = 0; i + 1 < N; ++i) g[i] = cfg->gain[i];
  double Pc[PL_MAX_STAGES], Tc, Ti;
  int64_t Pi[PL_MAX_STAGES];
  int st = plsolve::solve_fig1(N, cfg->service_time, g, b, cfg->vector_width, cfg->interarrival, cfg->deadline, Pc,
                               &Tc, Pi, &Ti);
  if (st == PL_EINVAL) return fail(PL_EINVAL, "gains must be > 0");
  if (st != PL_OK) return fail(PL_EINFEASIBLE, "Fig. 1 infeasible at tau0=%lld D=%lld", (long long)cfg->interarrival,
                               (long long)cfg->deadline);
  for (int i = 0; i < N; ++i) w_out[i] = Pi[i] - cfg->service_time[i];
  if (theta_out) plsolve::thresholds(N, g, Pi, cfg->interarrival, cfg->vector_width, theta_out);
  if (T_out) *T_out = Ti;
  if (T_cont) *T_cont = Tc;
  return PL_OK;
}

pl_status pl_solve_monolithic(const pl_config* cfg, uint32_t* M_out, double* T_out) {
  if (!cfg || !cfg->service_time || !M_out) return fail(PL_EINVAL, "NULL argument");
  if (!cfg->gain && cfg->n_stages > 1) return fail(PL_EINVAL, "solver needs gains");
  const int N = (int)cfg->n_stages;
  double g[PL_MAX_STAGES] = {0};
  for (int i = 0; i + 1 < N; ++i) g[i] = cfg->gain[i];
  double T;
  int st = plsolve::solve_fig2(N, cfg->service_time, g, cfg->vector_width, cfg->interarrival, cfg->deadline,
                               cfg->mono_b ? (double)cfg->mono_b : 1.0, cfg->mono_S > 0 ? cfg->mono_S : 1.0, M_out, &T);
  if (st != PL_OK) return fail(PL_EINFEASIBLE, "Fig. 2 infeasible at tau0=%lld D=%lld", (long long)cfg->interarrival,
                               (long long)cfg->deadline);
  if (T_out) *T_out = T;
  return PL_OK;
}

pl_status pl_pipeline_create(const pl_config* cfg, const pl_workload* wl, pl_pipeline** out) {
  if (!out) return fail(PL_EINVAL, "out is NULL");
  *out = nullptr;
  pl_status st = validate(cfg, wl);
  if (st != PL_OK) return st;
  pl_pipeline* pl = new (std::nothrow) pl_pipeline();
  if (!pl) return fail(PL_ENOMEM, "host allocation failed");
  const uint32_t N = cfg->n_stages;
  pl->cfg = *cfg;
  for (uint32_t i = 0; i < N; ++i) {
    pl->stages[i] = cfg->stages[i];
    pl->t[i] = cfg->service_time[i];
    pl->b[i] = cfg->b ? cfg->b[i] : 1u;
  }
  pl->cfg.stages = pl->stages;
  pl->cfg.service_time = pl->t;
  pl->cfg.b = pl->b;
  pl->have_g = cfg->gain != nullptr;
  for (uint32_t i = 0; i + 1 < N; ++i) pl->g[i] = cfg->gain ? cfg->gain[i] : 0.0;
  pl->cfg.gain = pl->have_g ? pl->g : nullptr;
  pl->dna = is_dna(cfg->stages[0].kind);
  pl->device = cfg->device;
  auto bail = [&](pl_status s) {
    std::string keep = g_err;
    free_all(pl);
    delete pl;
    g_err = keep;
    return s;
  };
  // ---- schedule parameters
  const uint32_t v = cfg->vector_width;
  if (cfg->policy == PL_FIXED_WAIT || cfg->policy == PL_THRESHOLD_SLACK) {
    if (cfg->wait_time) {
      for (uint32_t i = 0; i < N; ++i) pl->w[i] = cfg->wait_time[i];
    } else if (cfg->policy == PL_FIXED_WAIT || !cfg->wait_threshold) {
      if (!pl->have_g && N > 1) return bail(fail(PL_EINVAL, "wait_time missing and no gains to solve Fig. 1"));
      double T;
      st = pl_solve_enforced_waits(&pl->cfg, pl->w, nullptr, &T, nullptr);
      if (st != PL_OK) return bail(st);
    }
    if (cfg->wait_threshold) {
      for (uint32_t i = 0; i < N; ++i) pl->theta[i] = cfg->wait_threshold[i];
    } else if (cfg->policy == PL_THRESHOLD_SLACK) {
      if (!pl->have_g && N > 1) return bail(fail(PL_EINVAL, "wait_threshold missing and no gains"));
      int64_t P[PL_MAX_STAGES];
      for (uint32_t i = 0; i < N; ++i) P[i] = pl->t[i] + pl->w[i];
      plsolve::thresholds((int)N, pl->g, P, cfg->interarrival, v, pl->theta);
    }
  } else {
    pl->M = cfg->block_size;
    if (!pl->M) {
      if (!pl->have_g && N > 1) return bail(fail(PL_EINVAL, "block_size missing and no gains to solve Fig. 2"));
      double T;
      st = pl_solve_monolithic(&pl->cfg, &pl->M, &T);
      if (st != PL_OK) return bail(st);
    }
  }
  pl->cfg.wait_time = pl->w;
  pl->cfg.wait_threshold = pl->theta;
  // ---- device
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return bail(fail(PL_EDEVICE, "no CUDA device"));
  if (cfg->device < 0 || cfg->device >= ndev) return bail(fail(PL_EINVAL, "device %d of %d", cfg->device, ndev));
  if (cudaSetDevice(cfg->device) != cudaSuccess) return bail(fail(PL_EDEVICE, "cudaSetDevice failed"));
  cudaDeviceProp prop;
  cudaGetDeviceProperties(&prop, cfg->device);
  if (prop.major != 10) return bail(fail(PL_EDEVICE, "built for sm_100a; device is sm_%d%d", prop.major, prop.minor));

  DevParams& d = pl->dp;
  std::memset(&d, 0, sizeof d);
  d.N = (int)N;
  d.v = (int)v;
  d.policy = (int)cfg->policy;
  d.clock = (int)cfg->clock;
  for (uint32_t i = 0; i < N; ++i) {
    d.t[i] = pl->t[i];
    d.P[i] = pl->t[i] + pl->w[i];
    d.theta[i] = pl->theta[i] ? pl->theta[i] : 1u;
    int64_t r = pl->t[i];
    for (uint32_t j = i + 1; j < N; ++j) r += 2 * pl->t[j];   // R_i = t_i + 2 sum_{j>i} t_j (R-THRESH)
    d.R[i] = r + cfg->slack_guard;
  }
  d.D = cfg->deadline;
  d.tau = cfg->interarrival;
  d.tau_m = d.tau > 1 ? ~0ull / (uint64_t)d.tau : 0;
  for (uint32_t i = 0; i < N; ++i) d.P_m[i] = d.P[i] > 1 ? ~0ull / (uint64_t)d.P[i] : 0;
  d.M = pl->M;
  d.ns_per_unit = cfg->clock == PL_CLOCK_GLOBALTIMER ? cfg->ns_per_unit : 1.0;
  d.seed = cfg->seed;
  d.n_streams = (int)cfg->n_streams;
  d.flags = cfg->flags;
  for (uint32_t i = 0; i < N; ++i) {
    const pl_stage& s = pl->stages[i];
    DevStage& ds = d.st[i];
    ds.kind = s.kind;
    ds.max_out = s.max_out;
    for (int j = 0; j < 4; ++j) ds.ip[j] = s.iparam[j];
    ds.cfix = (s.kind == PL_FIXED_GAIN || s.kind == PL_KEEP_EVERY) ? (uint32_t)s.param : 0u;
    if (s.kind == PL_BERNOULLI) ds.thr[0] = prob_to_u64(s.param);
    if (s.kind == PL_POISSON_CAPPED)
      for (uint32_t j = 0; j < s.max_out; ++j) ds.thr[j] = prob_to_u64(poisson_cdf(s.param, (int)j));
  }
  // ---- DNA: query index (direct-address k-mer table; counting sort keeps q ascending)
  if (pl->dna) {
    pl->k = cfg->stages[0].iparam[0];
    pl->q_len = wl->q_len;
    pl->db_len = wl->db_len;
    const uint32_t nqw = (uint32_t)((wl->q_len + 15) / 16);
    pl->query.assign(wl->query, wl->query + nqw);
    const uint32_t K = 1u << (2 * pl->k);
    const uint32_t nq = (uint32_t)(wl->q_len - pl->k + 1);
    std::vector<uint16_t> off(K + 1, 0), pos(nq);
    std::vector<uint32_t> keys(nq);
    auto qb = [&](uint64_t j) { return (pl->query[j >> 4] >> ((j & 15) * 2)) & 3u; };
    for (uint32_t q = 0; q < nq; ++q) {
      uint32_t key = 0;
      for (int j = 0; j < pl->k; ++j) key = (key << 2) | qb(q + j);
      keys[q] = key;
      off[key + 1]++;
    }
    for (uint32_t j = 0; j < K; ++j) off[j + 1] += off[j];
    std::vector<uint16_t> fill(off.begin(), off.end() - 1);
    for (uint32_t q = 0; q < nq; ++q) pos[fill[keys[q]]++] = (uint16_t)q;
    // padded to whole 16-byte units: the kernel stages them with cp.async.bulk
    const size_t b_qo = ((K + 1) * 2 + 15) & ~size_t(15), b_qp = (nq * 2 + 15) & ~size_t(15),
                 b_qw = (nqw * 4 + 15) & ~size_t(15);
    if (cudaMalloc(&pl->d_qoff, b_qo) != cudaSuccess || cudaMalloc(&pl->d_qpos, b_qp) != cudaSuccess ||
        cudaMalloc(&pl->d_qw, b_qw) != cudaSuccess)
      return bail(fail(PL_ENOMEM, "query index allocation"));
    cudaMemset(pl->d_qoff, 0, b_qo);
    cudaMemset(pl->d_qpos, 0, b_qp);
    cudaMemset(pl->d_qw, 0, b_qw);
    cudaMemcpy(pl->d_qoff, off.data(), (K + 1) * 2, cudaMemcpyHostToDevice);
    cudaMemcpy(pl->d_qpos, pos.data(), nq * 2, cudaMemcpyHostToDevice);
    cudaMemcpy(pl->d_qw, pl->query.data(), nqw * 4, cudaMemcpyHostToDevice);
    d.k = pl->k;
    d.q_len = (int)wl->q_len;
    d.qoff = pl->d_qoff;
    d.qpos = pl->d_qpos;
    d.qwords = pl->d_qw;
    const uint64_t dbw = (wl->db_len + 15) / 16 + 8;     // padded: TMA copies whole 16-byte units
    if (cudaMalloc(&pl->d_db, dbw * 4) != cudaSuccess) return bail(fail(PL_ENOMEM, "DB allocation"));
    cudaMemset(pl->d_db, 0, dbw * 4);
    pl->db_alloc_words = dbw;
    // smem DB window per stream: its roots + k-1 overlap + halo on both sides, as a ring of
    // chunks refilled by TMA as the stream advances (executor.cu win_step).  Default: the whole
    // stream range when it fits in 16 chunks of 1024 words (64 KB), else a 64 KB sliding ring.
    const uint64_t R = wl->db_len >= (uint64_t)pl->k ? wl->db_len - pl->k + 1 : 0;
    const uint64_t per = (R + cfg->n_streams - 1) / cfg->n_streams;
    // halo: an extension walks at most q_len bases from its seed (Dna::right/left_limit), so
    // with q_len + 48 every walk of an interior root stays in the window (Dna::extend_win)
    d.win_halo = std::max<uint32_t>(512u, (uint32_t)wl->q_len + 48u);
    const uint32_t CH = cfg->window_chunk_words ? cfg->window_chunk_words : 1024u;
    if (!is_pow2(CH) || CH < 4) return bail(fail(PL_EINVAL, "window_chunk_words must be a power of 2 >= 4"));
    uint64_t words = (per + pl->k + 2 * d.win_halo) / 16 + 8;
    words = (words + 3) & ~3ull;
    const uint64_t chunks = (words + CH - 1) / CH + 1;     // + 1: chunks sit at absolute boundaries
    // a sliding ring of 8 chunks (32 KB = 128 K bases) holds far more than a stream's in-flight
    // roots plus the extension halo; the rest of the smem goes to the queues (below)
    uint32_t cap = CH * (chunks <= 16 ? next_pow2((uint32_t)chunks) : 8u);
    if (cfg->window_words) {
      if (!is_pow2(cfg->window_words) || cfg->window_words < 2 * CH)
        return bail(fail(PL_EINVAL, "window_words must be a power of 2 >= 2 * window_chunk_words"));
      cap = cfg->window_words;
    }
    d.win_cap = cap;
    d.win_lg = 0;
    while ((1u << d.win_lg) < CH) ++d.win_lg;
    pl->roots_cap = wl->db_len >= (uint64_t)pl->k ? wl->db_len - pl->k + 1 : 0;
  } else {
    pl->roots_cap = cfg->n_roots * cfg->n_streams;
  }
  // ---- queues
  const uint32_t S = cfg->n_streams;
  d.segcap = next_pow2(2 * v);
  uint32_t maxu = 1;
  for (uint32_t i = 1; i < N; ++i) {
    const uint32_t u = pl->stages[i - 1].max_out;
    if (u > maxu) maxu = u;
    uint32_t cap = cfg->queue_capacity ? cfg->queue_capacity : next_pow2(std::max(4 * v, v * (u + 1)));
    if (!is_pow2(cap)) return bail(fail(PL_EINVAL, "queue_capacity must be a power of 2"));
    d.cap_s[i] = cap;
  }
  d.cap_g = cfg->spill_capacity ? cfg->spill_capacity : (1u << 15);
  if (!is_pow2(d.cap_g)) return bail(fail(PL_EINVAL, "spill_capacity must be a power of 2"));
  if (d.cap_g < v * (maxu + 1)) return bail(fail(PL_EINVAL, "spill_capacity < v*(u+1) can deadlock"));
  for (uint32_t i = 1; i < N; ++i)
    if (d.cap_g < d.cap_s[i]) return bail(fail(PL_EINVAL, "spill_capacity smaller than the smem ring"));
  if (cfg->policy == PL_MONOLITHIC) {
    for (uint32_t i = 0; i < PL_MAX_STAGES; ++i) d.cap_s[i] = 0;
    d.segcap = 0;
    uint64_t mx = pl->M, cur = pl->M;
    for (uint32_t i = 0; i + 1 < N; ++i) {
      cur *= pl->stages[i].max_out;
      mx = std::max(mx, cur);
    }
    d.mono_cap = (uint32_t)std::min<uint64_t>(mx, 1u << 24);
    if (cudaMalloc(&pl->d_mono, (size_t)S * 2 * d.mono_cap * sizeof(uint2)) != cudaSuccess)
      return bail(fail(PL_ENOMEM, "monolithic buffers"));
    pl->block = std::min<uint32_t>(N * v, 1024);
  } else {
    if (N > 1 && cudaMalloc(&pl->d_spill, (size_t)S * N * d.cap_g * sizeof(uint2)) != cudaSuccess)
      return bail(fail(PL_ENOMEM, "spill rings (%u streams x %u edges x %u)", S, N, d.cap_g));
    pl->block = N * v;             // one warp group of v lanes per node (executor.cu run_node)
  }
  d.spill = pl->d_spill;
  d.mono_buf = pl->d_mono;
  pl->smem = pl_layout_enforced_host(d);
  // Spare shared memory deepens the smem ring behind the largest amplifier (the edge whose
  // producer has the largest u): a burst of u outputs per input -- or the backlog after a
  // platform stall -- then stays on chip instead of spilling to the HBM ring.
  if (!cfg->queue_capacity && cfg->policy != PL_MONOLITHIC && N > 1) {
    uint32_t e = 1;
    for (uint32_t i = 2; i < N; ++i)
      if (pl->stages[i - 1].max_out > pl->stages[e - 1].max_out) e = i;
    while (2 * d.cap_s[e] <= d.cap_g) {
      d.cap_s[e] *= 2;
      if (pl_layout_enforced_host(d) > 196 * 1024) { d.cap_s[e] /= 2; break; }
    }
    pl->smem = pl_layout_enforced_host(d);
  }
  // one CTA (stream) per SM: the two-per-SM variant (64 registers) spills and measured no gain
  // (tools/streams_scaling.py); it stays selectable through PL_CTAS_PER_SM=2
  d.ctas_per_sm = 1;
  // bit 1: node 0's leader paces and one barrier releases its lanes (instead of every warp
  // pacing itself): on c4 the executor issues 17 % fewer instructions at the same rate
  // (ncu, profiles/r02_bench_ab_leader_paced.json); PL_VARIANT overrides the experiment bits
  d.variant = 1u;
  if (const char* e = getenv("PL_VARIANT")) d.variant = (uint32_t)atoi(e);
  // physical clock: a stream's time origin is set this far after its CTA has staged its
  // inputs, so that every warp group is resident before the first arrival
  d.t0_offset_ns = 2048;
  if (const char* e = getenv("PL_T0_OFFSET_NS")) d.t0_offset_ns = (uint32_t)atoi(e);
  if (const char* e = getenv("PL_CTAS_PER_SM"))
    if (atoi(e) == 2 && pl->block <= 512 && 2 * (pl->smem + 4096) <= (uint32_t)prop.sharedMemPerMultiprocessor)
      d.ctas_per_sm = 2;
  if (pl->smem > 200 * 1024) return bail(fail(PL_EINVAL, "smem layout %u B exceeds budget; lower queue_capacity", pl->smem));
  // ---- outputs
  const uint64_t R = std::max<uint64_t>(pl->roots_cap, 1);
  if (cfg->flags & PL_REC_LATENCY) {
    if (cudaMalloc(&pl->d_lat, R * 8) != cudaSuccess || cudaMalloc(&pl->d_lat_ns, R * 8) != cudaSuccess)
      return bail(fail(PL_ENOMEM, "latency arrays"));
  }
  if (cfg->flags & PL_REC_TRACE) {
    if (cudaMalloc(&pl->d_trace, R * (N + 1) * 4) != cudaSuccess) return bail(fail(PL_ENOMEM, "trace array"));
  }
  d.log_cap = (cfg->flags & PL_REC_FIRINGS) ? (cfg->firing_log_capacity ? cfg->firing_log_capacity : (1u << 16)) : 0u;
  if (d.log_cap && cudaMalloc(&pl->d_flog, (size_t)S * d.log_cap * sizeof(pl_firing)) != cudaSuccess)
    return bail(fail(PL_ENOMEM, "firing log"));
  d.match_cap = cfg->match_capacity ? cfg->match_capacity : (1ull << 20);
  if (!pl->dna) d.match_cap = 1;
  pl->own_match_cap = d.match_cap;
  if (cudaMalloc(&pl->d_matches, d.match_cap * sizeof(pl_match)) != cudaSuccess ||
      cudaMalloc(&pl->d_stats, S * sizeof(CtaStats)) != cudaSuccess)
    return bail(fail(PL_ENOMEM, "output buffers"));
  cudaMemset(pl->d_stats, 0, S * sizeof(CtaStats));
  // run summary + match count, double-buffered: launch k accumulates into slot k & 1 and
  // zeroes the other slot for launch k+1, so a launch needs no host-side memset
  if (cudaMalloc(&pl->d_summary, 2 * 8 * 8) != cudaSuccess) return bail(fail(PL_ENOMEM, "summary"));
  cudaMemset(pl->d_summary, 0, 2 * 64);
  pl->slot = 0;
  pl->d_match_count = pl->d_summary + 6;
  d.lat = pl->d_lat;
  d.lat_ns = cfg->clock == PL_CLOCK_GLOBALTIMER ? pl->d_lat_ns : nullptr;
  if (!(cfg->flags & PL_REC_LATENCY)) d.lat_ns = nullptr;
  d.trace = pl->d_trace;
  d.matches = pl->d_matches;
  d.match_count = pl->d_summary + 6;
  d.flog = pl->d_flog;
  d.stats = pl->d_stats;
  d.summary = pl->d_summary;
  d.summary_next = pl->d_summary + 8;
  if (cfg->arrivals) {   // arrival process given as data (Poisson, L263): per root, per stream
    if (cfg->n_arrivals != pl->roots_cap)
      return bail(fail(PL_EINVAL, "n_arrivals %llu != root count %llu", (unsigned long long)cfg->n_arrivals,
                       (unsigned long long)pl->roots_cap));
    const uint64_t R = pl->roots_cap;
    for (uint32_t s = 0; s < S; ++s) {
      const uint64_t lo = R * s / S, hi = R * (s + 1) / S;
      for (uint64_t r = lo; r < hi; ++r)
        if (cfg->arrivals[r] < 0 || (r > lo && cfg->arrivals[r] < cfg->arrivals[r - 1]))
          return bail(fail(PL_EINVAL, "arrivals must be >= 0 and non-decreasing within a stream"));
    }
    if (cudaMalloc(&pl->d_arr, R * 8) != cudaSuccess) return bail(fail(PL_ENOMEM, "arrival times"));
    cudaMemcpy(pl->d_arr, cfg->arrivals, R * 8, cudaMemcpyHostToDevice);
    pl->h_arr.assign(cfg->arrivals, cfg->arrivals + R);
    pl->h2d += R * 8;
  }
  d.arr = pl->d_arr;
  cudaError_t e1 = pl_kernel_attributes(200 * 1024);
  if (e1 != cudaSuccess) return bail(fail(PL_EDEVICE, "cudaFuncSetAttribute: %s", cudaGetErrorString(e1)));
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) return bail(fail(PL_EDEVICE, "create: %s", cudaGetErrorString(e)));
  *out = pl;
  return PL_OK;
}

pl_status pl_pipeline_set_stream(pl_pipeline* pl, void* stream) {
  if (!pl) return fail(PL_EINVAL, "NULL pipeline");
  pl->stream = (cudaStream_t)stream;
  return PL_OK;
}

pl_status pl_pipeline_push(pl_pipeline* pl, const void* items, uint64_t n) {
  if (!pl) return fail(PL_EINVAL, "NULL pipeline");
  if (pl->live) return fail(PL_ESTATE, "a live run is executing: use pl_pipeline_push_stream / push_all");
  if (pl->drained) return fail(PL_ESTATE, "push after drain; call pl_pipeline_rewind");
  if (pl->dna) {
    if (!items) return fail(PL_EINVAL, "DNA push needs items");
    if (pl->d_db_bound) return fail(PL_ESTATE, "a device DB is bound");
    if (pl->pushed % 16) return fail(PL_EINVAL, "previous push was not a multiple of 16 bases");
    if (pl->pushed + n > pl->db_len) return fail(PL_EINVAL, "push exceeds db_len");
    cudaSetDevice(pl->device);
    const uint64_t words = (n + 15) / 16;
    CUDA_TRY(cudaMemcpyAsync(pl->d_db + pl->pushed / 16, items, words * 4, cudaMemcpyHostToDevice, pl->stream));
    // pl.h promises `items` may be reused on return: a copy from pageable memory is staged before
    // cudaMemcpyAsync returns, one from page-locked memory is not -- wait for that one
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, items) != cudaSuccess) cudaGetLastError();
    else if (at.type == cudaMemoryTypeHost) CUDA_TRY(cudaStreamSynchronize(pl->stream));
    pl->h2d += words * 4;
    pl->pushed += n;
  } else {
    if (items) return fail(PL_EINVAL, "random-gain push takes items == NULL");
    if (pl->pushed + n > pl->cfg.n_roots) return fail(PL_EINVAL, "push exceeds n_roots");
    pl->pushed += n;
  }
  return PL_OK;
}

pl_status pl_pipeline_bind_device(pl_pipeline* pl, const void* dev_items, uint64_t n) {
  if (!pl || !dev_items) return fail(PL_EINVAL, "NULL argument");
  if (!pl->dna) return fail(PL_EINVAL, "bind_device is for DNA pipelines");
  if (n > pl->db_len) return fail(PL_EINVAL, "bound DB longer than db_len");
  pl->d_db_bound = (const uint32_t*)dev_items;
  pl->bound_host = false;
  pl->pushed = n;
  pl->launched = false;
  return PL_OK;
}

pl_status pl_pipeline_bind_host(pl_pipeline* pl, const void* host_items, uint64_t n) {
  if (!pl || !host_items) return fail(PL_EINVAL, "NULL argument");
  if (!pl->dna) return fail(PL_EINVAL, "bind_host is for DNA pipelines");
  if (n > pl->db_len) return fail(PL_EINVAL, "bound DB longer than db_len");
  cudaSetDevice(pl->device);
  void* dptr = nullptr;
  cudaError_t e = cudaHostGetDevicePointer(&dptr, const_cast<void*>(host_items), 0);
  if (e != cudaSuccess || !dptr) {
    cudaGetLastError();
    return fail(PL_EINVAL, "host buffer is not pinned+mapped (cudaHostAlloc / cudaHostRegisterMapped)");
  }
  pl->d_db_bound = (const uint32_t*)dptr;
  pl->bound_host = true;
  pl->pushed = n;
  pl->launched = false;
  return PL_OK;
}

pl_status pl_pipeline_bind_results(pl_pipeline* pl, void* buf, uint64_t cap) {
  if (!pl) return fail(PL_EINVAL, "NULL pipeline");
  if (!buf) {
    pl->dp.matches = pl->d_matches;
    pl->dp.match_cap = pl->own_match_cap;
    return PL_OK;
  }
  if (!cap) return fail(PL_EINVAL, "cap must be > 0");
  cudaSetDevice(pl->device);
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, buf) != cudaSuccess) {
    cudaGetLastError();
    return fail(PL_EINVAL, "results buffer is neither device memory nor registered host memory");
  }
  void* dptr = buf;
  if (at.type == cudaMemoryTypeHost) {
    if (cudaHostGetDevicePointer(&dptr, buf, 0) != cudaSuccess || !dptr) {
      cudaGetLastError();
      return fail(PL_EINVAL, "host results buffer is not mapped (cudaHostAllocMapped / cudaHostRegisterMapped)");
    }
  } else if (at.type != cudaMemoryTypeDevice && at.type != cudaMemoryTypeManaged) {
    return fail(PL_EINVAL, "results buffer is neither device memory nor pinned host memory");
  }
  pl->dp.matches = (pl_match*)dptr;
  pl->dp.match_cap = cap;
  return PL_OK;
}

pl_status pl_pipeline_queue_peaks(pl_pipeline* pl, uint32_t* buf, uint64_t cap, uint64_t* n) {
  if (!pl || !n) return fail(PL_EINVAL, "NULL argument");
  const uint32_t S = pl->cfg.n_streams, N = pl->cfg.n_stages;
  if (!buf) { *n = (uint64_t)S * N; return PL_OK; }
  cudaSetDevice(pl->device);
  CUDA_TRY(cudaStreamSynchronize(pl->stream));
  std::vector<CtaStats> cs(S);
  CUDA_TRY(cudaMemcpy(cs.data(), pl->d_stats, S * sizeof(CtaStats), cudaMemcpyDeviceToHost));
  pl->d2h += S * sizeof(CtaStats);
  uint64_t w = 0;
  for (uint32_t s = 0; s < S; ++s)
    for (uint32_t i = 0; i < N && w < cap; ++i) buf[w++] = cs[s].max_queue[i];
  *n = w;
  return PL_OK;
}

namespace {
void decode_summary(const pl_pipeline* pl, const unsigned long long* h, uint32_t launch, pl_summary* out) {
  out->roots = h[0];
  out->miss_events = h[1];
  out->miss_events_ns = h[5];
  out->max_latency = (int64_t)h[2];
  out->max_latency_ns = (int64_t)h[3];
  out->errors = (uint32_t)h[4];
  out->matches = std::min<uint64_t>(h[6], pl->dp.match_cap);
  out->launches = launch;
  out->latency_outliers = h[7];
}
}  // namespace

pl_status pl_pipeline_summary(pl_pipeline* pl, pl_summary* out) {
  if (!pl || !out) return fail(PL_EINVAL, "NULL argument");
  cudaSetDevice(pl->device);
  unsigned long long h[8];
  CUDA_TRY(cudaMemcpyAsync(h, pl->d_match_count - 6, 64, cudaMemcpyDeviceToHost, pl->stream));
  CUDA_TRY(cudaStreamSynchronize(pl->stream));
  pl->d2h += 64;
  decode_summary(pl, h, pl->launches, out);
  return PL_OK;
}


pl_status pl_pipeline_step(pl_pipeline* pl, pl_summary* prev, int* has_prev) {
  if (!pl || !prev || !has_prev) return fail(PL_EINVAL, "NULL argument");
  cudaSetDevice(pl->device);
  if (!pl->h_step) {
    CUDA_TRY(cudaHostAlloc((void**)&pl->h_step, 2 * 8 * sizeof(unsigned long long), cudaHostAllocDefault));
    for (cudaEvent_t& e : pl->step_ev) CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  }
  const uint32_t b = (uint32_t)(pl->steps & 1u);
  pl_status st = pl_pipeline_launch(pl);
  if (st != PL_OK) return st;
  // the run's summary slot is copied before the next launch (which zeroes it) can start
  CUDA_TRY(cudaMemcpyAsync(pl->h_step + 8 * b, pl->d_match_count - 6, 64, cudaMemcpyDeviceToHost, pl->stream));
  CUDA_TRY(cudaEventRecord(pl->step_ev[b], pl->stream));
  pl->step_launch[b] = pl->launches;
  pl->d2h += 64;
  *has_prev = 0;
  if (pl->steps > 0) {   // the previous step's run: wait for it only, the new one keeps running
    const uint32_t pb = b ^ 1u;
    CUDA_TRY(cudaEventSynchronize(pl->step_ev[pb]));
    decode_summary(pl, pl->h_step + 8 * pb, pl->step_launch[pb], prev);
    *has_prev = 1;
  }
  ++pl->steps;
  return PL_OK;
}

pl_status pl_pipeline_step_finish(pl_pipeline* pl, pl_summary* last, int* has_last) {
  if (!pl || !last || !has_last) return fail(PL_EINVAL, "NULL argument");
  cudaSetDevice(pl->device);
  *has_last = 0;
  if (pl->steps > 0) {
    const uint32_t b = (uint32_t)((pl->steps - 1) & 1u);
    CUDA_TRY(cudaEventSynchronize(pl->step_ev[b]));
    decode_summary(pl, pl->h_step + 8 * b, pl->step_launch[b], last);
    *has_last = 1;
  }
  pl->steps = 0;
  return PL_OK;
}


// ------------------------------------------------------------------ live ingest
namespace {
constexpr uint32_t kBells = 16;
// Stream s's DB word range [wlo, whi): its roots plus the k-1 overlap and the extension halo on
// both sides, 16-byte aligned -- the same computation as the executor's cta_setup.
void stream_words_range(const pl_pipeline* pl, uint32_t s, uint32_t* lo_out, uint32_t* hi_out) {
  const DevParams& p = pl->dp;
  const uint64_t total = pl->db_len >= (uint64_t)pl->k ? pl->db_len - pl->k + 1 : 0;
  const uint64_t S = pl->cfg.n_streams;
  const uint64_t lo = (total * s) / S, hi = (total * (s + 1)) / S;
  int64_t wlo = 0, whi = 0;
  if (p.win_cap > 0 && hi > lo) {
    wlo = ((int64_t)lo - (int64_t)p.win_halo) >> 4;
    whi = (((int64_t)hi + p.k + (int64_t)p.win_halo) >> 4) + 1;
    wlo = wlo < 0 ? 0 : (wlo & ~3ll);
    whi = (whi + 3) & ~3ll;
    if (whi > (int64_t)pl->db_alloc_words) whi = (int64_t)pl->db_alloc_words & ~3ll;
    if (whi < wlo) whi = wlo;
  }
  *lo_out = (uint32_t)wlo;
  *hi_out = (uint32_t)whi;
}

// Stage words of stream s into its pinned host mirror (slot = word & (R-1), as on the device)
// and enqueue the copy of that slot range to the device ring.  The mirror's slots are reused on
// the same condition as the ring's (the device consumed them), which implies the copy was done.
cudaError_t stage_copy(pl_pipeline* pl, uint32_t s, uint32_t f, const uint32_t* words, uint32_t n) {
  const uint32_t R = pl->ring_words;
  uint32_t* h = pl->h_stage + (size_t)s * R + (f & (R - 1));
  if (words) std::memcpy(h, words, (size_t)n * 4);
  else std::memset(h, 0, (size_t)n * 4);
  return cudaMemcpyAsync(pl->d_ring + (size_t)s * R + (f & (R - 1)), h, (size_t)n * 4, cudaMemcpyHostToDevice,
                         pl->copy_stream);
}

// Ring the doorbells of streams [s0, s0 + count) behind every copy enqueued so far: their fronts
// go through a pinned slot (one of kBells, reused once its copy has completed) to d_front.
cudaError_t ring_bells(pl_pipeline* pl, uint32_t s0, uint32_t count) {
  const uint32_t S = pl->cfg.n_streams;
  const uint32_t j = (uint32_t)(pl->bell_next++ % kBells);
  cudaError_t e = cudaEventSynchronize(pl->bell_ev[j]);
  if (e != cudaSuccess) return e;
  uint32_t* slot = pl->h_bell + (size_t)j * S;
  std::memcpy(slot + s0, pl->lw_front.data() + s0, (size_t)count * 4);
  e = cudaMemcpyAsync(pl->d_front + s0, slot + s0, (size_t)count * 4, cudaMemcpyHostToDevice, pl->copy_stream);
  if (e != cudaSuccess) return e;
  return cudaEventRecord(pl->bell_ev[j], pl->copy_stream);
}

// Enqueue up to n words of stream s (as many as its ring has room for); *full = the ring had
// no room for the rest.
pl_status push_some(pl_pipeline* pl, uint32_t s, const uint32_t*& words, uint64_t& n, bool* full) {
  const uint32_t R = pl->ring_words;
  uint32_t& f = pl->lw_front[s];
  *full = false;
  auto room = [&]() {
    const uint32_t cons = std::max<uint32_t>(pl->lw_lo[s], (uint32_t)*(volatile uint32_t*)(pl->h_consumed + s));
    return (uint64_t)R - (uint64_t)(f - std::min(f, cons));
  };
  while (n > 0) {
    const uint64_t space = room();
    if (space == 0) { *full = true; break; }
    const uint32_t piece = (uint32_t)std::min<uint64_t>(std::min<uint64_t>(n, space), R - (f & (R - 1)));
    CUDA_TRY(stage_copy(pl, s, f, words, piece));
    f += piece;
    words += piece;
    n -= piece;
    pl->h2d += (uint64_t)piece * 4;
  }
  if (n == 0 && f == pl->lw_end[s] && f < pl->lw_hi[s]) {   // the stream's last words: zero-pad to hi
    const uint32_t pad = pl->lw_hi[s] - f;                    // (<= 11 words past the DB's end)
    if (room() < pad) { *full = true; return PL_OK; }
    const uint32_t first = std::min(pad, R - (f & (R - 1)));
    CUDA_TRY(stage_copy(pl, s, f, nullptr, first));
    if (pad > first) CUDA_TRY(stage_copy(pl, s, f + first, nullptr, pad - first));
    f += pad;
  }
  return PL_OK;
}

pl_status push_streams(pl_pipeline* pl, uint32_t s0, uint32_t count, const uint32_t* const* words,
                       const uint64_t* n, int nonblocking) {
  if (!pl) return fail(PL_EINVAL, "NULL pipeline");
  if (!pl->live) return fail(PL_ESTATE, "no live run (pl_pipeline_live_start)");
  if (!words || !n) return fail(PL_EINVAL, "NULL argument");
  const uint32_t R = pl->ring_words;
  for (uint32_t j = 0; j < count; ++j) {
    const uint32_t s = s0 + j;
    if (n[j] && !words[j]) return fail(PL_EINVAL, "stream %u: NULL words", s);
    if (n[j] && (uint64_t)pl->lw_front[s] + n[j] > pl->lw_end[s])
      return fail(PL_EINVAL, "stream %u: push of %llu words exceeds its range (%u left)", s,
                  (unsigned long long)n[j], pl->lw_end[s] - std::min(pl->lw_end[s], pl->lw_front[s]));
    if (nonblocking) {
      const uint32_t cons = std::max<uint32_t>(pl->lw_lo[s], (uint32_t)*(volatile uint32_t*)(pl->h_consumed + s));
      const uint64_t used = pl->lw_front[s] - std::min(pl->lw_front[s], cons);
      if (used + n[j] + 16 > R) return fail(PL_EAGAIN, "stream %u: ring full (%llu of %u words in use)", s,
                                            (unsigned long long)used, R);
    }
  }
  cudaSetDevice(pl->device);
  std::vector<const uint32_t*> w(words, words + count);
  std::vector<uint64_t> left(n, n + count);
  const auto t_start = std::chrono::steady_clock::now();
  for (;;) {
    bool any_full = false, progress = false;
    for (uint32_t j = 0; j < count; ++j) {
      const uint32_t s = s0 + j;
      const uint32_t f0 = pl->lw_front[s];
      bool full = false;
      pl_status st = push_some(pl, s, w[j], left[j], &full);
      if (st != PL_OK) return st;
      any_full |= full;
      progress |= pl->lw_front[s] != f0;
    }
    if (progress) CUDA_TRY(ring_bells(pl, s0, count));   // behind the data, in copy-stream order
    if (!any_full) break;
    if (std::chrono::steady_clock::now() - t_start > std::chrono::seconds(10))
      return fail(PL_EAGAIN, "live ring full for 10 s: the executor is not consuming");
    std::this_thread::yield();
  }
  return PL_OK;
}
}  // namespace

pl_status pl_pipeline_live_start(pl_pipeline* pl, uint32_t ring_words) {
  if (!pl) return fail(PL_EINVAL, "NULL pipeline");
  if (!pl->dna) return fail(PL_EINVAL, "live ingest is for DNA pipelines (items are DB words)");
  if (pl->live) return fail(PL_ESTATE, "a live run is already executing");
  if (pl->d_arr) return fail(PL_EINVAL, "live ingest takes arrivals at r * tau0 (no arrival array)");
  if (pl->cfg.flags & PL_CLUSTER_NODES) return fail(PL_EINVAL, "live ingest runs one CTA per stream (not PL_CLUSTER_NODES)");
  cudaSetDevice(pl->device);
  const uint32_t S = pl->cfg.n_streams;
  int sms = 0;
  CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, pl->device));
  const int per_sm = pl->dp.ctas_per_sm > 1 ? pl->dp.ctas_per_sm : 1;
  if ((int64_t)S > (int64_t)sms * per_sm)
    return fail(PL_EINVAL, "live ingest needs every stream resident at once (n_streams %u > %d)", S, sms * per_sm);
  const uint32_t CH = 1u << pl->dp.win_lg;
  uint32_t R = ring_words ? ring_words : std::max<uint32_t>(4 * pl->dp.win_cap, 1u << 16);
  if (!is_pow2(R) || R < 2 * pl->dp.win_cap || R < CH)
    return fail(PL_EINVAL, "ring_words must be a power of 2 >= 2 x the smem window (%u words)", pl->dp.win_cap);
  if (R != pl->ring_words) {
    if (pl->d_ring) cudaFree(pl->d_ring);
    if (pl->h_stage) cudaFreeHost(pl->h_stage);
    pl->d_ring = nullptr;
    pl->h_stage = nullptr;
    pl->ring_words = 0;
    if (cudaMalloc(&pl->d_ring, (size_t)S * R * 4) != cudaSuccess) return fail(PL_ENOMEM, "live rings (%u x %u words)", S, R);
    if (cudaHostAlloc((void**)&pl->h_stage, (size_t)S * R * 4, cudaHostAllocDefault) != cudaSuccess)
      return fail(PL_ENOMEM, "live ring mirror (pinned, %u x %u words)", S, R);
    pl->ring_words = R;
  }
  if (!pl->h_bell) {
    if (cudaHostAlloc((void**)&pl->h_bell, (size_t)kBells * S * 4, cudaHostAllocDefault) != cudaSuccess)
      return fail(PL_ENOMEM, "doorbell slots (pinned)");
    for (uint32_t j = 0; j < kBells; ++j) CUDA_TRY(cudaEventCreateWithFlags(&pl->bell_ev[j], cudaEventDisableTiming));
  }
  if (!pl->d_front && cudaMalloc(&pl->d_front, (size_t)S * 4) != cudaSuccess) return fail(PL_ENOMEM, "doorbells");
  if (!pl->h_consumed && cudaHostAlloc((void**)&pl->h_consumed, (size_t)S * 4, cudaHostAllocMapped) != cudaSuccess)
    return fail(PL_ENOMEM, "consumed watermarks (pinned)");
  if (!pl->copy_stream) CUDA_TRY(cudaStreamCreateWithFlags(&pl->copy_stream, cudaStreamNonBlocking));
  uint32_t* d_cons = nullptr;
  CUDA_TRY(cudaHostGetDevicePointer((void**)&d_cons, pl->h_consumed, 0));
  pl->lw_lo.resize(S);
  pl->lw_end.resize(S);
  pl->lw_hi.resize(S);
  pl->lw_front.resize(S);
  const uint32_t db_words = (uint32_t)((pl->db_len + 15) / 16);
  for (uint32_t s = 0; s < S; ++s) {
    stream_words_range(pl, s, &pl->lw_lo[s], &pl->lw_hi[s]);
    pl->lw_end[s] = std::max(pl->lw_lo[s], std::min(pl->lw_hi[s], db_words));
    pl->lw_front[s] = pl->lw_lo[s];
    pl->h_consumed[s] = pl->lw_lo[s];
  }
  // make sure no earlier copy on the copy stream is still in flight, then reset the doorbells
  CUDA_TRY(cudaStreamSynchronize(pl->copy_stream));
  CUDA_TRY(cudaMemcpy(pl->d_front, pl->lw_front.data(), (size_t)S * 4, cudaMemcpyHostToDevice));
  DevParams& d = pl->dp;
  pl->d_db_bound = nullptr;
  pl->bound_host = false;
  pl->pushed = pl->db_len;             // the run covers the whole stream; its words arrive by push
  d.live = 1;
  d.ring = pl->d_ring;
  d.ring_mask = R - 1;
  d.front = pl->d_front;
  d.consumed = d_cons;
  pl_status st = pl_pipeline_launch(pl);
  d.live = 0;                          // later non-live launches (the kernel took its own copy)
  if (st != PL_OK) return st;
  pl->live = true;
  pl->drained = false;
  return PL_OK;
}

pl_status pl_pipeline_stream_words(const pl_pipeline* pl, uint32_t stream, uint64_t* word_lo, uint64_t* word_hi) {
  if (!pl || !word_lo || !word_hi) return fail(PL_EINVAL, "NULL argument");
  if (!pl->dna) return fail(PL_EINVAL, "stream words exist for DNA pipelines only");
  if (stream >= pl->cfg.n_streams) return fail(PL_EINVAL, "stream %u >= n_streams %u", stream, pl->cfg.n_streams);
  uint32_t lo, hi;
  stream_words_range(pl, stream, &lo, &hi);
  const uint32_t db_words = (uint32_t)((pl->db_len + 15) / 16);
  *word_lo = lo;
  *word_hi = std::max(lo, std::min(hi, db_words));
  return PL_OK;
}

pl_status pl_pipeline_push_stream(pl_pipeline* pl, uint32_t stream, const uint32_t* words, uint64_t n,
                                  int nonblocking) {
  if (!pl) return fail(PL_EINVAL, "NULL pipeline");
  if (stream >= pl->cfg.n_streams) return fail(PL_EINVAL, "stream %u >= n_streams %u", stream, pl->cfg.n_streams);
  return push_streams(pl, stream, 1, &words, &n, nonblocking);
}

pl_status pl_pipeline_push_all(pl_pipeline* pl, const uint32_t* const* words, const uint64_t* n, int nonblocking) {
  if (!pl) return fail(PL_EINVAL, "NULL pipeline");
  return push_streams(pl, 0, pl->cfg.n_streams, words, n, nonblocking);
}

pl_status pl_pipeline_inject_stalls(pl_pipeline* pl, int64_t period_ns, int64_t len_ns) {
  if (!pl) return fail(PL_EINVAL, "NULL pipeline");
  if (len_ns < 0 || (len_ns > 0 && period_ns <= len_ns))
    return fail(PL_EINVAL, "stall injection needs 0 <= len_ns < period_ns");
  if (len_ns > 0 && pl->cfg.clock != PL_CLOCK_GLOBALTIMER) return fail(PL_EINVAL, "stall injection needs the physical clock");
  pl->dp.inj_period_ns = len_ns > 0 ? (uint64_t)period_ns : 1u;
  pl->dp.inj_len_ns = (uint64_t)len_ns;
  return PL_OK;
}

pl_status pl_pipeline_launch(pl_pipeline* pl) {
  if (!pl) return fail(PL_EINVAL, "NULL pipeline");
  if (pl->live) return fail(PL_ESTATE, "a live run is executing; pl_pipeline_drain ends it");
  cudaSetDevice(pl->device);
  DevParams& d = pl->dp;
  if (pl->dna) {
    d.db = pl->d_db_bound ? pl->d_db_bound : pl->d_db;
    d.db_len = pl->pushed;
    d.db_words = (uint32_t)((pl->pushed + 15) / 16);
    d.db_alloc_words = pl->d_db_bound ? d.db_words : pl->db_alloc_words;
    d.db_tma = pl->d_db_bound ? (((uintptr_t)pl->d_db_bound & 15u) == 0u) : 1u;
    d.total_roots = pl->pushed >= (uint64_t)pl->k ? pl->pushed - pl->k + 1 : 0;
  } else {
    d.total_roots = pl->pushed * pl->cfg.n_streams;
  }
  if (d.total_roots > pl->roots_cap) return fail(PL_EINVAL, "more roots than allocated");
  if (pl->d_arr && d.total_roots != pl->roots_cap)
    return fail(PL_EINVAL, "arrival times were given for %llu roots; push the whole stream",
                (unsigned long long)pl->roots_cap);
  d.summary = pl->d_summary + 8 * pl->slot;
  d.match_count = d.summary + 6;
  d.summary_next = pl->d_summary + 8 * (pl->slot ^ 1u);
  CUDA_TRY(pl_launch(d, pl->cfg.n_streams, pl->block, pl->smem, pl->stream));
  pl->d_match_count = d.summary + 6;       // readers see the slot of the last launch
  pl->slot ^= 1u;
  pl->launched = true;
  pl->launches++;
  return PL_OK;
}

pl_status pl_pipeline_drain(pl_pipeline* pl) {
  if (!pl) return fail(PL_EINVAL, "NULL pipeline");
  if (pl->live) {          // a live run ends once every stream's words were pushed
    for (uint32_t s = 0; s < pl->cfg.n_streams; ++s)
      if (pl->lw_front[s] < pl->lw_hi[s])
        return fail(PL_ESTATE, "live run: stream %u has %u of its %u words; push them all before drain", s,
                    pl->lw_front[s] - pl->lw_lo[s], pl->lw_hi[s] - pl->lw_lo[s]);
  } else if (!pl->launched) {     // nothing launched since create / rewind: run the pushed stream now
    pl_status s = pl_pipeline_launch(pl);
    if (s != PL_OK) return s;
  }
  CUDA_TRY(cudaStreamSynchronize(pl->stream));
  if (pl->live) pl->pushed = 0;   // the live words went to the rings, not to the handle's DB buffer
  pl->live = false;
  pl->drained = true;
  std::vector<CtaStats> cs(pl->cfg.n_streams);
  CUDA_TRY(cudaMemcpy(cs.data(), pl->d_stats, cs.size() * sizeof(CtaStats), cudaMemcpyDeviceToHost));
  pl->d2h += cs.size() * sizeof(CtaStats);
  uint32_t err = 0;
  for (auto& s : cs) err |= s.errors;
  if (err) return fail(PL_EOVERFLOW, "device reported overflow bits 0x%x (queue=1 match=2 log=4 seg=8 ingest-timeout=16 watchdog=32)", err);
  return PL_OK;
}

pl_status pl_pipeline_rewind(pl_pipeline* pl) {
  if (!pl) return fail(PL_EINVAL, "NULL pipeline");
  pl->drained = false;
  pl->launched = false;
  if (!pl->d_db_bound) pl->pushed = 0;
  return PL_OK;
}

pl_status pl_pipeline_stats(pl_pipeline* pl, pl_stats* out) {
  if (!pl || !out) return fail(PL_EINVAL, "NULL argument");
  cudaSetDevice(pl->device);
  CUDA_TRY(cudaStreamSynchronize(pl->stream));
  const uint32_t S = pl->cfg.n_streams, N = pl->cfg.n_stages;
  std::vector<CtaStats> cs(S);
  CUDA_TRY(cudaMemcpy(cs.data(), pl->d_stats, S * sizeof(CtaStats), cudaMemcpyDeviceToHost));
  pl->d2h += S * sizeof(CtaStats);
  std::memset(out, 0, sizeof *out);
  out->n_stages = N;
  out->n_streams = S;
  const int64_t tau = pl->cfg.interarrival;
  for (const CtaStats& s : cs) {
    out->roots += s.n_roots;
    const int64_t H = (int64_t)s.n_roots * tau;
    out->window += H;
    out->t_end += s.t_end;
    for (uint32_t i = 0; i < N; ++i) {
      out->firings[i] += s.firings[i];
      out->empty_firings[i] += s.empty[i];
      out->consumed[i] += s.consumed[i];
      out->produced[i] += s.produced[i];
      out->busy_ns[i] += s.busy_ns[i];
      out->spilled[i] += s.spilled[i];
      out->overruns[i] += s.overruns[i];
      out->stalls[i] += s.stalls[i];
      out->max_queue[i] = std::max(out->max_queue[i], s.max_queue[i]);
      out->max_lateness_ns[i] = std::max(out->max_lateness_ns[i], s.lateness[i]);
      out->sched_cycles[i] += s.sched_cycles[i];
      out->max_fire_ns[i] = std::max(out->max_fire_ns[i], s.max_fire_ns[i]);
      out->max_loop_ns[i] = std::max(out->max_loop_ns[i], s.max_loop_ns[i]);
      for (int k = 0; k < 6; ++k) out->phase_cycles[i][k] += s.phase_cycles[i][k];
      out->active_window[i] += s.active_win[i];   // computed per node by the executor
    }
    out->miss_events += s.miss_events;
    out->miss_events_ns += s.miss_events_ns;
    out->max_latency = std::max(out->max_latency, s.max_lat);
    out->max_latency_ns = std::max(out->max_latency_ns, s.max_lat_ns);
    out->wall_ns = std::max(out->wall_ns, s.wall_ns);
    out->errors |= s.errors;
    out->window_refills += s.win_refills;
    out->latency_outliers += s.agr_bad;
    out->latency_rel_err_max = std::max(out->latency_rel_err_max, (double)s.agr_ppm * 1e-6);
    out->ingest_waits += s.ingest_waits;
    out->max_ingest_wait_ns = std::max<int64_t>(out->max_ingest_wait_ns, s.ingest_max_ns);
  }
  unsigned long long mc = 0;
  CUDA_TRY(cudaMemcpy(&mc, pl->d_match_count, 8, cudaMemcpyDeviceToHost));
  pl->d2h += 8;
  out->matches = std::min<uint64_t>(mc, pl->dp.match_cap);
  double act = 0, act_ne = 0, busy = 0;
  for (uint32_t i = 0; i < N; ++i) {
    act += (double)out->active_window[i];
    busy += (double)out->busy_ns[i];
  }
  for (const CtaStats& s : cs)
    for (uint32_t i = 0; i < N; ++i) act_ne += (double)s.active_ne[i];
  const double denom = pl->cfg.policy == PL_MONOLITHIC ? (double)out->window : (double)N * (double)out->window;
  out->active_fraction = out->window ? act / denom : 0.0;
  out->active_fraction_nonempty = out->window ? act_ne / denom : 0.0;
  {   // drain-inclusive ratio over [0, T_end] per stream (SURVEY §8(c) C-D "Outputs"):
      // FIXED_WAIT charges every time-triggered slot m P_i < T_end clipped to T_end (L97; with
      // R-DRAIN only the slots m P_i < A_last) plus the drain firings; every other firing of
      // any policy ends by T_end and is charged t_i.
    double acc = 0, te_sum = 0;
    uint64_t r0 = 0;
    for (const CtaStats& s : cs) {
      const int64_t Te = s.t_end;
      te_sum += (double)Te;
      for (uint32_t i = 0; i < N; ++i) {
        const int64_t t = pl->t[i];
        if (pl->cfg.policy == PL_FIXED_WAIT) {
          const int64_t P = pl->t[i] + pl->w[i];
          int64_t K = Te > 0 ? (Te + P - 1) / P : 0;          // slots m P < T_end
          if (pl->cfg.flags & PL_EAGER_DRAIN) {
            const int64_t A_last = s.n_roots == 0 ? 0
                : (pl->h_arr.empty() ? (int64_t)(s.n_roots - 1) * tau : pl->h_arr[r0 + s.n_roots - 1]);
            K = std::min<int64_t>(K, (A_last + P - 1) / P);   // slots m P < A_last
            acc += (double)s.drain_firings[i] * (double)t;
          }
          if (K > 0) {
            const int64_t full = Te >= t ? std::min<int64_t>(K, (Te - t) / P + 1) : 0;   // m P + t <= T_end
            acc += (double)full * (double)t;
            for (int64_t m = full; m < K; ++m) acc += (double)std::min<int64_t>(t, Te - m * P);
          }
        } else {
          acc += (double)s.firings[i] * (double)t;
        }
      }
      r0 += s.n_roots;
    }
    const double dd = pl->cfg.policy == PL_MONOLITHIC ? te_sum : (double)N * te_sum;
    out->active_fraction_drain = dd > 0 ? acc / dd : 0.0;
  }
  if (out->wall_ns > 0) {
    const double procs = pl->cfg.policy == PL_MONOLITHIC ? 1.0 : (double)N;
    out->hw_busy_fraction = busy / (procs * (double)out->wall_ns * (double)S);
  }
  if ((pl->cfg.flags & PL_REC_LATENCY) && pl->d_lat) {
    std::vector<int64_t> lat(pl->dp.total_roots);
    if (!lat.empty()) {
      CUDA_TRY(cudaMemcpy(lat.data(), pl->d_lat, lat.size() * 8, cudaMemcpyDeviceToHost));
      std::vector<int64_t> latn;
      const bool phys = pl->cfg.clock == PL_CLOCK_GLOBALTIMER;
      if (phys) {
        latn.resize(lat.size());
        CUDA_TRY(cudaMemcpy(latn.data(), pl->d_lat_ns, latn.size() * 8, cudaMemcpyDeviceToHost));
      }
      const double Dns = (double)pl->cfg.deadline * pl->dp.ns_per_unit;
      for (size_t r = 0; r < lat.size(); ++r)
        out->misses += phys ? ((double)latn[r] > Dns) : (lat[r] > pl->cfg.deadline);
    }
  }
  out->launches = pl->launches;
  out->h2d_bytes = pl->h2d;
  out->d2h_bytes = pl->d2h;
  return PL_OK;
}

pl_status pl_pipeline_results(pl_pipeline* pl, pl_match* buf, uint64_t cap, uint64_t* n) {
  if (!pl || !n) return fail(PL_EINVAL, "NULL argument");
  cudaSetDevice(pl->device);
  CUDA_TRY(cudaStreamSynchronize(pl->stream));
  unsigned long long mc = 0;
  CUDA_TRY(cudaMemcpy(&mc, pl->d_match_count, 8, cudaMemcpyDeviceToHost));
  uint64_t cnt = std::min<uint64_t>(mc, pl->dp.match_cap);
  if (!buf) { *n = cnt; return PL_OK; }
  cnt = std::min(cnt, cap);
  if (cnt) CUDA_TRY(cudaMemcpy(buf, pl->dp.matches, cnt * sizeof(pl_match), cudaMemcpyDefault));
  pl->d2h += 8 + cnt * sizeof(pl_match);
  *n = cnt;
  return PL_OK;
}

pl_status pl_pipeline_latency(pl_pipeline* pl, int64_t* lat_units, int64_t* lat_ns, uint64_t cap, uint64_t* n) {
  if (!pl || !n) return fail(PL_EINVAL, "NULL argument");
  if (!(pl->cfg.flags & PL_REC_LATENCY)) return fail(PL_ESTATE, "PL_REC_LATENCY not enabled");
  cudaSetDevice(pl->device);
  CUDA_TRY(cudaStreamSynchronize(pl->stream));
  uint64_t R = pl->dp.total_roots;
  if (!lat_units) { *n = R; return PL_OK; }
  R = std::min(R, cap);
  if (R) CUDA_TRY(cudaMemcpy(lat_units, pl->d_lat, R * 8, cudaMemcpyDeviceToHost));
  if (lat_ns && R) {
    if (pl->cfg.clock == PL_CLOCK_GLOBALTIMER) CUDA_TRY(cudaMemcpy(lat_ns, pl->d_lat_ns, R * 8, cudaMemcpyDeviceToHost));
    else for (uint64_t r = 0; r < R; ++r) lat_ns[r] = -1;
  }
  *n = R;
  return PL_OK;
}

pl_status pl_pipeline_trace(pl_pipeline* pl, uint32_t* cnt, uint64_t cap, uint64_t* n) {
  if (!pl || !n) return fail(PL_EINVAL, "NULL argument");
  if (!(pl->cfg.flags & PL_REC_TRACE)) return fail(PL_ESTATE, "PL_REC_TRACE not enabled");
  cudaSetDevice(pl->device);
  CUDA_TRY(cudaStreamSynchronize(pl->stream));
  uint64_t E = pl->dp.total_roots * (pl->cfg.n_stages + 1);
  if (!cnt) { *n = E; return PL_OK; }
  E = std::min(E, cap);
  if (E) CUDA_TRY(cudaMemcpy(cnt, pl->d_trace, E * 4, cudaMemcpyDeviceToHost));
  *n = E;
  return PL_OK;
}

pl_status pl_pipeline_firings(pl_pipeline* pl, pl_firing* buf, uint64_t cap, uint64_t* n) {
  if (!pl || !n) return fail(PL_EINVAL, "NULL argument");
  if (!(pl->cfg.flags & PL_REC_FIRINGS)) return fail(PL_ESTATE, "PL_REC_FIRINGS not enabled");
  cudaSetDevice(pl->device);
  CUDA_TRY(cudaStreamSynchronize(pl->stream));
  const uint32_t S = pl->cfg.n_streams;
  std::vector<CtaStats> cs(S);
  CUDA_TRY(cudaMemcpy(cs.data(), pl->d_stats, S * sizeof(CtaStats), cudaMemcpyDeviceToHost));
  uint64_t total = 0;
  for (auto& s : cs) total += s.n_log;
  if (!buf) { *n = total; return PL_OK; }
  uint64_t w = 0;
  for (uint32_t s = 0; s < S && w < cap; ++s) {
    const uint64_t c = std::min<uint64_t>(cs[s].n_log, cap - w);
    if (c) CUDA_TRY(cudaMemcpy(buf + w, pl->d_flog + (uint64_t)s * pl->dp.log_cap, c * sizeof(pl_firing),
                               cudaMemcpyDeviceToHost));
    w += c;
  }
  *n = w;
  return PL_OK;
}

pl_status pl_stage_batch(pl_pipeline* pl, uint32_t stage, const void* in_dev, uint64_t n, uint64_t first_root,
                         void* out_dev, uint64_t cap, uint64_t* n_out, uint64_t* max_vec_cycles) {
  if (!pl || !n_out) return fail(PL_EINVAL, "NULL argument");
  if (stage >= pl->cfg.n_stages) return fail(PL_EINVAL, "stage %u out of range", stage);
  if (stage > 0 && n && !in_dev) return fail(PL_EINVAL, "stage > 0 needs input entries");
  if (pl->dna && pl->pushed < (uint64_t)pl->k) return fail(PL_ESTATE, "push or bind the DB first");
  if (v_too_big(pl)) return fail(PL_EINVAL, "vector_width > 256");
  cudaSetDevice(pl->device);
  DevParams d = pl->dp;
  if (pl->dna) {
    d.db = pl->d_db_bound ? pl->d_db_bound : pl->d_db;
    d.db_len = pl->pushed;
    d.db_words = (uint32_t)((pl->pushed + 15) / 16);
    d.total_roots = pl->pushed - pl->k + 1;
  } else {
    d.total_roots = first_root + n;
  }
  if (stage == 0 && pl->dna && first_root + n > d.total_roots)
    return fail(PL_EINVAL, "roots %llu..%llu beyond the DB's %llu roots", (unsigned long long)first_root,
                (unsigned long long)(first_root + n), (unsigned long long)d.total_roots);
  d.win_cap = 0;
  d.match_count = pl->d_match_count;
  d.summary = nullptr;
  d.summary_next = nullptr;
  if (!pl->d_scratch && cudaMalloc(&pl->d_scratch, 16) != cudaSuccess) return fail(PL_ENOMEM, "scratch");
  CUDA_TRY(cudaMemsetAsync(pl->d_scratch, 0, 16, pl->stream));
  if (stage == pl->cfg.n_stages - 1) CUDA_TRY(cudaMemsetAsync(pl->d_match_count, 0, 8, pl->stream));
  const uint32_t smem = pl_layout_enforced_host(d);
  CUDA_TRY(pl_launch_stage_batch(d, (int)stage, in_dev, n, first_root, out_dev, cap, pl->d_scratch, smem, pl->stream));
  unsigned long long h[2];
  CUDA_TRY(cudaMemcpyAsync(h, pl->d_scratch, 16, cudaMemcpyDeviceToHost, pl->stream));
  CUDA_TRY(cudaStreamSynchronize(pl->stream));
  if (stage == pl->cfg.n_stages - 1 && pl->dna) {   // the sink's records are the pipeline's matches
    const unsigned long long mc = std::min<unsigned long long>(h[0], pl->dp.match_cap);
    CUDA_TRY(cudaMemcpy(pl->d_match_count, &mc, 8, cudaMemcpyHostToDevice));
  }
  *n_out = h[0];
  if (max_vec_cycles) *max_vec_cycles = h[1];
  if (h[0] > cap && stage + 1 < pl->cfg.n_stages) return fail(PL_EOVERFLOW, "output capacity %llu < %llu",
                                                              (unsigned long long)cap, h[0]);
  return PL_OK;
}

pl_status pl_pipeline_params(const pl_pipeline* pl, int64_t* w_out, uint32_t* theta_out, uint32_t* M_out) {
  if (!pl) return fail(PL_EINVAL, "NULL pipeline");
  for (uint32_t i = 0; i < pl->cfg.n_stages; ++i) {
    if (w_out) w_out[i] = pl->w[i];
    if (theta_out) theta_out[i] = pl->dp.theta[i];
  }
  if (M_out) *M_out = pl->M;
  return PL_OK;
}

void pl_pipeline_destroy(pl_pipeline* pl) {
  if (!pl) return;
  cudaSetDevice(pl->device);
  cudaStreamSynchronize(pl->stream);
  free_all(pl);
  delete pl;
}

}  // extern "C"
