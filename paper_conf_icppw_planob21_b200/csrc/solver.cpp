// solver.cpp — host solvers for the paper's two optimisation problems.
//
// Fig. 1: minimise T(P) = (1/N) sum t_i/P_i, P_i = t_i + w_i,
//   s.t. P_0 <= v tau0 (L125/L145, reading A3), g_{i-1} P_i <= P_{i-1} (L131/L147),
//   sum b_i P_i <= D (L135/L149), P_i >= t_i.
// Exact continuous solve: with Q_i = G_i P_i (G_0 = 1, G_i = prod_{j<i} g_j) the
// chain constraints become Q_0 >= Q_1 >= ... >= Q_{N-1}, the objective
// sum c_i/Q_i (c_i = t_i G_i) and the deadline sum a_i Q_i <= D (a_i = b_i/G_i).
// For a deadline multiplier lambda the Lagrangian is separable convex under an
// isotonic order: pool-adjacent-violators gives the unbounded isotonic minimiser
// (block value sqrt(sum c / (lambda sum a))), which is then clipped to the
// order-compatible bounds [max_{j>=i} G_j t_j, v tau0].  lambda is found by
// bisection on the (monotone) deadline slack.  The integer answer (reading A17)
// is the best feasible point of two neighbourhood searches around the continuous
// optimum -- a chain-aware depth-first search, and a slack-absorption pass that gives
// one stage the largest value the others leave it -- ties broken towards the
// lexicographically smallest w.  Not a proof of integer optimality: it is checked
// against the oracle's exact search (tests/test_abi.py) where that search is exact.
// Fig. 2: exhaustive search over M while b M tau0 + S Tbar(M) <= D.
#include <cmath>
#include <cstdint>
#include <cstring>
#include <vector>

#include "pl_internal.h"

namespace plsolve {

static void gains(const double* g, int N, double* G) {
  G[0] = 1.0;
  for (int i = 1; i < N; ++i) G[i] = G[i - 1] * g[i - 1];   // left to right (R-FP)
}

static bool feasible(int N, const int64_t* t, const double* g, const uint32_t* b, uint32_t v, int64_t tau,
                     int64_t D, const int64_t* P) {
  for (int i = 0; i < N; ++i)
    if (P[i] < t[i]) return false;
  if ((double)P[0] > (double)v * (double)tau) return false;
  for (int i = 1; i < N; ++i)
    if ((double)P[i] * g[i - 1] > (double)P[i - 1]) return false;
  int64_t s = 0;
  for (int i = 0; i < N; ++i) s += (int64_t)b[i] * P[i];
  return s <= D;
}

static double objective(int N, const int64_t* t, const double* P) {
  double s = 0;
  for (int i = 0; i < N; ++i) s += (double)t[i] / P[i];
  return s / N;
}

// isotonic (non-increasing) minimiser of sum c_i/Q + lam a_i Q, clipped to [L_i, U]
static void iso_solve(int N, const double* c, const double* a, double lam, const double* L, double U,
                      double* Q) {
  double bc[PL_MAX_STAGES], ba[PL_MAX_STAGES], bv[PL_MAX_STAGES];
  int bs[PL_MAX_STAGES], bn = 0;
  for (int i = 0; i < N; ++i) {
    bc[bn] = c[i];
    ba[bn] = a[i];
    bs[bn] = 1;
    bv[bn] = lam > 0 ? std::sqrt(c[i] / (lam * a[i])) : INFINITY;
    ++bn;
    // non-increasing order: merge while a later block exceeds the earlier one
    while (bn > 1 && bv[bn - 1] > bv[bn - 2]) {
      bc[bn - 2] += bc[bn - 1];
      ba[bn - 2] += ba[bn - 1];
      bs[bn - 2] += bs[bn - 1];
      bv[bn - 2] = lam > 0 ? std::sqrt(bc[bn - 2] / (lam * ba[bn - 2])) : INFINITY;
      --bn;
    }
  }
  int k = 0;
  for (int j = 0; j < bn; ++j)
    for (int r = 0; r < bs[j]; ++r, ++k) {
      double q = bv[j];
      if (q > U) q = U;
      if (q < L[k]) q = L[k];
      Q[k] = q;
    }
}

int solve_fig1(int N, const int64_t* t, const double* g, const uint32_t* b, uint32_t v, int64_t tau, int64_t D,
               double* Pc, double* Tc, int64_t* Pi, double* Ti) {
  double G[PL_MAX_STAGES], c[PL_MAX_STAGES], a[PL_MAX_STAGES], L[PL_MAX_STAGES], Q[PL_MAX_STAGES];
  gains(g, N, G);
  for (int i = 0; i < N; ++i) {
    if (!(G[i] > 0)) return PL_EINVAL;
    c[i] = (double)t[i] * G[i];
    a[i] = (double)b[i] / G[i];
  }
  // order-compatible lower bounds: Q_i >= Q_j >= G_j t_j for j >= i
  for (int i = N - 1; i >= 0; --i) {
    L[i] = G[i] * (double)t[i];
    if (i + 1 < N && L[i + 1] > L[i]) L[i] = L[i + 1];
  }
  const double U = (double)v * (double)tau;
  if (L[0] > U * (1 + 1e-15)) return PL_EINFEASIBLE;
  auto slack = [&](double lam) {
    iso_solve(N, c, a, lam, L, U, Q);
    double s = 0;
    for (int i = 0; i < N; ++i) s += a[i] * Q[i];
    return s - (double)D;
  };
  double lo_s;
  {  // lam -> infinity: Q = L
    double s = 0;
    for (int i = 0; i < N; ++i) s += a[i] * L[i];
    lo_s = s - (double)D;
  }
  if (lo_s > 1e-9 * (double)D) return PL_EINFEASIBLE;
  if (slack(0.0) > 0) {
    double lam_lo = 1e-30, lam_hi = 1.0;
    while (slack(lam_hi) > 0) lam_hi *= 16.0;
    for (int it = 0; it < 400; ++it) {
      double mid = std::sqrt(lam_lo * lam_hi);
      if (slack(mid) > 0) lam_lo = mid; else lam_hi = mid;
      if (lam_hi / lam_lo < 1 + 1e-15) break;
    }
    slack(lam_hi);
  }
  for (int i = 0; i < N; ++i) Pc[i] = Q[i] / G[i];
  *Tc = objective(N, t, Pc);
  // integer search (reading A17): branch and bound, depth-first over stages.  Stage i tries
  // floor(P_i) - R .. floor(P_i) + R + 1 around the continuous optimum and the R+1 largest
  // integers allowed by the chain bound g_{i-1} P_i <= P_{i-1} of the chosen predecessor;
  // branches that cannot meet the deadline or beat the incumbent objective are cut.
  const int RW = 8;
  int64_t bestP[PL_MAX_STAGES], P[PL_MAX_STAGES];
  bool found = false;
  double best = 0;
  int64_t bsum_suffix_min[PL_MAX_STAGES + 1];
  double obj_suffix_lb[PL_MAX_STAGES + 1];
  bsum_suffix_min[N] = 0;
  obj_suffix_lb[N] = 0;
  for (int i = N - 1; i >= 0; --i) bsum_suffix_min[i] = bsum_suffix_min[i + 1] + (int64_t)b[i] * t[i];
  for (int i = N - 1; i >= 0; --i) {
    // P_i <= (D - sum_{j != i} b_j t_j) / b_i bounds t_i / P_i from below
    const double ub = (double)(D - (bsum_suffix_min[0] - (int64_t)b[i] * t[i])) / (double)b[i];
    obj_suffix_lb[i] = obj_suffix_lb[i + 1] + (ub > 0 ? (double)t[i] / ub : 0.0);
  }
  const int MAXC = 4 * RW + 4;
  struct Frame { int64_t cand[4 * 8 + 4]; int nc, k; int64_t bsum; double obj; };
  Frame fr[PL_MAX_STAGES];
  auto fill = [&](int i, int64_t prevP, int64_t bsum, double obj) {
    Frame& f = fr[i];
    f.nc = 0; f.k = 0; f.bsum = bsum; f.obj = obj;
    int64_t ub;
    if (i == 0) {
      ub = (int64_t)std::floor((double)v * (double)tau);
    } else {
      ub = (int64_t)std::floor((double)prevP / g[i - 1]);
      while (ub > 0 && (double)ub * g[i - 1] > (double)prevP) --ub;
      while ((double)(ub + 1) * g[i - 1] <= (double)prevP) ++ub;
    }
    const int64_t fl = (int64_t)std::floor(Pc[i]);
    int64_t c[4 * 8 + 4];
    int nc = 0;
    for (int d = 0; d <= RW; ++d) c[nc++] = ub - d;
    for (int d = -RW; d <= RW + 1; ++d) c[nc++] = fl + d;
    for (int j = 0; j < nc && f.nc < MAXC; ++j) {
      const int64_t x = c[j];
      if (x < t[i] || x > ub) continue;
      if (bsum + (int64_t)b[i] * x + bsum_suffix_min[i + 1] > D) continue;
      bool dup = false;
      for (int q = 0; q < f.nc; ++q) dup |= f.cand[q] == x;
      if (!dup) f.cand[f.nc++] = x;
    }
  };
  int depth = 0;
  fill(0, 0, 0, 0.0);
  while (depth >= 0) {
    Frame& f = fr[depth];
    if (f.k >= f.nc) { --depth; continue; }
    P[depth] = f.cand[f.k++];
    const int64_t bs = f.bsum + (int64_t)b[depth] * P[depth];
    const double ob = f.obj + (double)t[depth] / (double)P[depth];
    if (found && (ob + obj_suffix_lb[depth + 1]) / N > best * (1 + 1e-12)) continue;
    if (depth + 1 < N) {
      fill(depth + 1, P[depth], bs, ob);
      ++depth;
      continue;
    }
    if (!feasible(N, t, g, b, v, tau, D, P)) continue;
    double Pd[PL_MAX_STAGES];
    for (int i = 0; i < N; ++i) Pd[i] = (double)P[i];
    const double T = objective(N, t, Pd);
    bool better = !found || T < best;
    if (found && T == best) {   // tie -> lexicographically smallest w (= smallest P)
      better = false;
      for (int i = 0; i < N; ++i)
        if (P[i] != bestP[i]) { better = P[i] < bestP[i]; break; }
    }
    if (better) {
      found = true;
      best = T;
      std::memcpy(bestP, P, sizeof(int64_t) * N);
    }
  }
  // Slack absorption.  Rounding the other stages down can free more deadline units than the
  // window above reaches, so for every stage a (the one that absorbs the slack): enumerate the
  // other stages over floor(P_j) - RA .. floor(P_j) + RA + 1 and give P_a the LARGEST value the
  // constraints allow (t_a / P_a falls as P_a grows, so for fixed others that is optimal):
  // P_a <= v tau0 (a = 0), P_a <= P_{a-1} / g_{a-1}, g_a P_{a+1} <= P_a, b_a P_a <= D - rest.
  {
    const int RA = N <= 4 ? 8 : (N <= 5 ? 4 : (N <= 6 ? 2 : 1));
    const int span = 2 * RA + 2;
    int64_t Q2[PL_MAX_STAGES];
    for (int a = 0; a < N; ++a) {
      int64_t combos = 1;
      for (int j = 0; j < N - 1; ++j) combos *= span;
      for (int64_t code = 0; code < combos; ++code) {
        int64_t cc = code;
        int64_t rest = 0;
        bool ok = true;
        for (int j = 0; j < N && ok; ++j) {
          if (j == a) continue;
          Q2[j] = (int64_t)std::floor(Pc[j]) - RA + (cc % span);
          cc /= span;
          if (Q2[j] < t[j]) ok = false;
          rest += (int64_t)b[j] * Q2[j];
        }
        if (!ok) continue;
        int64_t ub = (D - rest) / (int64_t)b[a];
        if (D - rest < 0) continue;
        if (a == 0) ub = std::min<int64_t>(ub, (int64_t)std::floor((double)v * (double)tau));
        if (a > 0) {
          int64_t c2 = (int64_t)std::floor((double)Q2[a - 1] / g[a - 1]);
          while (c2 > 0 && (double)c2 * g[a - 1] > (double)Q2[a - 1]) --c2;
          while ((double)(c2 + 1) * g[a - 1] <= (double)Q2[a - 1]) ++c2;
          ub = std::min(ub, c2);
        }
        if (ub < t[a]) continue;
        Q2[a] = ub;
        if (!feasible(N, t, g, b, v, tau, D, Q2)) continue;
        double Pd[PL_MAX_STAGES];
        for (int i = 0; i < N; ++i) Pd[i] = (double)Q2[i];
        const double T = objective(N, t, Pd);
        bool better = !found || T < best;
        if (found && T == best) {
          better = false;
          for (int i = 0; i < N; ++i)
            if (Q2[i] != bestP[i]) { better = Q2[i] < bestP[i]; break; }
        }
        if (better) {
          found = true;
          best = T;
          std::memcpy(bestP, Q2, sizeof(int64_t) * N);
        }
      }
    }
  }
  if (!found) return PL_EINFEASIBLE;
  std::memcpy(Pi, bestP, sizeof(int64_t) * N);
  *Ti = best;
  return PL_OK;
}

void thresholds(int N, const double* g, const int64_t* P, int64_t tau, uint32_t v, uint32_t* theta) {
  double G[PL_MAX_STAGES];
  gains(g, N, G);
  for (int i = 0; i < N; ++i) {
    double x = std::floor(G[i] * (double)P[i] / (double)tau);
    if (x < 1) x = 1;
    if (x > v) x = v;
    theta[i] = (uint32_t)x;
  }
}

double tbar(int N, const int64_t* t, const double* g, uint32_t v, int64_t M) {
  double G[PL_MAX_STAGES];
  gains(g, N, G);
  double s = 0;
  for (int i = 0; i < N; ++i) s += std::ceil((double)M * G[i] / (double)v) * (double)t[i];
  return s;
}

int solve_fig2(int N, const int64_t* t, const double* g, uint32_t v, int64_t tau, int64_t D, double bb, double S,
               uint32_t* M_out, double* T_out) {
  bool found = false;
  double best = 0;
  int64_t bestM = 0;
  for (int64_t M = 1; M < (int64_t)1 << 31; ++M) {
    const double tb = tbar(N, t, g, v, M);
    if (bb * (double)M * (double)tau + S * tb > (double)D) break;
    if (tb <= (double)M * (double)tau) {
      const double obj = tb / ((double)M * (double)tau);
      if (!found || obj < best) { found = true; best = obj; bestM = M; }
    }
  }
  if (!found) return PL_EINFEASIBLE;
  *M_out = (uint32_t)bestM;
  *T_out = best;
  return PL_OK;
}

}  // namespace plsolve
