// selector.cpp -- workload classification, the Tab I policy, the selection
// algorithm and the SM split (§III-B; readings Q8-Q10, Q13 in
// DESIGN.md).  Pure host functions, exported through the C ABI so they can be
// checked against the oracle without a GPU.
#include <algorithm>
#include <cmath>
#include <functional>
#include <cstdint>
#include <limits>
#include <vector>

#include "../../include/slate.h"

namespace {

// Tab I exactly as printed; row = active kernel, column = candidate;
// order L_C, M_C, H_C, M_M, H_M; 1 = corun, 0 = solo.
const int kLiteral[5][5] = {
    {1, 1, 0, 1, 1},
    {1, 1, 0, 0, 1},
    {0, 0, 0, 0, 1},
    {1, 0, 1, 0, 0},
    {1, 1, 0, 0, 0},
};

int level(double frac, double lo, double hi) { return frac < lo ? 0 : (frac < hi ? 1 : 2); }

// solo time on s SMs, linear in throughput between samples, 0 throughput at 0 SMs
double interp(const uint32_t* sms, const double* ms, uint32_t n, double s) {
  if (n == 0) return std::numeric_limits<double>::infinity();
  if (s >= sms[n - 1]) return ms[n - 1];
  double s0 = 0, r0 = 0;
  for (uint32_t i = 0; i < n; ++i) {
    const double s1 = sms[i], r1 = 1.0 / ms[i];
    if (s <= s1) {
      const double r = r0 + (r1 - r0) * (s - s0) / (s1 - s0);
      return r <= 0 ? std::numeric_limits<double>::infinity() : 1.0 / r;
    }
    s0 = s1;
    r0 = r1;
  }
  return ms[n - 1];
}

}  // namespace

extern "C" {

uint32_t slate_classify(double hbm_frac, double fp32_frac, double tc_frac, uint32_t* c_level, uint32_t* m_level) {
  // Q9: memory L < 25% <= M < 85% <= H; compute (max of FP32, tensor) L < 1% <= M < 10% <= H
  const int m = level(hbm_frac, 0.25, 0.85);
  const int c = level(fp32_frac > tc_frac ? fp32_frac : tc_frac, 0.01, 0.10);
  if (c_level) *c_level = uint32_t(c);
  if (m_level) *m_level = uint32_t(m);
  // memory intensity has priority: H_M, M_M, else L_C/M_C/H_C by compute
  if (m == 2) return 4;
  if (m == 1) return 3;
  return uint32_t(c);
}

int slate_policy(uint32_t a, uint32_t b, int literal) {
  if (a > 4 || b > 4) return 0;
  if (literal) return kLiteral[a][b];
  // Q8: symmetric table, the upper triangle (holding the H_C row) authoritative
  return a <= b ? kLiteral[a][b] : kLiteral[b][a];
}

int slate_select(uint32_t active, const uint32_t* cats, const uint32_t* bypassed, uint32_t n, uint32_t max_bypass,
                 int literal) {
  // test J_{k+1} first, then the rest of the queue; -1 = run J_k solo
  for (uint32_t i = 0; i < n; ++i) {
    if (slate_policy(active, cats[i], literal)) return int(i);
    if (bypassed && bypassed[i] >= max_bypass) return -1;   // Q13: no look-ahead past a starving kernel
  }
  return -1;
}

uint32_t slate_saturation_sms(const uint32_t* sms, const double* ms, uint32_t n, uint32_t n_sms, double frac) {
  const double t_full = interp(sms, ms, n, double(n_sms));
  for (uint32_t s = 1; s <= n_sms; ++s)
    if (interp(sms, ms, n, double(s)) <= t_full / frac) return s;
  return n_sms;
}

// fluid model: completion times of A on n-s SMs and B on s SMs, the
// first to finish handing its SMs to the other (oracle selector.corun_times)
static void corun_times(const uint32_t* sms_a, const double* ms_a, uint32_t n_a, const uint32_t* sms_b,
                        const double* ms_b, uint32_t n_b, uint32_t n_sms, uint32_t s, double* t_a, double* t_b) {
  const double ta = interp(sms_a, ms_a, n_a, double(n_sms - s));
  const double tb = interp(sms_b, ms_b, n_b, double(s));
  if (tb <= ta) {
    *t_a = tb + (1.0 - tb / ta) * interp(sms_a, ms_a, n_a, n_sms);
    *t_b = tb;
  } else {
    *t_a = ta;
    *t_b = ta + (1.0 - ta / tb) * interp(sms_b, ms_b, n_b, n_sms);
  }
}

uint32_t slate_choose_split_obj(const uint32_t* sms_a, const double* ms_a, uint32_t n_a, const uint32_t* sms_b,
                                const double* ms_b, uint32_t n_b, uint32_t n_sms, uint32_t step, uint32_t lo_b,
                                uint32_t hi_b, uint32_t objective, double slack, double* makespan_ms, double* antt) {
  if (step == 0) step = 1;
  const double ta_full = interp(sms_a, ms_a, n_a, n_sms), tb_full = interp(sms_b, ms_b, n_b, n_sms);
  std::vector<uint32_t> cands;
  for (uint32_t s = step; s + step <= n_sms; s += step)
    if ((!lo_b || s >= lo_b) && (!hi_b || s <= hi_b)) cands.push_back(s);
  if (cands.empty())   // the bounds exclude every candidate: the bound nearest the range
    cands.push_back(std::min(std::max(step, lo_b ? lo_b : step), n_sms - step));
  std::vector<double> mk(cands.size()), an(cands.size());
  double best_t = std::numeric_limits<double>::infinity();
  size_t best = 0;
  for (size_t i = 0; i < cands.size(); ++i) {
    double a, b;
    corun_times(sms_a, ms_a, n_a, sms_b, ms_b, n_b, n_sms, cands[i], &a, &b);
    mk[i] = std::max(a, b);
    an[i] = 0.5 * (a / ta_full + b / tb_full);
    if (mk[i] < best_t - 1e-12) {
      best_t = mk[i];
      best = i;
    }
  }
  if (objective == SLATE_SPLIT_ANTT) {   // reading Q41: least ANTT within `slack` of the best makespan
    const double bound = best_t * (1.0 + slack);
    double best_a = std::numeric_limits<double>::infinity();
    for (size_t i = 0; i < cands.size(); ++i)
      if (mk[i] <= bound + 1e-12 && an[i] < best_a - 1e-12) {
        best_a = an[i];
        best = i;
      }
  }
  if (makespan_ms) *makespan_ms = mk[best];
  if (antt) *antt = an[best];
  return cands[best];
}

uint32_t slate_choose_split(const uint32_t* sms_a, const double* ms_a, uint32_t n_a, const uint32_t* sms_b,
                            const double* ms_b, uint32_t n_b, uint32_t n_sms, uint32_t step, uint32_t lo_b,
                            uint32_t hi_b, double* makespan_ms) {
  return slate_choose_split_obj(sms_a, ms_a, n_a, sms_b, ms_b, n_b, n_sms, step, lo_b, hi_b, SLATE_SPLIT_MAKESPAN,
                                0.0, makespan_ms, nullptr);
}

int slate_fluid_corun_obj(const uint32_t* sms_a, const double* ms_a, uint32_t n_a, double work_a,
                          const uint32_t* sms_b, const double* ms_b, uint32_t n_b, double work_b, uint32_t n_sms,
                          uint32_t step, uint32_t lo_b, uint32_t hi_b, double min_gain, uint32_t objective,
                          double slack, uint32_t* split, double* gain) {
  // job curves: `work` launches of the kernel, back to back on the same SMs
  std::vector<double> ja(ms_a, ms_a + n_a), jb(ms_b, ms_b + n_b);
  for (double& v : ja) v *= work_a;
  for (double& v : jb) v *= work_b;
  double t_co = 0;
  const uint32_t s = slate_choose_split_obj(sms_a, ja.data(), n_a, sms_b, jb.data(), n_b, n_sms, step, lo_b, hi_b,
                                            objective, slack, &t_co, nullptr);
  const double t_seq = interp(sms_a, ja.data(), n_a, n_sms) + interp(sms_b, jb.data(), n_b, n_sms);
  const double g = t_co > 0 ? t_seq / t_co : 0.0;
  if (split) *split = s;
  if (gain) *gain = g;
  return g >= min_gain ? 1 : 0;
}

int slate_fluid_corun(const uint32_t* sms_a, const double* ms_a, uint32_t n_a, double work_a, const uint32_t* sms_b,
                      const double* ms_b, uint32_t n_b, double work_b, uint32_t n_sms, uint32_t step, uint32_t lo_b,
                      uint32_t hi_b, double min_gain, uint32_t* split, double* gain) {
  return slate_fluid_corun_obj(sms_a, ms_a, n_a, work_a, sms_b, ms_b, n_b, work_b, n_sms, step, lo_b, hi_b, min_gain,
                               SLATE_SPLIT_MAKESPAN, 0.0, split, gain);
}

uint32_t slate_choose_iters(double solo_ms, uint32_t occ, uint32_t n_sms, uint32_t B, uint32_t cap, double budget_us) {
  if (B == 0 || occ == 0 || n_sms == 0) return 1;
  const double workers = double(occ) * n_sms;
  const double t_block_us = std::max(solo_ms * 1e3 * workers / B, 1e-3);
  const double it = std::min(std::floor(budget_us / t_block_us), std::floor(B / (2.0 * workers)));
  return uint32_t(std::max(1.0, std::min(double(cap ? cap : 1), it)));
}

// NEXT-4: k co-runners (oracle selector.corun_makespan_k / choose_split_k).
// curve i: npts[i] points sms[i][*] -> ms[i][*].
static double makespan_k(const uint32_t* const* sms, const double* const* ms, const uint32_t* npts, uint32_t k,
                         const uint32_t* shares) {
  std::vector<double> left(k, 1.0), s(k);
  std::vector<bool> alive(k, true);
  for (uint32_t i = 0; i < k; ++i) s[i] = shares[i];
  double t = 0;
  for (;;) {
    double dt = std::numeric_limits<double>::infinity();
    bool any = false;
    std::vector<double> rate(k, 0.0);
    for (uint32_t i = 0; i < k; ++i)
      if (alive[i]) {
        any = true;
        rate[i] = 1.0 / interp(sms[i], ms[i], npts[i], s[i]);
        dt = std::min(dt, left[i] / rate[i]);
      }
    if (!any) return t;
    t += dt;
    double freed = 0;
    std::vector<uint32_t> done;
    for (uint32_t i = 0; i < k; ++i)
      if (alive[i]) {
        if (left[i] - rate[i] * dt <= 1e-12) done.push_back(i);
        left[i] = std::max(0.0, left[i] - rate[i] * dt);
      }
    for (uint32_t i : done) {
      alive[i] = false;
      freed += s[i];
      s[i] = 0;
    }
    if (freed > 0) {
      int best = -1;
      double most = -1;
      for (uint32_t i = 0; i < k; ++i)
        if (alive[i]) {
          const double rem = left[i] * interp(sms[i], ms[i], npts[i], s[i]);
          if (rem > most) { most = rem; best = int(i); }
        }
      if (best >= 0) s[best] += freed;
    }
  }
}

double slate_corun_makespan_k(const uint32_t* const* sms, const double* const* ms, const uint32_t* npts, uint32_t k,
                              const uint32_t* shares) {
  return makespan_k(sms, ms, npts, k, shares);
}

double slate_choose_split_k(const uint32_t* const* sms, const double* const* ms, const uint32_t* npts, uint32_t k,
                            uint32_t n_sms, uint32_t step, uint32_t* shares_out) {
  if (k == 0 || step == 0 || n_sms / step < k) return -1.0;
  const uint32_t units = n_sms / step;
  std::vector<uint32_t> u(k, 1), best;
  double best_t = std::numeric_limits<double>::infinity();
  // enumerate compositions of `units` into k positive parts, lexicographic order
  std::vector<uint32_t> sh(k);
  std::function<void(uint32_t, uint32_t)> rec = [&](uint32_t pos, uint32_t rest) {
    if (pos == k - 1) {
      u[pos] = rest;
      for (uint32_t i = 0; i < k; ++i) sh[i] = u[i] * step;
      const double t = makespan_k(sms, ms, npts, k, sh.data());
      if (t < best_t - 1e-12) { best_t = t; best = sh; }
      return;
    }
    for (uint32_t v = 1; v + (k - 1 - pos) <= rest; ++v) {
      u[pos] = v;
      rec(pos + 1, rest - v);
    }
  };
  rec(0, units);
  for (uint32_t i = 0; i < k; ++i) shares_out[i] = best[i];
  return best_t;
}

// NEXT-4 (reading Q49): should the candidate (curve k) join a co-running group
// of k jobs on shares_cur?  At most one memory-intensive job per group (Q37);
// gain = (makespan_k(group) + T_candidate(n)) / makespan_{k+1}(best shares).
// oracle selector.kway_admit
int slate_kway_admit(const uint32_t* const* sms, const double* const* ms, const uint32_t* npts, const uint32_t* cats,
                     uint32_t k, const uint32_t* shares_cur, uint32_t n_sms, uint32_t step, double min_gain,
                     uint32_t* shares_out, double* gain) {
  if (gain) *gain = 0.0;
  uint32_t mem = 0;
  for (uint32_t i = 0; i <= k; ++i) mem += cats[i] >= 3 ? 1u : 0u;
  if (mem > 1 || k == 0) return 0;
  const double t_cur = makespan_k(sms, ms, npts, k, shares_cur);
  const double t_c = interp(sms[k], ms[k], npts[k], double(n_sms));
  const double t_new = slate_choose_split_k(sms, ms, npts, k + 1, n_sms, step, shares_out);
  if (t_new <= 0) return 0;
  const double g = (t_cur + t_c) / t_new;
  if (gain) *gain = g;
  return g >= min_gain ? 1 : 0;
}

}  // extern "C"
