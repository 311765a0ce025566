// predictor.cpp — duration model store (a9, a10): per-kernel LR and two-stage fused model.
//
// Per-kernel LR (§VI-C): X = a * blocks + b from a few measured points.
// Two-stage fused model (§VI-A/B, Eqs. 1-6): load ratio r = X_cd / X_tc (Eq. 1);
// normalised duration tau = T_fuse / X_tc is piecewise linear in r, one LR per stage, with
// the inflection at the opportune ratio (Fig. 10).  Reading: tau(r) =
// max(l1(r), l2(r)); fitted from samples at r in {0.1, 0.2, 1.8, 1.9}, refit
// online when the prediction error exceeds 10%.
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <utility>
#include <vector>

#include "runtime.h"
#include "tacker.h"

using namespace tkrt;

namespace {

struct Lr {
  std::vector<std::pair<double, double>> pts;
  bool fitted = false;
  double a = 0, b = 0;
};

struct Pair {
  std::vector<std::pair<double, double>> pts;  // (r, tau)
  bool fitted = false;
  double a1 = 0, b1 = 0, a2 = 0, b2 = 0;       // l_s(r) = a_s + b_s r
};

std::mutex g_mu;
std::map<std::string, Lr> g_lr;
std::map<std::string, Pair> g_pair;

// closed-form least squares y = slope*x + icpt
void ols(const std::vector<std::pair<double, double>> &p, double &slope, double &icpt) {
  const double n = (double)p.size();
  double mx = 0, my = 0;
  for (auto &q : p) mx += q.first, my += q.second;
  mx /= n;
  my /= n;
  double sxx = 0, sxy = 0;
  for (auto &q : p) sxx += (q.first - mx) * (q.first - mx), sxy += (q.first - mx) * (q.second - my);
  if (sxx == 0.0) {
    slope = 0;
    icpt = my;
    return;
  }
  slope = sxy / sxx;
  icpt = my - slope * mx;
}

// split < 0: the lower half of the samples (by r) starts as stage 1 — for the paper's training
// ratios {0.1, 0.2, 1.8, 1.9} that is {0.1, 0.2} vs {1.8, 1.9}, and it still works
// when coarse BE blocks shift every measured ratio to one side of 1.
bool fit_pair(Pair &P, double split) {
  std::vector<std::pair<double, double>> pts = P.pts, lo, hi;
  std::sort(pts.begin(), pts.end());
  if (pts.size() < 2) return false;
  if (split >= 0)
    for (auto &q : pts) (q.first <= split ? lo : hi).push_back(q);
  if (lo.empty() || hi.empty()) {   // median split (also the fallback for a one-sided split)
    lo.assign(pts.begin(), pts.begin() + pts.size() / 2);
    hi.assign(pts.begin() + pts.size() / 2, pts.end());
  }
  for (int it = 0; it < 16; ++it) {
    ols(lo, P.b1, P.a1);
    ols(hi, P.b2, P.a2);
    if (P.b1 == P.b2) break;
    const double rs = (P.a2 - P.a1) / (P.b1 - P.b2);
    std::vector<std::pair<double, double>> nlo, nhi;
    for (auto &q : pts) (q.first <= rs ? nlo : nhi).push_back(q);
    // each stage is a line through >= 2 samples (one LR per stage): a re-split leaving
    // a stage one sample would fix no slope (OLS slope 0, a flat stage)
    if (nlo.size() < 2 || nhi.size() < 2 || (nlo == lo && nhi == hi)) break;
    lo.swap(nlo);
    hi.swap(nhi);
  }
  // Fig. 10's stages are co-run (slope below the CD-solo stage's) then CD solo; fitted
  // slopes in the other order describe no such curve (max() would put the steeper first stage at
  // large r): one LR over all samples (reading 5)
  if (P.b1 >= P.b2) {
    ols(pts, P.b1, P.a1);
    P.a2 = P.a1;
    P.b2 = P.b1;
  }
  P.fitted = true;
  return true;
}

double pair_tau(const Pair &P, double r) { return std::max(P.a1 + P.b1 * r, P.a2 + P.b2 * r); }

bool key_ok(const char *k) { return k && *k && strlen(k) < 256; }

}  // namespace

namespace tkrt {
bool model_predict(const std::string &key, double x, double *y) {
  std::lock_guard<std::mutex> g(g_mu);
  auto it = g_lr.find(key);
  if (it == g_lr.end() || !it->second.fitted) return false;
  *y = it->second.a * x + it->second.b;
  return true;
}
bool pair_predict(const std::string &key, double x_tc, double x_cd, double *y) {
  std::lock_guard<std::mutex> g(g_mu);
  auto it = g_pair.find(key);
  if (it == g_pair.end() || !it->second.fitted || x_tc <= 0) return false;
  *y = x_tc * pair_tau(it->second, x_cd / x_tc);
  return true;
}
// Opportune load ratio of a pair (Fig. 10): the inflection r* = (a2 - a1) / (b1 - b2)
// of the two-stage model, where stage 1 (co-run, slope b1) meets stage 2 (CD solo, slope b2).
// False when the fitted stages do not form a convex two-stage curve (b1 >= b2) or r* <= 0.
bool pair_opportune(const std::string &key, double *r) {
  std::lock_guard<std::mutex> g(g_mu);
  auto it = g_pair.find(key);
  if (it == g_pair.end() || !it->second.fitted) return false;
  const Pair &P = it->second;
  if (!(P.b1 < P.b2)) return false;
  const double rs = (P.a2 - P.a1) / (P.b1 - P.b2);
  if (!(rs > 0) || !std::isfinite(rs)) return false;
  *r = rs;
  return true;
}
const std::string &fused_lc_key(tacker_fused_t f);
const std::string &fused_be_key(tacker_fused_t f);
const std::string &fused_pair_key(tacker_fused_t f);
int64_t fused_lc_tiles(tacker_fused_t f);
int64_t fused_be_blocks(tacker_fused_t f);
}  // namespace tkrt

extern "C" {

tacker_status tacker_model_add_sample(const char *key, double blocks, double ms) {
  if (!key_ok(key) || !std::isfinite(blocks) || !std::isfinite(ms)) return set_error("bad sample"), TACKER_EINVAL;
  std::lock_guard<std::mutex> g(g_mu);
  g_lr[key].pts.emplace_back(blocks, ms);
  return TACKER_OK;
}

tacker_status tacker_model_fit(const char *key, double *a_out, double *b_out) {
  if (!key_ok(key)) return set_error("bad key"), TACKER_EINVAL;
  std::lock_guard<std::mutex> g(g_mu);
  auto it = g_lr.find(key);
  if (it == g_lr.end() || it->second.pts.empty()) return set_error("no samples for %s", key), TACKER_ENOMODEL;
  ols(it->second.pts, it->second.a, it->second.b);
  it->second.fitted = true;
  if (a_out) *a_out = it->second.a;
  if (b_out) *b_out = it->second.b;
  return TACKER_OK;
}

tacker_status tacker_model_predict(const char *key, double blocks, double *ms_out) {
  if (!key_ok(key) || !ms_out) return set_error("bad argument"), TACKER_EINVAL;
  if (!model_predict(key, blocks, ms_out)) return set_error("no fitted model for %s", key), TACKER_ENOMODEL;
  return TACKER_OK;
}

tacker_status tacker_pair_add_sample(const char *key, double x_tc, double x_cd, double t_fused) {
  if (!key_ok(key) || !(x_tc > 0) || !(x_cd >= 0) || !(t_fused > 0)) return set_error("bad pair sample"), TACKER_EINVAL;
  std::lock_guard<std::mutex> g(g_mu);
  g_pair[key].pts.emplace_back(x_cd / x_tc, t_fused / x_tc);
  return TACKER_OK;
}

tacker_status tacker_pair_fit(const char *key, double coef_out[4]) {
  if (!key_ok(key)) return set_error("bad key"), TACKER_EINVAL;
  std::lock_guard<std::mutex> g(g_mu);
  auto it = g_pair.find(key);
  if (it == g_pair.end() || !fit_pair(it->second, -1.0))
    return set_error("pair %s needs at least 2 samples", key), TACKER_ENOMODEL;
  if (coef_out) {
    coef_out[0] = it->second.a1;
    coef_out[1] = it->second.b1;
    coef_out[2] = it->second.a2;
    coef_out[3] = it->second.b2;
  }
  return TACKER_OK;
}

tacker_status tacker_pair_predict(const char *key, double x_tc, double x_cd, double *ms_out) {
  if (!key_ok(key) || !ms_out) return set_error("bad argument"), TACKER_EINVAL;
  if (!pair_predict(key, x_tc, x_cd, ms_out)) return set_error("no fitted pair model for %s", key), TACKER_ENOMODEL;
  return TACKER_OK;
}

tacker_status tacker_pair_observe(const char *key, double x_tc, double x_cd, double t_meas, int32_t *refit_out) {
  if (!key_ok(key) || !(x_tc > 0) || !(t_meas > 0)) return set_error("bad argument"), TACKER_EINVAL;
  std::lock_guard<std::mutex> g(g_mu);
  auto it = g_pair.find(key);
  if (it == g_pair.end() || !it->second.fitted) return set_error("no fitted pair model for %s", key), TACKER_ENOMODEL;
  Pair &P = it->second;
  const double pred = x_tc * pair_tau(P, x_cd / x_tc);
  int32_t refit = 0;
  if (std::fabs(pred - t_meas) / t_meas > 0.10) {
    P.pts.emplace_back(x_cd / x_tc, t_meas / x_tc);
    double split = -1.0;
    if (P.b1 != P.b2) {
      const double rs = (P.a2 - P.a1) / (P.b1 - P.b2);
      if (rs > 0) split = rs;
    }
    fit_pair(P, split);
    refit = 1;
  }
  if (refit_out) *refit_out = refit;
  return TACKER_OK;
}

tacker_status tacker_model_clear(void) {
  std::lock_guard<std::mutex> g(g_mu);
  g_lr.clear();
  g_pair.clear();
  return TACKER_OK;
}

// Text format, one record per line:  L <key> <n> x y x y ...   /   P <key> <n> r tau ...
tacker_status tacker_model_save(const char *path) {
  if (!path) return set_error("null path"), TACKER_EINVAL;
  std::lock_guard<std::mutex> g(g_mu);
  FILE *f = fopen(path, "w");
  if (!f) return set_error("cannot open %s", path), TACKER_EINVAL;
  for (auto &kv : g_lr) {
    fprintf(f, "L %s %zu", kv.first.c_str(), kv.second.pts.size());
    for (auto &p : kv.second.pts) fprintf(f, " %.17g %.17g", p.first, p.second);
    fprintf(f, "\n");
  }
  for (auto &kv : g_pair) {
    fprintf(f, "P %s %zu", kv.first.c_str(), kv.second.pts.size());
    for (auto &p : kv.second.pts) fprintf(f, " %.17g %.17g", p.first, p.second);
    fprintf(f, "\n");
  }
  fclose(f);
  return TACKER_OK;
}

tacker_status tacker_model_load(const char *path) {
  if (!path) return set_error("null path"), TACKER_EINVAL;
  FILE *f = fopen(path, "r");
  if (!f) return set_error("cannot open %s", path), TACKER_EINVAL;
  std::lock_guard<std::mutex> g(g_mu);
  char kind[4], key[512];
  size_t n;
  while (fscanf(f, "%3s %511s %zu", kind, key, &n) == 3) {
    std::vector<std::pair<double, double>> pts(n);
    for (size_t i = 0; i < n; ++i)
      if (fscanf(f, "%lg %lg", &pts[i].first, &pts[i].second) != 2) {
        fclose(f);
        return set_error("corrupt model file"), TACKER_EINVAL;
      }
    if (kind[0] == 'L') {
      Lr &m = g_lr[key];
      m.pts = pts;
      ols(m.pts, m.a, m.b);
      m.fitted = !pts.empty();
    } else {
      Pair &P = g_pair[key];
      P.pts = pts;
      fit_pair(P, -1.0);
    }
  }
  fclose(f);
  return TACKER_OK;
}

tacker_status tacker_predict_duration(tacker_fused_t f, double *ms_out) {
  if (!f || !ms_out) return set_error("null argument"), TACKER_EINVAL;
  double xtc, xcd;
  if (!model_predict(fused_lc_key(f), (double)fused_lc_tiles(f), &xtc))
    return set_error("no LC model %s", fused_lc_key(f).c_str()), TACKER_ENOMODEL;
  if (fused_be_key(f).empty()) {
    *ms_out = xtc;
    return TACKER_OK;
  }
  if (!model_predict(fused_be_key(f), (double)fused_be_blocks(f), &xcd))
    return set_error("no BE model %s", fused_be_key(f).c_str()), TACKER_ENOMODEL;
  if (!pair_predict(fused_pair_key(f), xtc, xcd, ms_out))
    return set_error("no pair model %s", fused_pair_key(f).c_str()), TACKER_ENOMODEL;
  return TACKER_OK;
}

}  // extern "C"
