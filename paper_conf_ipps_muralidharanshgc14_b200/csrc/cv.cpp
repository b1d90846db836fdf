// cv.cpp — the generic Nitro layer (include/nitro.h §1): context, code
// variants, features, constraints, training inputs, offline training
// (exhaustive search + scaling + CV grid + RBF C-SVC), model I/O,
// selection and call; plus nitro_spmv_register, which
// plugs the five GPU SpMV variants into it.
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <limits>
#include <new>
#include <string>
#include <vector>

#include "nitro_internal.h"
#include "svm_internal.h"

struct nitro_context {
  int n_cv = 0;
};

namespace {

struct Variant {
  std::string name;
  nitro_variant_fn fn = nullptr;
  void *user = nullptr;
  std::vector<std::pair<nitro_constraint_fn, void *>> cons;
};
struct FeatureEntry {
  std::vector<std::string> names;
  nitro_feature_fn fn = nullptr;
  nitro_feature_group_fn gfn = nullptr;
  void *user = nullptr;
};

}  // namespace

struct nitro_cv {
  nitro_context *ctx = nullptr;
  std::string name;
  std::vector<Variant> variants;
  int default_id = 0;
  int model_nv = 0;  // variant count of a loaded model (a cv without registered variants)
  std::vector<FeatureEntry> feats;
  int n_feat = 0;
  std::vector<void *> inputs;
  bool frozen = false, trained = false;
  // training table
  int n_in = 0;
  std::vector<double> t_feat, t_cost;
  std::vector<int> t_label;
  // feature transform (nitro_cv_set_feature_transform): log1p of the features
  // in flog (bit j = feature j) before min-max scaling; fclip clips scaled
  // inputs to [-1, 1]
  uint32_t flog = 0;
  int fclip = 0;
  // model
  std::vector<double> lo, hi;
  double C = 1.0, gamma = 1.0, cv_acc = 0.0;
  nitro::SvmModel svm;
  // incremental tuning history (one entry per refit)
  std::vector<int> h_nlab, h_pick;
  std::vector<double> h_acc, h_perf;
};

using namespace nitro;

namespace {

constexpr double kInf = std::numeric_limits<double>::infinity();

// Training timeout: while an input is labelled, the variant being
// timed may stop early once its cost exceeds timeout_factor x the best cost
// seen so far on that input (nitro_cv_cost_cutoff).
thread_local double g_cost_cutoff = kInf;
struct CutoffScope {
  CutoffScope(double best, double factor) { g_cost_cutoff = (factor > 0 && best < kInf) ? factor * best : kInf; }
  ~CutoffScope() { g_cost_cutoff = kInf; }
};

nitro_status_t eval_features(nitro_cv *cv, const void *input, double *out) {
  int k = 0;
  for (auto &f : cv->feats) {
    if (f.fn) {
      out[k++] = f.fn(input, f.user);
    } else {
      const int n = (int)f.names.size();
      if (f.gfn(input, out + k, n, f.user) != 0)
        return fail(NITRO_E_INVALID_ARG, "feature group function failed: " + std::string(nitro_last_error()));
      k += n;
    }
  }
  return NITRO_OK;
}

bool allowed(const nitro_cv *cv, int v, const void *input) {
  for (auto &c : cv->variants[v].cons)
    if (!c.first(input, c.second)) return false;
  return true;
}

// feature j as the model sees it: log1p(x) for the features in flog (R11)
inline double tf(const nitro_cv *cv, int j, double x) {
  return (j < 32 && ((cv->flog >> j) & 1u)) ? std::log1p(x) : x;
}

void scale_row(const nitro_cv *cv, const double *f, double *out) {
  // x' = -1 + 2 (t(x) - lo) / (hi - lo); constant feature -> 0; clipped to
  // [-1, 1] when fclip (R11)
  for (int j = 0; j < cv->n_feat; ++j) {
    double v = cv->hi[j] == cv->lo[j] ? 0.0 : -1.0 + 2.0 * (tf(cv, j, f[j]) - cv->lo[j]) / (cv->hi[j] - cv->lo[j]);
    if (cv->fclip) v = v < -1.0 ? -1.0 : (v > 1.0 ? 1.0 : v);
    out[j] = v;
  }
}

int predict_raw(const nitro_cv *cv, const double *f) {
  std::vector<double> xs(cv->n_feat);
  scale_row(cv, f, xs.data());
  return svm_predict_one(cv->svm, xs.data());
}

void scale_from(nitro_cv *cv, const double *F, int n) {
  const int d = cv->n_feat;
  cv->lo.assign(d, kInf);
  cv->hi.assign(d, -kInf);
  for (int i = 0; i < n; ++i)
    for (int j = 0; j < d; ++j) {
      const double v = tf(cv, j, F[(size_t)i * d + j]);
      cv->lo[j] = std::min(cv->lo[j], v);
      cv->hi[j] = std::max(cv->hi[j], v);
    }
}

// grid + refit on the training table with the scaler already set
nitro_status_t fit_scaled(nitro_cv *cv, const nitro_train_opts &o);

nitro_status_t fit(nitro_cv *cv, const nitro_train_opts &o) {
  scale_from(cv, cv->t_feat.data(), cv->n_in);
  return fit_scaled(cv, o);
}

nitro_status_t fit_scaled(nitro_cv *cv, const nitro_train_opts &o) {
  const int n = cv->n_in, d = cv->n_feat;
  std::vector<double> Xs((size_t)n * d);
  for (int i = 0; i < n; ++i) scale_row(cv, &cv->t_feat[(size_t)i * d], &Xs[(size_t)i * d]);
  // inputs every variant failed on (label -1) carry no information: dropped
  std::vector<double> X;
  std::vector<int> y;
  for (int i = 0; i < n; ++i)
    if (cv->t_label[i] >= 0) {
      X.insert(X.end(), Xs.begin() + (size_t)i * d, Xs.begin() + (size_t)(i + 1) * d);
      y.push_back(cv->t_label[i]);
    }
  const int m = (int)y.size();
  if (m == 0) return fail(NITRO_E_STATE, "no labelled training input");
  // CV grid (R12): C ascending, gamma descending, strict improvement keeps the first
  double best = -1.0;
  int bc = o.log2c_lo, bg = o.log2g_hi;
  const int folds = std::max(2, std::min(o.folds, m));
  for (int lc = o.log2c_lo; lc <= o.log2c_hi; lc += o.log2c_step)
    for (int lg = o.log2g_hi; lg >= o.log2g_lo; lg -= o.log2g_step) {
      double acc = cv_accuracy_impl(m, d, X.data(), y.data(), std::ldexp(1.0, lc), std::ldexp(1.0, lg), o.tol, folds,
                                    o.seed);
      if (o.verbose) std::fprintf(stderr, "nitro: log2C=%d log2g=%d cv=%.4f\n", lc, lg, acc);
      if (acc > best) { best = acc; bc = lc; bg = lg; }
    }
  cv->C = std::ldexp(1.0, bc);
  cv->gamma = std::ldexp(1.0, bg);
  cv->cv_acc = best;
  svm_fit_impl(m, d, X.data(), y.data(), cv->C, cv->gamma, o.tol, cv->svm);
  cv->trained = true;
  cv->frozen = true;
  return NITRO_OK;
}

}  // namespace

#define GUARD_BEGIN try {
#define GUARD_END                                              \
  }                                                            \
  catch (const std::bad_alloc &) {                             \
    return fail(NITRO_E_OOM, "host allocation failed");       \
  }                                                            \
  catch (...) {                                                \
    return fail(NITRO_E_INVALID_ARG, "unexpected exception"); \
  }

extern "C" {

double nitro_cv_cost_cutoff(void) { return g_cost_cutoff; }

void nitro_train_opts_default(nitro_train_opts *o) {
  if (!o) return;
  o->folds = 5;
  o->seed = 0;
  o->tol = 1e-6;
  o->log2c_lo = -5; o->log2c_hi = 15; o->log2c_step = 2;
  o->log2g_lo = -15; o->log2g_hi = 3; o->log2g_step = 2;
  o->verbose = 0;
  o->timeout_factor = 20.0;
}

nitro_status_t nitro_context_create(nitro_context **out) {
  GUARD_BEGIN
  if (!out) return fail(NITRO_E_INVALID_ARG, "out is NULL");
  *out = new nitro_context();
  return NITRO_OK;
  GUARD_END
}
void nitro_context_destroy(nitro_context *ctx) { delete ctx; }

nitro_status_t nitro_cv_create(nitro_context *ctx, const char *name, nitro_cv **out) {
  GUARD_BEGIN
  if (!ctx || !out) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  nitro_cv *cv = new nitro_cv();
  cv->ctx = ctx;
  cv->name = name ? name : "";
  *out = cv;
  return NITRO_OK;
  GUARD_END
}
void nitro_cv_destroy(nitro_cv *cv) { delete cv; }  // never touches ctx (may already be gone)

nitro_status_t nitro_cv_add_variant(nitro_cv *cv, const char *name, nitro_variant_fn fn, void *user, int *out_id) {
  GUARD_BEGIN
  if (!cv || !fn) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  if (cv->frozen) return fail(NITRO_E_STATE, "code variant already trained");
  Variant v;
  v.name = name ? name : "";
  v.fn = fn;
  v.user = user;
  cv->variants.push_back(v);
  if (out_id) *out_id = (int)cv->variants.size() - 1;
  return NITRO_OK;
  GUARD_END
}

nitro_status_t nitro_cv_set_default(nitro_cv *cv, int id) {
  if (!cv || id < 0 || id >= (int)cv->variants.size()) return fail(NITRO_E_INVALID_ARG, "bad variant id");
  cv->default_id = id;
  return NITRO_OK;
}

nitro_status_t nitro_cv_set_feature_transform(nitro_cv *cv, uint32_t log_mask, int clip) {
  if (!cv) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  if (cv->frozen) return fail(NITRO_E_STATE, "code variant already trained");
  cv->flog = log_mask;
  cv->fclip = clip ? 1 : 0;
  return NITRO_OK;
}

nitro_status_t nitro_cv_add_feature(nitro_cv *cv, const char *name, nitro_feature_fn fn, void *user, int *out_id) {
  GUARD_BEGIN
  if (!cv || !fn) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  if (cv->frozen) return fail(NITRO_E_STATE, "code variant already trained");
  FeatureEntry f;
  f.names.push_back(name ? name : "");
  f.fn = fn;
  f.user = user;
  cv->feats.push_back(f);
  if (out_id) *out_id = cv->n_feat;
  cv->n_feat += 1;
  return NITRO_OK;
  GUARD_END
}

nitro_status_t nitro_cv_add_feature_group(nitro_cv *cv, const char *const *names, int n, nitro_feature_group_fn fn,
                                          void *user) {
  GUARD_BEGIN
  if (!cv || !fn || n <= 0) return fail(NITRO_E_INVALID_ARG, "bad argument");
  if (cv->frozen) return fail(NITRO_E_STATE, "code variant already trained");
  FeatureEntry f;
  for (int i = 0; i < n; ++i) f.names.push_back(names && names[i] ? names[i] : "");
  f.gfn = fn;
  f.user = user;
  cv->feats.push_back(f);
  cv->n_feat += n;
  return NITRO_OK;
  GUARD_END
}

nitro_status_t nitro_cv_add_constraint(nitro_cv *cv, int id, nitro_constraint_fn fn, void *user) {
  GUARD_BEGIN
  if (!cv || !fn || id < 0 || id >= (int)cv->variants.size()) return fail(NITRO_E_INVALID_ARG, "bad argument");
  cv->variants[id].cons.emplace_back(fn, user);
  return NITRO_OK;
  GUARD_END
}

nitro_status_t nitro_cv_add_training_input(nitro_cv *cv, void *input) {
  GUARD_BEGIN
  if (!cv) return fail(NITRO_E_INVALID_ARG, "NULL cv");
  if (cv->frozen) return fail(NITRO_E_STATE, "code variant already trained");
  cv->inputs.push_back(input);
  return NITRO_OK;
  GUARD_END
}

nitro_status_t nitro_cv_train(nitro_cv *cv, const nitro_train_opts *opts) {
  NITRO_NVTX("nitro_cv_train");
  GUARD_BEGIN
  if (!cv) return fail(NITRO_E_INVALID_ARG, "NULL cv");
  if (cv->variants.empty() || cv->n_feat == 0 || cv->inputs.empty())
    return fail(NITRO_E_STATE, "need variants, features and training inputs");
  nitro_train_opts o;
  if (opts) o = *opts; else nitro_train_opts_default(&o);
  const int n = (int)cv->inputs.size(), d = cv->n_feat, V = (int)cv->variants.size();
  cv->n_in = n;
  cv->t_feat.assign((size_t)n * d, 0.0);
  cv->t_cost.assign((size_t)n * V, kInf);
  cv->t_label.assign(n, -1);
  for (int i = 0; i < n; ++i) {
    void *in = cv->inputs[i];
    NITRO_TRY(eval_features(cv, in, &cv->t_feat[(size_t)i * d]));
    double best = kInf;
    for (int q = 0; q < V; ++q) {
      // exhaustive search; a failed constraint makes the cost infinite.
      // The default variant is timed first, so the training timeout has a
      // reference cost early; the label is the argmin whatever the order.
      const int v = q == 0 ? cv->default_id : (q <= cv->default_id ? q - 1 : q);
      double c = kInf;
      if (allowed(cv, v, in)) {
        const CutoffScope cs(best, o.timeout_factor);
        c = cv->variants[v].fn(in, cv->variants[v].user);
      }
      if (std::isnan(c)) c = kInf;
      cv->t_cost[(size_t)i * V + v] = c;
      best = std::min(best, c);
    }
    for (int v = 0; v < V; ++v)  // label = argmin, ties -> lowest id
      if (cv->t_label[i] < 0 ? cv->t_cost[(size_t)i * V + v] < kInf
                             : cv->t_cost[(size_t)i * V + v] < cv->t_cost[(size_t)i * V + cv->t_label[i]])
        cv->t_label[i] = v;
    if (o.verbose)
      std::fprintf(stderr, "nitro: input %d/%d label %d\n", i + 1, n, cv->t_label[i]);
  }
  return fit(cv, o);
  GUARD_END
}

nitro_status_t nitro_cv_train_from_table(nitro_cv *cv, int n_in, const double *feat, const double *cost,
                                         const nitro_train_opts *opts) {
  GUARD_BEGIN
  if (!cv || n_in <= 0 || !feat || !cost) return fail(NITRO_E_INVALID_ARG, "bad argument");
  if (cv->variants.empty() || cv->n_feat == 0) return fail(NITRO_E_STATE, "need variants and features");
  nitro_train_opts o;
  if (opts) o = *opts; else nitro_train_opts_default(&o);
  const int d = cv->n_feat, V = (int)cv->variants.size();
  cv->n_in = n_in;
  cv->t_feat.assign(feat, feat + (size_t)n_in * d);
  cv->t_cost.assign(cost, cost + (size_t)n_in * V);
  cv->t_label.assign(n_in, -1);
  for (int i = 0; i < n_in; ++i) {
    double best = kInf;
    for (int v = 0; v < V; ++v) {
      double c = cv->t_cost[(size_t)i * V + v];
      if (c < best) { best = c; cv->t_label[i] = v; }
    }
  }
  return fit(cv, o);
  GUARD_END
}

void nitro_itune_opts_default(nitro_itune_opts *o) {
  if (!o) return;
  o->init = 0;
  o->iters = 0;
  o->acc = 0.0;
  o->seed = 0;
  o->prob_folds = 5;
  o->n_test = 0;
  o->test_feat = nullptr;
  o->test_cost = nullptr;
}

nitro_status_t nitro_cv_itune(nitro_cv *cv, const nitro_train_opts *topts, const nitro_itune_opts *iopts) {
  NITRO_NVTX("nitro_cv_itune");
  GUARD_BEGIN
  if (!cv) return fail(NITRO_E_INVALID_ARG, "NULL cv");
  if (cv->variants.empty() || cv->n_feat == 0 || cv->inputs.empty())
    return fail(NITRO_E_STATE, "need variants, features and training inputs");
  nitro_train_opts o;
  if (topts) o = *topts; else nitro_train_opts_default(&o);
  nitro_itune_opts it;
  if (iopts) it = *iopts; else nitro_itune_opts_default(&it);
  if (it.n_test > 0 && (!it.test_feat || !it.test_cost)) return fail(NITRO_E_INVALID_ARG, "test set arrays missing");
  const int n = (int)cv->inputs.size(), d = cv->n_feat, V = (int)cv->variants.size();
  // 1. features of every input first: they are cheap next to running variants
  std::vector<double> F((size_t)n * d);
  for (int i = 0; i < n; ++i) NITRO_TRY(eval_features(cv, cv->inputs[i], &F[(size_t)i * d]));
  scale_from(cv, F.data(), n);  // the whole pool's features are known: scale with them
  // seeded order of the initial picks (same key as the CV folds, R15)
  std::vector<int> order(n);
  for (int i = 0; i < n; ++i) order[i] = i;
  const uint64_t s0 = [](uint64_t z) {
    z += 0x9E3779B97F4A7C15ULL; z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL; return z ^ (z >> 31);
  }(it.seed);
  auto key = [&](int i) {
    uint64_t z = s0 ^ (uint64_t)i;
    z += 0x9E3779B97F4A7C15ULL; z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL; return z ^ (z >> 31);
  };
  std::stable_sort(order.begin(), order.end(), [&](int a, int b) {
    const uint64_t ka = key(a), kb = key(b);
    return ka != kb ? ka < kb : a < b;
  });
  std::vector<char> done(n, 0);
  std::vector<int> labelled, label_of(n, -1);
  std::vector<double> cost((size_t)n * V, kInf);
  auto label_input = [&](int i) {  // exhaustive search on one input
    void *in = cv->inputs[i];
    double best = kInf;
    for (int q = 0; q < V; ++q) {  // default first (training timeout reference), as nitro_cv_train
      const int v = q == 0 ? cv->default_id : (q <= cv->default_id ? q - 1 : q);
      double c = kInf;
      if (allowed(cv, v, in)) {
        const CutoffScope cs(best, o.timeout_factor);
        c = cv->variants[v].fn(in, cv->variants[v].user);
      }
      if (std::isnan(c)) c = kInf;
      cost[(size_t)i * V + v] = c;
      best = std::min(best, c);
    }
    for (int v = 0; v < V; ++v)  // label = argmin, ties -> lowest id
      if (cost[(size_t)i * V + v] < kInf &&
          (label_of[i] < 0 || cost[(size_t)i * V + v] < cost[(size_t)i * V + label_of[i]]))
        label_of[i] = v;
    done[i] = 1;
    labelled.push_back(i);
  };
  auto distinct = [&]() {
    std::vector<char> seen(V, 0);
    int k = 0;
    for (int i : labelled)
      if (label_of[i] >= 0 && !seen[label_of[i]]) { seen[label_of[i]] = 1; ++k; }
    return k;
  };
  const int init = it.init > 0 ? it.init : V;
  size_t pos = 0;
  while (pos < order.size() && ((int)labelled.size() < init || distinct() < 2)) label_input(order[pos++]);
  // test-set labels (argmin of the given costs, ties -> lowest id)
  std::vector<int> tlab(std::max(it.n_test, 0), -1);
  for (int t = 0; t < it.n_test; ++t) {
    double b = kInf;
    for (int v = 0; v < V; ++v)
      if (it.test_cost[(size_t)t * V + v] < b) { b = it.test_cost[(size_t)t * V + v]; tlab[t] = v; }
  }
  cv->h_nlab.clear(); cv->h_pick.clear(); cv->h_acc.clear(); cv->h_perf.clear();
  int picks = 0;
  for (;;) {
    // refit on the labelled inputs (labelling order)
    const int m = (int)labelled.size();
    cv->n_in = m;
    cv->t_feat.resize((size_t)m * d);
    cv->t_cost.resize((size_t)m * V);
    cv->t_label.resize(m);
    for (int r = 0; r < m; ++r) {
      const int i = labelled[r];
      std::copy(&F[(size_t)i * d], &F[(size_t)(i + 1) * d], &cv->t_feat[(size_t)r * d]);
      std::copy(&cost[(size_t)i * V], &cost[(size_t)(i + 1) * V], &cv->t_cost[(size_t)r * V]);
      cv->t_label[r] = label_of[i];
    }
    NITRO_TRY(fit_scaled(cv, o));
    double acc = std::numeric_limits<double>::quiet_NaN(), perf = acc;
    if (it.n_test > 0) {
      int ok = 0, cnt = 0;
      double ps = 0.0;
      for (int t = 0; t < it.n_test; ++t) {
        if (tlab[t] < 0) continue;
        int v = predict_raw(cv, &it.test_feat[(size_t)t * d]);
        if (v < 0 || v >= V || !std::isfinite(it.test_cost[(size_t)t * V + v])) v = cv->default_id;
        ++cnt;
        ok += v == tlab[t];
        const double cs = it.test_cost[(size_t)t * V + v], cb = it.test_cost[(size_t)t * V + tlab[t]];
        ps += std::isfinite(cs) ? cb / cs : 0.0;
      }
      if (cnt) { acc = (double)ok / cnt; perf = ps / cnt; }
    }
    cv->h_nlab.push_back(m);
    cv->h_pick.push_back(-1);
    cv->h_acc.push_back(acc);
    cv->h_perf.push_back(perf);
    if (it.acc > 0 && acc >= it.acc) break;
    if (it.iters > 0 && picks >= it.iters) break;
    std::vector<int> pool;
    for (int i = 0; i < n; ++i)
      if (!done[i]) pool.push_back(i);
    if (pool.empty()) break;
    int pick = -1;
    if (cv->svm.const_label >= 0 || cv->svm.classes.size() < 2) {
      for (int i : order)
        if (!done[i]) { pick = i; break; }
    } else {
      // Best-vs-Second-Best: smallest gap between the two largest probabilities
      std::vector<double> X;
      std::vector<int> y;
      for (int i : labelled)
        if (label_of[i] >= 0) {
          std::vector<double> xs(d);
          scale_row(cv, &F[(size_t)i * d], xs.data());
          X.insert(X.end(), xs.begin(), xs.end());
          y.push_back(label_of[i]);
        }
      SvmModel pm;
      svm_fit_prob_impl((int)y.size(), d, X.data(), y.data(), cv->C, cv->gamma, o.tol,
                        std::max(2, it.prob_folds), it.seed, pm);
      const int k = (int)pm.classes.size();
      std::vector<double> xs(d), p(std::max(k, 1));
      double best_gap = kInf;
      for (int i : pool) {
        scale_row(cv, &F[(size_t)i * d], xs.data());
        svm_probability_impl(pm, xs.data(), p.data());
        double p1 = -kInf, p2 = -kInf;
        for (int c = 0; c < k; ++c) {
          if (p[c] > p1) { p2 = p1; p1 = p[c]; }
          else if (p[c] > p2) p2 = p[c];
        }
        const double gap = p1 - p2;
        if (gap < best_gap) { best_gap = gap; pick = i; }  // ties -> lowest input index
      }
    }
    cv->h_pick.back() = pick;
    label_input(pick);
    ++picks;
  }
  cv->trained = true;
  cv->frozen = true;
  return NITRO_OK;
  GUARD_END
}

nitro_status_t nitro_cv_itune_history(const nitro_cv *cv, int *n_steps, int *n_labelled, int *picked,
                                      double *test_acc, double *test_perf) {
  if (!cv || !n_steps) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  *n_steps = (int)cv->h_nlab.size();
  if (n_labelled) std::copy(cv->h_nlab.begin(), cv->h_nlab.end(), n_labelled);
  if (picked) std::copy(cv->h_pick.begin(), cv->h_pick.end(), picked);
  if (test_acc) std::copy(cv->h_acc.begin(), cv->h_acc.end(), test_acc);
  if (test_perf) std::copy(cv->h_perf.begin(), cv->h_perf.end(), test_perf);
  return NITRO_OK;
}

nitro_status_t nitro_cv_training_table(const nitro_cv *cv, int *n_in, double *cost, double *feat, int *label) {
  if (!cv) return fail(NITRO_E_INVALID_ARG, "NULL cv");
  if (n_in) *n_in = cv->n_in;
  if (cost) std::copy(cv->t_cost.begin(), cv->t_cost.end(), cost);
  if (feat) std::copy(cv->t_feat.begin(), cv->t_feat.end(), feat);
  if (label) std::copy(cv->t_label.begin(), cv->t_label.end(), label);
  return NITRO_OK;
}

nitro_status_t nitro_cv_model_info(const nitro_cv *cv, double *C, double *gamma, double *cv_acc, int *n_sv) {
  if (!cv) return fail(NITRO_E_INVALID_ARG, "NULL cv");
  if (!cv->trained) return fail(NITRO_E_STATE, "not trained");
  if (C) *C = cv->C;
  if (gamma) *gamma = cv->gamma;
  if (cv_acc) *cv_acc = cv->cv_acc;
  if (n_sv) {
    std::vector<char> is(cv->svm.n_train, 0);
    for (auto &p : cv->svm.pairs)
      for (int s : p.sv) is[s] = 1;
    int k = 0;
    for (char c : is) k += c;
    *n_sv = k;
  }
  return NITRO_OK;
}

nitro_status_t nitro_cv_num_features(const nitro_cv *cv, int *n) {
  if (!cv || !n) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  *n = cv->n_feat;
  return NITRO_OK;
}
nitro_status_t nitro_cv_num_variants(const nitro_cv *cv, int *n) {
  if (!cv || !n) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  *n = (int)cv->variants.size();
  return NITRO_OK;
}

// Model file: text, fp64 written with %.17g (round-trips exactly).
nitro_status_t nitro_cv_save_model(const nitro_cv *cv, const char *path) {
  if (!cv || !path) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  if (!cv->trained) return fail(NITRO_E_STATE, "not trained");
  FILE *f = std::fopen(path, "w");
  if (!f) return fail(NITRO_E_IO, std::string("cannot write ") + path);
  const SvmModel &m = cv->svm;
  std::fprintf(f, "NITRO_MODEL 2\n%d %d %d\n%u %d\n", cv->n_feat, (int)cv->variants.size(), cv->default_id,
               (unsigned)cv->flog, cv->fclip);
  for (int j = 0; j < cv->n_feat; ++j) std::fprintf(f, "%.17g %.17g\n", cv->lo[j], cv->hi[j]);
  std::fprintf(f, "%.17g %.17g %.17g\n", cv->C, cv->gamma, cv->cv_acc);
  std::fprintf(f, "%d %d %d %zu\n", m.d, m.n_train, m.const_label, m.classes.size());
  for (int c : m.classes) std::fprintf(f, "%d ", c);
  std::fprintf(f, "\n");
  for (size_t i = 0; i < m.X.size(); ++i) std::fprintf(f, "%.17g\n", m.X[i]);
  std::fprintf(f, "%zu\n", m.pairs.size());
  for (auto &p : m.pairs) {
    std::fprintf(f, "%d %d %.17g %zu\n", p.ca, p.cb, p.rho, p.sv.size());
    for (size_t t = 0; t < p.sv.size(); ++t) std::fprintf(f, "%d %.17g\n", p.sv[t], p.coef[t]);
  }
  bool ok = std::fclose(f) == 0;
  return ok ? NITRO_OK : fail(NITRO_E_IO, "write failed");
}

nitro_status_t nitro_cv_load_model(nitro_cv *cv, const char *path) {
  GUARD_BEGIN
  if (!cv || !path) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  FILE *f = std::fopen(path, "r");
  if (!f) return fail(NITRO_E_IO, std::string("cannot read ") + path);
  auto bad = [&](const char *why) { std::fclose(f); return fail(NITRO_E_IO, std::string("bad model file: ") + why); };
  int ver = 0, nf = 0, nv = 0, def = 0;
  if (std::fscanf(f, "NITRO_MODEL %d\n%d %d %d", &ver, &nf, &nv, &def) != 4 || (ver != 1 && ver != 2))
    return bad("header");
  unsigned flog = 0;
  int fclip = 0;
  if (ver >= 2 && std::fscanf(f, "%u %d", &flog, &fclip) != 2) return bad("feature transform");
  if (nf <= 0 || nf > 4096 || nv <= 0 || nv > 4096) return bad("feature / variant count");
  if (cv->n_feat && nf != cv->n_feat) return bad("feature count differs from this code variant");
  if (!cv->variants.empty() && nv != (int)cv->variants.size()) return bad("variant count differs");
  cv->flog = flog;
  cv->fclip = fclip;
  cv->lo.assign(nf, 0.0);
  cv->hi.assign(nf, 0.0);
  for (int j = 0; j < nf; ++j)
    if (std::fscanf(f, "%lg %lg", &cv->lo[j], &cv->hi[j]) != 2) return bad("scaler");
  if (std::fscanf(f, "%lg %lg %lg", &cv->C, &cv->gamma, &cv->cv_acc) != 3) return bad("params");
  SvmModel m;
  size_t ncls = 0;
  if (std::fscanf(f, "%d %d %d %zu", &m.d, &m.n_train, &m.const_label, &ncls) != 4) return bad("svm header");
  // every index the predictor follows is validated here (a stale or corrupted
  // file must give NITRO_E_IO, not out-of-bounds reads at predict time)
  if (m.d != nf) return bad("SVM dimension differs from the feature count");
  if (m.n_train < 0 || m.n_train > (1 << 24) || ncls > (size_t)nv) return bad("svm sizes");
  if (m.const_label >= nv || (m.const_label < 0 && ncls == 0)) return bad("constant label");
  m.classes.resize(ncls);
  for (auto &c : m.classes)
    if (std::fscanf(f, "%d", &c) != 1 || c < 0 || c >= nv) return bad("classes");
  m.X.resize((size_t)m.d * m.n_train);
  for (auto &x : m.X)
    if (std::fscanf(f, "%lg", &x) != 1) return bad("points");
  size_t np = 0;
  if (std::fscanf(f, "%zu", &np) != 1) return bad("pairs");
  m.pairs.resize(np);
  for (auto &p : m.pairs) {
    size_t ns = 0;
    if (std::fscanf(f, "%d %d %lg %zu", &p.ca, &p.cb, &p.rho, &ns) != 4) return bad("pair");
    if (p.ca < 0 || p.cb < 0 || (size_t)p.ca >= ncls || (size_t)p.cb >= ncls || ns > (size_t)m.n_train)
      return bad("pair classes");
    p.sv.resize(ns);
    p.coef.resize(ns);
    for (size_t t = 0; t < ns; ++t)
      if (std::fscanf(f, "%d %lg", &p.sv[t], &p.coef[t]) != 2 || p.sv[t] < 0 || p.sv[t] >= m.n_train)
        return bad("sv");
  }
  std::fclose(f);
  m.gamma = cv->gamma;
  cv->svm = std::move(m);
  cv->n_feat = nf;
  if (def >= 0 && def < nv && (int)cv->variants.size() == nv) cv->default_id = def;
  cv->model_nv = nv;
  cv->trained = true;
  cv->frozen = true;
  return NITRO_OK;
  GUARD_END
}

nitro_status_t nitro_cv_predict(nitro_cv *cv, const double *feat, const int *allowed_mask, int *out_variant) {
  GUARD_BEGIN
  if (!cv || !feat || !out_variant) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  if (!cv->trained) return fail(NITRO_E_STATE, "select before train/load");
  int v = predict_raw(cv, feat);
  const int nvar = cv->variants.empty() ? cv->model_nv : (int)cv->variants.size();
  if (v < 0 || v >= nvar || (allowed_mask && !allowed_mask[v])) v = cv->default_id;
  *out_variant = v;
  return NITRO_OK;
  GUARD_END
}

nitro_status_t nitro_cv_select(nitro_cv *cv, const void *input, int *out_variant, double *out_feat) {
  NITRO_NVTX("nitro_cv_select");
  GUARD_BEGIN
  if (!cv || !out_variant) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  if (!cv->trained) return fail(NITRO_E_STATE, "select before train/load");
  std::vector<double> f(cv->n_feat);
  NITRO_TRY(eval_features(cv, input, f.data()));
  int v = predict_raw(cv, f.data());
  if (v < 0 || v >= (int)cv->variants.size() || !allowed(cv, v, input)) v = cv->default_id;
  *out_variant = v;
  if (out_feat) std::copy(f.begin(), f.end(), out_feat);
  return NITRO_OK;
  GUARD_END
}

nitro_status_t nitro_cv_call(nitro_cv *cv, void *input, int *out_variant, double *out_cost) {
  NITRO_NVTX("nitro_cv_call");
  GUARD_BEGIN
  int v = 0;
  NITRO_TRY(nitro_cv_select(cv, input, &v, nullptr));
  double c = cv->variants[v].fn(input, cv->variants[v].user);
  if (out_variant) *out_variant = v;
  if (out_cost) *out_cost = c;
  return NITRO_OK;
  GUARD_END
}

// ---------------------------------------------------------------- SpMV registration
static double spmv_variant_fn(void *input, void *user) {
  nitro_spmv_input *in = (nitro_spmv_input *)input;
  const int v = (int)(intptr_t)user;
  double t = kInf;
  if (!in || !in->A || !in->d_x || !in->d_y) return kInf;
  // training timeout: stop the reps once the median passes the cv's cutoff
  if (nitro::time_variant(in->A, v, in->d_x, in->d_y, std::max(in->warmup, 0), in->reps > 0 ? in->reps : 1,
                          in->flush_l2, nitro_cv_cost_cutoff(), &t, nullptr, nullptr) != NITRO_OK)
    return kInf;
  return t;
}
static int spmv_feature_group(const void *input, double *out, int n, void *) {
  const nitro_spmv_input *in = (const nitro_spmv_input *)input;
  if (!in || !in->A || n != 7) return 1;
  nitro_spmv_feat f;
  if (nitro_spmv_features(in->A, &f) != NITRO_OK) return 1;
  out[0] = (double)f.nnz; out[1] = (double)f.rows; out[2] = f.mean; out[3] = f.sd;
  out[4] = f.max_dev; out[5] = f.dia_fill; out[6] = f.ell_fill;
  return 0;
}
static int spmv_constraint(const void *input, void *user) {
  const nitro_spmv_input *in = (const nitro_spmv_input *)input;
  int ok = 0;
  if (!in || !in->A) return 0;
  if (nitro_spmv_allowed(in->A, (int)(intptr_t)user, &ok) != NITRO_OK) return 0;
  return ok;
}

nitro_status_t nitro_spmv_register(nitro_cv *cv) {
  GUARD_BEGIN
  if (!cv) return fail(NITRO_E_INVALID_ARG, "NULL cv");
  if (!cv->variants.empty() || cv->n_feat != 0) return fail(NITRO_E_STATE, "register on a fresh code variant");
  static const char *vn[NITRO_NUM_VARIANTS] = {"csr_scalar", "csr_vector", "ell", "dia", "hyb"};
  for (int v = 0; v < NITRO_NUM_VARIANTS; ++v)
    NITRO_TRY(nitro_cv_add_variant(cv, vn[v], spmv_variant_fn, (void *)(intptr_t)v, nullptr));
  static const char *fn[7] = {"nnz", "rows", "mean", "sd", "max_dev", "dia_fill", "ell_fill"};
  NITRO_TRY(nitro_cv_add_feature_group(cv, fn, 7, spmv_feature_group, nullptr));
  NITRO_TRY(nitro_cv_add_constraint(cv, NITRO_DIA, spmv_constraint, (void *)(intptr_t)NITRO_DIA));
  NITRO_TRY(nitro_cv_add_constraint(cv, NITRO_ELL, spmv_constraint, (void *)(intptr_t)NITRO_ELL));
  // features scaled to [-1, 1] as the paper states; the log1p + clip
  // extension (R11x) is opt-in: nitro_cv_set_feature_transform
  return nitro_cv_set_default(cv, NITRO_CSR_VECTOR);
  GUARD_END
}

}  // extern "C"
