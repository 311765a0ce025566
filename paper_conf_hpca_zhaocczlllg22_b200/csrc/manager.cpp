// manager.cpp — Tacker's runtime QoS-aware kernel manager (a11; §VII).
//
// Per LC kernel of the oldest active query:
//   * Eq. 9: at the first issue of the newest query Q,
//       Thr = T_qos - T_queue - T_ori_solo(Q) - sum_i T_lc_i(remaining, earlier queries),
//     T_queue = issue time - arrival (reading).  "Thr close to 0" ->
//     Q runs direct: Thr <= max(direct_eps, shortest ready BE head) (direct_rule MIN_BE, default).
//   * Only the newest query fuses/reorders; params.fuse_older (reading 18): an older
//     query too, within min(its Thr, Eq. 9 of every later active query) - older_margin_ms.
//   * CUDA-core LC kernel (NEXT-2, reading 17): the same Eq. 8 over ready BE tensor-core heads,
//     the pair model evaluated with X_tc = the BE kernel, X_cd = the LC kernel.
//   * TC kernel: Eq. 8 over the ready BE heads with a fitted pair model:
//       Ttc + Tcd > Tk_fuse  &&  Tk_fuse - Ttc < Thr;  max Tgain = Tcd - (Tk_fuse - Ttc)
//     (P:2045-2056), ties -> lowest app index; Thr -= Tk_fuse - Ttc.
//   * Original launch (if not fused), then reorder ready BE heads with Ttmp < Thr:
//     only after an unfused LC kernel (the paper's rule, default), after every LC kernel
//     (reorder_rule ALWAYS, reading 6) or never.
//   * Baymax policy: identical with fusion disabled ("static scheduling").
//   * Idle GPU (paper silent): one ready BE head no longer than idle_cap.
//   * PTB slicing (params.slice_be, reading 13): a fused launch may carry only a slice of the BE
//     head kernel's remaining blocks, sized so that X_cd(n) = t_floor + t_block n (the kernel's
//     LR, §VI-C) puts the pair at its opportune ratio r* (Fig. 10); the head stays
//     the head until its last block is issued.  Reorder / idle launches issue the whole rest.
// In simulation mode every kernel takes its predicted time on a serial virtual stream (the
// discrete-event reference oracle/manager_ref.py follows the same rules); in GPU mode the
// manager launches on its stream and observes completion with CUDA events.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstring>
#include <deque>
#include <memory>
#include <array>
#include <map>
#include <set>
#include <string>
#include <tuple>
#include <vector>

#include "runtime.h"
#include "tacker.h"

namespace tkrt {
bool make_keys(const tacker_lc_desc *lc, const tacker_be_desc *be, int warp_split, std::string *lk, std::string *bk,
               std::string *pk);
bool blacklist_op(const std::string &be_key, int op);
}
using namespace tkrt;

namespace {

struct Query {
  int id;
  double arrival;
  // the query's kernels, shared by every query of a batch submission (a trace of 10^4 queries of
  // one service holds one copy)
  std::shared_ptr<const std::vector<tacker_lc_kernel>> kv;
  const std::vector<tacker_lc_kernel> &ks() const { return *kv; }
  size_t pos = 0;
  bool issued = false, direct = false, has_thr = false;
  double thr = 0;
  double done_at = -1;
  cudaEvent_t last_ev = nullptr;  // GPU mode: event after its last kernel
  double remaining() const {
    double s = 0;
    for (size_t i = pos; i < kv->size(); ++i) s += (*kv)[i].t_pred_ms;
    return s;
  }
};

struct App {
  std::vector<tacker_be_kernel> ks;
  size_t pos = 0;
  double ready_at = 0;
  int64_t completed = 0;
  int64_t done = 0;                // blocks of the head kernel already issued (PTB slices)
  const tacker_be_kernel &head() const { return ks[pos % ks.size()]; }
};

// Per-kernel LR of a PTB slice of n blocks (§VI-C)
double slice_ms(const tacker_be_kernel &b, int64_t n) { return b.t_floor_ms + b.t_block_ms * (double)n; }
// predicted standalone time of what is left of an app's head kernel
double rem_ms(const App &A) {
  const tacker_be_kernel &b = A.head();
  return A.done == 0 ? b.t_pred_ms : slice_ms(b, b.n_blocks - A.done);
}

}  // namespace

struct tacker_manager_s {
  int policy;
  tacker_manager_params prm;
  cudaStream_t stream;
  double now = 0;
  bool external_clock = false;
  std::chrono::steady_clock::time_point t0;
  cudaEvent_t base_ev = nullptr;
  std::vector<Query> queries;        // by id
  std::vector<int> pending;          // ids not yet admitted, arrival order
  size_t next_pending = 0;
  std::deque<int> active;
  std::vector<App> apps;
  tacker_manager_stats st{};
  std::vector<tacker_fused_t> owned;      // fused handles built by the manager
  // per (LC operands, BE kernel) pair: model-store key and fused handle, so a decision does no
  // string formatting / handle lookup (the manager loop is host-latency bound for 10 us kernels)
  struct PairEntry {
    bool keyed = false;
    std::string pk;
    tacker_fused_t f = nullptr;
  };
  std::map<std::tuple<const void *, const void *, const void *, int, size_t>, PairEntry> pairs;
  // reverse fusion (NEXT-2): keyed by the LC CUDA-core descriptor's bytes and (app, kernel)
  std::map<std::tuple<std::string, int, size_t>, PairEntry> rpairs;
  std::set<std::string> prepared_cd;   // LC CUDA-core descriptors already prepared
  // in-flight cap: launches issued vs launches known complete, observed through stream events
  // recorded every ev_every launches (and after launches whose completion is needed), so the
  // stream is not cut by an event after every ~10 us kernel (events block launch overlap)
  struct Mark {
    cudaEvent_t e;
    int64_t upto;
  };
  std::deque<Mark> marks;
  int64_t launched = 0, marked_upto = 0, completed_upto = 0, ev_every = 1;
  std::vector<cudaEvent_t> free_events;
  std::map<cudaEvent_t, int> refs;
  struct Observed {
    cudaEvent_t start, end;
    std::string pair_key;
    double x_tc, x_cd, t_pred;
  };
  std::deque<Observed> observed;   // fused launches awaiting their measured duration
  int64_t refits = 0;
  int idle_rr = 0;                 // idle launches: the next app in round-robin order
  size_t prepared = 0;                                   // queries visited by tacker_manager_prepare
  std::set<std::array<const void *, 3>> prepared_lc;     // LC operand triples already prepared
  double be_work_ms = 0;           // sum of standalone (predicted) times of issued BE kernels
  double pred_err_sum = 0;         // sum |predicted - measured| / measured over fused launches
  int64_t pred_err_n = 0;
  struct Timed {
    cudaEvent_t start, end;
    int cls;
  };
  std::deque<Timed> timed;         // sampled launches: device time per class
  double class_ms[4] = {0, 0, 0, 0};   // summed over the timed sample
  int64_t class_timed[4] = {0, 0, 0, 0};
  int64_t class_n[4] = {0, 0, 0, 0};   // every launch

  std::vector<tacker_trace_rec> trace;   // decision trace (tacker_manager_trace_enable)
  int64_t trace_cap = 0, trace_dropped = 0;
  double trace_tf[TACKER_TRACE_MAX_APPS];  // Tk_fuse per app evaluated by the current decision
  uint32_t trace_ready = 0;                // BE apps whose head was ready at the current decision

  double host_ns[3] = {0, 0, 0};   // poll, launch + event calls, whole step
  int64_t host_steps = 0;

  bool sim() const { return prm.simulate != 0; }
};

namespace {
// accumulates the wall time of a scope into a manager counter (GPU mode host profile)
struct HostTimer {
  double &acc;
  std::chrono::steady_clock::time_point t0;
  explicit HostTimer(double &a) : acc(a), t0(std::chrono::steady_clock::now()) {}
  ~HostTimer() { acc += std::chrono::duration<double, std::nano>(std::chrono::steady_clock::now() - t0).count(); }
};
}  // namespace

static bool sliceable(const tacker_manager_s *m, const tacker_be_kernel &b) {
  return m->policy == TACKER_POLICY_TACKER && m->prm.slice_be && !b.is_tc && b.n_blocks > 1 && b.t_block_ms > 0;
}

// Bookkeeping of n issued blocks of app A's head kernel (n < 0: the whole rest, which completes
// the kernel).  BE work is counted in standalone milliseconds: a slice of n of N blocks is
// n/N of the kernel's standalone time, so the slices of a kernel add up to the whole kernel.
static void issue_be(tacker_manager_s *m, App &A, int64_t n) {
  const tacker_be_kernel &b = A.head();
  if (n >= 0 && b.n_blocks > 1 && A.done + n < b.n_blocks) {
    m->be_work_ms += b.t_pred_ms * (double)n / (double)b.n_blocks;
    A.done += n;
    return;
  }
  m->be_work_ms += A.done == 0 ? b.t_pred_ms : b.t_pred_ms * (double)(b.n_blocks - A.done) / (double)b.n_blocks;
  A.done = 0;
  A.pos++;
  A.completed++;
  m->st.be_kernels_done++;
}

static double host_now(tacker_manager_s *m) {
  if (m->external_clock || m->sim()) return m->now;
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - m->t0).count();
}

static cudaEvent_t get_event(tacker_manager_s *m) {
  if (!m->free_events.empty()) {
    cudaEvent_t e = m->free_events.back();
    m->free_events.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}

// GPU completion time of an event on the manager clock (ms since creation)
static double event_time(tacker_manager_s *m, cudaEvent_t e) {
  float ms = 0;
  cudaEventElapsedTime(&ms, m->base_ev, e);
  return (double)ms;
}

// Events are reference counted (in flight / an app's pending kernel / a query's last kernel)
// and recycled when the last reference drops.
static cudaEvent_t ref(tacker_manager_s *m, cudaEvent_t e) {
  m->refs[e]++;
  return e;
}
static void unref(tacker_manager_s *m, cudaEvent_t e) {
  auto it = m->refs.find(e);
  if (it != m->refs.end() && --it->second == 0) {
    m->refs.erase(it);
    m->free_events.push_back(e);
  }
}

static void poll(tacker_manager_s *m) {
  if (m->sim()) return;
  HostTimer ht(m->host_ns[0]);
  while (!m->marks.empty() && cudaEventQuery(m->marks.front().e) == cudaSuccess) {
    m->completed_upto = m->marks.front().upto;
    unref(m, m->marks.front().e);
    m->marks.pop_front();
  }
  while (!m->timed.empty() && cudaEventQuery(m->timed.front().end) == cudaSuccess) {
    auto &t = m->timed.front();
    float ms = 0;
    cudaEventElapsedTime(&ms, t.start, t.end);
    m->class_ms[t.cls] += ms;
    m->class_timed[t.cls]++;
    unref(m, t.start);
    unref(m, t.end);
    m->timed.pop_front();
  }
  while (!m->observed.empty() && cudaEventQuery(m->observed.front().end) == cudaSuccess) {
    auto &o = m->observed.front();
    float ms = 0;
    cudaEventElapsedTime(&ms, o.start, o.end);
    int32_t refit = 0;
    if (ms > 0) {
      m->pred_err_sum += std::fabs(o.t_pred - ms) / ms;
      m->pred_err_n++;
    }
    if (ms > 0 && tacker_pair_observe(o.pair_key.c_str(), o.x_tc, o.x_cd, ms, &refit) == TACKER_OK && refit)
      m->refits++;
    unref(m, o.start);
    unref(m, o.end);
    m->observed.pop_front();
  }
  for (int id : m->active) {
    Query &q = m->queries[id];
    if (q.pos == q.ks().size() && q.done_at < 0 && q.last_ev && cudaEventQuery(q.last_ev) == cudaSuccess) {
      q.done_at = event_time(m, q.last_ev);
      unref(m, q.last_ev);
      q.last_ev = nullptr;
      m->st.lc_queries_done++;
    }
  }
}

// A BE application's head kernel is ready once its predecessor has been issued: in GPU mode the
// manager's single stream orders an app's kernels, so the next one may be fused or reordered
// right away (as on the simulator's serial virtual stream, where ready_at is the issue end);
// the in-flight cap bounds how far the host runs ahead.
static bool app_ready(tacker_manager_s *m, const App &a, double t) {
  if (m->sim()) return a.ready_at <= t;
  return true;
}

// pair-model key of (TC kernel k, BE CUDA-core kernel b); false for a blacklisted BE kernel (NEXT-1,
// never considered for fusion)
static bool pair_key(const tacker_lc_kernel &k, const tacker_be_kernel &b, std::string *pk) {
  std::string lk, bk;
  const int ws = b.warp_split ? b.warp_split : 16;
  if (!make_keys(&k.lc, &b.be, ws, &lk, &bk, pk)) return false;
  return !blacklist_op(bk, -1);
}
static bool pair_time(const tacker_lc_kernel &k, const tacker_be_kernel &b, double *tf) {
  std::string pk;
  if (!pair_key(k, b, &pk)) return false;
  return pair_predict(pk, k.t_pred_ms, b.t_pred_ms, tf);
}

static bool sliceable(const tacker_manager_s *m, const tacker_be_kernel &b);

// ---- reverse fusion (NEXT-2): LC CUDA-core kernel k (the fused kernel's CUDA-core part) with
// BE tensor-core kernel b (its tcgen05 part); the pair model takes X_tc = b, X_cd = k.
static int rev_ws(const tacker_lc_kernel &k) { return k.warp_split ? k.warp_split : 16; }
static bool rpair_key(const tacker_lc_kernel &k, const tacker_be_kernel &b, std::string *pk) {
  std::string lk, bk;
  return make_keys(&b.tc, &k.cd, rev_ws(k), &lk, &bk, pk);
}
static std::string cd_bytes(const tacker_be_desc &d) {
  return std::string(reinterpret_cast<const char *>(&d), sizeof d);
}
static tacker_manager_s::PairEntry &rpair_entry(tacker_manager_s *m, const tacker_lc_kernel &k, int app, size_t kidx) {
  const tacker_be_kernel &b = m->apps[app].ks[kidx];
  auto &e = m->rpairs[std::make_tuple(cd_bytes(k.cd), app, kidx)];
  if (!e.keyed) {
    e.keyed = true;
    if (!rpair_key(k, b, &e.pk)) e.pk.clear();
  }
  return e;
}
static tacker_status rfused_handle(tacker_manager_s *m, const tacker_lc_kernel &k, int app, size_t kidx,
                                   tacker_fused_t *out) {
  auto &pe = rpair_entry(m, k, app, kidx);
  if (pe.f) {
    *out = pe.f;
    return TACKER_OK;
  }
  const tacker_be_kernel &b = m->apps[app].ks[kidx];
  tacker_status s = tacker_fuse(&b.tc, &k.cd, rev_ws(k), tacker_ratio{0, 0}, out);
  if (s == TACKER_OK) {
    pe.f = *out;
    m->owned.push_back(*out);
  }
  return s;
}

// keyed by the LC operands and (app, kernel index): stable across reallocation of the app list
static tacker_manager_s::PairEntry &pair_entry(tacker_manager_s *m, const tacker_lc_kernel &k, int app, size_t kidx) {
  const tacker_be_kernel &b = m->apps[app].ks[kidx];
  auto &e = m->pairs[std::make_tuple(k.lc.A, k.lc.B, k.lc.D, app, kidx)];
  if (!e.keyed) {
    e.keyed = true;
    if (!pair_key(k, b, &e.pk)) e.pk.clear();
  }
  return e;
}

// Blocks of the head kernel of A that a fused launch with TC kernel k should carry: the
// smallest n with X_cd(n) >= r* X_tc (clamped to the remaining blocks), or -1 = the whole rest
// (slicing off, kernel not sliceable, or no opportune ratio for the pair).
static int64_t slice_blocks(const tacker_manager_s *m, const App &A, const std::string &pk, double ttc) {
  const tacker_be_kernel &b = A.head();
  if (!sliceable(m, b)) return -1;
  double rt = m->prm.slice_ratio;
  if (!(rt > 0) && !pair_opportune(pk, &rt)) return -1;
  const int64_t R = b.n_blocks - A.done;
  int64_t n = (int64_t)std::ceil((rt * ttc - b.t_floor_ms) / b.t_block_ms - 1e-9);
  n = std::max<int64_t>(1, std::min<int64_t>(n, R));
  return n < R ? n : -1;
}

// ---------------------------------------------------------------- GPU launches
static tacker_status launch_lc(tacker_manager_s *m, const tacker_lc_kernel &k) {
  HostTimer ht(m->host_ns[1]);
  if (k.is_tc) return tacker_launch_original(&k.lc, nullptr, reinterpret_cast<tacker_stream_t>(m->stream));
  return tacker_launch_original(nullptr, &k.cd, reinterpret_cast<tacker_stream_t>(m->stream));
}

// the rest of app A's head kernel (the whole kernel when no slice of it was issued yet)
static tacker_status launch_be(tacker_manager_s *m, const App &A) {
  HostTimer ht(m->host_ns[1]);
  const tacker_be_kernel &b = A.head();
  if (b.is_tc) return tacker_launch_original(&b.tc, nullptr, reinterpret_cast<tacker_stream_t>(m->stream));
  if (A.done == 0) return tacker_launch_original(nullptr, &b.be, reinterpret_cast<tacker_stream_t>(m->stream));
  tacker_be_desc d = b.be;
  d.block_offset = b.be.block_offset + (int32_t)A.done;
  d.orig_blocks = (int32_t)(b.n_blocks - A.done);
  return tacker_launch_original(nullptr, &d, reinterpret_cast<tacker_stream_t>(m->stream));
}

// Fused handle of (LC kernel, BE kernel) from the manager's cache, built on first use.
static tacker_status fused_handle(tacker_manager_s *m, const tacker_lc_kernel &k, int app, size_t kidx,
                                  tacker_fused_t *out) {
  auto &pe = pair_entry(m, k, app, kidx);
  if (pe.f) {
    *out = pe.f;
    return TACKER_OK;
  }
  const tacker_be_kernel &b = m->apps[app].ks[kidx];
  const int ws = b.warp_split ? b.warp_split : 16;
  tacker_status s = tacker_fuse(&k.lc, &b.be, ws, tacker_ratio{0, 0}, out);
  if (s == TACKER_OK) {
    pe.f = *out;
    m->owned.push_back(*out);
  }
  return s;
}

// TC kernel k fused with n blocks of app A's head kernel (n < 0: the whole rest)
static tacker_status launch_fused(tacker_manager_s *m, const tacker_lc_kernel &k, int app, int64_t n) {
  HostTimer ht(m->host_ns[1]);
  const App &A = m->apps[app];
  const tacker_be_kernel &b = A.head();
  tacker_fused_t f = nullptr;
  tacker_status s = fused_handle(m, k, app, A.pos % A.ks.size(), &f);
  if (s) return s;
  if (A.done == 0 && n < 0) return tacker_launch_fused(f, reinterpret_cast<tacker_stream_t>(m->stream));
  return tacker_launch_fused_slice(f, (int64_t)b.be.block_offset + A.done, n < 0 ? b.n_blocks - A.done : n,
                                   reinterpret_cast<tacker_stream_t>(m->stream));
}

// After a launch: count it, and record a stream event when one is needed at this point (force:
// the launch is timed, observed or ends a query) or ev_every launches have gone unmarked.
static cudaEvent_t mark(tacker_manager_s *m, bool force) {
  m->launched++;
  if (!force && m->launched - m->marked_upto < m->ev_every) return nullptr;
  HostTimer ht(m->host_ns[1]);
  cudaEvent_t e = get_event(m);
  cudaEventRecord(e, m->stream);
  m->marks.push_back(tacker_manager_s::Mark{ref(m, e), m->launched});
  m->marked_upto = m->launched;
  return e;
}
// Per-class device time (stats.class_ms): every launch is counted, one launch in kTimeEvery of
// each class is bracketed by events (a start event costs a host API call per launch, and the
// manager loop of a 53-kernel query is host-latency sensitive); the class total is the sampled
// mean x the count.  Fused launches are always timed: the online refit needs each one.
static constexpr int64_t kTimeEvery = 16;
// start event of a launch (the stream reaches it when the previous kernel has finished), or
// nullptr when this launch is not in the timed sample
static cudaEvent_t begin(tacker_manager_s *m, int cls, bool always = false) {
  if (!always && m->class_n[cls]++ % kTimeEvery != 0) return nullptr;
  if (always) m->class_n[cls]++;
  HostTimer ht(m->host_ns[1]);
  cudaEvent_t e = get_event(m);
  cudaEventRecord(e, m->stream);
  return e;
}
static void track(tacker_manager_s *m, cudaEvent_t start, cudaEvent_t end, int cls) {
  if (start) m->timed.push_back(tacker_manager_s::Timed{ref(m, start), ref(m, end), cls});
}

extern "C" {

tacker_status tacker_manager_create(int32_t policy, const tacker_manager_params *params, tacker_stream_t stream,
                                    tacker_manager_t *out) {
  if (!out || !params) return set_error("null argument"), TACKER_EINVAL;
  if (policy != TACKER_POLICY_TACKER && policy != TACKER_POLICY_BAYMAX) return set_error("bad policy"), TACKER_EINVAL;
  auto *m = new (std::nothrow) tacker_manager_s();
  if (!m) return TACKER_ENOMEM;
  m->policy = policy;
  m->prm = *params;
  if (m->prm.max_inflight < 1) m->prm.max_inflight = 1;
  m->ev_every = std::max(1, m->prm.max_inflight / 2);
  m->stream = reinterpret_cast<cudaStream_t>(stream);
  m->t0 = std::chrono::steady_clock::now();
  if (!m->sim()) {
    cudaError_t e = cudaEventCreate(&m->base_ev);
    if (e == cudaSuccess) e = cudaEventRecord(m->base_ev, m->stream);
    if (e != cudaSuccess) {
      delete m;
      return cuda_fail("manager events", e);
    }
  }
  *out = m;
  return TACKER_OK;
}

tacker_status tacker_manager_destroy(tacker_manager_t m) {
  if (!m) return TACKER_OK;
  if (!m->sim()) {
    cudaStreamSynchronize(m->stream);
    for (auto f : m->owned) tacker_fused_destroy(f);
    for (auto &mk : m->marks) cudaEventDestroy(mk.e);
    for (auto e : m->free_events) cudaEventDestroy(e);
    if (m->base_ev) cudaEventDestroy(m->base_ev);
  }
  delete m;
  return TACKER_OK;
}

static tacker_status submit_query(tacker_manager_t m, Query &&Q, int32_t *id);

tacker_status tacker_manager_submit_lc(tacker_manager_t m, const tacker_lc_query *q, double arrival_ms, int32_t *id) {
  if (!m || !q || q->n_kernels <= 0 || !q->kernels) return set_error("bad query"), TACKER_EINVAL;
  Query Q;
  Q.id = (int)m->queries.size();
  Q.arrival = arrival_ms;
  Q.kv = std::make_shared<const std::vector<tacker_lc_kernel>>(q->kernels, q->kernels + q->n_kernels);
  return submit_query(m, std::move(Q), id);
}

static tacker_status submit_query(tacker_manager_t m, Query &&Q, int32_t *id) {
  const double arrival_ms = Q.arrival;
  m->queries.push_back(std::move(Q));
  Query &Qr = m->queries.back();
  // keep pending sorted by arrival (stable): scan from the back, so queries submitted in arrival
  // order append in O(1)
  size_t pos = m->pending.size();
  while (pos > m->next_pending && m->queries[m->pending[pos - 1]].arrival > arrival_ms) --pos;
  m->pending.insert(m->pending.begin() + (long)pos, Qr.id);
  if (id) *id = Qr.id;
  return TACKER_OK;
}

tacker_status tacker_manager_submit_lc_batch(tacker_manager_t m, const tacker_lc_query *q, const double *arrivals_ms,
                                             int64_t n, int32_t *first_id) {
  if (!m || !q || n < 0 || (n > 0 && !arrivals_ms)) return set_error("bad query batch"), TACKER_EINVAL;
  if (q->n_kernels <= 0 || !q->kernels) return set_error("bad query"), TACKER_EINVAL;
  if (first_id) *first_id = (int32_t)m->queries.size();
  m->queries.reserve(m->queries.size() + (size_t)n);
  auto kv = std::make_shared<const std::vector<tacker_lc_kernel>>(q->kernels, q->kernels + q->n_kernels);
  for (int64_t i = 0; i < n; ++i) {
    Query Q;
    Q.id = (int)m->queries.size();
    Q.arrival = arrivals_ms[i];
    Q.kv = kv;
    if (tacker_status s = submit_query(m, std::move(Q), nullptr)) return s;
  }
  return TACKER_OK;
}

tacker_status tacker_manager_submit_be(tacker_manager_t m, const tacker_be_app *app, int32_t *id) {
  if (!m || !app || app->n_kernels <= 0 || !app->kernels) return set_error("bad BE app"), TACKER_EINVAL;
  if (m->apps.size() >= TACKER_MAX_APPS) return set_error("too many BE apps"), TACKER_ERESOURCE;
  for (int32_t i = 0; i < app->n_kernels; ++i) {
    const tacker_be_kernel &b = app->kernels[i];
    if (b.is_tc && (b.is_cd || b.tc.kind == TACKER_LC_NONE))
      return set_error("BE kernel %d: is_tc needs is_cd == 0 and a tensor-core descriptor", i), TACKER_EINVAL;
  }
  App A;
  A.ks.assign(app->kernels, app->kernels + app->n_kernels);
  A.ready_at = m->now;
  m->apps.push_back(A);
  if (id) *id = (int)m->apps.size() - 1;
  return TACKER_OK;
}

tacker_status tacker_manager_set_clock(tacker_manager_t m, double now_ms) {
  if (!m) return set_error("null manager"), TACKER_EINVAL;
  m->now = now_ms;
  m->external_clock = true;
  return TACKER_OK;
}

static tacker_status step_impl(tacker_manager_t m, double qos, double *headroom, tacker_decision *out) {
  HostTimer ht(m->host_ns[2]);
  for (double &x : m->trace_tf) x = NAN;
  m->host_steps++;
  memset(out, 0, sizeof *out);
  out->action = TACKER_DEC_NOTHING;
  out->query = out->lc_index = out->fused_app = -1;
  poll(m);
  const double t = host_now(m);
  m->now = t;
  out->t_start_ms = out->t_end_ms = t;
  while (m->next_pending < m->pending.size() && m->queries[m->pending[m->next_pending]].arrival <= t)
    m->active.push_back(m->pending[m->next_pending++]);
  // retire finished queries
  while (!m->active.empty()) {
    Query &q = m->queries[m->active.front()];
    if (q.pos < q.ks().size()) break;
    if (m->sim() || q.done_at >= 0) m->active.pop_front();
    else break;
  }
  if (!m->sim() && m->launched - m->completed_upto >= m->prm.max_inflight) return TACKER_OK;   // stream is busy

  // oldest query with kernels still to issue
  int qid = -1;
  for (int id : m->active)
    if (m->queries[id].pos < m->queries[id].ks().size()) {
      qid = id;
      break;
    }
  std::vector<int> heads;
  m->trace_ready = 0;
  for (size_t a = 0; a < m->apps.size(); ++a)
    if (app_ready(m, m->apps[a], t)) {
      heads.push_back((int)a);
      if (a < TACKER_TRACE_MAX_APPS) m->trace_ready |= 1u << a;
    }

  if (qid < 0) {
    // idle GPU (or only tails of earlier queries still running): one bounded BE kernel, the apps
    // taken round robin from the one after the last idle launch (no app starves behind another)
    std::rotate(heads.begin(), std::lower_bound(heads.begin(), heads.end(), m->idle_rr), heads.end());
    for (int a : heads) {
      const double tt = rem_ms(m->apps[a]);
      if (m->prm.idle_cap_ms > 0 && tt > m->prm.idle_cap_ms) continue;
      if (!m->active.empty()) break;   // do not delay a running query's completion
      out->action = TACKER_DEC_IDLE_BE;
      out->n_reorder = 1;
      out->reorder_apps[0] = a;
      m->idle_rr = a + 1;
      App &A = m->apps[a];
      if (m->sim()) {
        m->now += tt;
        A.ready_at = m->now;
      } else {
        cudaEvent_t e0 = begin(m, TACKER_CLASS_BE);
        tacker_status s = launch_be(m, A);
        if (s) return s;
        track(m, e0, mark(m, e0 != nullptr), TACKER_CLASS_BE);
      }
      issue_be(m, A, -1);
      m->st.idle_be++;
      out->t_end_ms = m->now;
      return TACKER_OK;
    }
    if (m->sim()) {   // advance the virtual clock to the next event
      double nxt = INFINITY;
      if (m->next_pending < m->pending.size()) nxt = m->queries[m->pending[m->next_pending]].arrival;
      for (auto &A : m->apps)
        if (A.ready_at > t) nxt = std::min(nxt, A.ready_at);
      if (std::isfinite(nxt)) m->now = nxt;
      out->t_end_ms = m->now;
    }
    return TACKER_OK;
  }

  Query &q = m->queries[qid];
  const bool newest = (qid == m->active.back());
  const bool older_ok = m->prm.fuse_older != 0;
  if (!q.issued) {
    q.issued = true;
    if (newest || older_ok) {
      double earlier = 0;   // remaining predicted time of the active queries ahead of q
      for (int id : m->active) {
        if (id == qid) break;
        earlier += m->queries[id].remaining();
      }
      q.thr = qos - (t - q.arrival) - q.remaining() - earlier;   // Eq. 9
      q.has_thr = true;
      // "Thr close to 0": reading TACKER_DIRECT_MIN_BE = not even the shortest
      // ready BE head fits the headroom
      double bound = m->prm.direct_eps_ms;
      if (m->prm.direct_rule == TACKER_DIRECT_MIN_BE && !heads.empty()) {
        double mn = INFINITY;
        for (int a : heads) mn = std::min(mn, rem_ms(m->apps[a]));
        bound = std::max(bound, mn);
      }
      q.direct = q.thr <= bound;
    }
  }
  const bool allow = (newest || older_ok) && q.has_thr && !q.direct;
  double thr = q.has_thr ? q.thr : 0.0;
  if (allow && headroom && !std::isnan(*headroom)) thr = *headroom;
  // reading 18: an older query spends at most the smallest headroom of itself and of every later
  // active query (Eq. 9 of each at time t)
  const double thr_in = thr;
  if (allow && !newest) {
    double ahead = 0;
    bool after = false;
    for (int id : m->active) {
      const Query &o = m->queries[id];
      ahead += o.remaining();
      if (after) thr = std::min(thr, qos - (t - o.arrival) - ahead);
      if (id == qid) after = true;
    }
    thr -= m->prm.older_margin_ms;
  }
  const double thr_eff = thr;
  const tacker_lc_kernel &k = q.ks()[q.pos];
  const double ttc = k.t_pred_ms;

  int fused = -1;
  int64_t best_n = -1;
  double best_gain = 0, best_tf = 0, best_tcd = 0;
  if (allow && m->policy == TACKER_POLICY_TACKER && k.is_tc) {
    for (int a : heads) {
      const App &A = m->apps[a];
      const tacker_be_kernel &b = A.head();
      if (!b.is_cd) continue;
      const std::string &pk = pair_entry(m, k, a, A.pos % A.ks.size()).pk;
      if (pk.empty()) continue;
      const int64_t n = slice_blocks(m, A, pk, ttc);
      const double tcd = n < 0 ? rem_ms(A) : slice_ms(b, n);
      double tf;
      if (!pair_predict(pk, ttc, tcd, &tf)) continue;
      if (a < TACKER_TRACE_MAX_APPS) m->trace_tf[a] = tf;
      if (ttc + tcd > tf && tf - ttc < thr) {   // Eq. 8
        const double gain = tcd - (tf - ttc);
        if (fused < 0 || gain > best_gain) {
          fused = a;
          best_gain = gain;
          best_tf = tf;
          best_tcd = tcd;
          best_n = n;
        }
      }
    }
  }
  // NEXT-2 reverse fusion: the LC kernel is a CUDA-core kernel and a ready BE head a tensor-core
  // kernel; Eq. 8 unchanged with t_lc = ttc, t_be = the BE kernel's time (the model's X_tc)
  bool reverse = false;
  if (allow && m->policy == TACKER_POLICY_TACKER && !k.is_tc && !m->prm.no_reverse_fusion) {
    for (int a : heads) {
      const App &A = m->apps[a];
      const tacker_be_kernel &b = A.head();
      if (!b.is_tc) continue;
      const std::string &pk = rpair_entry(m, k, a, A.pos % A.ks.size()).pk;
      if (pk.empty()) continue;
      const double tbe = b.t_pred_ms;
      double tf;
      if (!pair_predict(pk, tbe, ttc, &tf)) continue;
      if (a < TACKER_TRACE_MAX_APPS) m->trace_tf[a] = tf;
      if (ttc + tbe > tf && tf - ttc < thr) {   // Eq. 8
        const double gain = tbe - (tf - ttc);
        if (fused < 0 || gain > best_gain) {
          fused = a;
          best_gain = gain;
          best_tf = tf;
          best_tcd = tbe;
          best_n = -1;
          reverse = true;
        }
      }
    }
  }
  std::vector<int> reorder;
  if (fused >= 0) thr -= best_tf - ttc;
  // Reorder: the ready heads with Ttmp < Thr after an LC kernel that was not fused
  // (the paper's rule, TACKER_REORDER_UNFUSED); TACKER_REORDER_ALWAYS (reading 6) also after a
  // fused launch ("both adaptive kernel fusion and kernel reorder").
  const int32_t rr = m->prm.reorder_rule;
  if (allow && rr != TACKER_REORDER_NEVER && !(rr == TACKER_REORDER_UNFUSED && fused >= 0)) {
    for (int a : heads) {
      if (a == fused) continue;
      const double tt = rem_ms(m->apps[a]);
      if (tt < thr) {
        reorder.push_back(a);
        thr -= tt;
      }
    }
  }
  if (allow) q.thr = thr_in - (thr_eff - thr);   // what this decision spent

  // execute
  out->query = qid;
  out->lc_index = (int)q.pos;
  out->fused_app = fused;
  out->fused_blocks = fused >= 0 ? best_n : 0;
  out->gain_ms = fused >= 0 ? best_gain : 0;
  out->thr_ms = thr;
  out->reverse = reverse ? 1 : 0;
  if (headroom) *headroom = thr;
  if (fused >= 0) {
    App &A = m->apps[fused];
    if (m->sim()) {
      m->now += best_tf;
      A.ready_at = m->now;
    } else {
      cudaEvent_t e0 = begin(m, TACKER_CLASS_FUSED, true);
      tacker_status s;
      if (reverse) {
        HostTimer ht(m->host_ns[1]);
        tacker_fused_t f = nullptr;
        s = rfused_handle(m, k, fused, A.pos % A.ks.size(), &f);
        if (s == TACKER_OK) s = tacker_launch_fused(f, reinterpret_cast<tacker_stream_t>(m->stream));
      } else {
        s = launch_fused(m, k, fused, best_n);
      }
      if (s) return s;
      cudaEvent_t e = mark(m, true);
      track(m, e0, e, TACKER_CLASS_FUSED);
      if (q.pos + 1 == q.ks().size()) q.last_ev = ref(m, e);
      // online model update from the measured co-run: (X_tc, X_cd) of the pair
      if (reverse) {
        const std::string &pk = rpair_entry(m, k, fused, A.pos % A.ks.size()).pk;
        m->observed.push_back(tacker_manager_s::Observed{ref(m, e0), ref(m, e), pk, best_tcd, ttc, best_tf});
      } else {
        const std::string &pk = pair_entry(m, k, fused, A.pos % A.ks.size()).pk;
        m->observed.push_back(tacker_manager_s::Observed{ref(m, e0), ref(m, e), pk, ttc, best_tcd, best_tf});
      }
    }
    issue_be(m, A, best_n);
    m->st.fused_launches++;
    if (reverse) m->st.reverse_fused++;
    out->action = TACKER_DEC_FUSED;
  } else {
    if (m->sim()) {
      m->now += ttc;
    } else {
      cudaEvent_t e0 = begin(m, k.is_tc ? TACKER_CLASS_LC_TC : TACKER_CLASS_LC_CD);
      tacker_status s = launch_lc(m, k);
      if (s) return s;
      const bool last = q.pos + 1 == q.ks().size();
      cudaEvent_t e = mark(m, e0 != nullptr || last);
      track(m, e0, e, k.is_tc ? TACKER_CLASS_LC_TC : TACKER_CLASS_LC_CD);
      if (last) q.last_ev = ref(m, e);
    }
    m->st.original_lc++;
    out->action = reorder.empty() ? TACKER_DEC_ORIGINAL_LC : TACKER_DEC_REORDER_BE;
  }
  q.pos++;
  if (m->sim() && q.pos == q.ks().size()) {
    q.done_at = m->now;
    m->st.lc_queries_done++;
  }
  for (int a : reorder) {
    App &A = m->apps[a];
    if (m->sim()) {
      m->now += rem_ms(A);
      A.ready_at = m->now;
    } else {
      cudaEvent_t e0 = begin(m, TACKER_CLASS_BE);
      tacker_status s = launch_be(m, A);
      if (s) return s;
      track(m, e0, mark(m, e0 != nullptr), TACKER_CLASS_BE);
    }
    issue_be(m, A, -1);
    m->st.reordered_be++;
    if (out->n_reorder < TACKER_MAX_REORDER) out->reorder_apps[out->n_reorder++] = a;
  }
  out->t_end_ms = m->now;
  return TACKER_OK;
}

tacker_status tacker_manager_step(tacker_manager_t m, double qos, double *headroom, tacker_decision *out) {
  if (!m || !out) return set_error("null argument"), TACKER_EINVAL;
  tacker_status s = step_impl(m, qos, headroom, out);
  if (s != TACKER_OK || m->trace_cap <= 0 || out->action == TACKER_DEC_NOTHING) return s;
  if ((int64_t)m->trace.size() >= m->trace_cap) {
    m->trace_dropped++;
    return s;
  }
  tacker_trace_rec r;
  memset(&r, 0, sizeof r);
  r.t_ms = out->t_start_ms;
  r.n_active = (int32_t)m->active.size();
  r.first_active = m->active.empty() ? -1 : m->active.front();
  r.active_contiguous = 1;
  for (size_t i = 0; i < m->active.size(); ++i)
    if (m->active[i] != r.first_active + (int32_t)i) r.active_contiguous = 0;
  r.direct = out->query >= 0 && m->queries[out->query].direct ? 1 : 0;
  r.n_apps = (int32_t)std::min<size_t>(m->apps.size(), TACKER_TRACE_MAX_APPS);
  r.ready_mask = m->trace_ready;
  for (int a = 0; a < TACKER_TRACE_MAX_APPS; ++a) r.tk_fuse_ms[a] = m->trace_tf[a];
  r.d = *out;
  m->trace.push_back(r);
  return s;
}

tacker_status tacker_manager_trace_enable(tacker_manager_t m, int64_t capacity) {
  if (!m || capacity < 0) return set_error("bad trace capacity"), TACKER_EINVAL;
  m->trace.clear();
  m->trace.reserve((size_t)capacity);
  m->trace_cap = capacity;
  m->trace_dropped = 0;
  return TACKER_OK;
}

tacker_status tacker_manager_trace_count(tacker_manager_t m, int64_t *stored, int64_t *dropped) {
  if (!m || !stored || !dropped) return set_error("null argument"), TACKER_EINVAL;
  *stored = (int64_t)m->trace.size();
  *dropped = m->trace_dropped;
  return TACKER_OK;
}

tacker_status tacker_manager_trace_get(tacker_manager_t m, int64_t i, tacker_trace_rec *out) {
  if (!m || !out || i < 0 || i >= (int64_t)m->trace.size()) return set_error("bad trace index"), TACKER_EINVAL;
  *out = m->trace[(size_t)i];
  return TACKER_OK;
}

// Fused handles of every (TC kernel in ks, CUDA-core kernel of a BE app) pair the predictor has
// a model for: the only pairs Eq. 8 can admit.  Queries of one service share their kernels, so
// only LC operand triples not seen before are visited.
static tacker_status prepare_kernels(tacker_manager_s *m, const tacker_lc_kernel *ks, size_t n) {
  for (size_t i = 0; i < n; ++i) {
    const tacker_lc_kernel &k = ks[i];
    if (!k.is_tc) {
      // reverse pairs (NEXT-2): this CUDA-core kernel with every BE tensor-core kernel
      if (m->prm.no_reverse_fusion || !m->prepared_cd.insert(cd_bytes(k.cd)).second) continue;
      for (size_t a = 0; a < m->apps.size(); ++a)
        for (size_t j = 0; j < m->apps[a].ks.size(); ++j) {
          const tacker_be_kernel &b = m->apps[a].ks[j];
          std::string pk;
          double tf;
          if (!b.is_tc || !rpair_key(k, b, &pk) || !pair_predict(pk, b.t_pred_ms, k.t_pred_ms, &tf)) continue;
          tacker_fused_t f = nullptr;
          tacker_status s = rfused_handle(m, k, (int)a, j, &f);
          if (s != TACKER_OK && s != TACKER_ERESOURCE && s != TACKER_EUNSUPPORTED) return s;
        }
      continue;
    }
    if (!m->prepared_lc.insert({k.lc.A, k.lc.B, k.lc.D}).second) continue;
    for (size_t a = 0; a < m->apps.size(); ++a)
      for (size_t j = 0; j < m->apps[a].ks.size(); ++j) {
        const tacker_be_kernel &b = m->apps[a].ks[j];
        double tf;
        if (!b.is_cd || !pair_time(k, b, &tf)) continue;
        tacker_fused_t f = nullptr;
        tacker_status s = fused_handle(m, k, (int)a, j, &f);
        if (s != TACKER_OK && s != TACKER_ERESOURCE && s != TACKER_EUNSUPPORTED) return s;
      }
  }
  return TACKER_OK;
}

tacker_status tacker_manager_prepare(tacker_manager_t m, const tacker_lc_query *q) {
  if (!m) return set_error("null manager"), TACKER_EINVAL;
  if (m->sim() || m->policy != TACKER_POLICY_TACKER) return TACKER_OK;
  if (q) {
    if (q->n_kernels < 0 || (q->n_kernels > 0 && !q->kernels)) return set_error("bad query"), TACKER_EINVAL;
    return prepare_kernels(m, q->kernels, (size_t)q->n_kernels);
  }
  const std::vector<tacker_lc_kernel> *last = nullptr;
  for (; m->prepared < m->queries.size(); ++m->prepared) {
    const Query &Q = m->queries[m->prepared];
    if (Q.kv.get() == last) continue;   // same kernels as the previous query (a batch submission)
    last = Q.kv.get();
    if (tacker_status s = prepare_kernels(m, Q.ks().data(), Q.ks().size())) return s;
  }
  return TACKER_OK;
}

tacker_status tacker_manager_run(tacker_manager_t m, double qos, double t_end_ms, int64_t max_decisions) {
  if (!m) return set_error("null manager"), TACKER_EINVAL;
  if (tacker_status s = tacker_manager_prepare(m, nullptr)) return s;
  int64_t n = 0;
  tacker_decision d;
  for (;;) {
    double thr = NAN;
    tacker_status s = tacker_manager_step(m, qos, &thr, &d);
    if (s) return s;
    if (d.action != TACKER_DEC_NOTHING && max_decisions > 0 && ++n >= max_decisions) break;
    poll(m);
    const bool all_done = m->st.lc_queries_done == (int64_t)m->queries.size();
    if (all_done && m->now >= t_end_ms) break;
    if (m->sim() && all_done && m->next_pending >= m->pending.size()) break;
  }
  if (!m->sim()) {
    cudaError_t e = cudaStreamSynchronize(m->stream);
    if (e != cudaSuccess) return cuda_fail("manager run sync", e);
    poll(m);
  }
  return TACKER_OK;
}

tacker_status tacker_manager_run_until(tacker_manager_t m, double qos, double t_until_ms) {
  if (!m) return set_error("null manager"), TACKER_EINVAL;
  if (tacker_status s = tacker_manager_prepare(m, nullptr)) return s;
  tacker_decision d;
  for (;;) {
    if ((m->sim() ? m->now : host_now(m)) >= t_until_ms) break;
    double thr = NAN;
    if (tacker_status s = tacker_manager_step(m, qos, &thr, &d)) return s;
    if (m->sim() && d.action == TACKER_DEC_NOTHING && m->next_pending >= m->pending.size() &&
        m->st.lc_queries_done == (int64_t)m->queries.size())
      break;   // nothing left to simulate
    poll(m);
  }
  return TACKER_OK;
}

tacker_status tacker_manager_stats_get(tacker_manager_t m, tacker_manager_stats *o) {
  if (!m || !o) return set_error("null argument"), TACKER_EINVAL;
  poll(m);
  *o = m->st;
  o->now_ms = m->sim() ? m->now : host_now(m);
  o->model_refits = m->refits;
  o->pred_err_sum = m->pred_err_sum;
  o->be_work_ms = m->be_work_ms;
  o->pred_err_n = m->pred_err_n;
  o->host_poll_ms = m->host_ns[0] * 1e-6;
  o->host_launch_ms = m->host_ns[1] * 1e-6;
  o->host_decide_ms = m->host_ns[2] * 1e-6;   // whole step (includes its poll and launches)
  o->host_steps = m->host_steps;
  for (int c = 0; c < 4; ++c) {
    o->class_ms[c] = m->class_timed[c] ? m->class_ms[c] / (double)m->class_timed[c] * (double)m->class_n[c] : 0.0;
    o->class_launches[c] = m->class_n[c];
  }
  return TACKER_OK;
}

tacker_status tacker_manager_query_latency(tacker_manager_t m, int32_t id, double *lat) {
  if (!m || !lat || id < 0 || id >= (int)m->queries.size()) return set_error("bad query id"), TACKER_EINVAL;
  poll(m);
  const Query &q = m->queries[id];
  *lat = q.done_at >= 0 ? q.done_at - q.arrival : -1.0;
  return TACKER_OK;
}

}  // extern "C"
