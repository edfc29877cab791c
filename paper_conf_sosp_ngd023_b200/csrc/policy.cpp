// See policy.h.  Rule-for-rule the state machine of SURVEY.md §8(c) C2.
#include "policy.h"

#include <algorithm>
#include <cassert>
#include <climits>
#include <stdexcept>

namespace paella {

Policy::Policy(const Cfg& c) : cfg_(c) {
  launches_.resize(kLaunchSlots);
  free_.assign((c.streams + 63) / 64, 0);
  for (uint32_t s = 0; s < c.streams; ++s) free_[s / 64] |= 1ull << (s % 64);
  Dt_.assign(c.num_clients, 0);
  unfinished_.assign(c.num_clients, 0);
  per_client_.resize(c.num_clients);
  models_.resize(kMaxModels);   // never reallocated: models are added while dispatching
  vs_kernels_.resize(kMaxModels);
  model_total_.assign(kMaxModels, 0);
  tb_sum_.resize(kMaxModels);
  tb_cnt_.resize(kMaxModels);
  live_by_model_.resize(kMaxModels);
}

void Policy::add_model(uint32_t mid, const std::vector<PolicyLayer>& layers) {
  if (mid >= kMaxModels) throw std::runtime_error("too many models");
  models_[mid] = layers;
  uint32_t nv = 1;
  for (const auto& l : layers) {
    if (l.vs >= MAX_VS) throw std::runtime_error("too many virtual streams");
    nv = std::max(nv, l.vs + 1);
  }
  vs_kernels_[mid].assign(nv, {});
  for (uint32_t k = 0; k < layers.size(); ++k) vs_kernels_[mid][layers[k].vs].push_back(k);
  int64_t t = 0;
  for (const auto& l : layers) t += l.tbar;
  model_total_[mid] = t;
  tb_sum_[mid].assign(layers.size(), 0);
  tb_cnt_[mid].assign(layers.size(), kProfileRuns);
  for (size_t l = 0; l < layers.size(); ++l) tb_sum_[mid][l] = layers[l].tbar * kProfileRuns;
  if (!layers.empty()) {
    auto it = std::lower_bound(totals_.begin(), totals_.end(), t);
    if (it == totals_.end() || *it != t) totals_.insert(it, t);
  }
}

// Stream-priority classes (B200 adaptation, reading B200-Q2; identical to
// oracle/sim.py Policy.job_class): the number of registered models whose whole-job
// T-bar sum is strictly below R_j, clamped to K-1; a deficit-override pick -> 0.
uint32_t Policy::job_class(const PolicyJob& j) const {
  const uint32_t K = cfg_.prio_classes;
  if (K <= 1 || over_) return 0;
  uint32_t c = (uint32_t)(std::lower_bound(totals_.begin(), totals_.end(), j.R) - totals_.begin());
  return c < K - 1 ? c : K - 1;
}

int Policy::lowest_free_in_class(uint32_t c) const {
  for (uint32_t s = 0; s < cfg_.streams; ++s)
    if ((free_[s / 64] >> (s % 64) & 1) && stream_class(s, cfg_.prio_classes, cfg_.streams) == c) return (int)s;
  return -1;
}

// The job's lowest-index active kernel that may be dispatched now, or -1 (identical to
// oracle Policy.head): the next kernel of a virtual stream whose cross-stream
// dependencies have completed and whose stream is idle -- or, with launch-ahead D > 0,
// whose oldest in-flight kernel is fully placed (running) with at most D in flight
// (la_unplaced: at most D in flight, placement not required).
int64_t Policy::head(const PolicyJob& j) const {
  if (!j.live || j.cursor >= models_[j.model].size()) return -1;
  const auto& ml = models_[j.model];
  const auto& vk = vs_kernels_[j.model];
  int64_t best = -1;
  for (uint32_t v = 0; v < j.nvs; ++v) {
    if (j.vs_next[v] >= vk[v].size()) continue;
    const uint32_t k = vk[v][j.vs_next[v]];
    bool deps_done = true;
    for (uint32_t d : ml[k].cross) deps_done &= j.state[d] == 2;
    if (!deps_done) continue;
    const uint32_t infl = j.vs_infl[v];
    if (infl > 0) {
      if (cfg_.lookahead == 0 || infl > cfg_.lookahead) continue;
      if (cfg_.la_unplaced) {
        if (best < 0 || (int64_t)k < best) best = k;
        continue;
      }
      const uint32_t oldest = j.vs_uid[v][0];
      const PolicyLaunch& L = launches_[oldest % kLaunchSlots];
      if (!L.live || L.uid != oldest || (L.p > L.f ? L.p : L.f) < L.grid) continue;
    }
    if (best < 0 || (int64_t)k < best) best = k;
  }
  return best;
}

// bring the ready structures in line with is_ready(j)
void Policy::refresh(PolicyJob& j) {
  bool r = is_ready(j);
  if (r && !j.in_ready) make_ready(j);
  else if (!r && j.in_ready) make_unready(j);
}

void Policy::observe(uint32_t uid, int64_t d) {
  PolicyLaunch& L = launches_[uid % kLaunchSlots];
  if (!L.live || L.uid != uid) throw std::runtime_error("observation for unknown launch");
  L.obs = d;
  L.has_obs = true;
}

// NEXT-4 (identical to oracle Policy._refine): fold the launch's observed duration into
// the running average of its (model, layer) T-bar and shift R_j of every live job that
// has not dispatched that layer yet by the change.
void Policy::refine(const PolicyLaunch& L) {
  if (!cfg_.online_tbar || !L.has_obs) return;
  const uint32_t m = jobs_[L.job].model, lay = L.layer;
  tb_sum_[m][lay] += L.obs;
  tb_cnt_[m][lay] += 1;
  const int64_t nv = tb_sum_[m][lay] / tb_cnt_[m][lay];
  const int64_t delta = nv - models_[m][lay].tbar;
  models_[m][lay].tbar = nv;
  if (delta == 0) return;
  for (uint32_t id : live_by_model_[m]) {
    PolicyJob& j = jobs_[id];
    if (j.state[lay] != 0) continue;   // already dispatched
    const bool rdy = j.in_ready;
    if (rdy) make_unready(j);
    active_erase(j);
    j.R += delta;
    work_ += delta;
    active_insert(j);
    if (rdy) make_ready(j);
  }
}

// ready-set order key: SRPT (R_j), SJF (the model's whole-job T-bar sum), RR (uid of the
// job's last issued kernel, -1 = never); ties (seq, id).  Identical to oracle Policy.pick.
int64_t Policy::order_key(const PolicyJob& j) const {
  if (cfg_.policy == POL_SJF) return model_total_[j.model];
  if (cfg_.policy == POL_RR) return j.rr;
  return j.R;
}

// the order of the job cap (oracle Policy.eligible): the policy's total order (SRPT R_j,
// SJF model T-bar sum, RR last issued uid, FIFO arrival only), or arrival only with
// cap_fifo; ties (seq, id)
int64_t Policy::active_key(const PolicyJob& j) const {
  return (cfg_.policy == POL_FIFO || cfg_.cap_fifo) ? 0 : order_key(j);
}
void Policy::active_erase(const PolicyJob& j) {
  if (cfg_.max_active) active_.erase(std::make_tuple(active_key(j), j.seq, j.id));
}
void Policy::active_insert(const PolicyJob& j) {
  if (cfg_.max_active && j.cursor < models_[j.model].size()) active_.emplace(active_key(j), j.seq, j.id);
}

void Policy::make_ready(PolicyJob& j) {
  j.in_ready = true;
  srpt_.emplace(order_key(j), j.seq, j.id);
  fifo_.emplace(j.seq, j.id);
  per_client_[j.client].emplace(j.seq, j.id);
}

void Policy::make_unready(PolicyJob& j) {
  j.in_ready = false;
  srpt_.erase(std::make_tuple(order_key(j), j.seq, j.id));
  fifo_.erase(std::make_pair(j.seq, j.id));
  per_client_[j.client].erase(std::make_pair(j.seq, j.id));
}

void Policy::arrival(uint32_t job_id, uint32_t client, uint32_t model) {
  if (unfinished_[client] == 0) Dt_[client] = -Omega_;   // C2-Q11: idle client restarts at 0
  unfinished_[client] += 1;
  if (jobs_.size() <= job_id) jobs_.resize(job_id + 1 + jobs_.size());
  PolicyJob& j = jobs_[job_id];
  j = PolicyJob();
  j.id = job_id;
  j.client = client;
  j.model = model;
  j.state.assign(models_[model].size(), 0);
  j.nvs = (uint32_t)vs_kernels_[model].size();
  j.seq = next_seq_++;
  int64_t R = 0;
  for (const auto& l : models_[model]) R += l.tbar;
  j.R = R;
  j.live = true;
  j.model_pos = (uint32_t)live_by_model_[model].size();
  live_by_model_[model].push_back(job_id);
  work_ += R;
  live_jobs_ += 1;
  active_insert(j);
  refresh(j);
}

bool Policy::record(uint32_t type, uint32_t uid, uint32_t n, int64_t* job_done) {
  *job_done = -1;
  PolicyLaunch& L = launches_[uid % kLaunchSlots];
  if (!L.live || L.uid != uid) throw std::runtime_error("record for unknown launch");
  O_ -= 1;
  uint32_t old = L.p > L.f ? L.p : L.f;
  const PolicyLayer& lay = models_[jobs_[L.job].model][L.layer];
  if (type == 1) {
    L.p += n;
  } else if (type == 2) {
    L.f += n;
    for (int r = 0; r < NRES; ++r) U_[r] -= (int64_t)n * lay.demand[r];
  } else {
    throw std::runtime_error("bad record type");
  }
  uint32_t now = L.p > L.f ? L.p : L.f;
  Q_ -= (int64_t)(now - old);
  if (L.p > L.grid || L.f > L.grid) throw std::runtime_error("record count exceeds grid");
  PolicyJob& j = jobs_[L.job];
  if (L.f != L.grid) {
    if (cfg_.lookahead) refresh(j);   // a fully placed predecessor may free a launch-ahead
    return false;
  }
  L.live = false;
  refine(L);
  j.done += 1;
  j.state[L.layer] = 2;
  const uint32_t v = models_[j.model][L.layer].vs;
  // drop the uid from the stream's in-flight list (completions of one stream may be
  // consumed out of issue order: the drain visits launches in any order)
  {
    uint32_t* u = j.vs_uid[v];
    uint32_t n = j.vs_infl[v], i = 0;
    while (i < n && u[i] != L.uid) ++i;
    if (i == n) throw std::runtime_error("completion of a launch not in flight on its stream");
    for (; i + 1 < n; ++i) u[i] = u[i + 1];
  }
  j.vs_infl[v] -= 1;
  if (j.vs_infl[v] == 0) {           // drained: its CUDA stream is free
    free_[L.stream / 64] |= 1ull << (L.stream % 64);
    j.vs_stream[v] = -1;
    j.vs_last[v] = (int32_t)L.stream;
  }
  if (j.done == models_[j.model].size()) {
    if (j.in_ready) make_unready(j);
    j.live = false;
    auto& lm = live_by_model_[j.model];   // swap-remove from the model's live list
    jobs_[lm.back()].model_pos = j.model_pos;
    lm[j.model_pos] = lm.back();
    lm.pop_back();
    unfinished_[j.client] -= 1;
    live_jobs_ -= 1;
    *job_done = j.id;
  } else {
    refresh(j);
  }
  return true;
}

int Policy::lowest_free() const {
  for (size_t w = 0; w < free_.size(); ++w)
    if (free_[w]) return (int)(w * 64 + __builtin_ctzll(free_[w]));
  return -1;
}

// B200-Q6 (max_active = K): the first ready job among the K first jobs of active_ (the
// policy's order over live jobs with kernels left to issue); false if none is ready
bool Policy::pick_capped(uint32_t* job_id) const {
  uint32_t k = 0;
  if (cfg_.cap_fifo && cfg_.policy != POL_FIFO) {
    // the cap admits in arrival order; among its ready jobs the policy's order decides
    bool found = false;
    std::tuple<int64_t, uint64_t, uint32_t> best{};
    for (auto it = active_.begin(); it != active_.end() && k < cfg_.max_active; ++it, ++k) {
      const PolicyJob& j = jobs_[std::get<2>(*it)];
      if (!j.in_ready) continue;
      const auto key = std::make_tuple(order_key(j), j.seq, j.id);
      if (!found || key < best) {
        best = key;
        found = true;
      }
    }
    if (found) *job_id = std::get<2>(best);
    return found;
  }
  for (auto it = active_.begin(); it != active_.end() && k < cfg_.max_active; ++it, ++k) {
    const uint32_t id = std::get<2>(*it);
    if (jobs_[id].in_ready) {
      *job_id = id;
      return true;
    }
  }
  return false;
}

bool Policy::pick(uint32_t* job_id) {
  over_ = false;
  if (srpt_.empty()) return false;
  if (cfg_.policy != POL_SRPT_DEFICIT && cfg_.max_active) return pick_capped(job_id);
  if (cfg_.policy == POL_FIFO) {
    *job_id = fifo_.begin()->second;
    return true;
  }
  if (cfg_.policy == POL_SJF || cfg_.policy == POL_RR) {   // pure orders, no deficit rule
    *job_id = std::get<2>(*srpt_.begin());
    return true;
  }
  // c* = argmax (D_c, -c) over clients with a ready job
  int cstar = -1;
  int64_t best = 0;
  for (uint32_t c = 0; c < cfg_.num_clients; ++c) {
    if (per_client_[c].empty()) continue;
    int64_t d = Dt_[c] + Omega_;
    if (cstar < 0 || d > best) {
      cstar = (int)c;
      best = d;
    }
  }
  bool over = false;
  if (cfg_.theta != INT64_MAX) {
    // theta * N without overflow: huge thresholds are never exceeded
    if (cfg_.theta <= INT64_MAX / (int64_t)cfg_.num_clients)
      over = best > cfg_.theta * (int64_t)cfg_.num_clients;
  }
  over_ = over;
  if (over) {
    *job_id = per_client_[cstar].begin()->second;   // oldest ready job of c* (overrides the cap too)
  } else if (cfg_.max_active) {
    return pick_capped(job_id);
  } else {
    *job_id = std::get<2>(*srpt_.begin());           // SRPT: (R, seq, id)
  }
  return true;
}

bool Policy::predicate(uint32_t grid) const {
  bool all_below = true;
  for (int r = 0; r < NRES; ++r)
    if (!(U_[r] < cfg_.capacity[r])) all_below = false;
  bool fits = (Q_ < cfg_.slack) || all_below;
  int64_t recs = 2 * (int64_t)((grid + cfg_.group - 1) / cfg_.group);
  bool ring_ok = O_ + recs <= cfg_.ring_capacity;
  return fits && ring_ok;
}

void Policy::decide(std::vector<Issue>* out) {
  for (;;) {
    uint32_t jid;
    if (!pick(&jid)) {
      last_stop_ = srpt_.empty() ? 0 : 4;   // 4: ready jobs, all outside the job cap
      break;
    }
    PolicyJob& j = jobs_[jid];
    const uint32_t k = (uint32_t)head(j);
    const uint32_t v = models_[j.model][k].vs;
    int s0 = lowest_free();
    if (j.vs_infl[v] == 0 && s0 < 0) {
      last_stop_ = 1;
      break;
    }
    const PolicyLayer& lay = models_[j.model][k];
    if (!predicate(lay.grid)) {
      int64_t recs = 2 * (int64_t)((lay.grid + cfg_.group - 1) / cfg_.group);
      last_stop_ = O_ + recs <= cfg_.ring_capacity ? 2 : 3;
      break;
    }
    uint32_t uid = next_uid_++;
    uint32_t stream;
    if (j.vs_infl[v] > 0) {
      stream = (uint32_t)j.vs_stream[v];   // launch-ahead: queued behind its predecessor
    } else {
      const uint32_t c = job_class(j);
      const uint32_t K = cfg_.prio_classes, P = cfg_.streams;
      const int32_t last = j.vs_last[v];
      if (last >= 0 && (free_[last / 64] >> (last % 64) & 1) && stream_class((uint32_t)last, K, P) == c) {
        stream = (uint32_t)last;
      } else {
        int sc = lowest_free_in_class(c);
        stream = sc >= 0 ? (uint32_t)sc : (uint32_t)s0;
      }
      free_[stream / 64] &= ~(1ull << (stream % 64));
      j.vs_stream[v] = (int32_t)stream;
    }
    PolicyLaunch& L = launches_[uid % kLaunchSlots];
    if (L.live) throw std::runtime_error("launch slot table overflow");
    L.uid = uid;
    L.job = jid;
    L.layer = k;
    L.grid = lay.grid;
    L.stream = stream;
    L.p = L.f = 0;
    L.has_obs = false;
    L.live = true;
    for (int r = 0; r < NRES; ++r) U_[r] += (int64_t)lay.grid * lay.demand[r];
    Q_ += lay.grid;
    O_ += 2 * (int64_t)((lay.grid + cfg_.group - 1) / cfg_.group);
    make_unready(j);
    active_erase(j);
    j.R -= lay.tbar;
    work_ -= lay.tbar;
    j.state[k] = 1;
    j.vs_uid[v][j.vs_infl[v]] = uid;
    j.vs_infl[v] += 1;
    j.vs_next[v] += 1;
    j.cursor += 1;
    j.last_uid = uid;
    j.rr = uid;   // after make_unready above: the ready-set key changes only out of the set
    active_insert(j);
    Dt_[j.client] -= (int64_t)cfg_.num_clients;
    Omega_ += 1;
    out->push_back(Issue{uid, jid, L.layer, stream});
    refresh(j);   // not ready until its new kernel is fully placed
  }
}

}  // namespace paella
