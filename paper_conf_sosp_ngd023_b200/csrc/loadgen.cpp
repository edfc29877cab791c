// Open-loop load generator (benchmark harness), see paella_loadgen in paella.h.
// Client side of the paper's channels: predict() with a pointer into the client's
// shared region (P1039-1061) and readResult(NONBLOCK) polling (P1147-1155).
#include <errno.h>

#include <atomic>
#include <cstring>
#include <thread>
#include <time.h>
#include <vector>

#include "engine.h"

using namespace paella;

extern "C" int64_t paella_loadgen(paella_t* p, const paella_req_t* reqs, uint32_t n, size_t stride,
                                  uint32_t slots_per_client, const void* const* const* copy_inputs, int64_t t0_ns,
                                  int64_t* jct_ns, int64_t* elapsed_ns) {
  Paella* P = (Paella*)p;
  if (!P || !reqs || !jct_ns || slots_per_client == 0) return -EINVAL;
  const uint32_t N = P->cfg.num_clients;
  if ((size_t)slots_per_client * stride > P->region_bytes) return -EINVAL;
  std::vector<std::vector<uint32_t>> free_slots(N);
  for (uint32_t c = 0; c < N; ++c)
    for (uint32_t s = slots_per_client; s-- > 0;) free_slots[c].push_back(s);
  // req_id -> (request index, slot)
  struct Pend {
    uint32_t idx, slot;
  };
  std::vector<std::vector<std::pair<uint64_t, Pend>>> pend(N);
  std::vector<uint8_t> sink(1 << 16);
  const int64_t t0 = t0_ns ? t0_ns : now_ns();
  uint32_t next = 0, done = 0;
  // per-client FIFO of requests that arrived but found no free slot
  std::vector<std::vector<uint32_t>> waiting(N);
  for (uint32_t i = 0; i < n; ++i) jct_ns[i] = -1;
  auto try_submit = [&](uint32_t i) -> bool {
    const paella_req_t& r = reqs[i];
    auto& fs = free_slots[r.client];
    if (fs.empty()) return false;
    uint32_t slot = fs.back();
    Model* m = P->models[r.model].get();
    uint8_t* io = P->region[r.client] + (size_t)slot * stride;
    if (copy_inputs) std::memcpy(io, copy_inputs[r.model][r.input_idx], m->input_bytes);
    int64_t rid = paella_submit_at(p, r.client, r.model, io, m->input_bytes + m->output_bytes, 0, t0 + r.t_ns);
    if (rid < 0) return false;
    fs.pop_back();
    pend[r.client].push_back({(uint64_t)rid, Pend{i, slot}});
    return true;
  };
  while (done < n) {
    int64_t now = now_ns();
    // arrivals due now (open loop: the schedule never waits for completions)
    while (next < n && t0 + reqs[next].t_ns <= now) {
      uint32_t c = reqs[next].client;
      if (c >= N) return -EINVAL;
      if (!waiting[c].empty() || !try_submit(next)) waiting[c].push_back(next);
      ++next;
    }
    // completions
    for (uint32_t c = 0; c < N; ++c) {
      for (;;) {
        int32_t st = 0;
        int64_t rid = paella_poll_completion(p, c, PAELLA_NONBLOCK, &st);
        if (rid < 0) break;
        int64_t tdone = now_ns();
        auto& v = pend[c];
        size_t k = 0;
        while (k < v.size() && v[k].first != (uint64_t)rid) ++k;
        if (k == v.size()) continue;
        Pend pd = v[k].second;
        v[k] = v.back();
        v.pop_back();
        const paella_req_t& r = reqs[pd.idx];
        Model* m = P->models[r.model].get();
        if (copy_inputs) {   // the client reads its logits out of the shared region
          uint8_t* io = P->region[c] + (size_t)pd.slot * stride;
          std::memcpy(sink.data(), io + m->input_bytes, std::min<size_t>(m->output_bytes, sink.size()));
        }
        jct_ns[pd.idx] = st == 0 ? tdone - (t0 + r.t_ns) : -1;
        free_slots[c].push_back(pd.slot);
        ++done;
        // a freed slot admits the oldest waiting request of this client
        while (!waiting[c].empty() && try_submit(waiting[c].front())) waiting[c].erase(waiting[c].begin());
      }
    }
  }
  if (elapsed_ns) *elapsed_ns = now_ns() - t0;
  return done;
}

extern "C" int paella_bench_wait(paella_t* p, uint32_t client_id, uint32_t model_id, uint32_t n, int64_t gap_ns,
                                 uint32_t poll_flags, size_t stride, uint32_t slots, int64_t* jct_ns,
                                 double* waiter_cpu_frac) {
  Paella* P = (Paella*)p;
  if (!P || !jct_ns || !waiter_cpu_frac || client_id >= P->cfg.num_clients || model_id >= P->nmodels.load() ||
      slots == 0 || (size_t)slots * stride > P->region_bytes)
    return -EINVAL;
  Model* m = P->models[model_id].get();
  std::vector<std::atomic<int64_t>> t_sub(n);
  std::vector<std::atomic<uint32_t>> slot_free(slots);
  for (auto& f : slot_free) f.store(1);
  std::vector<uint32_t> slot_of(n, 0);
  std::atomic<uint32_t> done{0};
  std::atomic<int64_t> seq0{-1};   // req_id sequence number of request 0 (ids are per-client seqs)
  double cpu_frac = 0;
  std::thread waiter([&] {
    timespec c0, c1;
    clock_gettime(CLOCK_THREAD_CPUTIME_ID, &c0);
    const int64_t w0 = now_ns();
    while (done.load() < n) {
      int32_t st = 0;
      int64_t rid = paella_poll_completion(p, client_id, poll_flags, &st);
      if (rid < 0) {
        if (rid == -EAGAIN) continue;
        break;
      }
      const int64_t t = now_ns();
      while (seq0.load(std::memory_order_acquire) < 0) {
      }
      const uint32_t i = (uint32_t)(((uint64_t)rid & 0xFFFFFFFFFFFFull) - (uint64_t)seq0.load());
      if (i >= n) continue;
      jct_ns[i] = st == 0 ? t - t_sub[i].load(std::memory_order_acquire) : -1;
      slot_free[slot_of[i]].store(1, std::memory_order_release);
      done.fetch_add(1);
    }
    clock_gettime(CLOCK_THREAD_CPUTIME_ID, &c1);
    const double cpu = (c1.tv_sec - c0.tv_sec) + (c1.tv_nsec - c0.tv_nsec) * 1e-9;
    cpu_frac = cpu / ((now_ns() - w0) * 1e-9);
  });
  int64_t due = now_ns();
  int rc = 0;
  for (uint32_t i = 0; i < n && rc == 0; ++i) {
    due += gap_ns;
    while (now_ns() < due) {
    }
    uint32_t s = i % slots;
    while (!slot_free[s].load(std::memory_order_acquire)) {
    }
    slot_free[s].store(0);
    slot_of[i] = s;
    t_sub[i].store(now_ns(), std::memory_order_release);
    uint8_t* io = P->region[client_id] + (size_t)s * stride;
    int64_t rid = paella_submit(p, client_id, model_id, io, m->input_bytes + m->output_bytes, 0);
    if (rid < 0) rc = (int)rid;
    else if (i == 0) seq0.store((int64_t)((uint64_t)rid & 0xFFFFFFFFFFFFull), std::memory_order_release);
  }
  if (rc) done.store(n);
  waiter.join();
  *waiter_cpu_frac = cpu_frac;
  return rc;
}
