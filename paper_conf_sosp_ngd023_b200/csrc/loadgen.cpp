// Open-loop load generator (benchmark harness), see paella_loadgen in paella.h.
// Client side of the paper's channels: predict() with a pointer into the client's
// shared region (P1039-1061) and readResult(NONBLOCK) polling (P1147-1155).
#include <errno.h>

#include <cstring>
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
