// Lock-free single-producer / single-consumer ring living in shared memory.
//
// Client -> dispatcher submission queue and dispatcher -> client completion queue
// (P1030-1033 §5: "each client obtains a shared memory region when setting up the
// connection"; P1062-1065: the dispatcher polls each queue round-robin;
// P1144-1155 §5.3: completions).  Head and tail sit on their own cache lines; the
// producer publishes a slot with a release store of tail, the consumer frees it
// with a release store of head.  Slots are fixed-size PODs.
#pragma once
#include <atomic>
#include <cstddef>
#include <cstdint>
#include <cstring>

namespace paella {

struct alignas(64) SubmitSlot {     // 64 B, SURVEY.md §8(a) a1
  uint64_t req_id;
  uint32_t model_id;
  uint32_t flags;
  uint64_t io_off;                  // offset of io inside the client's region
  uint64_t len;
  int64_t t_sched_ns;               // scheduled arrival (CLOCK_MONOTONIC)
  int64_t route_w[2];               // router's W snapshot of the two candidates (ng > 1)
  uint32_t route_meta;              // g0 | g1 << 8 | route << 16 (ng > 1), logged as ROUTE
  uint32_t pad;
};
static_assert(sizeof(SubmitSlot) == 64, "slot size");

struct alignas(32) CompleteSlot {   // 32 B
  uint64_t req_id;
  int32_t status;
  uint32_t gpu;
  int64_t t_done_ns;
  uint64_t pad;
};
static_assert(sizeof(CompleteSlot) == 32, "slot size");

template <typename T>
struct SpscRing {
  // lives at the start of a shared mapping, followed by the slots
  alignas(64) std::atomic<uint64_t> tail;   // written by the producer
  alignas(64) std::atomic<uint64_t> head;   // written by the consumer
  alignas(64) uint64_t cap;                 // power of two
  uint64_t mask;
  // producer-side cache of head, consumer-side cache of tail (each touched by one side)
  alignas(64) uint64_t head_cache;
  alignas(64) uint64_t tail_cache;
  alignas(64) T slots[1];

  static size_t bytes(uint64_t cap) { return offsetof(SpscRing, slots) + cap * sizeof(T); }

  void init(uint64_t c) {
    tail.store(0, std::memory_order_relaxed);
    head.store(0, std::memory_order_relaxed);
    cap = c;
    mask = c - 1;
    head_cache = 0;
    tail_cache = 0;
  }

  // producer
  bool push(const T& v) {
    uint64_t t = tail.load(std::memory_order_relaxed);
    if (t - head_cache >= cap) {
      head_cache = head.load(std::memory_order_acquire);
      if (t - head_cache >= cap) return false;
    }
    slots[t & mask] = v;
    tail.store(t + 1, std::memory_order_release);
    return true;
  }

  // consumer: pointer to the oldest slot or nullptr
  const T* peek() {
    uint64_t h = head.load(std::memory_order_relaxed);
    if (h == tail_cache) {
      tail_cache = tail.load(std::memory_order_acquire);
      if (h == tail_cache) return nullptr;
    }
    return &slots[h & mask];
  }
  void pop() { head.store(head.load(std::memory_order_relaxed) + 1, std::memory_order_release); }

  uint64_t size() const {
    return tail.load(std::memory_order_acquire) - head.load(std::memory_order_acquire);
  }
};

}  // namespace paella
