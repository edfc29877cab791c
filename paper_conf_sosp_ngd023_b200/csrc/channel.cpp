// Client <-> Paella memory channels: layout, predict() and readResult(), and the
// out-of-process client API (paella_client_*).  See channel.h.
#include "channel.h"

#include <errno.h>
#include <fcntl.h>
#include <linux/futex.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <sys/syscall.h>
#include <time.h>
#include <unistd.h>

#include <cstring>
#include <new>

namespace paella {

static size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

size_t channel_layout(ShmHeader* h, uint32_t num_clients, uint32_t num_gpus, uint32_t submit_slots,
                      size_t region_bytes) {
  const size_t page = 4096;
  size_t off = align_up(sizeof(ShmHeader), page);
  h->num_clients = num_clients;
  h->num_gpus = num_gpus;
  h->submit_slots = submit_slots;
  h->region_bytes = region_bytes;
  for (uint32_t c = 0; c < num_clients; ++c) {
    h->region_off[c] = off;
    off = align_up(off + region_bytes, page);
  }
  for (uint32_t g = 0; g < num_gpus; ++g)
    for (uint32_t c = 0; c < num_clients; ++c) {
      h->sub_off[g][c] = off;
      off = align_up(off + SpscRing<SubmitSlot>::bytes(submit_slots), 64);
      h->done_off[g][c] = off;
      off = align_up(off + SpscRing<CompleteSlot>::bytes(submit_slots), 64);
    }
  h->total_bytes = align_up(off, page);
  return h->total_bytes;
}

void channel_init(const Channel& ch, const ShmHeader& layout, uint32_t route) {
  ShmHeader* h = new (ch.hdr) ShmHeader();   // atomics value-initialised (the mapping is zeroed)
  h->abi = PAELLA_ABI_VERSION;
  h->num_clients = layout.num_clients;
  h->num_gpus = layout.num_gpus;
  h->submit_slots = layout.submit_slots;
  h->route = route;
  h->total_bytes = layout.total_bytes;
  h->region_bytes = layout.region_bytes;
  std::memcpy(h->region_off, layout.region_off, sizeof h->region_off);
  std::memcpy(h->sub_off, layout.sub_off, sizeof h->sub_off);
  std::memcpy(h->done_off, layout.done_off, sizeof h->done_off);
  for (uint32_t g = 0; g < h->num_gpus; ++g)
    for (uint32_t c = 0; c < h->num_clients; ++c) {
      ch.sub(g, c)->init(h->submit_slots);
      ch.done(g, c)->init(h->submit_slots);
    }
  std::atomic_thread_fence(std::memory_order_release);
  h->magic = SHM_MAGIC;
}

int64_t channel_submit(const Channel& ch, uint32_t client_id, uint32_t model_id, void* io, size_t len, uint32_t flags,
                       int64_t t_sched, std::vector<paella_route_rec_t>* route_log) {
  ShmHeader* H = ch.hdr;
  if (H->shutting.load(std::memory_order_acquire)) return -ESHUTDOWN;
  if (client_id >= H->num_clients) return -EINVAL;
  if (model_id >= H->nmodels.load(std::memory_order_acquire)) return -EINVAL;
  const ModelPub& m = H->models[model_id];
  uint8_t* base = ch.region(client_id);
  uint8_t* b = (uint8_t*)io;
  if (b < base || b + len > base + H->region_bytes || b + len < b) return -EFAULT;   // P1060-1061
  if (len < m.input_bytes + m.output_bytes) return -EINVAL;
  if (((uintptr_t)io & 15) != 0) return -EINVAL;
  ClientPub& C = H->client[client_id];
  const uint64_t seq = C.seq.fetch_add(1);
  const uint64_t req_id = ((uint64_t)client_id << 48) | (seq & ((1ull << 48) - 1));
  // route: least outstanding work W_g, ties to the lowest index;
  // W_g = published sum of R_j + unadmitted submissions x the model's whole-job T-bar.
  // A failed GPU (err != 0) is never chosen; -EIO once none is left.
  uint32_t gsel = 0;
  const uint32_t ng = H->num_gpus;
  SubmitSlot s{};
  if (ng > 1) {
    int64_t work[PAELLA_MAX_GPUS] = {0}, pend[PAELLA_MAX_GPUS] = {0}, W[PAELLA_MAX_GPUS] = {0};
    uint32_t alive = 0;
    for (uint32_t g = 0; g < ng; ++g) {
      GpuPub& pub = H->gpu[g];
      if (pub.err.load(std::memory_order_acquire) == 0) alive |= 1u << g;
      // pending before work: an admission moves a job from the first to the second
      pend[g] = (int64_t)(pub.submitted.load(std::memory_order_relaxed) - pub.admitted.load(std::memory_order_acquire));
      work[g] = pub.work.load(std::memory_order_acquire);
      W[g] = work[g] + pend[g] * m.total_tbar;
    }
    if (!alive) return -EIO;
    auto least = [&]() {
      uint32_t best = ng;
      for (uint32_t g = 0; g < ng; ++g)
        if ((alive >> g & 1) && (best == ng || W[g] < W[best])) best = g;
      return best;
    };
    uint32_t g0 = 0, g1 = 0;
    if (H->route == PAELLA_ROUTE_ROUND_ROBIN) {
      // the client's next GPU in cyclic order, skipping failed ones
      uint32_t k = 0;
      do {
        gsel = C.rr_next.fetch_add(1, std::memory_order_relaxed) % ng;
      } while (!(alive >> gsel & 1) && ++k < ng);
      g0 = g1 = gsel;
    } else if (H->route == PAELLA_ROUTE_POWER_OF_TWO) {
      paella_route_pair(req_id, ng, &g0, &g1);
      const uint32_t lo = g0 < g1 ? g0 : g1, hi = g0 < g1 ? g1 : g0;
      if ((alive >> lo & 1) && (alive >> hi & 1)) gsel = W[hi] < W[lo] ? hi : lo;
      else if (alive >> lo & 1) gsel = lo;
      else if (alive >> hi & 1) gsel = hi;
      else gsel = least();
    } else {
      gsel = g0 = g1 = least();
    }
    s.route_w[0] = W[g0];
    s.route_w[1] = W[g1];
    s.route_meta = g0 | (g1 << 8) | (H->route << 16);
    if (route_log) {
      paella_route_rec_t rr{};
      rr.req_id = req_id;
      rr.route = H->route;
      rr.chosen = gsel;
      rr.g0 = g0;
      rr.g1 = g1;
      rr.num_gpus = ng;
      rr.model = model_id;
      rr.alive = alive;
      rr.tbar_model = m.total_tbar;
      for (uint32_t g = 0; g < ng; ++g) {
        rr.work[g] = work[g];
        rr.pending[g] = pend[g];
      }
      route_log->push_back(rr);
    }
  } else if (H->gpu[0].err.load(std::memory_order_acquire)) {
    return -EIO;
  }
  s.req_id = req_id;
  s.model_id = model_id;
  s.flags = flags;
  s.io_off = (uint64_t)(b - base);
  s.len = len;
  s.t_sched_ns = t_sched;
  SpscRing<SubmitSlot>* q = ch.sub(gsel, client_id);
  for (;;) {
    if (q->push(s)) break;
    if (flags & PAELLA_NONBLOCK) return -EAGAIN;
    if (H->shutting.load(std::memory_order_acquire)) return -ESHUTDOWN;
  }
  H->gpu[gsel].submitted.fetch_add(1, std::memory_order_relaxed);
  return (int64_t)s.req_id;
}

void channel_wake(ShmHeader* H, uint32_t client) {
  ClientPub& C = H->client[client];
  C.wake_seq.fetch_add(1, std::memory_order_release);
  if (C.sleepers.load(std::memory_order_acquire) != 0)   // shared futex: the waiter may be another process
    syscall(SYS_futex, reinterpret_cast<uint32_t*>(&C.wake_seq), FUTEX_WAKE, INT32_MAX, nullptr, nullptr, 0);
}

int64_t channel_poll(const Channel& ch, uint32_t client_id, uint32_t flags, int32_t* status) {
  ShmHeader* H = ch.hdr;
  if (client_id >= H->num_clients) return -EINVAL;
  ClientPub& C = H->client[client_id];
  const uint32_t ng = H->num_gpus;
  int64_t spin_start = 0;
  for (;;) {
    const uint32_t r0 = C.poll_rr.load(std::memory_order_relaxed);
    for (uint32_t k = 0; k < ng; ++k) {
      const uint32_t g = (r0 + k) % ng;
      SpscRing<CompleteSlot>* q = ch.done(g, client_id);
      const CompleteSlot* c = q->peek();
      if (c) {
        const int64_t id = (int64_t)c->req_id;
        if (status) *status = c->status;
        q->pop();
        C.poll_rr.store((g + 1) % ng, std::memory_order_relaxed);
        return id;
      }
    }
    // every GPU failed and every submission has been answered: nothing will come
    bool all_dead = true;
    for (uint32_t g = 0; g < ng; ++g)
      all_dead &= H->gpu[g].err.load(std::memory_order_acquire) != 0 &&
                  H->gpu[g].popped.load(std::memory_order_acquire) >= H->gpu[g].submitted.load(std::memory_order_acquire);
    if (all_dead) {
      bool empty = true;   // re-check: a completion may have landed since the scan
      for (uint32_t k = 0; k < ng && empty; ++k) empty = ch.done(k, client_id)->peek() == nullptr;
      if (empty) return -EIO;
      continue;
    }
    if (flags & PAELLA_NONBLOCK) return -EAGAIN;
    if (H->shutting.load(std::memory_order_acquire)) return -ESHUTDOWN;
    if (flags & PAELLA_HYBRID) {
      // spin ~20 us after the last wake-up, then sleep until the next hint/completion
      const uint32_t seen = C.wake_seq.load(std::memory_order_acquire);
      if (spin_start == 0) spin_start = now_ns();
      if (now_ns() - spin_start < 20000) continue;
      C.sleepers.fetch_add(1, std::memory_order_acq_rel);
      bool empty = true;   // re-check after announcing the sleep (no lost wake-up)
      for (uint32_t k = 0; k < ng && empty; ++k) empty = ch.done(k, client_id)->peek() == nullptr;
      if (empty && C.wake_seq.load(std::memory_order_acquire) == seen) {
        timespec ts{0, 2000000};   // 2 ms cap: shutdown and error paths need no wake-up
        syscall(SYS_futex, reinterpret_cast<uint32_t*>(&C.wake_seq), FUTEX_WAIT, seen, &ts, nullptr, 0);
      }
      C.sleepers.fetch_sub(1, std::memory_order_acq_rel);
      spin_start = now_ns();
    }
  }
}

}  // namespace paella

using namespace paella;

// ---------------------------------------------------------------------------
// out-of-process clients (include/paella.h "client processes")
// ---------------------------------------------------------------------------
struct paella_client_s {
  Channel ch;
  size_t bytes = 0;
  uint32_t id = 0;
};

extern "C" {

int paella_client_attach(const char* path, uint32_t client_id, paella_client_t** out) {
  if (!path || !out) return -EINVAL;
  const int fd = open(path, O_RDWR | O_CLOEXEC);
  if (fd < 0) return -errno;
  struct stat st;
  if (fstat(fd, &st) != 0 || (size_t)st.st_size < sizeof(ShmHeader)) {
    close(fd);
    return -EINVAL;
  }
  void* p = mmap(nullptr, (size_t)st.st_size, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  close(fd);
  if (p == MAP_FAILED) return -ENOMEM;
  ShmHeader* h = (ShmHeader*)p;
  if (h->magic != SHM_MAGIC || h->abi != PAELLA_ABI_VERSION || h->total_bytes != (uint64_t)st.st_size ||
      client_id >= h->num_clients) {
    munmap(p, (size_t)st.st_size);
    return -EINVAL;
  }
  uint32_t expect = 0;   // one process per client id (the channels are single-producer)
  if (!h->client[client_id].attached.compare_exchange_strong(expect, 1)) {
    munmap(p, (size_t)st.st_size);
    return -EBUSY;
  }
  auto* c = new paella_client_s();
  c->ch.hdr = h;
  c->ch.base = (uint8_t*)p;
  c->bytes = (size_t)st.st_size;
  c->id = client_id;
  *out = c;
  return 0;
}

int paella_client_region_of(paella_client_t* c, void** base, size_t* bytes) {
  if (!c) return -EINVAL;
  if (base) *base = c->ch.region(c->id);
  if (bytes) *bytes = c->ch.hdr->region_bytes;
  return 0;
}

int paella_client_model_io(paella_client_t* c, uint32_t model_id, size_t* input_bytes, size_t* output_bytes) {
  if (!c || model_id >= c->ch.hdr->nmodels.load(std::memory_order_acquire)) return -EINVAL;
  if (input_bytes) *input_bytes = c->ch.hdr->models[model_id].input_bytes;
  if (output_bytes) *output_bytes = c->ch.hdr->models[model_id].output_bytes;
  return 0;
}

int64_t paella_client_submit(paella_client_t* c, uint32_t model_id, void* io, size_t len, uint32_t flags) {
  if (!c) return -EINVAL;
  return channel_submit(c->ch, c->id, model_id, io, len, flags, now_ns(), nullptr);
}

int64_t paella_client_poll(paella_client_t* c, uint32_t flags, int32_t* status) {
  if (!c) return -EINVAL;
  return channel_poll(c->ch, c->id, flags, status);
}

int paella_client_detach(paella_client_t* c) {
  if (!c) return -EINVAL;
  c->ch.hdr->client[c->id].attached.store(0, std::memory_order_release);
  munmap(c->ch.base, c->bytes);
  delete c;
  return 0;
}

}  // extern "C"
