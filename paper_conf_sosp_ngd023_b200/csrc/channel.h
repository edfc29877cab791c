// Client <-> Paella memory channels (§5, P1030-1033: "each client obtains a
// shared memory region when setting up the connection"; §5.1 P1039-1068 predict();
// §5.3 P1144-1171 readResult()).
//
// Everything a client needs lives in ONE shared mapping (a memfd the engine creates):
// a header with the published routing state of every GPU dispatcher, the registered
// models' io sizes and the per-client sequence / wake-up words; then every client's io
// region; then the per-(GPU, client) submission and completion rings.  The engine maps
// it at paella_init; a client in another process maps the same file
// (paella_client_attach) and runs the SAME submit / poll code on its own view, so a
// request is a store into shared memory whether it comes from the engine's process or
// not.  All offsets are relative to the mapping (addresses differ per process).
#pragma once
#include <atomic>
#include <cstdint>
#include <vector>

#include "../../include/paella.h"
#include "spsc.h"

namespace paella {

constexpr uint64_t SHM_MAGIC = 0x50414C4C41534D31ull;   // "PALLASM1"
constexpr uint32_t SHM_MAX_MODELS = 256;

// what a dispatcher publishes for the router and failure handling
struct alignas(64) GpuPub {
  std::atomic<int64_t> work;         // W_g: sum of R_j over its live jobs (after each decide)
  std::atomic<uint64_t> admitted;    // submissions it admitted
  std::atomic<uint64_t> submitted;   // submissions routed to it (incremented by clients)
  std::atomic<uint64_t> popped;      // submissions taken out of its rings (any outcome)
  std::atomic<int32_t> err;          // != 0: failed (-EIO) or hung (-ETIMEDOUT)
};

struct ModelPub {
  uint64_t input_bytes, output_bytes;
  int64_t total_tbar;                // whole-job T-bar sum (the router's backlog estimate)
};

struct alignas(64) ClientPub {
  std::atomic<uint64_t> seq;         // request sequence (req_id = client << 48 | seq)
  std::atomic<uint32_t> rr_next;     // round-robin router position
  std::atomic<uint32_t> poll_rr;     // completion-ring scan start
  std::atomic<uint32_t> wake_seq;    // hybrid wait: bumped on hints and completions (futex word)
  std::atomic<uint32_t> sleepers;    // threads sleeping on wake_seq
  std::atomic<uint32_t> attached;    // an out-of-process client holds this id
};

struct ShmHeader {
  uint64_t magic;
  uint32_t abi, num_clients, num_gpus, submit_slots, route, pad;
  uint64_t total_bytes, region_bytes;
  uint64_t region_off[PAELLA_MAX_CLIENTS];
  uint64_t sub_off[PAELLA_MAX_GPUS][PAELLA_MAX_CLIENTS];
  uint64_t done_off[PAELLA_MAX_GPUS][PAELLA_MAX_CLIENTS];
  GpuPub gpu[PAELLA_MAX_GPUS];
  alignas(64) std::atomic<uint32_t> nmodels;
  std::atomic<uint32_t> shutting;
  ModelPub models[SHM_MAX_MODELS];
  ClientPub client[PAELLA_MAX_CLIENTS];
};

// one process's view of the shared channels
struct Channel {
  ShmHeader* hdr = nullptr;
  uint8_t* base = nullptr;
  uint8_t* region(uint32_t c) const { return base + hdr->region_off[c]; }
  SpscRing<SubmitSlot>* sub(uint32_t g, uint32_t c) const {
    return reinterpret_cast<SpscRing<SubmitSlot>*>(base + hdr->sub_off[g][c]);
  }
  SpscRing<CompleteSlot>* done(uint32_t g, uint32_t c) const {
    return reinterpret_cast<SpscRing<CompleteSlot>*>(base + hdr->done_off[g][c]);
  }
};

// lay out a channel mapping for the configuration: fills the header's offsets and
// sizes; returns the total bytes (regions page aligned)
size_t channel_layout(ShmHeader* h, uint32_t num_clients, uint32_t num_gpus, uint32_t submit_slots,
                      size_t region_bytes);
// initialise a freshly mapped (zeroed) channel: header fields, rings
void channel_init(const Channel& ch, const ShmHeader& layout, uint32_t route);

// predict() (P1039-1061): range check, req id, route, push (see include/paella.h)
int64_t channel_submit(const Channel& ch, uint32_t client, uint32_t model, void* io, size_t len, uint32_t flags,
                       int64_t t_sched, std::vector<paella_route_rec_t>* route_log);
// readResult() (P1144-1171): first available completion of the client
int64_t channel_poll(const Channel& ch, uint32_t client, uint32_t flags, int32_t* status);
// hybrid wait: bump the client's futex word; a syscall only if a thread sleeps on it
void channel_wake(ShmHeader* h, uint32_t client);

int64_t now_ns();

}  // namespace paella
