// Internal structures of the Paella runtime (host side).
#pragma once
#include <atomic>
#include <cstdint>
#include <cstdio>
#include <deque>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "../../include/paella.h"
#include "channel.h"
#include "common.h"
#include "kernels.h"
#include "policy.h"
#include "spsc.h"

namespace paella {

// one kernel of a model's chain (one per non-concat node, plus the ingest)
struct KernelInst {
  uint32_t kind = 0;
  int32_t node = -1;           // graph node it computes (-1 = ingest)
  uint32_t grid[3] = {1, 1, 1};
  uint32_t block = 256;
  uint32_t smem = 0;           // dynamic shared memory
  uint32_t regs = 32, static_smem = 0, tmem_cols = 0;
  LayerArgs proto{};           // shapes/flags; pointers patched per GPU / slot
  int32_t in_buf = -1, out_buf = -1, res_buf = -1;
  size_t w_off = 0, w_bytes = 0;       // packed weights in the model's weight blob
  size_t b_off = 0, ps_off = 0, pz_off = 0;   // fp32 bias / prologue scale / shift
  bool has_pro = false;
  int64_t tbar = 0;
  uint64_t flops = 0, bytes = 0;
  int64_t demand[NRES] = {1, 0, 0, 0, 0};
  // NEXT-4 intra-job concurrency (Fig. 7 waitlists, P906-951): the kernels whose
  // outputs this one reads (through concats and fused GAPs), its virtual stream, and
  // whether a kernel on another virtual stream consumes its output (then its exit count
  // is a release: the consumer is launched on another CUDA stream once it is seen)
  std::vector<uint32_t> deps;
  uint32_t vs = 0;
  bool xout = false;
  uint32_t grid_total() const { return grid[0] * grid[1] * grid[2]; }
};

struct Buffer {
  uint32_t c, h, w;
  size_t off, bytes;
};

struct TmapStore {           // CUtensorMap storage (64-byte aligned, 128 bytes)
  alignas(64) uint8_t b[128];
};

struct ModelGpu {
  void* weights = nullptr;     // device blob (packed weights + fp32 vectors)
  void* workspace = nullptr;   // slots * slot_bytes (+1 isolated slot)
  // split-K partial sums (fp32, TC_BN x TC_BM per output tile, all zero between uses):
  // the isolated slot's (sized for any split of any layer: autotuning, forced splits)
  // and the serving slots' (sized for the chosen splits); per virtual stream (NEXT-4
  // branches of one job run concurrently)
  float* splitk_iso = nullptr;
  float* splitk_slots = nullptr;
  std::vector<std::vector<LayerArgs>> args;   // [slot][kernel]
  std::vector<uint32_t> free_slots;
  std::vector<TmapStore> tmaps;   // per kernel (tcgen05 conv weights)
  uint8_t* bmaps = nullptr;       // device: [slot][kernel] im2col tensor maps (LF_TMA_B), 128 B each
};

struct Model {
  std::string name;
  uint32_t id = 0, dtype = 0;
  std::vector<paella_node_t> nodes;       // shapes/attrs (host param pointers not kept)
  std::vector<std::vector<int32_t>> node_inputs;
  std::vector<int32_t> buf_of;            // node -> buffer
  std::vector<uint32_t> coff;             // node -> channel offset in its buffer
  std::vector<Buffer> bufs;
  size_t slot_bytes = 0;
  std::vector<KernelInst> kernels;
  std::vector<uint8_t> blob;              // host copy of the packed parameters
  size_t input_bytes = 0, output_bytes = 0;
  uint32_t in_c = 0, in_h = 0, in_w = 0, out_n = 0;
  std::vector<ModelGpu> gpu;
  int64_t total_tbar = 0;
  uint32_t n_vs = 1;          // virtual streams of the DAG (1 = a chain)
};

struct JobRec {
  uint64_t req_id = 0;
  uint32_t client = 0, model = 0, slot = 0;
  uint8_t* io = nullptr;
  int64_t t_sched = 0;
  bool live = false;
  // naive mode
  uint32_t stream = 0;
  void* event = nullptr;
  uint8_t event_recorded = 0;  // set by the launcher thread (__atomic builtins)
  // counter mode, relaxed exits: when the job's in-flight kernels have
  // all completed and the policy released its stream, an event is recorded on that
  // stream; if the job's next kernel is issued on another stream, that stream waits
  // for the event (stream order carries the data dependency, reading C2-Q19)
  // (per virtual stream, NEXT-4: a job may hold several streams)
  void* rel_ev[MAX_VS] = {nullptr, nullptr, nullptr, nullptr};
  uint8_t rel_recorded[MAX_VS] = {0, 0, 0, 0};
  int32_t rel_stream[MAX_VS] = {-1, -1, -1, -1};
};

struct Paella;

// a launch handed from the dispatcher to a launcher thread
struct LaunchDesc {
  const KernelInst* k;
  LayerArgs a;
  InstrArgs ia;
  const void* tmap;
  void* event;                 // kind 1: record this event on the stream
  uint8_t* recorded;
  uint32_t stream, dtype;
  uint8_t instr, kind;         // kind 0 = kernel, 1 = event record, 2 = wait for a recorded event
  int64_t t_push;              // PAELLA_LAUNCH_STATS: host time the dispatcher queued it
};

// plain (in-process) single-producer / single-consumer queue
template <typename T>
struct SpscQ {
  std::vector<T> buf;
  uint64_t mask = 0;
  alignas(64) std::atomic<uint64_t> tail{0};
  alignas(64) std::atomic<uint64_t> head{0};
  void init(uint64_t cap) {
    buf.resize(cap);
    mask = cap - 1;
  }
  bool push(const T& v) {
    uint64_t t = tail.load(std::memory_order_relaxed);
    if (t - head.load(std::memory_order_acquire) > mask) return false;
    buf[t & mask] = v;
    tail.store(t + 1, std::memory_order_release);
    return true;
  }
  T* peek() {
    uint64_t h = head.load(std::memory_order_relaxed);
    if (h == tail.load(std::memory_order_acquire)) return nullptr;
    return &buf[h & mask];
  }
  void pop() { head.store(head.load(std::memory_order_relaxed) + 1, std::memory_order_release); }
};

struct Launcher {
  SpscQ<LaunchDesc> q;
  std::thread th;
  // PAELLA_LAUNCH_STATS (diagnosis): kernel launches, time queued before the call and
  // time inside cudaLaunchKernelExC, histograms in 0.5 us bins (last bin: >= 100 us)
  uint64_t n = 0;
  std::vector<uint64_t> h_queue = std::vector<uint64_t>(201, 0), h_call = std::vector<uint64_t>(201, 0);
};

// device backend: real CUDA GPU or CPU fake
struct Backend {
  virtual ~Backend() {}
  virtual int init() = 0;
  virtual Rec* ring() = 0;          // host view of the notification ring
  virtual void launch(const KernelInst& k, const LayerArgs& a, const InstrArgs& ia, uint32_t stream,
                      uint32_t dtype, bool instr) = 0;
  virtual void advance() {}         // fake: progress virtual time
  virtual int error() { return 0; }
  virtual uint32_t* tail_dev() = 0;
  virtual uint32_t* ctr_dev() = 0;
  virtual void* ring_dev() = 0;
  // naive mode completion detection
  virtual void record_event(uint32_t stream, void** ev) = 0;
  virtual void record_existing(uint32_t stream, void* ev) = 0;   // re-record a created event
  virtual void wait_event(uint32_t stream, void* ev) = 0;
  virtual bool event_done(void* ev) = 0;
  virtual void release_event(void* ev) = 0;
  virtual void sync() {}
};

struct Gpu {
  static constexpr uint32_t kObsSlots = 8192;   // = Policy::kLaunchSlots
  std::vector<int64_t> first_place_ns = std::vector<int64_t>(kObsSlots, 0);   // NEXT-4
  Paella* P = nullptr;
  uint32_t index = 0;       // instance-local index
  int device = 0;           // CUDA ordinal
  std::unique_ptr<Backend> be;
  std::unique_ptr<Policy> policy;
  uint64_t head = 0;        // notification ring consumer index
  uint32_t cap = 0, log2cap = 0;
  std::vector<uint32_t> ctr_base;   // running base per counter slot
  // counter-mode notification: launches in flight and their slots
  struct CtrLive {
    uint32_t uid, slot, base, grid, p, f;   // p, f: counts already turned into records
  };
  bool ctr_mode = false;
  std::vector<CtrLive> ctr_live;
  std::vector<uint32_t> ctr_free;           // free counter-mode slots
  std::vector<uint32_t> ctr_mbase;          // running base per counter-mode slot
  std::vector<JobRec> jobs;         // indexed by job id (dense)
  std::vector<uint32_t> free_job_ids;
  uint32_t next_job = 0;
  std::vector<SpscRing<SubmitSlot>*> sub;     // per client (in the shared channel mapping)
  std::vector<SpscRing<CompleteSlot>*> done;  // per client
  std::thread thread;
  std::atomic<bool> stop{false};
  // published in the shared channel header for every client process: W_g, admissions,
  // submissions, pops, and err (!= 0: this GPU failed (-EIO) or hung (-ETIMEDOUT); it
  // only completes submissions with -EIO from then on: dead mode)
  GpuPub* pub = nullptr;
  // completions the client's ring could not take yet (never blocks the dispatcher)
  std::vector<std::deque<CompleteSlot>> overflow;
  int64_t last_progress_ns = 0;     // watchdog: last time a record was consumed (or nothing was due)
  // model registration is applied by the dispatcher thread itself (no data race with
  // decide(); the MODEL events are ordered with the rest of the log)
  std::mutex inbox_mu;
  std::vector<std::pair<uint32_t, std::vector<PolicyLayer>>> inbox;
  std::atomic<uint32_t> inbox_n{0};          // models posted
  std::atomic<uint32_t> models_applied{0};   // models the dispatcher has added to its policy
  uint32_t rr_start = 0;
  // globaltimer -> host clock (C3): device_ns ~= host_ns + clk_offset; rtt < 0 = not calibrated
  int64_t clk_offset = 0, clk_rtt = -1, clk_res = 0, clk_at = 0;   // clk_at: host time of the sample
  bool clk_pending = false;           // paella_clock_sync -> the dispatcher logs it (inbox_mu)
  int64_t clk_new[4] = {0, 0, 0, 0};
  std::atomic<uint64_t> clk_req{0}, clk_applied{0};
  FILE* log = nullptr;
  bool log_times = false;
  uint32_t naive_uid = 0;   // PAELLA_NAIVE_INSTR diagnosis: launch counter of the naive path   // PAELLA_TRACE_TIMES: host-time events (EV_TIME) for timelines
  std::mutex log_mu;
  paella_stats_t stats{};   // written by the dispatcher thread only
  // paella_stats: a caller bumps st_req; the dispatcher copies stats into st_snap (under
  // st_mu) and publishes st_ack; after the thread's last write it sets loop_done, so a
  // caller can read stats directly (release/acquire, no data race -- ThreadSanitizer run)
  std::atomic<uint64_t> st_req{0}, st_ack{0};
  std::atomic<bool> loop_done{false};
  std::mutex st_mu;
  paella_stats_t st_snap{};
  std::vector<Issue> issues;
  // isolated runs (profiling, parity tests): private ring, counters and stream
  Rec* prof_ring_h = nullptr;
  void* prof_ring_d = nullptr;
  uint32_t* prof_tail = nullptr;
  Rec* prof_devring = nullptr;     // device-memory ring of isolated runs
  void* trace_buf = nullptr;       // debug phase timestamps
  void* flush_buf = nullptr;       // L2-cold timing: overwritten before each timed launch
  uint32_t* prof_ctr = nullptr;
  std::vector<uint32_t> prof_base;
  uint32_t prof_uid = 0;
  void* prof_stream = nullptr;
  void* stage_in = nullptr;    // pinned mapped staging for isolated-run io
  size_t stage_bytes = 0;
  std::mutex iso_mu;
  std::vector<uint32_t> naive_inflight;   // job ids in naive mode
  // live event timing of one kernel kind (roofline)
  struct EvPair {
    void* e0;
    void* e1;
    uint64_t bytes, flops;
  };
  std::vector<EvPair> ev_free;
  std::vector<EvPair> ev_pending;   // FIFO by launch order
  size_t ev_head = 0;
  // launcher threads (cfg.launch_threads)
  std::vector<std::unique_ptr<Launcher>> launchers;
  std::atomic<bool> launchers_stop{false};
  std::thread noise;   // PAELLA_LAUNCH_NOISE_US (diagnosis): background launches of an empty kernel
  std::atomic<int> launch_err{0};
};

struct Paella {
  paella_config_t cfg{};
  uint32_t sms = 148;
  std::vector<std::unique_ptr<Gpu>> gpus;
  std::vector<std::unique_ptr<Model>> models;   // capacity reserved; published via nmodels
  std::atomic<uint32_t> nmodels{0};
  std::mutex reg_mu;
  // the client channels (channel.h): one shared memfd mapping holding the header
  // (routing state, model io sizes, per-client words), the io regions and the rings
  Channel ch;
  int shm_fd = -1;
  size_t shm_bytes = 0;
  std::vector<uint8_t*> region;                 // client io regions (into ch)
  size_t region_bytes = 0;
  int64_t capacity[NRES];
  // routing log (multi-GPU, cfg.route_log_path): every decision with the full W_g
  // snapshot it was taken on, one vector per client (written by that client's thread)
  std::vector<std::vector<paella_route_rec_t>> route_log;
};

// planner (plan.cpp)
int plan_model(Paella* P, const paella_model_desc_t* d, Model* m);
uint32_t tc_tmem_cols();

// time
int64_t now_ns();

}  // namespace paella
