// Paella runtime: C ABI, per-GPU dispatcher threads, notification-ring drain,
// client channels, router, event log, CUDA and fake backends.
//
// Paper map:  dispatcher on a dedicated core (§5 P1024-1033, §7 P1331-1332);
// client->Paella shm queues polled round-robin (§5.1 P1062-1068); Paella->GPU
// launches with the original config + instrumentation params + a substituted
// stream from a pool (§5.2 P1080-1098); notifQ polling and INVALID reset
// (P1100-1113); flow control by delaying dispatch (P1115-1119); readResult with
// NONBLOCK / EAGAIN (§5.3 P1144-1155); scheduling policy (§6, policy.cpp).
#include <errno.h>
#include <fcntl.h>
#include <pthread.h>
#include <sched.h>
#include <sys/mman.h>
#include <time.h>
#include <unistd.h>

#include <algorithm>
#include <array>
#include <climits>
#include <cstdarg>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <queue>

#include <cuda_runtime.h>

#include <linux/futex.h>
#include <sys/syscall.h>
#include <unistd.h>
#include <climits>

#include "engine.h"

namespace paella {

// Under a profiler (Nsight Compute injects itself through CUDA_INJECTION64_PATH) every
// launch is serialised and replayed: a persistent warp (the notification mirror / proxy)
// never returns and a kernel spinning on a host flag the host sets only after the
// launch calls return (the timing gate) deadlocks.  Both are switched off then:
// notifications take the direct ring path, timing runs ungated.
static bool profiled() {
  static const bool p = std::getenv("CUDA_INJECTION64_PATH") != nullptr || std::getenv("NV_NSIGHT_INJECTION_TRANSPORT_TYPE") != nullptr ||
                        std::getenv("NV_TPS_LAUNCH_TOKEN") != nullptr || std::getenv("PAELLA_PROFILED") != nullptr;
  return p;
}
static bool no_gate() { return profiled() || std::getenv("PAELLA_NO_GATE") != nullptr; }
static bool no_proxy_env() { return profiled() || std::getenv("PAELLA_NO_PROXY") != nullptr; }
// diagnosis: run the counter mirror warp next to the naive baseline (its cost alone)
static bool naive_mirror_env() { return std::getenv("PAELLA_NAIVE_MIRROR") != nullptr; }
// diagnosis: the naive baseline launches the INSTRUMENTED kernels, counting into a scratch
// counter table laid out like counter mode's (nobody reads it): the device-side cost of
// the instrumentation alone, without the dispatcher
static bool naive_instr_env() { return std::getenv("PAELLA_NAIVE_INSTR") != nullptr; }

int64_t now_ns() {
  timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return (int64_t)ts.tv_sec * 1000000000ll + ts.tv_nsec;
}

// cheap timestamps for the dispatcher's busy-time accounting (stats.busy_ns)
static inline uint64_t ticks() {
#if defined(__x86_64__)
  return __builtin_ia32_rdtsc();
#else
  return (uint64_t)now_ns();
#endif
}
static double ns_per_tick() {
  static const double r = [] {
#if defined(__x86_64__)
    const int64_t n0 = now_ns();
    const uint64_t c0 = ticks();
    timespec ts{0, 20000000};
    nanosleep(&ts, nullptr);
    return (double)(now_ns() - n0) / (double)(ticks() - c0);
#else
    return 1.0;
#endif
  }();
  return r;
}

// ---------------------------------------------------------------------------
// event log (replay input for oracle/sim.py::replay; format in DESIGN.md)
// ---------------------------------------------------------------------------
enum : uint32_t { EV_ARRIVAL = 1, EV_RECORD = 2, EV_BATCH_END = 3, EV_ISSUE = 4, EV_COMPLETE = 5, EV_OBSERVE = 6, EV_ROUTE = 7,
                  EV_CLOCK = 8, EV_TIME = 9,
                  EV_CONFIG = 100, EV_CAPACITY = 101, EV_MODEL = 110, EV_LAYER = 111, EV_DEMAND = 112, EV_DEP = 113,
                  EV_VS = 114 };

struct LogEv {
  uint32_t type, a;
  uint64_t b, c, d;
};
static_assert(sizeof(LogEv) == 32, "log event");

static inline void logev(Gpu* g, uint32_t type, uint32_t a, uint64_t b, uint64_t c, uint64_t d) {
  if (!g->log) return;
  LogEv e{type, a, b, c, d};
  fwrite(&e, sizeof e, 1, g->log);
}

// ---------------------------------------------------------------------------
// fake backend: a CPU model of a GPU that synthesises ring records
// ---------------------------------------------------------------------------
struct FakeBackend : Backend {
  struct FK {
    uint32_t uid, grid, stream, placed = 0, sc = 0, ec = 0;
    int64_t demand[NRES];
    int64_t dur;
  };
  uint32_t sms, cap, log2cap, G, nstreams;
  int64_t per_sm[NRES] = {32, 64, 65536, 233472, 512};
  std::vector<std::array<int64_t, NRES>> freeres;
  std::vector<Rec> ringmem;
  uint32_t tail = 0;
  std::vector<uint32_t> ctr;
  std::vector<std::deque<FK*>> streams;
  struct End {
    int64_t t;
    uint64_t seq;
    FK* k;
    uint32_t sm;
    bool operator>(const End& o) const { return t != o.t ? t > o.t : seq > o.seq; }
  };
  std::priority_queue<End, std::vector<End>, std::greater<End>> ends;
  uint64_t seq = 0;
  int64_t now = 0, dt;
  std::vector<void*> evs;

  // fault injection (paella_config_t.fake_fault): record / launch ordinals, 1-based
  uint32_t fault = PAELLA_FAULT_NONE, fault_arg = 0;
  uint64_t rec_seq = 0, launch_seq = 0;
  std::vector<std::pair<uint32_t, uint64_t>> torn_pending;   // (slot, w1) landing next advance()

  FakeBackend(uint32_t s, uint32_t c, uint32_t l2, uint32_t g, uint32_t P, int64_t d, uint32_t f, uint32_t fa)
      : sms(s), cap(c), log2cap(l2), G(g), nstreams(P), dt(d), fault(f), fault_arg(fa) {}
  int init() override {
    freeres.assign(sms, {});
    for (auto& f : freeres)
      for (int r = 0; r < NRES; ++r) f[r] = per_sm[r];
    ringmem.assign(cap, Rec{0, 0});
    ctr.assign(2 * NCTR, 0);
    streams.resize(nstreams + 1);
    return 0;
  }
  Rec* ring() override { return ringmem.data(); }
  uint32_t* tail_dev() override { return &tail; }
  uint32_t* ctr_dev() override { return ctr.data(); }
  void* ring_dev() override { return ringmem.data(); }
  void put(uint32_t type, uint32_t n, uint32_t uid, uint32_t group) {
    uint32_t idx = tail++;
    Rec r = rec_encode(type, n, 0, idx >> log2cap, uid, (uint64_t)now, group);
    Rec& slot = ringmem[idx & (cap - 1)];
    if (fault == PAELLA_FAULT_TORN) {   // first half now, second half next iteration
      reinterpret_cast<volatile uint64_t*>(&slot)[0] = r.w0;
      torn_pending.emplace_back(idx & (cap - 1), r.w1);
    } else {
      slot = r;
    }
  }
  void emit(FK* k, uint32_t type, uint32_t count) {
    uint32_t r = count % G;
    if (r == 0 || count == k->grid) {
      // DROP counts COMPLETION records only (a lost PLACEMENT is absorbed by p_eff =
      // max(p, f)); the other faults count every record
      const bool counted = fault != PAELLA_FAULT_DROP || type == REC_COMPLETION;
      const bool hit = counted && ++rec_seq == fault_arg;
      if (hit && fault == PAELLA_FAULT_DROP) return;   // lost on the way to the ring
      const uint32_t n = r == 0 ? G : r, grp = (count - 1) / G;
      put(hit && fault == PAELLA_FAULT_CORRUPT ? 7u : type, n, k->uid, grp);
      if (hit && fault == PAELLA_FAULT_DUP) put(type, n, k->uid, grp);
    }
  }
  void launch(const KernelInst& k, const LayerArgs&, const InstrArgs& ia, uint32_t stream, uint32_t,
              bool) override {
    FK* f = new FK();
    f->uid = ia.uid;
    f->grid = k.grid_total();
    f->stream = stream;
    for (int r = 0; r < NRES; ++r) f->demand[r] = k.demand[r];
    f->dur = k.tbar > 0 ? k.tbar : 1000;
    if (fault == PAELLA_FAULT_HANG && ++launch_seq == fault_arg) f->dur = INT64_MAX / 4;   // never ends
    streams[stream].push_back(f);
  }
  void place() {
    for (auto& q : streams) {
      if (q.empty()) continue;
      FK* k = q.front();
      while (k->placed < k->grid) {
        int sm = -1;
        for (uint32_t i = 0; i < sms && sm < 0; ++i) {
          bool ok = true;
          for (int r = 0; r < NRES; ++r) ok &= freeres[i][r] >= k->demand[r];
          if (ok) sm = (int)i;
        }
        if (sm < 0) break;
        for (int r = 0; r < NRES; ++r) freeres[sm][r] -= k->demand[r];
        k->placed++;
        k->sc++;
        emit(k, REC_PLACEMENT, k->sc);
        ends.push(End{now + k->dur, seq++, k, (uint32_t)sm});
      }
    }
  }
  void advance() override {
    for (auto& tp : torn_pending) reinterpret_cast<volatile uint64_t*>(&ringmem[tp.first])[1] = tp.second;
    torn_pending.clear();
    now += dt;
    while (!ends.empty() && ends.top().t <= now) {
      End e = ends.top();
      ends.pop();
      for (int r = 0; r < NRES; ++r) freeres[e.sm][r] += e.k->demand[r];
      e.k->ec++;
      emit(e.k, REC_COMPLETION, e.k->ec);
      if (e.k->ec == e.k->grid) {
        streams[e.k->stream].pop_front();
        delete e.k;
      }
    }
    place();
  }
  // naive mode is a CUDA-only baseline; on the fake device jobs finish at once
  void record_event(uint32_t, void** ev) override { *ev = nullptr; }
  void record_existing(uint32_t, void*) override {}
  void wait_event(uint32_t, void*) override {}
  bool event_done(void*) override { return true; }
  void release_event(void*) override {}
};

// ---------------------------------------------------------------------------
// CUDA backend
// ---------------------------------------------------------------------------
// one launch of kernel k: split-K tcgen05 convs are thread-block clusters
static bool is_tc(uint32_t kind) {
  return kind == KIND_CONV_TC || kind == KIND_CONV_TC_PRO || kind == KIND_CONV_TC128 || kind == KIND_CONV_TC_M64;
}
static uint32_t tc_bn(uint32_t kind) { return kind == KIND_CONV_TC128 ? TC_BN_WIDE : TC_BN; }

// pdl: programmatic dependent launch (programmatic stream serialization).  Measured on
// B200 (tools/launch_quantum.cu, profiles/launch_quantum_r1.txt): a kernel queued
// behind another on the same stream starts on a ~2.05 us quantum with a plain launch
// (a 1 us kernel costs 4.1 us back to back) but 0.6 us after its predecessor with
// PDL.  Every kernel executes griddepcontrol.wait before touching its inputs
// (instr.cuh), and none triggers early, so the dependency semantics are unchanged:
// the successor's blocks are placed only once the predecessor has completed.
static cudaError_t cuda_launch(KernelFn fn, const KernelInst& k, void** args, cudaStream_t s, bool pdl) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(k.grid[0], k.grid[1], k.grid[2]);
  cfg.blockDim = dim3(k.block);
  cfg.dynamicSmemBytes = k.smem;
  cfg.stream = s;
  cudaLaunchAttribute at[2];
  uint32_t n = 0;
  if (is_tc(k.kind) && k.proto.ksplit > 1) {
    at[n].id = cudaLaunchAttributeClusterDimension;
    at[n].val.clusterDim.x = 1;
    at[n].val.clusterDim.y = 1;
    at[n].val.clusterDim.z = k.proto.ksplit;
    ++n;
  } else if (k.kind == KIND_GAPFC) {
    at[n].id = cudaLaunchAttributeClusterDimension;
    at[n].val.clusterDim.x = GAPFC_CLUSTER;
    at[n].val.clusterDim.y = 1;
    at[n].val.clusterDim.z = 1;
    ++n;
  }
  if (pdl) {
    at[n].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[n].val.programmaticStreamSerializationAllowed = 1;
    ++n;
  }
  if (n == 0) return cudaLaunchKernel((const void*)fn, cfg.gridDim, cfg.blockDim, args, k.smem, s);
  cfg.attrs = at;
  cfg.numAttrs = n;
  return cudaLaunchKernelExC(&cfg, (const void*)fn, args);
}

struct CudaBackend : Backend {
  int dev;
  uint32_t cap, nstreams;
  Rec* ring_h = nullptr;
  Rec* ring_d = nullptr;      // device view of the pinned host ring
  // notification proxy: kernels write to dev_ring (device memory); one persistent warp
  // forwards to the host ring, so no kernel pays the PCIe write on its exit path
  bool proxy = false;
  bool mirror = false;         // counter mode: kernels only count, k_notify_mirror copies
  uint32_t* ctr_m = nullptr;   // device: NCTR_SUB tables of NCTR_M x {start, end}
  uint32_t* mirror_h = nullptr;   // pinned, mapped host copy
  uint32_t* mirror_d = nullptr;
  bool pdl = true;             // programmatic dependent launches (off for the naive baseline)
  uint32_t prio_classes = 1;   // stream-priority classes (set before init)
  Rec* dev_ring = nullptr;
  uint32_t* proxy_ctl = nullptr;     // pinned mapped: [0] stop flag, [16] heartbeat
  cudaStream_t proxy_stream = nullptr;
  uint32_t* tail = nullptr;   // device
  uint32_t* ctr = nullptr;    // device, 2*NCTR
  std::vector<cudaStream_t> streams;
  KernelFn tab[2][2][KIND_COUNT];   // [dtype][instr][kind]
  int err_ = 0;
  CudaBackend(int d, uint32_t c, uint32_t P, bool px, bool mir)
      : dev(d), cap(c), nstreams(P), proxy(px && !mir), mirror(mir) {}
  bool proxy_running = false;
  uint32_t* ctl_d = nullptr;
  int setup_proxy(cudaStream_t s) {
    if (mirror) {
      if (cudaMalloc(&ctr_m, NCTR_SUB * 2 * NCTR_M * sizeof(uint32_t)) != cudaSuccess) return -ENOMEM;
      cudaMemsetAsync(ctr_m, 0, NCTR_SUB * 2 * NCTR_M * sizeof(uint32_t), s);
      if (cudaHostAlloc((void**)&mirror_h, NCTR_SUB * 2 * NCTR_M * sizeof(uint32_t),
                        cudaHostAllocMapped | cudaHostAllocPortable) !=
          cudaSuccess)
        return -ENOMEM;
      std::memset(mirror_h, 0, NCTR_SUB * 2 * NCTR_M * sizeof(uint32_t));
      cudaHostGetDevicePointer((void**)&mirror_d, mirror_h, 0);
    } else {
      if (cudaMalloc(&dev_ring, (size_t)cap * sizeof(Rec)) != cudaSuccess) return -ENOMEM;
      cudaMemsetAsync(dev_ring, 0, (size_t)cap * sizeof(Rec), s);
    }
    if (cudaHostAlloc((void**)&proxy_ctl, 256, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess)
      return -ENOMEM;
    std::memset(proxy_ctl, 0, 256);
    cudaHostGetDevicePointer((void**)&ctl_d, proxy_ctl, 0);
    int least = 0, greatest = 0;   // the forwarding warp outranks every pool stream
    cudaDeviceGetStreamPriorityRange(&least, &greatest);
    if (cudaStreamCreateWithPriority(&proxy_stream, cudaStreamNonBlocking, greatest) != cudaSuccess) return -EIO;
    return 0;
  }
  // dispatcher thread: (re)start the forwarding warp when records may be outstanding
  void ensure_proxy() {
    if (!proxy && !mirror) return;
    if (proxy_running) {
      if (__atomic_load_n(&proxy_ctl[32], __ATOMIC_ACQUIRE) == 0) return;
      proxy_running = false;   // it left after an idle spell
    }
    __atomic_store_n(&proxy_ctl[32], 0u, __ATOMIC_RELEASE);
    if (const char* pace = std::getenv("PAELLA_MIRROR_PACE_NS"))
      __atomic_store_n(&proxy_ctl[8], (uint32_t)atoi(pace), __ATOMIC_RELEASE);
    const Rec* src = dev_ring;
    Rec* dst = ring_d;
    uint32_t mask = cap - 1, l2 = 0;
    while ((1u << l2) < cap) ++l2;
    volatile uint32_t* st = ctl_d;
    void* args[5] = {(void*)&src, (void*)&dst, (void*)&mask, (void*)&l2, (void*)&st};
    const uint4* mc = (const uint4*)ctr_m;
    uint4* mh = (uint4*)mirror_d;
    void* margs[3] = {(void*)&mc, (void*)&mh, (void*)&st};
    if (cudaLaunchKernel(mirror ? (const void*)mirror_kernel() : (const void*)proxy_kernel(), dim3(1), dim3(32),
                         mirror ? margs : args, 0, proxy_stream) == cudaSuccess)
      proxy_running = true;
    else if (!err_)
      err_ = (int)cudaErrorLaunchFailure;
  }
  void stop_proxy() {
    if (!proxy_ctl) return;
    __atomic_store_n(&proxy_ctl[0], 1u, __ATOMIC_SEQ_CST);
    if (proxy_stream) cudaStreamSynchronize(proxy_stream);
    proxy_running = false;
  }
  int init() override {
    if (cudaSetDevice(dev) != cudaSuccess) return -ENODEV;
    if (cudaHostAlloc((void**)&ring_h, (size_t)cap * sizeof(Rec), cudaHostAllocMapped | cudaHostAllocPortable) !=
        cudaSuccess)
      return -ENOMEM;
    std::memset(ring_h, 0, (size_t)cap * sizeof(Rec));
    if (cudaHostGetDevicePointer((void**)&ring_d, ring_h, 0) != cudaSuccess) return -EIO;
    if (cudaMalloc(&tail, 256) != cudaSuccess) return -ENOMEM;
    if (cudaMalloc(&ctr, 2 * NCTR * sizeof(uint32_t)) != cudaSuccess) return -ENOMEM;
    streams.resize(nstreams);
    // stream-priority classes: class c of Policy::stream_class -> hardware priority
    // greatest + c (clamped to the device's range; class 0 = highest)
    int least = 0, greatest = 0;
    cudaDeviceGetStreamPriorityRange(&least, &greatest);
    for (uint32_t i = 0; i < nstreams; ++i) {
      int prio = 0;
      if (prio_classes > 1) {
        prio = greatest + (int)Policy::stream_class(i, prio_classes, nstreams);
        if (prio > least) prio = least;
      }
      if (cudaStreamCreateWithPriority(&streams[i], cudaStreamNonBlocking, prio) != cudaSuccess) return -EIO;
    }
    if (const char* rot = std::getenv("PAELLA_STREAM_ROT"))   // diagnosis: logical -> physical stream
      if (nstreams) std::rotate(streams.begin(), streams.begin() + (atoi(rot) % nstreams), streams.end());
    cudaMemsetAsync(tail, 0, 256, streams[0]);
    cudaMemsetAsync(ctr, 0, 2 * NCTR * sizeof(uint32_t), streams[0]);
    KernelFn tc_i[4], tc_p[4];
    simt_kernel_table(tab[0][1], tab[0][0], tab[1][1], tab[1][0]);
    tc_kernel_table(tc_i, tc_p);
    tab[0][1][KIND_CONV_TC] = tc_i[0];
    tab[0][0][KIND_CONV_TC] = tc_p[0];
    tab[0][1][KIND_CONV_TC_PRO] = tc_i[1];
    tab[0][0][KIND_CONV_TC_PRO] = tc_p[1];
    tab[0][1][KIND_CONV_TC128] = tc_i[2];
    tab[0][0][KIND_CONV_TC128] = tc_p[2];
    tab[0][1][KIND_CONV_TC_M64] = tc_i[3];
    tab[0][0][KIND_CONV_TC_M64] = tc_p[3];
    for (int i = 0; i < 2; ++i)
      tab[1][i][KIND_CONV_TC] = tab[1][i][KIND_CONV_TC_PRO] = tab[1][i][KIND_CONV_TC128] = tab[1][i][KIND_CONV_TC_M64] =
          nullptr;
    if (proxy || mirror) {
      int rc = setup_proxy(streams[0]);
      if (rc) return rc;
    }
    // stream-scoped: another engine's forwarding warp may be resident on this device
    return cudaStreamSynchronize(streams[0]) == cudaSuccess ? 0 : -EIO;
  }
  ~CudaBackend() override {
    cudaSetDevice(dev);
    stop_proxy();
    if (proxy_stream) cudaStreamDestroy(proxy_stream);
    if (dev_ring) cudaFree(dev_ring);
    if (ctr_m) cudaFree(ctr_m);
    if (mirror_h) cudaFreeHost(mirror_h);
    if (proxy_ctl) cudaFreeHost(proxy_ctl);
    for (auto& s : streams) cudaStreamDestroy(s);
    if (ring_h) cudaFreeHost(ring_h);
    if (tail) cudaFree(tail);
    if (ctr) cudaFree(ctr);
  }
  Rec* ring() override { return ring_h; }
  uint32_t* tail_dev() override { return tail; }
  uint32_t* ctr_dev() override { return ctr; }
  void* ring_dev() override { return proxy ? (void*)dev_ring : (void*)ring_d; }
  KernelFn fn(uint32_t kind, uint32_t dtype, bool instr) { return tab[dtype][instr ? 1 : 0][kind]; }
  void launch(const KernelInst& k, const LayerArgs& a, const InstrArgs& ia, uint32_t stream, uint32_t dtype,
              bool instr) override {
    void* args[3] = {(void*)&a, (void*)&ia, (void*)k_tmap(k)};
    cudaError_t e = cuda_launch(fn(k.kind, dtype, instr), k, args, streams[stream], pdl);
    if (e != cudaSuccess && !err_) err_ = (int)e;
  }
  // the tensor map of a tcgen05 conv is stored right after its KernelInst's proto
  // in per-GPU storage; set by the engine before launch through this hook
  const void* cur_tmap = nullptr;
  const void* k_tmap(const KernelInst&) { return cur_tmap; }
  int error() override {
    if (err_) return err_;
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) err_ = (int)e;
    return err_;
  }
  void record_event(uint32_t stream, void** ev) override {
    cudaEvent_t e;
    cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
    cudaEventRecord(e, streams[stream]);
    *ev = e;
  }
  void record_existing(uint32_t stream, void* ev) override { cudaEventRecord((cudaEvent_t)ev, streams[stream]); }
  void wait_event(uint32_t stream, void* ev) override { cudaStreamWaitEvent(streams[stream], (cudaEvent_t)ev, 0); }
  bool event_done(void* ev) override { return cudaEventQuery((cudaEvent_t)ev) == cudaSuccess; }
  void release_event(void* ev) override { cudaEventDestroy((cudaEvent_t)ev); }
  void sync() override {
    for (auto& s : streams) cudaStreamSynchronize(s);
  }
};

// per-(model, gpu) tensor maps for tcgen05 weights (defined in kernels_tc.cu)
int make_weight_tmap(void* weights, uint32_t rows, uint32_t kpad, uint32_t box_rows, void* out128);
int make_im2col_tmap(const void* in, const LayerArgs& a, uint32_t bn, void* out128);


// ---------------------------------------------------------------------------
// helpers
// ---------------------------------------------------------------------------
static InstrArgs make_instr(Gpu* g, uint32_t uid, uint32_t grid, bool last, bool instr, bool xout) {
  InstrArgs ia{};
  ia.ring = (Rec*)g->be->ring_dev();
  ia.tail = g->be->tail_dev();
  ia.mask = g->cap - 1;
  ia.log2cap = g->log2cap;
  ia.uid = uid;
  ia.group = g->P->cfg.group_size;
  ia.flags = INSTR_ON | (last ? INSTR_LAST : 0);
  if (g->P->cfg.naive && instr) {   // PAELLA_NAIVE_INSTR (diagnosis)
    ia.ctr = g->be->ctr_dev() + 2 * (uid % NCTR_M);
    ia.ctr_stride = 2 * NCTR_M;
    ia.flags |= INSTR_CTR | (last ? 0u : INSTR_RELAXED);
    return ia;
  }
  if (g->ctr_mode && instr) {
    // counter mode: a free slot of the mirrored counter table (> P x (lookahead + 1)
    // slots, so one is always free); the slot returns when its last block has exited
    uint32_t slot = g->ctr_free.back();
    g->ctr_free.pop_back();
    ia.ctr = static_cast<CudaBackend*>(g->be.get())->ctr_m + 2 * slot;
    ia.ctr_stride = 2 * NCTR_M;
    ia.base = g->ctr_mbase[slot];
    g->ctr_mbase[slot] += grid;
    if (last && std::getenv("PAELLA_LAST_SYS")) ia.flags |= INSTR_SYSREL;
    ia.flags |= INSTR_CTR;
    // the job's data dependencies are carried by streams -- except towards a consumer on
    // another virtual stream (NEXT-4), launched once this kernel's final count is seen
    if (!last && !xout) ia.flags |= INSTR_RELAXED;
    g->ctr_live.push_back(Gpu::CtrLive{uid, slot, ia.base, grid, 0, 0});
    return ia;
  }
  uint32_t slot = uid % NCTR;
  ia.ctr = g->be->ctr_dev() + 2 * slot;
  ia.base = g->ctr_base[slot];
  g->ctr_base[slot] += grid;
  return ia;
}

static bool launch_stats_env() {
  static const bool on = std::getenv("PAELLA_LAUNCH_STATS") != nullptr;
  return on;
}

static void launcher_push(Gpu* g, const LaunchDesc& d0) {
  Launcher* L = g->launchers[d0.stream % g->launchers.size()].get();
  LaunchDesc d = d0;
  d.t_push = launch_stats_env() ? now_ns() : 0;
  while (!L->q.push(d)) {
  }
}

static void launch_stats_print(Gpu* g) {
  auto pct = [](const std::vector<uint64_t>& h, uint64_t n, double q) {
    uint64_t c = 0;
    for (size_t i = 0; i < h.size(); ++i) {
      c += h[i];
      if (c >= q * n) return 0.5 * (double)i;
    }
    return 100.0;
  };
  for (size_t i = 0; i < g->launchers.size(); ++i) {
    const Launcher* L = g->launchers[i].get();
    if (!L->n) continue;
    fprintf(stderr, "[paella] gpu %u launcher %zu: %llu launches, queued p50 %.1f p99 %.1f us, call p50 %.1f p90 %.1f p99 %.1f us\n",
            g->index, i, (unsigned long long)L->n, pct(L->h_queue, L->n, 0.5), pct(L->h_queue, L->n, 0.99),
            pct(L->h_call, L->n, 0.5), pct(L->h_call, L->n, 0.9), pct(L->h_call, L->n, 0.99));
  }
}

// launcher thread: performs the CUDA launches of the streams it owns, in order
static void launcher_main(Gpu* g, Launcher* L) {
  cudaSetDevice(g->device);
  auto* cb = static_cast<CudaBackend*>(g->be.get());
  for (;;) {
    LaunchDesc* d = L->q.peek();
    if (!d) {
      if (g->launchers_stop.load(std::memory_order_acquire) && !L->q.peek()) break;
      continue;
    }
    if (d->kind == 0) {
      void* args[3] = {(void*)&d->a, (void*)&d->ia, (void*)d->tmap};
      const int64_t t0 = d->t_push ? now_ns() : 0;
      cudaError_t e = cuda_launch(cb->fn(d->k->kind, d->dtype, d->instr != 0), *d->k, args, cb->streams[d->stream], cb->pdl);
      if (e != cudaSuccess) g->launch_err.store((int)e);
      if (d->t_push) {
        const int64_t t1 = now_ns();
        L->n++;
        L->h_queue[std::min<int64_t>(200, (t0 - d->t_push) / 500)]++;
        L->h_call[std::min<int64_t>(200, (t1 - t0) / 500)]++;
      }
    } else if (d->kind == 1) {
      cudaEventRecord((cudaEvent_t)d->event, cb->streams[d->stream]);
      __atomic_store_n(d->recorded, (uint8_t)1, __ATOMIC_RELEASE);
    } else {
      // the record is on another launcher's stream: it must have been issued first
      while (!__atomic_load_n(d->recorded, __ATOMIC_ACQUIRE)) {
      }
      cudaStreamWaitEvent(cb->streams[d->stream], (cudaEvent_t)d->event, 0);
    }
    L->q.pop();
  }
}

static void do_launch(Gpu* g, Model* m, uint32_t slot, uint32_t layer, uint32_t uid, uint32_t stream, bool instr) {
  const KernelInst& k = m->kernels[layer];
  InstrArgs ia = make_instr(g, uid, k.grid_total(), layer + 1 == m->kernels.size(), instr,
                            g->P->cfg.branches && k.xout);
  const paella_config_t& cfg = g->P->cfg;
  if (!g->launchers.empty()) {
    LaunchDesc d;
    d.k = &k;
    d.a = m->gpu[g->index].args[slot][layer];
    d.ia = ia;
    d.tmap = is_tc(k.kind) ? m->gpu[g->index].tmaps[layer].b : nullptr;
    d.event = nullptr;
    d.recorded = nullptr;
    d.stream = stream;
    d.dtype = m->dtype;
    d.instr = instr ? 1 : 0;
    d.kind = 0;
    launcher_push(g, d);
    return;
  }
  Gpu::EvPair ep{nullptr, nullptr, 0, 0};
  CudaBackend* cb = nullptr;
  if (cfg.device == PAELLA_DEVICE_CUDA) {
    cb = static_cast<CudaBackend*>(g->be.get());
    cb->cur_tmap = is_tc(k.kind) ? m->gpu[g->index].tmaps[layer].b : nullptr;
    if (cfg.event_time_kind == k.kind + 1 && !g->ev_free.empty()) {
      ep = g->ev_free.back();
      g->ev_free.pop_back();
      ep.bytes = k.bytes;
      ep.flops = k.flops;
      cudaEventRecord((cudaEvent_t)ep.e0, cb->streams[stream]);
    }
  }
  g->be->launch(k, m->gpu[g->index].args[slot][layer], ia, stream, m->dtype, instr);
  if (ep.e0) {
    cudaEventRecord((cudaEvent_t)ep.e1, cb->streams[stream]);
    g->ev_pending.push_back(ep);
  }
}

// harvest completed event-timed launches (in launch order; stops at the first pending)
static void harvest_events(Gpu* g) {
  while (g->ev_head < g->ev_pending.size()) {
    Gpu::EvPair& ep = g->ev_pending[g->ev_head];
    if (cudaEventQuery((cudaEvent_t)ep.e1) != cudaSuccess) break;
    float ms = 0;
    cudaEventElapsedTime(&ms, (cudaEvent_t)ep.e0, (cudaEvent_t)ep.e1);
    g->stats.ev_launches++;
    g->stats.ev_ns += (uint64_t)((double)ms * 1e6);
    g->stats.ev_bytes += ep.bytes;
    g->stats.ev_flops += ep.flops;
    g->ev_free.push_back(ep);
    g->ev_head++;
  }
  if (g->ev_head == g->ev_pending.size()) {
    g->ev_pending.clear();
    g->ev_head = 0;
  }
}

// hybrid completion path: bump the client's futex word; a syscall only if it sleeps
static void wake_client(Paella* P, uint32_t client) { channel_wake(P->ch.hdr, client); }

// Completion to the client's ring; if the ring is full (the client is not polling) the
// completion waits in a per-client overflow queue, in order, and the dispatcher moves
// on (it never blocks on a client).
static void push_completion(Gpu* g, uint32_t client, uint64_t req_id, int32_t status) {
  CompleteSlot cs{};
  cs.req_id = req_id;
  cs.status = status;
  cs.gpu = g->index;
  cs.t_done_ns = now_ns();
  auto& ov = g->overflow[client];
  if (!ov.empty() || !g->done[client]->push(cs)) ov.push_back(cs);
  wake_client(g->P, client);
}

static void flush_overflow(Gpu* g) {
  for (uint32_t c = 0; c < g->overflow.size(); ++c) {
    auto& ov = g->overflow[c];
    bool moved = false;
    while (!ov.empty() && g->done[c]->push(ov.front())) {
      ov.pop_front();
      moved = true;
    }
    if (moved) wake_client(g->P, c);
  }
}

static void finish_job(Gpu* g, uint32_t jid, int32_t status) {
  JobRec& j = g->jobs[jid];
  Model* m = g->P->models[j.model].get();
  push_completion(g, j.client, j.req_id, status);
  m->gpu[g->index].free_slots.push_back(j.slot);
  j.live = false;
  g->free_job_ids.push_back(jid);
  g->stats.completed++;
  logev(g, EV_COMPLETE, 0, jid, (uint64_t)now_ns(), 0);
}

// admit one submission; false = no workspace (leave it in the ring)
static bool admit(Gpu* g, uint32_t client, const SubmitSlot& s) {
  Paella* P = g->P;
  Model* m = P->models[s.model_id].get();
  ModelGpu& mg = m->gpu[g->index];
  if (mg.free_slots.empty()) return false;
  // a job id first (ids come back when jobs finish), then the workspace slot
  if (g->free_job_ids.empty() && g->next_job >= g->jobs.capacity()) return false;
  uint32_t slot = mg.free_slots.back();
  mg.free_slots.pop_back();
  uint32_t jid;
  if (!g->free_job_ids.empty()) {
    jid = g->free_job_ids.back();
    g->free_job_ids.pop_back();
  } else {
    jid = g->next_job++;
    g->jobs.resize(g->next_job);
  }
  // The policy requires job ids in admission order only for tie-breaks via seq;
  // ids themselves may be reused once a job is done.
  JobRec& j = g->jobs[jid];
  j.req_id = s.req_id;
  j.client = client;
  j.model = s.model_id;
  j.slot = slot;
  j.io = P->region[client] + s.io_off;
  j.t_sched = s.t_sched_ns;
  j.live = true;
  for (uint32_t v = 0; v < MAX_VS; ++v) j.rel_stream[v] = -1;
  auto& args = mg.args[slot];
  args.front().in = j.io;                           // ingest reads client memory
  args.back().out = j.io + m->input_bytes;           // last kernel writes the logits in place
  g->stats.admitted++;
  if (P->gpus.size() > 1) logev(g, EV_ROUTE, s.route_meta, s.req_id, (uint64_t)s.route_w[0], (uint64_t)s.route_w[1]);
  logev(g, EV_ARRIVAL, client, jid, s.model_id, (uint64_t)s.t_sched_ns);
  if (P->cfg.naive) {
    // CUDA-MS baseline: every kernel of the job enters stream jid % P now
    uint32_t st = jid % P->cfg.stream_pool;
    j.stream = st;
    const bool ninstr = naive_instr_env();
    for (uint32_t l = 0; l < m->kernels.size(); ++l) {
      do_launch(g, m, slot, l, ninstr ? g->naive_uid++ : 0, st, ninstr);
      g->stats.launches++;
    }
    if (!g->launchers.empty()) {
      cudaEventCreateWithFlags((cudaEvent_t*)&j.event, cudaEventDisableTiming);
      __atomic_store_n(&j.event_recorded, (uint8_t)0, __ATOMIC_RELAXED);
      LaunchDesc d{};
      d.event = j.event;
      d.recorded = &j.event_recorded;
      d.stream = st;
      d.kind = 1;
      launcher_push(g, d);
    } else {
      g->be->record_event(st, &j.event);
      j.event_recorded = 1;
    }
    g->naive_inflight.push_back(jid);
  } else {
    g->policy->arrival(jid, client, s.model_id);
  }
  return true;
}

static void observe_before_record(Gpu* g, uint32_t type, uint32_t uid, uint32_t n);

static uint32_t drain_ring(Gpu* g) {
  Rec* ring = g->be->ring();
  uint32_t n = 0;
  for (;;) {
    Rec* r = ring + (g->head & (g->cap - 1));
    uint32_t lap = (uint32_t)(g->head >> g->log2cap);
    uint32_t want = rec_tag(lap);
    volatile uint64_t* vr = reinterpret_cast<volatile uint64_t*>(r);
    uint64_t w0 = vr[0];
    if ((w0 & 0xff) == REC_INVALID || ((w0 >> 24) & 0xff) != want) break;
    uint64_t w1 = vr[1];
    if ((w1 >> 56) != want) {   // torn: the second half has not landed yet
      g->stats.torn_retries++;
      break;
    }
    RecFields f = rec_decode(w0, w1);
    vr[0] = 0;                  // INVALID (P1110-1113)
    vr[1] = 0;
    g->head++;
    n++;
    g->stats.records++;
    observe_before_record(g, f.type, f.uid, f.count);   // OBSERVE precedes its RECORD in the log
    logev(g, EV_RECORD, f.type, f.uid, f.count, f.gtimer | ((uint64_t)f.group << 40) | ((uint64_t)f.smid << 56));
    int64_t done = -1;
    g->policy->record(f.type, f.uid, f.count, &done);
    if (done >= 0) finish_job(g, (uint32_t)done, 0);
  }
  return n;
}

// NEXT-4 (online T-bar): before the policy consumes a record, note when a launch's
// first PLACEMENT was seen; right before its final COMPLETION, hand the policy (and the
// event log) the observed duration.
static void observe_before_record(Gpu* g, uint32_t type, uint32_t uid, uint32_t n) {
  if (!g->P->cfg.online_tbar) return;
  const PolicyLaunch& L = g->policy->launch(uid);
  if (!L.live || L.uid != uid) return;
  int64_t& t0 = g->first_place_ns[uid % Gpu::kObsSlots];
  if (type == REC_PLACEMENT && L.p == 0 && L.f == 0) t0 = now_ns();
  if (type == REC_COMPLETION && L.f + n == L.grid) {
    if (L.p == 0 && L.f == 0) t0 = now_ns();   // completion seen before any placement
    const int64_t d = std::max<int64_t>(1, now_ns() - t0);
    logev(g, EV_OBSERVE, 0, uid, (uint64_t)d, 0);
    g->policy->observe(uid, d);
  }
}

// Counter mode, relaxed exits: a launch of a live job completed; if that left the job
// with nothing in flight, the policy released its stream -> record the release event
// there (in stream order right after the job's kernels)
static void maybe_release(Gpu* g, uint32_t uid) {
  const PolicyLaunch& pl = g->policy->launch(uid);
  const PolicyJob& pj = g->policy->job(pl.job);
  const uint32_t v = g->policy->model(pj.model)[pl.layer].vs;
  if (pj.vs_stream[v] >= 0) return;   // still in flight (launch-ahead): stream order holds
  JobRec& j = g->jobs[pl.job];
  const uint32_t s = pl.stream;
  j.rel_stream[v] = (int32_t)s;
  g->stats.rel_events++;
  if (!g->launchers.empty()) {
    if (!j.rel_ev[v]) cudaEventCreateWithFlags((cudaEvent_t*)&j.rel_ev[v], cudaEventDisableTiming);
    __atomic_store_n(&j.rel_recorded[v], (uint8_t)0, __ATOMIC_RELAXED);
    LaunchDesc d{};
    d.event = j.rel_ev[v];
    d.recorded = &j.rel_recorded[v];
    d.stream = s;
    d.kind = 1;
    launcher_push(g, d);
  } else {
    if (!j.rel_ev[v]) g->be->record_event(s, &j.rel_ev[v]);
    else g->be->record_existing(s, j.rel_ev[v]);
    j.rel_recorded[v] = 1;
  }
}

// Counter mode: turn the progress of every in-flight launch's mirrored {start, end}
// counters into the group-of-G records the ring would carry (group g of a launch
// covers counts (gG, min((g+1)G, grid)] and is reported once all of them are in;
// Fig. 6's aggregation, reading C2-Q2), in launch order, PLACEMENT before COMPLETION.
static uint32_t drain_counters(Gpu* g) {
  auto* cb = static_cast<CudaBackend*>(g->be.get());
  const uint32_t G = g->P->cfg.group_size;
  uint32_t n = 0;
  for (size_t i = 0; i < g->ctr_live.size();) {
    Gpu::CtrLive& L = g->ctr_live[i];
    // the launch's counts (the mirror warp publishes them summed over the NCTR_SUB tables)
    const uint64_t v = *reinterpret_cast<volatile uint64_t*>(cb->mirror_h + 2 * L.slot);
    const uint32_t st = (uint32_t)v, en = (uint32_t)(v >> 32);
    uint32_t cnt[2] = {st - L.base, en - L.base};
    uint32_t* seen[2] = {&L.p, &L.f};
    bool finished = false;
    for (int t = 0; t < 2; ++t) {
      const uint32_t now = cnt[t];
      if (now > L.grid) continue;   // not yet published for this use of the slot
      while (*seen[t] < now) {
        const uint32_t grp = *seen[t] / G;
        const uint32_t end = std::min((grp + 1) * G, L.grid);
        if (now < end) break;       // group incomplete
        const uint32_t cnt_g = end - grp * G;
        const uint32_t type = t == 0 ? REC_PLACEMENT : REC_COMPLETION;
        *seen[t] = end;
        n++;
        g->stats.records++;
        observe_before_record(g, type, L.uid, cnt_g);   // OBSERVE precedes its RECORD in the log
        logev(g, EV_RECORD, type, L.uid, cnt_g, ((uint64_t)grp << 40) | (0xFFull << 56));
        if (g->log_times) logev(g, EV_TIME, 1 + type, L.uid, (uint64_t)now_ns(), end);   // count seen (host)
        int64_t done = -1;
        const bool complete = g->policy->record(type, L.uid, cnt_g, &done);
        if (done >= 0)
          finish_job(g, (uint32_t)done, 0);
        else if (complete)
          maybe_release(g, L.uid);
      }
      if (t == 1 && L.f == L.grid) finished = true;
    }
    if (finished) {
      g->ctr_free.push_back(L.slot);
      g->ctr_live[i] = g->ctr_live.back();
      g->ctr_live.pop_back();
    } else {
      ++i;
    }
  }
  return n;
}

static void decide_and_launch(Gpu* g) {
  if (const uint32_t d = g->P->cfg.decide_delay_ns) {   // injected scheduler delay (Fig. 9)
    const int64_t until = now_ns() + d;
    while (now_ns() < until) {
    }
  }
  g->issues.clear();
  g->policy->decide(&g->issues);
  if (!g->issues.empty() && g->P->cfg.device == PAELLA_DEVICE_CUDA)
    static_cast<CudaBackend*>(g->be.get())->ensure_proxy();
  g->stats.decide_calls++;
  g->stats.stop_reason[g->policy->last_stop()]++;
  g->stats.sum_ready += g->policy->ready_count();
  g->stats.sum_live_jobs += g->policy->live_jobs();
  g->stats.sum_Q += (uint64_t)(g->policy->Q() > 0 ? g->policy->Q() : 0);
  for (const Issue& is : g->issues) {
    JobRec& j = g->jobs[is.job];
    Model* m = g->P->models[j.model].get();
    logev(g, EV_ISSUE, is.stream, is.uid, is.job, is.layer);
    if (g->log_times) logev(g, EV_TIME, 0, is.uid, (uint64_t)now_ns(), 0);   // decision time (host)
    const uint32_t v = g->policy->model(j.model)[is.layer].vs;
    if (j.rel_stream[v] >= 0) {
      if ((uint32_t)j.rel_stream[v] != is.stream) {   // moved: wait for the previous stream's release
        g->stats.xstream_waits++;
        if (!g->launchers.empty()) {
          LaunchDesc d{};
          d.event = j.rel_ev[v];
          d.recorded = &j.rel_recorded[v];
          d.stream = is.stream;
          d.kind = 2;
          launcher_push(g, d);
        } else {
          g->be->wait_event(is.stream, j.rel_ev[v]);
        }
      }
      j.rel_stream[v] = -1;
    }
    do_launch(g, m, j.slot, is.layer, is.uid, is.stream, g->P->cfg.instrument != 0);
    g->stats.launches++;
    if (is.layer + 1 == m->kernels.size()) wake_client(g->P, j.client);   // "almost finished" hint
  }
}

// Models posted by paella_register_model: added to this GPU's policy and logged by the
// dispatcher thread itself, between two loop iterations.
static void apply_inbox(Gpu* g) {
  if (g->st_req.load(std::memory_order_acquire) != g->st_ack.load(std::memory_order_relaxed)) {
    const uint64_t req = g->st_req.load(std::memory_order_acquire);
    {
      std::lock_guard<std::mutex> lk(g->st_mu);
      g->st_snap = g->stats;
    }
    g->st_ack.store(req, std::memory_order_release);
  }
  if (g->clk_req.load(std::memory_order_acquire) != g->clk_applied.load(std::memory_order_relaxed)) {
    std::lock_guard<std::mutex> lk(g->inbox_mu);
    if (g->clk_pending) {
      g->clk_offset = g->clk_new[0];
      g->clk_rtt = g->clk_new[1];
      g->clk_res = g->clk_new[2];
      g->clk_at = g->clk_new[3];
      logev(g, EV_CLOCK, g->index | ((uint32_t)std::min<int64_t>(g->clk_res, 0xFFFFFF) << 8), (uint64_t)g->clk_offset,
            (uint64_t)g->clk_rtt, (uint64_t)g->clk_at);
      g->clk_pending = false;
    }
    g->clk_applied.store(g->clk_req.load(std::memory_order_acquire), std::memory_order_release);
  }
  const uint32_t posted = g->inbox_n.load(std::memory_order_acquire);
  if (g->models_applied.load(std::memory_order_relaxed) == posted) return;
  std::vector<std::pair<uint32_t, std::vector<PolicyLayer>>> todo;
  {
    std::lock_guard<std::mutex> lk(g->inbox_mu);
    todo.swap(g->inbox);
  }
  for (auto& mt : todo) {
    const uint32_t nm = mt.first;
    const auto& layers = mt.second;
    g->policy->add_model(nm, layers);
    logev(g, EV_MODEL, nm, layers.size(), 0, 0);
    for (uint32_t l = 0; l < layers.size(); ++l) {
      logev(g, EV_LAYER, nm, l, layers[l].grid, (uint64_t)layers[l].tbar);
      logev(g, EV_DEMAND, nm, l, ((uint64_t)layers[l].demand[1] << 32) | (uint64_t)layers[l].demand[2],
            ((uint64_t)layers[l].demand[3] << 32) | (uint64_t)layers[l].demand[4]);
      if (g->P->cfg.branches) {   // NEXT-4: the DAG (virtual stream + cross-stream dependencies)
        logev(g, EV_VS, nm, l, layers[l].vs, 0);
        for (uint32_t d : layers[l].cross) logev(g, EV_DEP, nm, l, d, 0);
      }
    }
    if (g->log) fflush(g->log);
    g->models_applied.fetch_add(1, std::memory_order_release);
  }
}

// Fail this GPU: every live job completes with `status` (-EIO: a CUDA error or an
// inconsistent notification stream; -ETIMEDOUT: the watchdog).  The router stops
// sending work here (submit_impl checks err).
static void fail_gpu(Gpu* g, int status, const char* why) {
  fprintf(stderr, "[paella] GPU %u failed (%s): live jobs complete with %d\n", g->index, why, status);
  g->pub->err.store(status, std::memory_order_release);
  for (uint32_t jid = 0; jid < g->jobs.size(); ++jid)
    if (g->jobs[jid].live) finish_job(g, jid, status);
  g->naive_inflight.clear();
  if (g->log) fflush(g->log);
}

// Dead mode: the GPU is not used any more, but submissions that were routed here before
// the router noticed still get an answer (-EIO), and models keep being acknowledged.
static void dead_loop(Gpu* g) {
  const uint32_t N = g->P->cfg.num_clients;
  while (!g->stop.load(std::memory_order_acquire)) {
    apply_inbox(g);
    for (uint32_t c = 0; c < N; ++c) {
      const SubmitSlot* s;
      while ((s = g->sub[c]->peek()) != nullptr) {
        push_completion(g, c, s->req_id, -EIO);
        g->sub[c]->pop();
        g->pub->popped.fetch_add(1, std::memory_order_release);
      }
    }
    flush_overflow(g);
    struct timespec ts{0, 20000};
    nanosleep(&ts, nullptr);
  }
}

static void dispatch_loop(Gpu* g) {
  Paella* P = g->P;
  const uint32_t N = P->cfg.num_clients;
  const bool dbg = std::getenv("PAELLA_DEBUG") != nullptr;
  const int64_t watchdog_ns = (int64_t)P->cfg.watchdog_ms * 1000000;
  g->last_progress_ns = now_ns();
  uint64_t busy_ticks = 0;
  (void)ns_per_tick();
  for (;;) {
    const uint64_t it0 = ticks();
    if ((g->stats.loop_iters & 4095) == 0) g->stats.busy_ns = (uint64_t)(busy_ticks * ns_per_tick());
    g->stats.loop_iters++;
    if (dbg && (g->stats.loop_iters % 50000000) == 0) {
      fprintf(stderr, "[dbg gpu%u] iters=%lu admitted=%lu", g->index, (unsigned long)g->stats.loop_iters,
              (unsigned long)g->stats.admitted);
      for (uint32_t c = 0; c < N; ++c) fprintf(stderr, " sub[%u]=%lu", c, (unsigned long)g->sub[c]->size());
      uint32_t nm = P->nmodels.load();
      for (uint32_t m = 0; m < nm; ++m)
        fprintf(stderr, " free[%u]=%zu", m, P->models[m]->gpu[g->index].free_slots.size());
      fprintf(stderr, " live=%lu\n", (unsigned long)g->policy->live_jobs());
    }
    if ((g->stats.loop_iters & 63) == 0) {
      apply_inbox(g);
      flush_overflow(g);
      if (!g->ev_pending.empty()) harvest_events(g);
    }
    g->be->advance();
    uint32_t nev = 0;
    // 1. client rings, round-robin, starting after the last client served (C2-Q16)
    bool stopping = g->stop.load(std::memory_order_acquire);
    if (!stopping) {
      uint32_t nm = P->nmodels.load(std::memory_order_acquire);
      for (uint32_t k = 0; k < N; ++k) {
        uint32_t c = (g->rr_start + k) % N;
        SpscRing<SubmitSlot>* q = g->sub[c];
        const SubmitSlot* s;
        bool served = false;
        while ((s = q->peek()) != nullptr) {
          if (s->model_id >= nm) {
            // submit validated the id against nmodels, so the model is published: this
            // iteration loaded nmodels before the submission was pushed; reload it
            nm = P->nmodels.load(std::memory_order_acquire);
            if (s->model_id >= nm) break;
          }
          if (!admit(g, c, *s)) break;
          q->pop();
          g->pub->popped.fetch_add(1, std::memory_order_release);
          nev++;
          served = true;
        }
        if (served) g->rr_start = (c + 1) % N;
      }
      g->pub->admitted.store(g->stats.admitted, std::memory_order_release);
    }
    if (P->cfg.naive) {
      bool progressed = false;
      for (size_t i = 0; i < g->naive_inflight.size();) {
        uint32_t jid = g->naive_inflight[i];
        if (__atomic_load_n(&g->jobs[jid].event_recorded, __ATOMIC_ACQUIRE) && g->be->event_done(g->jobs[jid].event)) {
          g->be->release_event(g->jobs[jid].event);
          finish_job(g, jid, 0);
          g->naive_inflight[i] = g->naive_inflight.back();
          g->naive_inflight.pop_back();
          progressed = true;
        } else {
          ++i;
        }
      }
      if (progressed || g->naive_inflight.empty()) {
        if (watchdog_ns) g->last_progress_ns = now_ns();
      } else if (watchdog_ns && (g->stats.loop_iters & 1023) == 0 && now_ns() - g->last_progress_ns > watchdog_ns) {
        fail_gpu(g, -ETIMEDOUT, "watchdog: no job completed");
        return;
      }
      if (g->be->error() || g->launch_err.load(std::memory_order_relaxed)) {
        fail_gpu(g, -EIO, "CUDA error");
        return;
      }
      if (progressed || nev) busy_ticks += ticks() - it0;
      if (stopping && g->naive_inflight.empty()) return;
      if (naive_mirror_env() && (g->stats.loop_iters & 1023) == 0 && !g->naive_inflight.empty())
        static_cast<CudaBackend*>(g->be.get())->ensure_proxy();
      continue;
    }
    // 2. notification ring (keep the forwarding warp alive while records are due)
    if (P->cfg.device == PAELLA_DEVICE_CUDA && g->policy->O() > 0 && (g->stats.loop_iters & 1023) == 0)
      static_cast<CudaBackend*>(g->be.get())->ensure_proxy();
    const uint32_t nrec = g->ctr_mode ? drain_counters(g) : drain_ring(g);
    nev += nrec;
    // watchdog: records are due (launches in flight) but none arrived for too long
    if (nrec || g->policy->O() == 0) {
      if (watchdog_ns) g->last_progress_ns = now_ns();
    } else if (watchdog_ns && (g->stats.loop_iters & 1023) == 0 && now_ns() - g->last_progress_ns > watchdog_ns) {
      fail_gpu(g, -ETIMEDOUT, "watchdog: in-flight launches report no progress");
      return;
    }
    // 3. decide (the batch boundary is logged for replay, C2-Q17)
    if (nev) {
      logev(g, EV_BATCH_END, 0, 0, 0, 0);
      if (g->log_times) logev(g, EV_TIME, 1, 0, (uint64_t)now_ns(), 0);   // records consumed (host)
      decide_and_launch(g);
      g->pub->work.store(g->policy->outstanding_work(), std::memory_order_release);
      busy_ticks += ticks() - it0;
    }
    int e = g->be->error();
    if (!e) e = g->launch_err.load(std::memory_order_relaxed);
    if (e) {
      fail_gpu(g, -EIO, "CUDA error");
      return;
    }
    if (stopping && g->policy->live_jobs() == 0) return;
  }
}

static void dispatcher_main(Gpu* g) {
  Paella* P = g->P;
  if (P->cfg.device == PAELLA_DEVICE_CUDA) cudaSetDevice(g->device);
  if (P->cfg.dispatcher_cpus) {
    cpu_set_t cs;
    CPU_ZERO(&cs);
    CPU_SET(P->cfg.dispatcher_cpus[g->index], &cs);
    pthread_setaffinity_np(pthread_self(), sizeof cs, &cs);
    // a dedicated core with SCHED_FIFO (PAELLA_DISPATCHER_FIFO=<prio>);
    // only with a pinned core, so the spinning dispatcher cannot starve migrating threads
    if (const char* fifo = std::getenv("PAELLA_DISPATCHER_FIFO")) {
      sched_param sp{};
      sp.sched_priority = atoi(fifo);
      int rc = pthread_setschedparam(pthread_self(), SCHED_FIFO, &sp);
      if (rc) fprintf(stderr, "[paella] dispatcher %u: SCHED_FIFO %d refused (%s)\n", g->index, sp.sched_priority,
                      strerror(rc));
    }
  }
  if (P->cfg.device == PAELLA_DEVICE_CUDA && P->cfg.event_time_kind) {
    for (int i = 0; i < 512; ++i) {
      cudaEvent_t a, b;
      cudaEventCreate(&a);
      cudaEventCreate(&b);
      g->ev_free.push_back(Gpu::EvPair{a, b, 0, 0});
    }
  }
  // An inconsistent notification stream (a record for an unknown launch, a count beyond
  // the grid, an invalid type: a device or transport fault) makes the policy throw; that
  // fails this GPU's jobs with -EIO instead of terminating the process.
  try {
    dispatch_loop(g);
  } catch (const std::exception& ex) {
    fail_gpu(g, -EIO, ex.what());
  }
  if (g->pub->err.load(std::memory_order_acquire)) dead_loop(g);
  g->loop_done.store(true, std::memory_order_release);
}

// globaltimer -> host clock calibration: n ping-pongs with
// k_clock_probe through mapped memory; the sample with the smallest round trip gives
// offset = globaltimer - midpoint of the host send/receive times (CLOCK_MONOTONIC), so
// device_ns ~= host_ns + offset within +- rtt/2; the probe also measures the timer's
// resolution.  Not under a profiler (the probe waits for the host).
static int clock_sync(Gpu* g, uint32_t n, int64_t* off, int64_t* rtt, int64_t* res, int64_t* at) {
  if (profiled()) return -ENOTSUP;
  if (cudaSetDevice(g->device) != cudaSuccess) return -EIO;
  void* buf = nullptr;
  if (cudaHostAlloc(&buf, 4096, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) return -ENOMEM;
  std::memset(buf, 0, 4096);
  volatile uint32_t* flag = (volatile uint32_t*)buf;
  volatile uint64_t* out = (volatile uint64_t*)((uint8_t*)buf + 64);
  void *flag_d = nullptr, *out_d = nullptr;
  cudaHostGetDevicePointer(&flag_d, (void*)flag, 0);
  cudaHostGetDevicePointer(&out_d, (void*)out, 0);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  void* args[3] = {(void*)&flag_d, (void*)&out_d, (void*)&n};
  int rc = cudaLaunchKernel((const void*)clock_kernel(), dim3(1), dim3(1), args, 0, s) == cudaSuccess ? 0 : -EIO;
  int64_t best = INT64_MAX, boff = 0;
  for (uint32_t i = 0; i < n && rc == 0; ++i) {
    const int64_t t0 = now_ns();
    __atomic_store_n((uint32_t*)flag, i + 1, __ATOMIC_SEQ_CST);
    while (out[i] == 0) {
      if (now_ns() - t0 > 2000000000ll) {
        rc = -ETIMEDOUT;
        break;
      }
    }
    const int64_t t1 = now_ns();
    if (rc == 0 && t1 - t0 < best) {
      best = t1 - t0;
      boff = (int64_t)out[i] - (t0 + (t1 - t0) / 2);
      *at = t0 + (t1 - t0) / 2;
    }
  }
  __atomic_store_n((uint32_t*)flag, n, __ATOMIC_SEQ_CST);   // release the probe in any case
  if (cudaStreamSynchronize(s) != cudaSuccess && rc == 0) rc = -EIO;
  if (rc == 0) {
    *off = boff;
    *rtt = best;
    *res = (int64_t)out[n];
  }
  cudaStreamDestroy(s);
  cudaFreeHost(buf);
  return rc;
}

// ---------------------------------------------------------------------------
// shared memory helpers
// ---------------------------------------------------------------------------
// The client channels (channel.h) in one memfd mapping: other processes attach to it
// through /proc/<pid>/fd/<fd> (paella_channel_path / paella_client_attach).
static int channel_create(Paella* P) {
  const paella_config_t& cfg = P->cfg;
  ShmHeader layout{};
  const size_t total = channel_layout(&layout, cfg.num_clients, cfg.num_gpus, cfg.submit_slots, P->region_bytes);
  const int fd = (int)syscall(SYS_memfd_create, "paella-channels", 0u);
  if (fd < 0) return -errno;
  if (ftruncate(fd, (off_t)total) != 0) {
    close(fd);
    return -ENOMEM;
  }
  void* p = mmap(nullptr, total, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  if (p == MAP_FAILED) {
    close(fd);
    return -ENOMEM;
  }
  P->shm_fd = fd;
  P->shm_bytes = total;
  P->ch.hdr = (ShmHeader*)p;
  P->ch.base = (uint8_t*)p;
  channel_init(P->ch, layout, cfg.route);
  return 0;
}

static uint32_t ilog2(uint32_t x) {
  uint32_t l = 0;
  while ((1u << l) < x) ++l;
  return l;
}

static int setup_model_gpu(Paella* P, Model* m, Gpu* g);

}  // namespace paella

using namespace paella;

// ===========================================================================
// C ABI
// ===========================================================================
extern "C" {

int paella_init(const paella_config_t* cfg_in, paella_t** out) {
  if (!cfg_in || !out || cfg_in->abi_version != PAELLA_ABI_VERSION) return -EINVAL;
  paella_config_t cfg = *cfg_in;
  if (cfg.num_gpus < 1 || cfg.num_gpus > PAELLA_MAX_GPUS) return -EINVAL;
  if (cfg.num_clients < 1 || cfg.num_clients > PAELLA_MAX_CLIENTS) return -EINVAL;
  if (cfg.policy > PAELLA_POLICY_RR || cfg.device > PAELLA_DEVICE_FAKE) return -EINVAL;
  if (cfg.group_size == 0) cfg.group_size = 16;
  if (cfg.group_size > 16) return -EINVAL;
  if (cfg.ring_capacity == 0) cfg.ring_capacity = 65536;
  if (cfg.ring_capacity & (cfg.ring_capacity - 1)) return -EINVAL;
  if (cfg.stream_pool == 0) cfg.stream_pool = 32;
  if (cfg.stream_pool > 1024) return -EINVAL;
  if (cfg.submit_slots == 0) cfg.submit_slots = 1024;
  if (cfg.submit_slots & (cfg.submit_slots - 1)) return -EINVAL;
  if (cfg.max_jobs_per_model == 0) cfg.max_jobs_per_model = 128;
  if (cfg.client_region_bytes == 0) cfg.client_region_bytes = 64ull << 20;
  if (cfg.fake_time_scale_ns == 0) cfg.fake_time_scale_ns = 500;
  if (cfg.fairness_threshold < 0) return -EINVAL;
  if (cfg.lookahead > 7) return -EINVAL;   // in-flight uid list per virtual stream: 8
  if (cfg.prio_classes == 0) cfg.prio_classes = 1;
  if (cfg.notify_mode > PAELLA_NOTIFY_RING) return -EINVAL;
  // counter mode: in-flight launches (<= P x (lookahead + 1)) must fit the slot table
  if (cfg.notify_mode == PAELLA_NOTIFY_COUNTERS &&
      (uint64_t)(cfg.stream_pool ? cfg.stream_pool : 32) * (cfg.lookahead + 1) >= NCTR_M)
    return -EINVAL;
  if (cfg.prio_classes > cfg.stream_pool && cfg.stream_pool != 0) return -EINVAL;
  if (cfg.launch_threads > 16) return -EINVAL;
  if (cfg.max_jobs_per_model > 4096) return -EINVAL;   // job ids: 65,536 per GPU
  if (cfg.fake_fault > PAELLA_FAULT_CORRUPT || cfg.branches > 1 || cfg.lookahead_unplaced > 1 ||
      cfg.cap_arrival_order > 1)
    return -EINVAL;

  auto P = std::make_unique<Paella>();
  P->cfg = cfg;
  if (cfg.device == PAELLA_DEVICE_CUDA) {
    // 32 hardware work queues (the default is 8) for every system, so
    // the stream pool's 32 streams map onto distinct queues.  Effective only if this
    // process has not initialised CUDA yet (an existing value is kept).
    setenv("CUDA_DEVICE_MAX_CONNECTIONS", "32", 0);
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess || n < (int)(cfg.first_gpu + cfg.num_gpus)) return -ENODEV;
    cudaDeviceProp prop;
    cudaGetDeviceProperties(&prop, cfg.first_gpu);
    if (prop.major != 10) return -ENODEV;
    P->sms = prop.multiProcessorCount;
    int smem_sm = prop.sharedMemPerMultiprocessor;
    P->capacity[0] = (int64_t)P->sms * prop.maxBlocksPerMultiProcessor;
    P->capacity[1] = (int64_t)P->sms * (prop.maxThreadsPerMultiProcessor / 32);
    P->capacity[2] = (int64_t)P->sms * prop.regsPerMultiprocessor;
    P->capacity[3] = (int64_t)P->sms * smem_sm;
    P->capacity[4] = (int64_t)P->sms * 512;
  } else {
    P->sms = cfg.fake_sms ? cfg.fake_sms : 148;
    int64_t per[NRES] = {32, 64, 65536, 233472, 512};
    for (int r = 0; r < NRES; ++r) P->capacity[r] = (int64_t)P->sms * per[r];
  }
  if (cfg.slack_blocks == 0) P->cfg.slack_blocks = P->sms;
  P->models.resize(256);

  // client channels: regions (page-locked and mapped into every GPU) and rings in one
  // shared mapping (P1030-1033: each client's shared memory region)
  P->region_bytes = cfg.client_region_bytes;
  if (int rc = channel_create(P.get())) return rc;
  for (uint32_t c = 0; c < cfg.num_clients; ++c) {
    uint8_t* r = P->ch.region(c);
    if (cfg.device == PAELLA_DEVICE_CUDA) {
      cudaSetDevice(cfg.first_gpu);
      if (cudaHostRegister(r, P->region_bytes, cudaHostRegisterPortable | cudaHostRegisterMapped) != cudaSuccess)
        return -ENOMEM;
    }
    P->region.push_back(r);
  }
  P->route_log.resize(cfg.num_clients);

  // NUMA placement: a GPU's pinned notification ring and counter
  // mirror are first touched by a thread running on that GPU's dispatcher core, so
  // they land on the dispatcher's (= the GPU's, when the caller picks NUMA-local
  // cores) memory node; the caller's affinity is restored afterwards
  cpu_set_t saved_mask;
  const bool numa_pin = cfg.dispatcher_cpus != nullptr &&
                        pthread_getaffinity_np(pthread_self(), sizeof saved_mask, &saved_mask) == 0;
  struct RestoreMask {
    bool on;
    cpu_set_t* m;
    ~RestoreMask() {
      if (on) pthread_setaffinity_np(pthread_self(), sizeof *m, m);
    }
  } restore{numa_pin, &saved_mask};
  for (uint32_t gi = 0; gi < cfg.num_gpus; ++gi) {
    if (numa_pin) {
      cpu_set_t cs;
      CPU_ZERO(&cs);
      CPU_SET(cfg.dispatcher_cpus[gi], &cs);
      pthread_setaffinity_np(pthread_self(), sizeof cs, &cs);
    }
    auto g = std::make_unique<Gpu>();
    g->P = P.get();
    g->index = gi;
    g->device = (int)(cfg.first_gpu + gi);
    g->cap = cfg.ring_capacity;
    g->log2cap = ilog2(cfg.ring_capacity);
    g->ctr_base.assign(NCTR, 0);
    g->overflow.resize(cfg.num_clients);
    // never reallocated: launcher threads hold pointers into job records
    g->jobs.reserve(65536);
    if (cfg.device == PAELLA_DEVICE_CUDA)
      g->be.reset(new CudaBackend(g->device, g->cap, cfg.stream_pool,
                                  cfg.no_proxy == 0 && !no_proxy_env(),
                                  cfg.no_proxy == 0 && cfg.notify_mode == PAELLA_NOTIFY_COUNTERS &&
                                      (!cfg.naive || naive_mirror_env()) && !no_proxy_env()));
    if (cfg.device == PAELLA_DEVICE_CUDA) {
      auto* cb = static_cast<CudaBackend*>(g->be.get());
      cb->pdl = (!cfg.naive || cfg.naive_pdl) && !cfg.no_pdl && !std::getenv("PAELLA_NO_PDL");
      cb->prio_classes = cfg.naive ? 1 : cfg.prio_classes;
      if (cb->mirror) {
        g->ctr_mode = true;
        g->ctr_mbase.assign(NCTR_M, 0);
        for (uint32_t sl = NCTR_M; sl-- > 0;) g->ctr_free.push_back(sl);
      }
    }
    else
      g->be.reset(new FakeBackend(P->sms, g->cap, g->log2cap, cfg.group_size, cfg.stream_pool,
                                  cfg.fake_time_scale_ns, gi == 0 ? cfg.fake_fault : 0u, cfg.fake_fault_arg));
    int rc = g->be->init();
    if (rc) return rc;
    Policy::Cfg pc;
    pc.num_clients = cfg.num_clients;
    pc.policy = cfg.policy;
    pc.theta = cfg.fairness_threshold;
    pc.slack = P->cfg.slack_blocks;
    pc.group = cfg.group_size;
    pc.ring_capacity = cfg.ring_capacity;
    pc.streams = cfg.stream_pool;
    pc.lookahead = cfg.lookahead;
    pc.prio_classes = cfg.naive ? 1 : cfg.prio_classes;
    pc.online_tbar = cfg.online_tbar;
    pc.max_active = cfg.max_active_jobs;
    pc.la_unplaced = cfg.lookahead_unplaced ? 1u : 0u;
    pc.cap_fifo = cfg.cap_arrival_order ? 1u : 0u;
    for (int r = 0; r < NRES; ++r) pc.capacity[r] = P->capacity[r];
    if (cfg.device == PAELLA_DEVICE_CUDA &&
        (static_cast<CudaBackend*>(g->be.get())->proxy || static_cast<CudaBackend*>(g->be.get())->mirror)) {
      // the resident proxy / mirror warp: 1 block, 1 warp, its registers, the 1 KB reservation
      const int64_t proxy[NRES] = {1, 1, 160 * 32, 1024, 0};   // mirror warp: <= 160 regs/thread
      for (int r = 0; r < NRES; ++r) pc.capacity[r] -= proxy[r];
    }
    g->policy.reset(new Policy(pc));
    g->pub = &P->ch.hdr->gpu[gi];
    for (uint32_t c = 0; c < cfg.num_clients; ++c) {
      g->sub.push_back(P->ch.sub(gi, c));
      g->done.push_back(P->ch.done(gi, c));
    }
    if (cfg.event_log_path) {
      char path[4096];
      snprintf(path, sizeof path, cfg.event_log_path, gi);
      g->log = fopen(path, "wb");
      g->log_times = std::getenv("PAELLA_TRACE_TIMES") != nullptr;
      if (!g->log) return -EINVAL;
      setvbuf(g->log, nullptr, _IOFBF, 1 << 20);
      logev(g.get(), EV_CONFIG, cfg.num_clients, cfg.policy, (uint64_t)cfg.fairness_threshold,
            ((uint64_t)P->cfg.slack_blocks << 32) | cfg.group_size);
      logev(g.get(), EV_CONFIG + 0, 0xFFFFFFFFu, cfg.ring_capacity, cfg.stream_pool,
            ((uint64_t)pc.prio_classes << 32) | cfg.lookahead);
      logev(g.get(), EV_CONFIG + 0, 0xFFFFFFFEu, cfg.online_tbar, cfg.max_active_jobs,
            cfg.branches | ((uint64_t)(cfg.lookahead_unplaced ? 1 : 0) << 8) |
                ((uint64_t)(cfg.cap_arrival_order ? 1 : 0) << 9));
      for (int r = 0; r < NRES; ++r) logev(g.get(), EV_CAPACITY, (uint32_t)r, (uint64_t)pc.capacity[r], 0, 0);
    }
    if (cfg.device == PAELLA_DEVICE_CUDA &&
        clock_sync(g.get(), 32, &g->clk_offset, &g->clk_rtt, &g->clk_res, &g->clk_at) == 0)
      logev(g.get(), EV_CLOCK, gi | ((uint32_t)std::min<int64_t>(g->clk_res, 0xFFFFFF) << 8), (uint64_t)g->clk_offset,
            (uint64_t)g->clk_rtt, (uint64_t)g->clk_at);
    P->gpus.push_back(std::move(g));
  }
  if (numa_pin) {
    pthread_setaffinity_np(pthread_self(), sizeof saved_mask, &saved_mask);
    restore.on = false;
  }
  for (auto& g : P->gpus) {
    if (cfg.device == PAELLA_DEVICE_CUDA && cfg.launch_threads > 0) {
      for (uint32_t i = 0; i < cfg.launch_threads; ++i) {
        auto L = std::make_unique<Launcher>();
        L->q.init(8192);
        g->launchers.push_back(std::move(L));
      }
      for (auto& L : g->launchers) L->th = std::thread(launcher_main, g.get(), L.get());
    }
    if (cfg.device == PAELLA_DEVICE_CUDA && std::getenv("PAELLA_LAUNCH_NOISE_US")) {
      // diagnosis: host launches during kernel execution -- an empty 1-block kernel on its
      // own stream every N us until shutdown
      const int64_t period = (int64_t)(atof(std::getenv("PAELLA_LAUNCH_NOISE_US")) * 1000);
      const int burst = std::getenv("PAELLA_LAUNCH_NOISE_BURST") ? atoi(std::getenv("PAELLA_LAUNCH_NOISE_BURST")) : 1;
      Gpu* gp = g.get();
      gp->noise = std::thread([gp, period, burst] {
        cudaSetDevice(gp->device);
        cudaStream_t s;
        cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
        auto* cb = static_cast<CudaBackend*>(gp->be.get());
        KernelFn f = cb->fn(KIND_EMPTY, 0, false);
        LayerArgs la{};
        InstrArgs ia{};
        void* args[2] = {(void*)&la, (void*)&ia};
        int64_t next = now_ns();
        while (!gp->launchers_stop.load(std::memory_order_acquire) && !gp->stop.load(std::memory_order_acquire)) {
          for (int b = 0; b < burst; ++b) cudaLaunchKernel((const void*)f, dim3(1), dim3(32), args, 0, s);
          next += period;
          while (now_ns() < next) {
          }
        }
        cudaStreamSynchronize(s);
        cudaStreamDestroy(s);
      });
    }
    g->thread = std::thread(dispatcher_main, g.get());
  }
  *out = (paella_t*)P.release();
  return 0;
}

int paella_client_region(paella_t* p, uint32_t client_id, void** base, size_t* bytes) {
  Paella* P = (Paella*)p;
  if (!P || client_id >= P->cfg.num_clients) return -EINVAL;
  if (base) *base = P->region[client_id];
  if (bytes) *bytes = P->region_bytes;
  return 0;
}

int paella_register_model(paella_t* p, const paella_model_desc_t* desc, uint32_t* model_id) {
  Paella* P = (Paella*)p;
  if (!P || !desc || !desc->name) return -EINVAL;
  std::lock_guard<std::mutex> lk(P->reg_mu);
  uint32_t nm = P->nmodels.load();
  for (uint32_t i = 0; i < nm; ++i)
    if (P->models[i]->name == desc->name) return -EEXIST;
  if (nm >= P->models.size()) return -ENOMEM;
  auto m = std::make_unique<Model>();
  m->id = nm;
  int rc = plan_model(P, desc, m.get());
  if (rc) return rc;
  for (auto& k : m->kernels) {
    if (2ull * ((k.grid_total() + P->cfg.group_size - 1) / P->cfg.group_size) > P->cfg.ring_capacity)
      return -EINVAL;
  }
  m->gpu.resize(P->gpus.size());
  for (auto& g : P->gpus) {
    rc = setup_model_gpu(P, m.get(), g.get());
    if (rc) return rc;
  }
  // policy tables + log (identical T-bar on every GPU: profiled on GPU 0)
  std::vector<PolicyLayer> layers;
  m->total_tbar = 0;
  for (auto& k : m->kernels) {
    PolicyLayer L;
    L.grid = k.grid_total();
    for (int r = 0; r < NRES; ++r) L.demand[r] = k.demand[r];
    L.tbar = k.tbar;
    if (P->cfg.branches) {   // NEXT-4: virtual streams; else the chain of the paper's jobs
      L.vs = k.vs;
      for (uint32_t d : k.deps)
        if (m->kernels[d].vs != k.vs) L.cross.push_back(d);
    }
    m->total_tbar += k.tbar;
    layers.push_back(L);
  }
  Model* mp = m.get();
  P->models[nm] = std::move(m);
  // each dispatcher adds the model to its own policy on its own thread (apply_inbox);
  // the model is published (nmodels) once every dispatcher has it
  for (auto& g : P->gpus) {
    std::lock_guard<std::mutex> lk2(g->inbox_mu);
    g->inbox.emplace_back(nm, layers);
    g->inbox_n.fetch_add(1, std::memory_order_release);
  }
  for (auto& g : P->gpus)
    while (g->models_applied.load(std::memory_order_acquire) < nm + 1) {
      if (g->stop.load(std::memory_order_acquire)) return -ESHUTDOWN;
      std::this_thread::yield();
    }
  (void)mp;
  if (nm >= SHM_MAX_MODELS) return -ENOMEM;
  ModelPub& pubm = P->ch.hdr->models[nm];   // io sizes and T-bar for every client process
  pubm.input_bytes = mp->input_bytes;
  pubm.output_bytes = mp->output_bytes;
  pubm.total_tbar = mp->total_tbar;
  P->nmodels.store(nm + 1, std::memory_order_release);
  P->ch.hdr->nmodels.store(nm + 1, std::memory_order_release);
  if (model_id) *model_id = nm;
  return 0;
}

int paella_route_pair(uint64_t req_id, uint32_t num_gpus, uint32_t* g0, uint32_t* g1) {
  if (num_gpus == 0 || num_gpus > PAELLA_MAX_GPUS || !g0 || !g1) return -EINVAL;
  uint64_t z = req_id + 0x9E3779B97F4A7C15ull;   // splitmix64, one step from state req_id
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  z ^= z >> 31;
  if (num_gpus == 1) {
    *g0 = *g1 = 0;
    return 0;
  }
  *g0 = (uint32_t)(z % num_gpus);
  *g1 = (uint32_t)((*g0 + 1 + (z >> 32) % (num_gpus - 1)) % num_gpus);
  return 0;
}

static int64_t submit_impl(Paella* P, uint32_t client_id, uint32_t model_id, void* io, size_t len, uint32_t flags,
                           int64_t t_sched) {
  if (!P) return -EINVAL;
  if (client_id >= P->cfg.num_clients) return -EINVAL;
  return channel_submit(P->ch, client_id, model_id, io, len, flags, t_sched,
                        P->cfg.route_log_path && P->gpus.size() > 1 ? &P->route_log[client_id] : nullptr);
}

int64_t paella_submit(paella_t* p, uint32_t client_id, uint32_t model_id, void* io, size_t len, uint32_t flags) {
  return submit_impl((Paella*)p, client_id, model_id, io, len, flags, now_ns());
}

int64_t paella_submit_at(paella_t* p, uint32_t client_id, uint32_t model_id, void* io, size_t len, uint32_t flags,
                         int64_t t_sched_ns) {
  return submit_impl((Paella*)p, client_id, model_id, io, len, flags, t_sched_ns);
}

int64_t paella_poll_completion(paella_t* p, uint32_t client_id, uint32_t flags, int32_t* status) {
  Paella* P = (Paella*)p;
  if (!P || client_id >= P->cfg.num_clients) return -EINVAL;
  return channel_poll(P->ch, client_id, flags, status);
}

int paella_channel_path(paella_t* p, char* buf, size_t n) {
  Paella* P = (Paella*)p;
  if (!P || !buf || n == 0 || P->shm_fd < 0) return -EINVAL;
  const int k = snprintf(buf, n, "/proc/%d/fd/%d", (int)getpid(), P->shm_fd);
  return k > 0 && (size_t)k < n ? 0 : -ENAMETOOLONG;
}

// routing log of every client (cfg.route_log_path), rewritten in full
static int write_route_logs(Paella* P) {
  if (!P->cfg.route_log_path) return 0;
  for (uint32_t c = 0; c < P->route_log.size(); ++c) {
    char path[4096];
    snprintf(path, sizeof path, P->cfg.route_log_path, c);
    FILE* f = fopen(path, "wb");
    if (!f) return -EINVAL;
    const auto& v = P->route_log[c];
    if (!v.empty()) fwrite(v.data(), sizeof(paella_route_rec_t), v.size(), f);
    fclose(f);
  }
  return 0;
}

int paella_shutdown(paella_t* p) {
  Paella* P = (Paella*)p;
  if (!P) return -EINVAL;
  P->ch.hdr->shutting.store(1, std::memory_order_release);
  for (auto& g : P->gpus) g->stop.store(true, std::memory_order_release);
  for (auto& g : P->gpus)
    if (g->thread.joinable()) g->thread.join();
  for (auto& g : P->gpus) {
    g->launchers_stop.store(true, std::memory_order_release);
    for (auto& L : g->launchers)
      if (L->th.joinable()) L->th.join();
    if (g->noise.joinable()) g->noise.join();
    if (launch_stats_env()) launch_stats_print(g.get());
    if (P->cfg.device == PAELLA_DEVICE_CUDA) {
      cudaSetDevice(g->device);
      static_cast<CudaBackend*>(g->be.get())->stop_proxy();
      g->be->sync();
      if (g->prof_stream) {   // isolated-run resources (ensure_iso)
        cudaStreamSynchronize((cudaStream_t)g->prof_stream);
        cudaStreamDestroy((cudaStream_t)g->prof_stream);
        g->prof_stream = nullptr;
        cudaFreeHost(g->prof_ring_h);
        cudaFreeHost(g->stage_in);
        cudaFree(g->prof_tail);
        cudaFree(g->prof_ctr);
        cudaFree(g->prof_devring);
        cudaFree(g->trace_buf);
      }
      if (g->flush_buf) cudaFree(g->flush_buf);
    }
  }
  write_route_logs(P);
  // requests never admitted complete with -ECANCELED
  for (auto& g : P->gpus) {
    flush_overflow(g.get());
    for (uint32_t c = 0; c < P->cfg.num_clients; ++c) {
      const SubmitSlot* s;
      while ((s = g->sub[c]->peek()) != nullptr) {
        CompleteSlot cs{};
        cs.req_id = s->req_id;
        cs.status = -ECANCELED;
        g->done[c]->push(cs);
        g->sub[c]->pop();
      }
    }
    if (g->log) {
      fclose(g->log);
      g->log = nullptr;
    }
  }
  for (uint32_t i = 0; i < P->nmodels.load(); ++i) {
    Model* m = P->models[i].get();
    for (size_t gi = 0; gi < P->gpus.size(); ++gi) {
      if (P->cfg.device == PAELLA_DEVICE_CUDA) {
        cudaSetDevice(P->gpus[gi]->device);
        cudaFree(m->gpu[gi].weights);
        cudaFree(m->gpu[gi].workspace);
        if (m->gpu[gi].splitk_iso) cudaFree(m->gpu[gi].splitk_iso);
        if (m->gpu[gi].splitk_slots) cudaFree(m->gpu[gi].splitk_slots);
        if (m->gpu[gi].bmaps) cudaFree(m->gpu[gi].bmaps);
      } else {
        free(m->gpu[gi].weights);
        free(m->gpu[gi].workspace);
      }
    }
  }
  if (P->cfg.device == PAELLA_DEVICE_CUDA)
    for (auto* r : P->region) cudaHostUnregister(r);
  P->gpus.clear();
  munmap(P->ch.base, P->shm_bytes);
  if (P->shm_fd >= 0) close(P->shm_fd);
  delete P;
  return 0;
}

int paella_flush_log(paella_t* p) {
  Paella* P = (Paella*)p;
  if (!P) return -EINVAL;
  for (auto& g : P->gpus)
    if (g->log) fflush(g->log);
  return write_route_logs(P);
}

int paella_model_info(paella_t* p, uint32_t model_id, paella_model_info_t* info) {
  Paella* P = (Paella*)p;
  if (!P || !info || model_id >= P->nmodels.load()) return -EINVAL;
  Model* m = P->models[model_id].get();
  info->n_kernels = (uint32_t)m->kernels.size();
  info->input_bytes = m->input_bytes;
  info->output_bytes = m->output_bytes;
  info->weight_bytes = m->blob.size();
  info->total_tbar_ns = m->total_tbar;
  return 0;
}

int paella_kernel_info(paella_t* p, uint32_t model_id, uint32_t k, paella_kernel_info_t* info) {
  Paella* P = (Paella*)p;
  if (!P || !info || model_id >= P->nmodels.load()) return -EINVAL;
  Model* m = P->models[model_id].get();
  if (k >= m->kernels.size()) return -EINVAL;
  const KernelInst& ki = m->kernels[k];
  info->grid = ki.grid_total();
  info->block = ki.block;
  info->smem = ki.smem + ki.static_smem;
  info->regs = ki.regs;
  info->tmem_cols = ki.tmem_cols;
  info->kind = ki.kind;
  info->tbar_ns = ki.tbar;
  info->flops = ki.flops;
  info->bytes = ki.bytes;
  info->vs = ki.vs;
  info->n_deps = (uint32_t)ki.deps.size();
  for (uint32_t i = 0; i < ki.deps.size() && i < 8; ++i) info->deps[i] = ki.deps[i];
  return 0;
}

const char* paella_kernel_name(uint32_t kind) {
  static const char* names[] = {"ingest", "conv_simt", "conv_tcgen05", "dwconv", "maxpool",
                                "avgpool", "gap", "fc_gemv", "empty", "conv_tcgen05_pro", "gap_fc", "spin",
                                "conv_tcgen05_n128", "conv_tcgen05_m64"};
  return kind < KIND_COUNT ? names[kind] : "?";
}

int paella_check_counters(paella_t* p, uint32_t gpu, uint32_t* slots_checked) {
  Paella* P = (Paella*)p;
  if (!P || gpu >= P->gpus.size()) return -EINVAL;
  if (P->cfg.device != PAELLA_DEVICE_CUDA) return -ENODEV;
  Gpu* g = P->gpus[gpu].get();
  if (!g->ctr_mode) return -ENOTSUP;
  if (g->policy->live_jobs() != 0 || !g->ctr_live.empty()) return -EBUSY;
  auto* cb = static_cast<CudaBackend*>(g->be.get());
  std::vector<uint32_t> dev(NCTR_SUB * 2 * NCTR_M), mir(NCTR_SUB * 2 * NCTR_M);
  cudaSetDevice(g->device);
  if (cudaMemcpy(dev.data(), cb->ctr_m, dev.size() * 4, cudaMemcpyDeviceToHost) != cudaSuccess) return -EIO;
  std::memcpy(mir.data(), (const void*)cb->mirror_h, mir.size() * 4);
  int bad = 0;
  uint32_t used = 0;
  for (uint32_t s = 0; s < NCTR_M; ++s) {
    const uint32_t want = g->ctr_mbase[s];   // sum of the grids of every launch counted on slot s
    if (want) ++used;
    uint32_t d0 = 0, d1 = 0;
    for (uint32_t t = 0; t < NCTR_SUB; ++t) {
      d0 += dev[t * 2 * NCTR_M + 2 * s];
      d1 += dev[t * 2 * NCTR_M + 2 * s + 1];
    }
    const uint32_t m0 = mir[2 * s], m1 = mir[2 * s + 1];   // the mirror holds the sums
    // device counters AND their host mirror: every block entered and exited exactly once
    if (d0 != want || d1 != want || m0 != want || m1 != want) ++bad;
  }
  if (slots_checked) *slots_checked = used;
  return bad;
}

int paella_clock_sync(paella_t* p, uint32_t gpu) {
  Paella* P = (Paella*)p;
  if (!P || gpu >= P->gpus.size()) return -EINVAL;
  if (P->cfg.device != PAELLA_DEVICE_CUDA) return -ENODEV;
  Gpu* g = P->gpus[gpu].get();
  int64_t off, rtt, res, at;
  int rc = clock_sync(g, 32, &off, &rtt, &res, &at);
  if (rc) return rc;
  {
    std::lock_guard<std::mutex> lk(g->inbox_mu);   // applied by the dispatcher thread (log order)
    g->clk_pending = true;
    g->clk_new[0] = off;
    g->clk_new[1] = rtt;
    g->clk_new[2] = res;
    g->clk_new[3] = at;
  }
  const uint64_t seen = g->clk_applied.load(std::memory_order_acquire);
  g->clk_req.fetch_add(1, std::memory_order_release);
  while (g->clk_applied.load(std::memory_order_acquire) == seen) {
    if (g->stop.load(std::memory_order_acquire)) return -ESHUTDOWN;
    std::this_thread::yield();
  }
  return 0;
}

int paella_clock_info(paella_t* p, uint32_t gpu, int64_t* offset_ns, int64_t* rtt_ns, int64_t* resolution_ns) {
  Paella* P = (Paella*)p;
  if (!P || gpu >= P->gpus.size()) return -EINVAL;
  if (P->cfg.device != PAELLA_DEVICE_CUDA) return -ENODEV;
  Gpu* g = P->gpus[gpu].get();
  if (g->clk_rtt < 0) return -ENOTSUP;
  if (offset_ns) *offset_ns = g->clk_offset;
  if (rtt_ns) *rtt_ns = g->clk_rtt;
  if (resolution_ns) *resolution_ns = g->clk_res;
  return 0;
}

int paella_stats(paella_t* p, uint32_t gpu, paella_stats_t* st) {
  Paella* P = (Paella*)p;
  if (!P || !st || gpu >= P->gpus.size()) return -EINVAL;
  Gpu* g = P->gpus[gpu].get();
  // ask the dispatcher thread for a snapshot (apply_inbox runs every 64 loop iterations)
  // unless it has finished; a thread that was never started has written nothing
  if (g->thread.joinable() && !g->loop_done.load(std::memory_order_acquire)) {
    const uint64_t seen = g->st_ack.load(std::memory_order_acquire);
    g->st_req.fetch_add(1, std::memory_order_release);
    while (g->st_ack.load(std::memory_order_acquire) == seen && !g->loop_done.load(std::memory_order_acquire))
      std::this_thread::yield();
  }
  if (g->loop_done.load(std::memory_order_acquire) || !g->thread.joinable()) {
    *st = g->stats;
  } else {
    std::lock_guard<std::mutex> lk(g->st_mu);
    *st = g->st_snap;
  }
  st->outstanding_work_ns = g->pub->work.load();
  return 0;
}

}  // extern "C"

// ===========================================================================
// per-GPU model setup, isolated runs, profiling
// ===========================================================================
namespace paella {

static int ensure_iso(Gpu* g) {
  if (g->prof_ring_h) return 0;
  const uint32_t cap = 1u << 16;
  if (cudaSetDevice(g->device) != cudaSuccess) return -EIO;
  if (cudaHostAlloc((void**)&g->prof_ring_h, cap * sizeof(Rec), cudaHostAllocMapped | cudaHostAllocPortable))
    return -ENOMEM;
  std::memset(g->prof_ring_h, 0, cap * sizeof(Rec));
  cudaHostGetDevicePointer(&g->prof_ring_d, g->prof_ring_h, 0);
  if (cudaMalloc(&g->prof_tail, 256) || cudaMalloc(&g->prof_ctr, NCTR_SUB * 2 * NCTR * sizeof(uint32_t))) return -ENOMEM;
  g->prof_base.assign(NCTR, 0);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  g->prof_stream = s;
  cudaMemsetAsync(g->prof_tail, 0, 256, s);
  cudaMemsetAsync(g->prof_ctr, 0, NCTR_SUB * 2 * NCTR * sizeof(uint32_t), s);
  // isolated runs write their records to device memory (as served kernels do through
  // the proxy); nobody consumes them except the round-trip benchmark's direct ring
  if (cudaMalloc(&g->prof_devring, cap * sizeof(Rec))) return -ENOMEM;
  cudaMemsetAsync(g->prof_devring, 0, cap * sizeof(Rec), s);
  if (cudaMalloc(&g->trace_buf, 16 * 8 * 8192)) return -ENOMEM;
  g->stage_bytes = 16u << 20;
  if (cudaHostAlloc(&g->stage_in, g->stage_bytes, cudaHostAllocMapped | cudaHostAllocPortable)) return -ENOMEM;
  return cudaStreamSynchronize(s) == cudaSuccess ? 0 : -EIO;
}

// the ring isolated runs write to: device memory when served kernels go through the
// notification proxy (same cost as in serving), else the pinned host ring
static Rec* iso_ring(Gpu* g) {
  auto* cb = static_cast<CudaBackend*>(g->be.get());
  return cb->proxy ? g->prof_devring : (Rec*)g->prof_ring_d;
}

// launch kernel `l` of model m from the isolated slot on the profiling stream
static InstrArgs iso_instr(Gpu* g, uint32_t grid, uint32_t group, bool last);

static void iso_launch(Gpu* g, Model* m, uint32_t l, bool instr) {
  const KernelInst& k = m->kernels[l];
  InstrArgs ia = iso_instr(g, k.grid_total(), g->P->cfg.group_size, l + 1 == m->kernels.size());
  uint32_t iso_slot = (uint32_t)m->gpu[g->index].args.size() - 1;
  auto* cb = static_cast<CudaBackend*>(g->be.get());
  const void* tm = is_tc(k.kind) ? m->gpu[g->index].tmaps[l].b : nullptr;
  void* args[3] = {(void*)&m->gpu[g->index].args[iso_slot][l], (void*)&ia, (void*)tm};
  cuda_launch(cb->fn(k.kind, m->dtype, instr), k, args, (cudaStream_t)g->prof_stream, cb->pdl);
}

static int iso_run(Gpu* g, Model* m, const void* input, void* output, int64_t* kernel_ns, bool instr) {
  int rc = ensure_iso(g);
  if (rc) return rc;
  cudaSetDevice(g->device);
  uint8_t* st = (uint8_t*)g->stage_in;
  if (m->input_bytes + m->output_bytes > g->stage_bytes) return -ENOMEM;
  if (input) std::memcpy(st, input, m->input_bytes);
  std::memset(st + m->input_bytes, 0, m->output_bytes);
  ModelGpu& mg = m->gpu[g->index];
  auto& args = mg.args.back();
  args.front().in = st;
  args.back().out = st + m->input_bytes;
  cudaStream_t s = (cudaStream_t)g->prof_stream;
  std::vector<cudaEvent_t> ev;
  volatile uint32_t* gate = (volatile uint32_t*)(st + g->stage_bytes - 64);
  if (kernel_ns) {
    // gate the stream so the chain runs back to back: events then time the device,
    // not the host's launch rate
    *gate = 0;
    const volatile uint32_t* gd = nullptr;
    cudaHostGetDevicePointer((void**)&gd, (void*)gate, 0);
    void* gargs[1] = {(void*)&gd};
    if (!no_gate())
      cudaLaunchKernel((const void*)gate_kernel(), dim3(1), dim3(1), gargs, 0, s);
    ev.resize(m->kernels.size() + 1);
    for (auto& e : ev) cudaEventCreate(&e);
    cudaEventRecord(ev[0], s);
  }
  // debug: PAELLA_TRACE_KERNEL=<k> -> per-CTA phase timestamps of tcgen05 conv k
  int trace_k = std::getenv("PAELLA_TRACE_KERNEL") ? atoi(std::getenv("PAELLA_TRACE_KERNEL")) : -1;
  uint64_t* trbuf = nullptr;
  LayerArgs saved{};
  if (trace_k >= 0 && trace_k < (int)m->kernels.size() &&
      (is_tc(m->kernels[trace_k].kind) || m->kernels[trace_k].kind == KIND_GAPFC)) {
    trbuf = (uint64_t*)g->trace_buf;
    cudaMemsetAsync(trbuf, 0, 16 * 8 * m->kernels[trace_k].grid_total(), s);
    saved = args[trace_k];
    args[trace_k].flags |= LF_TRACE;
    args[trace_k].trace = trbuf;
  } else {
    trace_k = -1;
  }
  for (uint32_t l = 0; l < m->kernels.size(); ++l) {
    iso_launch(g, m, l, instr);
    if (kernel_ns) cudaEventRecord(ev[l + 1], s);
  }
  if (kernel_ns) {
    std::atomic_thread_fence(std::memory_order_seq_cst);
    *gate = 1;
  }
  cudaError_t e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) {
    fprintf(stderr, "paella: isolated run failed: %s\n", cudaGetErrorString(e));
    return -EIO;
  }
  if (trace_k >= 0) {
    cudaStreamSynchronize(s);
    uint32_t nb = m->kernels[trace_k].grid_total();
    std::vector<uint64_t> h(16 * nb);
    cudaMemcpyAsync(h.data(), trbuf, h.size() * 8, cudaMemcpyDeviceToHost, s);
    cudaStreamSynchronize(s);
    args[trace_k] = saved;
    uint64_t t0 = UINT64_MAX;
    for (uint32_t b = 0; b < nb; ++b) t0 = std::min(t0, h[16 * b]);
    const bool head = m->kernels[trace_k].kind == KIND_GAPFC;
    const char* names_tc[16] = {"entry", "setup", "full0", "mma_done", "accb", "epi_done", "pre_exit", "exit",
                                "tmem2smem", "pre_bar", "post_bar", "inited", "tma_issued", "b_issued", "reduced", "peers01"};
    const char* names_head[16] = {"entry", "pdl_done", "pooled", "bar1", "gathered", "fc_done", "stored", "exit",
                                  "-", "-", "-", "-", "-", "-", "-", "-"};
    const char* const* names = head ? names_head : names_tc;
    fprintf(stderr, "trace kernel %d grid %u (ns from first CTA entry): phase min/med/max\n", trace_k, nb);
    const int order_tc[16] = {0, 11, 12, 13, 1, 2, 3, 4, 8, 9, 10, 15, 14, 5, 6, 7};
    const int order_head[16] = {0, 1, 2, 3, 4, 5, 6, 7, 8, 8, 8, 8, 8, 8, 8, 8};
    const int* order = head ? order_head : order_tc;
    for (int oi = 0; oi < 16; ++oi) {
      int ph = order[oi];
      std::vector<int64_t> v;
      for (uint32_t b = 0; b < nb; ++b)
        if (h[16 * b + ph]) v.push_back((int64_t)(h[16 * b + ph] - t0));
      if (v.empty()) continue;
      std::sort(v.begin(), v.end());
      fprintf(stderr, "  %-9s %7lld %7lld %7lld\n", names[ph], (long long)v.front(), (long long)v[v.size() / 2],
              (long long)v.back());
    }
  }
  if (kernel_ns) {
    for (uint32_t l = 0; l < m->kernels.size(); ++l) {
      float ms = 0;
      cudaEventElapsedTime(&ms, ev[l], ev[l + 1]);
      kernel_ns[l] = (int64_t)((double)ms * 1e6);
    }
    for (auto& x : ev) cudaEventDestroy(x);
  }
  if (output) std::memcpy(output, st + m->input_bytes, m->output_bytes);
  return 0;
}

static volatile uint32_t* gate_ptr(Gpu* g, const volatile uint32_t** dev);
static void launch_gate(Gpu* g, const volatile uint32_t* gd);
static InstrArgs iso_instr(Gpu* g, uint32_t grid, uint32_t group, bool last);

// Device time of kernel l: `reps` back-to-back launches of it (PDL, as served) behind a
// gate on the profiling stream, timed with CUDA events; ns per launch, -1 on error.
static int64_t time_layer(Gpu* g, Model* m, uint32_t l, bool instr, uint32_t reps) {
  cudaSetDevice(g->device);
  cudaStream_t s = (cudaStream_t)g->prof_stream;
  auto* cb = static_cast<CudaBackend*>(g->be.get());
  const uint32_t iso_slot = (uint32_t)m->gpu[g->index].args.size() - 1;
  const KernelInst& k = m->kernels[l];
  reps = std::min(reps, 256u);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const volatile uint32_t* gd;
  volatile uint32_t* gate = gate_ptr(g, &gd);
  *gate = 0;
  launch_gate(g, gd);
  cudaEventRecord(e0, s);
  const void* tm = is_tc(k.kind) ? m->gpu[g->index].tmaps[l].b : nullptr;
  for (uint32_t r = 0; r < reps; ++r) {
    InstrArgs ia = iso_instr(g, k.grid_total(), g->P->cfg.group_size, l + 1 == m->kernels.size());
    void* args[3] = {(void*)&m->gpu[g->index].args[iso_slot][l], (void*)&ia, (void*)tm};
    cuda_launch(cb->fn(k.kind, m->dtype, instr), k, args, s, cb->pdl);
  }
  cudaEventRecord(e1, s);
  std::atomic_thread_fence(std::memory_order_seq_cst);
  *gate = 1;
  int64_t ns = -1;
  if (cudaStreamSynchronize(s) == cudaSuccess) {
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    ns = (int64_t)((double)ms * 1e6 / reps);
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  return ns;
}

// L2-cold device time of kernel l (L2-cold vs L2-warm): before each of
// `reps` launches a 2 x L2-sized buffer is overwritten on the same stream (the kernel's
// weights and inputs are evicted), and only the kernel itself is timed (events around
// each launch); ns per launch (median), -1 on error.
static int64_t time_layer_cold(Gpu* g, Model* m, uint32_t l, bool instr, uint32_t reps) {
  cudaSetDevice(g->device);
  cudaStream_t s = (cudaStream_t)g->prof_stream;
  auto* cb = static_cast<CudaBackend*>(g->be.get());
  const uint32_t iso_slot = (uint32_t)m->gpu[g->index].args.size() - 1;
  const KernelInst& k = m->kernels[l];
  const size_t flush_bytes = 256ull << 20;
  if (!g->flush_buf && cudaMalloc(&g->flush_buf, flush_bytes) != cudaSuccess) return -1;
  reps = std::min(reps, 64u);
  std::vector<cudaEvent_t> ev(2 * reps);
  for (auto& e : ev) cudaEventCreate(&e);
  const void* tm = is_tc(k.kind) ? m->gpu[g->index].tmaps[l].b : nullptr;
  for (uint32_t r = 0; r < reps; ++r) {
    cudaMemsetAsync(g->flush_buf, (int)(r & 0xff), flush_bytes, s);
    InstrArgs ia = iso_instr(g, k.grid_total(), g->P->cfg.group_size, l + 1 == m->kernels.size());
    void* args[3] = {(void*)&m->gpu[g->index].args[iso_slot][l], (void*)&ia, (void*)tm};
    cudaEventRecord(ev[2 * r], s);
    cuda_launch(cb->fn(k.kind, m->dtype, instr), k, args, s, false);
    cudaEventRecord(ev[2 * r + 1], s);
  }
  int64_t ns = -1;
  if (cudaStreamSynchronize(s) == cudaSuccess) {
    std::vector<int64_t> t(reps);
    for (uint32_t r = 0; r < reps; ++r) {
      float ms = 0;
      cudaEventElapsedTime(&ms, ev[2 * r], ev[2 * r + 1]);
      t[r] = (int64_t)((double)ms * 1e6);
    }
    std::nth_element(t.begin(), t.begin() + reps / 2, t.end());
    ns = t[reps / 2];
  }
  for (auto& e : ev) cudaEventDestroy(e);
  return ns;
}

// Split-K autotuning of the tcgen05 convs (GPU 0, at registration, before T-bar is
// profiled): every admissible split (power of two, <= 16 = the cluster limit, >= 1
// k-block per split, <= one wave at 2 CTAs/SM) is timed as served (instrumented, PDL
// chain) with each split-K reduction (in L2, or over DSMEM: neither wins on every layer,
// profiles/r2/splitk_*); a larger split must win by >= 5 % (it occupies more SMs under
// load).  PAELLA_SPLITS_FILE: a cache of the choices ("model layer split [dsmem]"
// lines): read if it exists (profiling runs reuse the served configuration without
// re-timing), appended to otherwise.
static int autotune_splits(Gpu* g, Model* m) {
  if (std::getenv("PAELLA_NO_AUTOTUNE") || std::getenv("PAELLA_NOSPLIT")) return 0;
  auto& mg = m->gpu[g->index];
  const char* cache = std::getenv("PAELLA_SPLITS_FILE");
  if (cache) {
    if (FILE* f = std::fopen(cache, "r")) {
      char line[512], name[256];
      unsigned l, sp, dsm;
      bool any = false;
      while (std::fgets(line, sizeof line, f)) {
        const int n = std::sscanf(line, "%255s %u %u %u", name, &l, &sp, &dsm);
        if (n < 3) continue;
        if (m->name != name || l >= m->kernels.size() || !is_tc(m->kernels[l].kind)) continue;
        if (m->kernels[l].kind == KIND_CONV_TC128) continue;   // 128-pixel tiles never split
        KernelInst& k = m->kernels[l];
        const uint32_t fl = (n == 4 && dsm) ? (k.proto.flags | LF_SPLIT_DSMEM) : (k.proto.flags & ~LF_SPLIT_DSMEM);
        k.proto.ksplit = sp;
        k.proto.flags = fl;
        k.grid[2] = sp;
        for (auto& A : mg.args) {
          A[l].ksplit = sp;
          A[l].flags = fl;
        }
        any = true;
      }
      std::fclose(f);
      if (any) return 0;
    }
  }
  if (iso_run(g, m, nullptr, nullptr, nullptr, true)) return -EIO;
  for (uint32_t l = 0; l < m->kernels.size(); ++l) {
    KernelInst& k = m->kernels[l];
    if (!is_tc(k.kind) || k.kind == KIND_CONV_TC128) continue;   // 128-pixel tiles never split
    const uint32_t nk = k.proto.kpad / TC_BK, tiles = k.proto.tiles_m * k.proto.tiles_n;
    auto set = [&](uint32_t sp, bool dsm) {
      k.proto.ksplit = sp;
      k.proto.flags = dsm ? (k.proto.flags | LF_SPLIT_DSMEM) : (k.proto.flags & ~LF_SPLIT_DSMEM);
      k.grid[2] = sp;
      for (auto& A : mg.args) {
        A[l].ksplit = sp;
        A[l].flags = k.proto.flags;
      }
    };
    const uint32_t orig = k.proto.ksplit;
    // PAELLA_SPLIT_DSMEM forces the DSMEM reduction, PAELLA_SPLIT_L2 the L2 one
    const bool only_dsm = std::getenv("PAELLA_SPLIT_DSMEM") != nullptr, only_l2 = std::getenv("PAELLA_SPLIT_L2") != nullptr;
    // a doubled split must beat the best so far by this factor (percent of its time):
    // it doubles the CTAs (device work) of the layer, which serving under load pays for.
    // Measured on the C-3 bench (profiles/r2/diag/split_gain): 95 % -> 65 % raises X_dev
    // 11.4 k -> 15.8 k req/s and req/s at the p99 SLO ~3.3 k -> ~5.0 k, for ~11 % more
    // isolated latency
    static const int64_t gain = std::getenv("PAELLA_SPLIT_GAIN") ? atoi(std::getenv("PAELLA_SPLIT_GAIN")) : 65;
    uint32_t best = orig;
    bool best_dsm = (k.proto.flags & LF_SPLIT_DSMEM) != 0;
    int64_t best_t = INT64_MAX;
    for (uint32_t sp = 1; sp <= 16 && sp <= nk && tiles * sp <= 2 * g->P->sms; sp *= 2) {
      int64_t t_sp = INT64_MAX;
      bool dsm_sp = false;
      for (int dsm = 0; dsm < 2; ++dsm) {
        if ((dsm && only_l2) || (!dsm && only_dsm) || (dsm && sp == 1)) continue;
        set(sp, dsm != 0);
        time_layer(g, m, l, true, 8);   // warm
        const int64_t t = time_layer(g, m, l, true, 40);
        if (t < 0) return -EIO;
        if (t < t_sp) {
          t_sp = t;
          dsm_sp = dsm != 0;
        }
      }
      if (t_sp == INT64_MAX) continue;
      if (best_t == INT64_MAX || t_sp * 100 < best_t * gain) {
        best_t = t_sp;
        best = sp;
        best_dsm = dsm_sp;
      }
    }
    set(best, best_dsm && best > 1);
    if (cache)
      if (FILE* f = std::fopen(cache, "a")) {
        std::fprintf(f, "%s %u %u %u\n", m->name.c_str(), l, best, best_dsm && best > 1 ? 1u : 0u);
        std::fclose(f);
      }
    if (std::getenv("PAELLA_AUTOTUNE_LOG"))
      fprintf(stderr, "autotune %s layer %u: nk %u tiles %u split %u -> %u%s (%lld ns)\n", m->name.c_str(), l, nk,
              tiles, orig, best, best_dsm && best > 1 ? " dsmem" : "", (long long)best_t);
  }
  return 0;
}

// Split-K partial-sum workspaces (ModelGpu::splitk_*; the tcgen05 conv reduces its
// split-K partials in L2 with bulk fp32 reductions): per virtual stream, room for the
// largest tile grid among the layers that may split there (iso: any tcgen05 layer --
// autotuning and forced splits run in the isolated slot; else the layers whose chosen
// split is > 1), TC_BN x TC_BM floats per output tile.  Zeroed once; every owner CTA
// re-zeroes the sums it consumed, so the region is all zero between launches.
static int splitk_workspace(Model* m, ModelGpu& mg, bool iso) {
  constexpr size_t kTile = (size_t)TC_BN * TC_BM;   // (KIND_CONV_TC128 never splits)
  uint32_t nvs = 1;
  for (const auto& k : m->kernels)
    if (is_tc(k.kind)) nvs = std::max(nvs, k.vs + 1);
  std::vector<size_t> off(nvs, 0), tiles(nvs, 0);
  for (const auto& k : m->kernels)
    if (is_tc(k.kind) && k.kind != KIND_CONV_TC128 && (iso || k.proto.ksplit > 1))
      tiles[k.vs] = std::max<size_t>(tiles[k.vs], (size_t)k.proto.tiles_m * k.proto.tiles_n);
  size_t per = 0;
  for (uint32_t v = 0; v < nvs; ++v) {
    off[v] = per;
    per += tiles[v] * kTile;
  }
  if (per == 0) return 0;
  const size_t first = iso ? mg.args.size() - 1 : 0, nsl = iso ? 1 : mg.args.size() - 1;
  float* ws = nullptr;
  if (cudaMalloc((void**)&ws, nsl * per * sizeof(float))) return -ENOMEM;
  cudaMemset(ws, 0, nsl * per * sizeof(float));
  if (cudaStreamSynchronize(0) != cudaSuccess) return -EIO;   // legacy-stream memset vs. our streams
  (iso ? mg.splitk_iso : mg.splitk_slots) = ws;
  for (size_t s = 0; s < nsl; ++s)
    for (uint32_t l = 0; l < m->kernels.size(); ++l)
      if (is_tc(m->kernels[l].kind)) mg.args[first + s][l].ws = ws + s * per + off[m->kernels[l].vs];
  return 0;
}

static int setup_model_gpu(Paella* P, Model* m, Gpu* g) {
  ModelGpu& mg = m->gpu[g->index];
  const uint32_t slots = P->cfg.max_jobs_per_model;
  const size_t nslot = slots + 1;   // + the isolated slot
  const bool cuda = P->cfg.device == PAELLA_DEVICE_CUDA;
  uint8_t* wdev;
  uint8_t* wsp;
  if (cuda) {
    cudaSetDevice(g->device);
    if (cudaMalloc((void**)&wdev, m->blob.size() + 256)) return -ENOMEM;
    cudaMemcpy(wdev, m->blob.data(), m->blob.size(), cudaMemcpyHostToDevice);
    if (cudaMalloc((void**)&wsp, nslot * m->slot_bytes)) return -ENOMEM;
    cudaMemset(wsp, 0, nslot * m->slot_bytes);
    cudaStreamSynchronize(0);   // legacy-stream memset vs. our non-blocking streams
  } else {
    wdev = (uint8_t*)malloc(m->blob.size() + 256);
    wsp = (uint8_t*)calloc(1, 256);   // the fake device never touches activations
  }
  mg.weights = wdev;
  mg.workspace = wsp;
  auto& tmaps = mg.tmaps;
  tmaps.resize(m->kernels.size());
  // per-kernel attributes -> Table-1 demand
  for (uint32_t l = 0; l < m->kernels.size(); ++l) {
    KernelInst& k = m->kernels[l];
    if (cuda) {
      auto* cb = static_cast<CudaBackend*>(g->be.get());
      KernelFn f = cb->fn(k.kind, m->dtype, true);
      if (!f) return -EINVAL;
      cudaFuncAttributes fa;
      if (cudaFuncGetAttributes(&fa, (const void*)f)) return -EIO;
      if (k.smem > 48 * 1024) {
        cudaFuncSetAttribute((const void*)f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)k.smem);
        cudaFuncSetAttribute((const void*)cb->fn(k.kind, m->dtype, false),
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)k.smem);
      }
      if (is_tc(k.kind)) {   // split-K clusters of up to 16 CTAs
        cudaFuncSetAttribute((const void*)f, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        cudaFuncSetAttribute((const void*)cb->fn(k.kind, m->dtype, false),
                             cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
      }
      // constant per-SM capacity for Table-1 accounting: maximum carveout (hard part #4)
      cudaFuncSetAttribute((const void*)f, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
      cudaFuncSetAttribute((const void*)cb->fn(k.kind, m->dtype, false),
                           cudaFuncAttributePreferredSharedMemoryCarveout, 100);
      k.regs = (uint32_t)fa.numRegs;
      k.static_smem = (uint32_t)fa.sharedSizeBytes;
      if (is_tc(k.kind)) {
        if (make_weight_tmap(wdev + k.w_off, k.proto.tiles_m * TC_BM, k.proto.kpad, k.proto.a_rows, tmaps[l].b)) return -EIO;
      }
    } else {
      k.regs = 64;
      k.static_smem = 0;
    }
    uint32_t warps = (k.block + 31) / 32;
    uint32_t regs_warp = (k.regs * 32 + 255) / 256 * 256;
    k.demand[0] = 1;
    k.demand[1] = warps;
    k.demand[2] = (int64_t)regs_warp * warps;
    k.demand[3] = (int64_t)((k.static_smem + k.smem + 1024 + 127) / 128 * 128);
    k.demand[4] = k.tmem_cols;
  }
  // per-slot argument blocks
  mg.args.assign(nslot, {});
  for (size_t s = 0; s < nslot; ++s) {
    uint8_t* base = wsp + (cuda ? s * m->slot_bytes : 0);
    auto& A = mg.args[s];
    A.resize(m->kernels.size());
    for (uint32_t l = 0; l < m->kernels.size(); ++l) {
      const KernelInst& k = m->kernels[l];
      LayerArgs a = k.proto;
      auto bp = [&](int32_t b) -> void* { return b >= 0 ? (void*)(base + m->bufs[b].off) : nullptr; };
      if (k.kind != KIND_INGEST) a.in = bp(k.in_buf);
      a.out = bp(k.out_buf);
      a.res = bp(k.res_buf);
      a.w = wdev + k.w_off;
      a.bias = (const float*)(wdev + k.b_off);
      a.pro_scale = k.has_pro ? (const float*)(wdev + k.ps_off) : nullptr;
      a.pro_shift = k.has_pro ? (const float*)(wdev + k.pz_off) : nullptr;
      A[l] = a;
    }
  }
  // LF_TMA_B layers: one im2col tensor map per (slot, layer) -- the input address differs
  // per slot -- in device memory, addressed from the layer's arguments
  if (cuda) {
    const size_t L = m->kernels.size();
    bool any = false;
    for (const auto& k : m->kernels) any |= is_tc(k.kind) && (k.proto.flags & LF_TMA_B);
    if (any) {
      std::vector<TmapStore> h(nslot * L);
      if (cudaMalloc((void**)&mg.bmaps, h.size() * sizeof(TmapStore))) return -ENOMEM;
      for (size_t s = 0; s < nslot; ++s)
        for (uint32_t l = 0; l < L; ++l) {
          const KernelInst& k = m->kernels[l];
          LayerArgs& A = mg.args[s][l];
          if (!is_tc(k.kind) || !(A.flags & LF_TMA_B)) continue;
          const uint32_t bn = k.kind == KIND_CONV_TC128 ? TC_BN_WIDE : TC_BN;
          if (make_im2col_tmap(A.in, A, bn, h[s * L + l].b)) {
            A.flags &= ~LF_TMA_B;   // the encoder rejected the shape: LDGSTS gather
            continue;
          }
          A.bmap = mg.bmaps + (s * L + l) * sizeof(TmapStore);
        }
      if (cudaMemcpy(mg.bmaps, h.data(), h.size() * sizeof(TmapStore), cudaMemcpyHostToDevice)) return -EIO;
    }
  }
  mg.free_slots.clear();
  for (uint32_t s = slots; s-- > 0;) mg.free_slots.push_back(s);
  if (cuda) {
    const int rc = splitk_workspace(m, mg, true);
    if (rc) return rc;
  }
  // split factors: GPU 0 tunes them (the other GPUs are set up afterwards from the
  // tuned prototypes), then the serving slots' workspaces are sized for them
  if (g->index == 0 && cuda && autotune_splits(g, m)) return -EIO;
  if (cuda) {
    const int rc = splitk_workspace(m, mg, false);
    if (rc) return rc;
  }
  // profile T-bar (P1249-1254; reading C2-Q15): GPU 0 measures, others copy
  if (g->index == 0) {
    uint32_t runs = 20;
    if (cuda) {
      std::vector<int64_t> t(m->kernels.size()), acc(m->kernels.size(), 0);
      for (int w = 0; w < 5; ++w)
        if (iso_run(g, m, nullptr, nullptr, nullptr, true)) return -EIO;
      for (uint32_t r = 0; r < runs; ++r) {
        if (iso_run(g, m, nullptr, nullptr, t.data(), true)) return -EIO;
        for (size_t l = 0; l < t.size(); ++l) acc[l] += t[l];
      }
      for (size_t l = 0; l < t.size(); ++l) m->kernels[l].tbar = std::max<int64_t>(1, acc[l] / runs);
    } else {
      // fake device: analytic block duration, used as its own "profile"
      for (auto& k : m->kernels) k.tbar = 2000 + 40 * (int64_t)((k.grid_total() + P->sms - 1) / P->sms) * 1000 / 1000;
    }
  }
  return 0;
}

}  // namespace paella

extern "C" {

int paella_run_isolated(paella_t* p, uint32_t gpu, uint32_t model_id, const void* input, void* output,
                        int64_t* kernel_ns) {
  Paella* P = (Paella*)p;
  if (!P || gpu >= P->gpus.size() || model_id >= P->nmodels.load()) return -EINVAL;
  if (P->cfg.device != PAELLA_DEVICE_CUDA) return -ENODEV;
  Gpu* g = P->gpus[gpu].get();
  std::lock_guard<std::mutex> lk(g->iso_mu);
  return iso_run(g, P->models[model_id].get(), input, output, kernel_ns, P->cfg.instrument != 0);
}

int paella_debug_node(paella_t* p, uint32_t gpu, uint32_t model_id, uint32_t node, float* out) {
  Paella* P = (Paella*)p;
  if (!P || gpu >= P->gpus.size() || model_id >= P->nmodels.load() || !out) return -EINVAL;
  if (P->cfg.device != PAELLA_DEVICE_CUDA) return -ENODEV;
  Model* m = P->models[model_id].get();
  if (node >= m->nodes.size() || m->buf_of[node] < 0) return -EINVAL;
  Gpu* g = P->gpus[gpu].get();
  const paella_node_t& nd = m->nodes[node];
  const Buffer& b = m->bufs[m->buf_of[node]];
  const size_t es = m->dtype == PAELLA_DTYPE_BF16 ? 2 : 4;
  std::vector<uint8_t> h(b.bytes);
  cudaSetDevice(g->device);
  uint8_t* base = (uint8_t*)m->gpu[gpu].workspace + (m->gpu[gpu].args.size() - 1) * m->slot_bytes;
  if (cudaMemcpy(h.data(), base + b.off, b.bytes, cudaMemcpyDeviceToHost)) return -EIO;
  uint32_t C = nd.op == PAELLA_OP_INPUT ? nd.c : nd.c;
  uint32_t co = m->coff[node];
  for (uint32_t c = 0; c < C; ++c)
    for (uint32_t p2 = 0; p2 < nd.h * nd.w; ++p2) {
      size_t idx = (size_t)p2 * b.c + co + c;
      float v;
      if (es == 2) {
        uint32_t u = (uint32_t)((uint16_t*)h.data())[idx] << 16;
        std::memcpy(&v, &u, 4);
      } else {
        v = ((float*)h.data())[idx];
      }
      out[(size_t)c * nd.h * nd.w + p2] = v;
    }
  return 0;
}

}  // extern "C"

// ===========================================================================
// device-only timing and notification microbenchmarks
// ===========================================================================
namespace paella {

static volatile uint32_t* gate_ptr(Gpu* g, const volatile uint32_t** dev) {
  volatile uint32_t* gate = (volatile uint32_t*)((uint8_t*)g->stage_in + g->stage_bytes - 64);
  cudaHostGetDevicePointer((void**)dev, (void*)gate, 0);
  return gate;
}

static void launch_gate(Gpu* g, const volatile uint32_t* gd) {
  if (no_gate()) return;
  void* gargs[1] = {(void*)&gd};
  cudaLaunchKernel((const void*)gate_kernel(), dim3(1), dim3(1), gargs, 0, (cudaStream_t)g->prof_stream);
}

static InstrArgs iso_instr(Gpu* g, uint32_t grid, uint32_t group, bool last) {
  InstrArgs ia{};
  ia.ring = iso_ring(g);
  ia.tail = g->prof_tail;
  uint32_t uid = g->prof_uid++;
  uint32_t slot = uid % NCTR;
  ia.ctr = g->prof_ctr + 2 * slot;
  ia.ctr_stride = 2 * NCTR;
  ia.mask = (1u << 16) - 1;
  ia.log2cap = 16;
  ia.base = g->prof_base[slot];
  g->prof_base[slot] += grid;
  ia.uid = uid;
  ia.group = group;
  ia.flags = INSTR_ON | (last ? INSTR_LAST : 0);
  if (last && std::getenv("PAELLA_LAST_SYS")) ia.flags |= INSTR_SYSREL;
  if (static_cast<CudaBackend*>(g->be.get())->mirror)   // as in serving
    ia.flags |= INSTR_CTR | (last ? 0u : INSTR_RELAXED);
  return ia;
}

}  // namespace paella

extern "C" {

// X_dev (SURVEY.md 8(d) "Throughput"): device-only saturation of a request mix, no
// dispatcher.  One CUDA graph per (model, stream) holds the model's uninstrumented
// kernel chain (PDL edges, as served) on workspace slot = stream; the requests of `seq`
// are replayed as graph launches round-robin over `streams` streams, all enqueued at
// once (overload); rate = requests / elapsed (CUDA events).
int paella_bench_xdev(paella_t* p, uint32_t gpu, const uint32_t* models, uint32_t n_models, const uint32_t* seq,
                      uint32_t n, uint32_t streams, double* req_per_s) {
  Paella* P = (Paella*)p;
  if (!P || gpu >= P->gpus.size() || !models || !seq || !req_per_s || n == 0 || streams == 0 || streams > 64)
    return -EINVAL;
  if (P->cfg.device != PAELLA_DEVICE_CUDA) return -ENODEV;
  Gpu* g = P->gpus[gpu].get();
  std::lock_guard<std::mutex> lk(g->iso_mu);
  int rc = ensure_iso(g);
  if (rc) return rc;
  for (uint32_t i = 0; i < n_models; ++i)
    if (models[i] >= P->nmodels.load() || P->cfg.max_jobs_per_model < streams) return -EINVAL;
  for (uint32_t i = 0; i < n; ++i)
    if (seq[i] >= n_models) return -EINVAL;
  cudaSetDevice(g->device);
  auto* cb = static_cast<CudaBackend*>(g->be.get());
  std::vector<cudaStream_t> ss(streams);
  for (auto& s : ss) cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  std::vector<cudaGraphExec_t> ex((size_t)n_models * streams, nullptr);
  uint8_t* st = (uint8_t*)g->stage_in;   // every request reads the same staged input
  std::memset(st, 0, 2 << 20);
  for (uint32_t mi = 0; mi < n_models && rc == 0; ++mi) {
    Model* m = P->models[models[mi]].get();
    ModelGpu& mg = m->gpu[gpu];
    for (uint32_t s = 0; s < streams && rc == 0; ++s) {
      std::vector<LayerArgs> A = mg.args[s];          // slot s, private copy of the parameters
      A.front().in = st;
      A.back().out = st + (8 << 20);   // past the largest input
      cudaGraph_t graph;
      if (cudaStreamBeginCapture(ss[s], cudaStreamCaptureModeThreadLocal) != cudaSuccess) rc = -EIO;
      for (uint32_t l = 0; l < m->kernels.size() && rc == 0; ++l) {
        const KernelInst& k = m->kernels[l];
        InstrArgs ia{};
        const void* tm = is_tc(k.kind) ? mg.tmaps[l].b : nullptr;
        void* args[3] = {(void*)&A[l], (void*)&ia, (void*)tm};
        if (cuda_launch(cb->fn(k.kind, m->dtype, false), k, args, ss[s], true) != cudaSuccess) rc = -EIO;
      }
      if (cudaStreamEndCapture(ss[s], &graph) != cudaSuccess) rc = -EIO;
      if (rc == 0 && cudaGraphInstantiate(&ex[(size_t)mi * streams + s], graph, 0) != cudaSuccess) rc = -EIO;
      if (rc == 0) cudaGraphDestroy(graph);
    }
  }
  if (rc == 0) {
    // warm every graph once, then the timed overload
    for (size_t i = 0; i < ex.size(); ++i) cudaGraphLaunch(ex[i], ss[i % streams]);
    for (auto& s : ss) cudaStreamSynchronize(s);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0, ss[0]);
    for (uint32_t s = 1; s < streams; ++s) cudaStreamWaitEvent(ss[s], e0, 0);
    for (uint32_t i = 0; i < n; ++i) {
      const uint32_t s = i % streams;
      cudaGraphLaunch(ex[(size_t)seq[i] * streams + s], ss[s]);
    }
    std::vector<cudaEvent_t> done(streams);
    for (uint32_t s = 0; s < streams; ++s) {
      cudaEventCreateWithFlags(&done[s], cudaEventDisableTiming);
      cudaEventRecord(done[s], ss[s]);
      cudaStreamWaitEvent(ss[0], done[s], 0);
    }
    cudaEventRecord(e1, ss[0]);
    if (cudaEventSynchronize(e1) != cudaSuccess) rc = -EIO;
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    *req_per_s = n / (ms * 1e-3);
    for (auto& e : done) cudaEventDestroy(e);
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
  }
  for (auto& x : ex)
    if (x) cudaGraphExecDestroy(x);
  for (auto& s : ss) cudaStreamDestroy(s);
  return rc;
}

int paella_time_kernels(paella_t* p, uint32_t gpu, uint32_t model_id, uint32_t instrumented, uint32_t reps,
                        int64_t* kernel_ns) {
  Paella* P = (Paella*)p;
  if (!P || gpu >= P->gpus.size() || model_id >= P->nmodels.load() || !kernel_ns || reps == 0) return -EINVAL;
  if (P->cfg.device != PAELLA_DEVICE_CUDA) return -ENODEV;
  Gpu* g = P->gpus[gpu].get();
  std::lock_guard<std::mutex> lk(g->iso_mu);
  Model* m = P->models[model_id].get();
  int rc = iso_run(g, m, nullptr, nullptr, nullptr, true);   // materialise valid activations
  if (rc) return rc;
  for (uint32_t l = 0; l < m->kernels.size(); ++l) {
    kernel_ns[l] = (instrumented & PAELLA_TIME_L2_COLD) ? time_layer_cold(g, m, l, instrumented & 1u, reps)
                                                        : time_layer(g, m, l, instrumented & 1u, reps);
    if (kernel_ns[l] < 0) return -EIO;
  }
  return 0;
}

int paella_bench_empty(paella_t* p, uint32_t gpu, uint32_t grid, uint32_t block, uint32_t instrumented,
                       uint32_t group, uint32_t iters, double* ns_per_launch) {
  Paella* P = (Paella*)p;
  if (!P || gpu >= P->gpus.size() || !ns_per_launch || iters == 0 || group == 0 || group > 16) return -EINVAL;
  if (P->cfg.device != PAELLA_DEVICE_CUDA) return -ENODEV;
  Gpu* g = P->gpus[gpu].get();
  std::lock_guard<std::mutex> lk(g->iso_mu);
  int rc = ensure_iso(g);
  if (rc) return rc;
  cudaSetDevice(g->device);
  cudaStream_t s = (cudaStream_t)g->prof_stream;
  auto* cb = static_cast<CudaBackend*>(g->be.get());
  KernelFn f = cb->fn(KIND_EMPTY, 0, instrumented != 0);
  LayerArgs la{};
  // experiment: PAELLA_BENCH_DEVRING=1 writes the records to device memory instead of
  // the pinned host ring (isolates the cost of the PCIe write + kernel-end flush)
  Rec* devring = std::getenv("PAELLA_BENCH_DIRECT") ? (Rec*)g->prof_ring_d : g->prof_devring;
  const volatile uint32_t* gd;
  volatile uint32_t* gate = gate_ptr(g, &gd);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  // gated batches stay well below the driver's pending-launch queue depth (a full
  // queue would block the host while the gate blocks the GPU)
  const uint32_t batch = 256;
  double total_ms = 0;
  for (uint32_t done = 0; done < iters; done += batch) {
    uint32_t nb = std::min(batch, iters - done);
    *gate = 0;
    launch_gate(g, gd);
    cudaEventRecord(e0, s);
    for (uint32_t i = 0; i < nb; ++i) {
      InstrArgs ia = iso_instr(g, grid, group, false);
      if (devring) ia.ring = devring;
      void* args[2] = {(void*)&la, (void*)&ia};
      cudaLaunchKernel((const void*)f, dim3(grid), dim3(block), args, 0, s);
    }
    cudaEventRecord(e1, s);
    std::atomic_thread_fence(std::memory_order_seq_cst);
    *gate = 1;
    if (cudaStreamSynchronize(s) != cudaSuccess) return -EIO;
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    total_ms += ms;
  }
  float ms = (float)total_ms;
  *ns_per_launch = (double)ms * 1e6 / iters;
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  return 0;
}

int paella_bench_roundtrip(paella_t* p, uint32_t gpu, uint32_t n, int64_t* place_ns, int64_t* complete_ns) {
  Paella* P = (Paella*)p;
  if (!P || gpu >= P->gpus.size() || !place_ns || !complete_ns) return -EINVAL;
  if (P->cfg.device != PAELLA_DEVICE_CUDA) return -ENODEV;
  Gpu* g = P->gpus[gpu].get();
  std::lock_guard<std::mutex> lk(g->iso_mu);
  int rc = ensure_iso(g);
  if (rc) return rc;
  cudaSetDevice(g->device);
  cudaStream_t s = (cudaStream_t)g->prof_stream;
  cudaStreamSynchronize(s);
  auto* cb = static_cast<CudaBackend*>(g->be.get());
  KernelFn f = cb->fn(KIND_EMPTY, 0, true);
  LayerArgs la{};
  // consume from the current device tail
  uint32_t tail = 0;
  cudaMemcpy(&tail, g->prof_tail, 4, cudaMemcpyDeviceToHost);
  uint64_t head = tail;
  const uint32_t mask = (1u << 16) - 1;
  for (uint32_t i = 0; i < n; ++i) {
    InstrArgs ia = iso_instr(g, 1, 1, false);
    ia.ring = (Rec*)g->prof_ring_d;   // direct write to the pinned host ring
    ia.flags &= ~(INSTR_CTR | INSTR_RELAXED);   // records, also when serving uses counter mode
    void* args[2] = {(void*)&la, (void*)&ia};
    int64_t t0 = now_ns();
    cudaLaunchKernel((const void*)f, dim3(1), dim3(32), args, 0, s);
    for (int want = 0; want < 2; ++want) {
      volatile uint64_t* r = (volatile uint64_t*)(g->prof_ring_h + (head & mask));
      uint32_t tag = rec_tag((uint32_t)(head >> 16));
      int64_t tstart = now_ns();
      for (;;) {
        uint64_t w0 = r[0];
        if ((w0 & 0xff) != 0 && ((w0 >> 24) & 0xff) == tag && (r[1] >> 56) == tag) break;
        if (now_ns() - tstart > 1000000000ll) return -ETIMEDOUT;
      }
      int64_t t = now_ns() - t0;
      uint64_t w0 = r[0];
      r[0] = 0;
      r[1] = 0;
      if ((w0 & 0xff) == REC_PLACEMENT)
        place_ns[i] = t;
      else
        complete_ns[i] = t;
      head++;
    }
  }
  return cudaStreamSynchronize(s) == cudaSuccess ? 0 : -EIO;
}

}  // extern "C"
