/*
 * paella.h -- C ABI of the B200-native Paella hot path.
 *
 * Paella (SOSP '23, "Low-latency Model Serving with Software-defined GPU
 * Scheduling"): many concurrent batch-1 inference jobs run on instrumented kernels
 * that report thread-block placement and completion through a host-mapped
 * notification ring; a software dispatcher (one pinned core per GPU) tracks SM
 * occupancy and decides kernel issue order with SRPT on remaining-time estimates
 * bounded by deficit-counter fairness, instead of the GPU's FIFO hardware queues.
 *
 * Citations are PAPER.md line numbers ("P123") with the section they fall in.
 *
 *   paella_init           -- service start-up; one dispatcher thread per GPU (P1024-1033 §5)
 *   paella_register_model -- "users add new job definitions to the Paella service"
 *                            (P1036-1038 §5.1); profiling runs fix T-bar (P1249-1254 §6)
 *   paella_submit         -- predict(model_name, len, io_ptr, options) -> req_id
 *                            (P1039-1056 §5.1); range check [io, io+len) (P1060-1061)
 *   paella_poll_completion-- readResult(options) -> first available completion id,
 *                            NONBLOCK -> negative EAGAIN (P1144-1155 §5.3)
 *   paella_shutdown       -- stop admitting, drain, free
 *
 * Conventions: every call returns >= 0 on success and -errno on failure ("it may
 * return the negative code EAGAIN", P1155).  No call takes or returns framework
 * (torch) types: plain host pointers and sizes only.
 *
 * Threading: one thread per client_id at a time (each client's submission and
 * completion queues are single-producer/single-consumer); different clients may
 * call concurrently.  The dispatcher threads are internal.
 *
 * Ownership: the io buffer passed to paella_submit is LENT to the library from
 * submit until paella_poll_completion returns that req_id; its layout is
 * [input | output] (Fig. 8, P992-996: output = io_ptr + INPUT_SIZE).  The input is
 * fp32 NCHW (1 x C x H x W); the output is fp32 logits.  The ingest kernel reads
 * the input straight from that (page-locked, device-mapped) client memory and the
 * last kernel writes the output in place ("pinned output", P1016).  The library
 * owns device weights, per-job workspaces, rings and streams.
 */
#ifndef PAELLA_H_
#define PAELLA_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PAELLA_ABI_VERSION 2u   /* 2: paella_config_t.lookahead_unplaced, cap_arrival_order */
#define PAELLA_NOTIFY_COUNTERS 0u
#define PAELLA_NOTIFY_RING     1u

/* policies (P1222-1323 §6; FIFO = the Paella-SS-like ablation of Table 3, P1349) */
#define PAELLA_POLICY_SRPT_DEFICIT 0u
#define PAELLA_POLICY_FIFO         1u
#define PAELLA_POLICY_SJF          2u   /* ablation (NEXT-2, Table 3): shortest whole job first */
#define PAELLA_POLICY_RR           3u   /* ablation: kernel-granular round robin over ready jobs */

/* routing across GPUs */
#define PAELLA_ROUTE_LEAST_WORK    0u
#define PAELLA_ROUTE_ROUND_ROBIN   1u
#define PAELLA_ROUTE_POWER_OF_TWO  2u   /* power-of-two choices: the lower W_g of two GPUs
                                          drawn from the request id (paella_route_pair) */

/* device backends */
#define PAELLA_DEVICE_CUDA 0u   /* real sm_100a GPUs */
#define PAELLA_DEVICE_FAKE 1u   /* CPU model of a GPU that synthesises ring records
                                   (tests of dispatcher / router / replay without a GPU) */

/* dtypes of a model's compute path */
#define PAELLA_DTYPE_BF16 0u    /* bf16 activations, fp32 accumulate, tcgen05 for conv */
#define PAELLA_DTYPE_FP32 1u    /* fp32 everything, SIMT FFMA, no TF32 */

/* flags */
#define PAELLA_NONBLOCK 1u      /* submit: -EAGAIN if the ring is full; poll: -EAGAIN if none */
#define PAELLA_HYBRID   2u      /* poll: hybrid interrupt/poll wait (P1157-1171): spin ~20 us,
                                   then sleep on a futex until the dispatcher issues the
                                   LAST kernel of one of this client's jobs (the "almost
                                   finished" hint) or pushes a completion, then spin again */

/* maximum sizes */
#define PAELLA_MAX_GPUS    8u
#define PAELLA_MAX_CLIENTS 64u

typedef struct paella_s paella_t;  /* opaque, owned by the library */

typedef struct {
  uint32_t abi_version;          /* = PAELLA_ABI_VERSION */
  uint32_t device;               /* PAELLA_DEVICE_CUDA | PAELLA_DEVICE_FAKE */
  uint32_t num_gpus;             /* 1..8; one dispatcher thread per GPU */
  uint32_t first_gpu;            /* CUDA ordinal of GPU 0 of this instance */
  uint32_t num_clients;          /* N of the deficit rule (P1290-1296); fixed */
  uint32_t policy;               /* PAELLA_POLICY_* */
  int64_t  fairness_threshold;   /* theta, in kernel dispatches; INT64_MAX = pure SRPT */
  uint32_t slack_blocks;         /* B (P1300-1304); 0 = default (SM count) */
  uint32_t group_size;           /* G in 1..16 (P1138-1142); 0 = default 16 */
  uint32_t ring_capacity;        /* notification ring slots, power of two; 0 = 65536 */
  uint32_t stream_pool;          /* P CUDA streams per GPU (P1090-1098); 0 = 32 */
  uint32_t route;                /* PAELLA_ROUTE_* */
  uint32_t submit_slots;         /* per-(client,GPU) submission ring slots, pow2; 0 = 1024 */
  uint32_t max_jobs_per_model;   /* in-flight job workspaces per model per GPU; 0 = 128 */
  uint32_t instrument;           /* 1 = instrumented kernels (Paella); 0 = uninstrumented twin */
  uint32_t naive;                /* 1 = naive baseline: no dispatcher decisions, every kernel
                                    of a job is launched at admission onto stream
                                    job % stream_pool (CUDA-MS, Table 3 P1343-1344) */
  size_t   client_region_bytes;  /* shared io region per client, created here; 0 = 64 MiB */
  const int32_t* dispatcher_cpus;/* num_gpus core ids to pin the dispatchers to, or NULL */
  const char* event_log_path;    /* binary event log for replay (printf pattern "%u" = GPU
                                    index), or NULL */
  uint32_t fake_sms;             /* FAKE device: SM count (0 = 148) */
  uint32_t fake_time_scale_ns;   /* FAKE device: virtual ns per poll iteration (0 = 500) */
  uint32_t event_time_kind;      /* 0 = off; k+1 = the dispatcher brackets every launch of
                                    kernel kind k with CUDA events on its stream and sums
                                    the durations (paella_stats ev_*): the live roofline */
  uint32_t lookahead;            /* NEXT-1 launch-ahead depth: 0 = the paper's semantics (a
                                    job's next kernel is dispatched after the previous one's
                                    final COMPLETION); D in 1..7 = once the job's OLDEST
                                    in-flight kernel is fully placed (running) and <= D are in
                                    flight, the next kernel is queued behind it on the same
                                    stream (with PDL it starts ~0.6 us after its predecessor) */
  uint32_t launch_threads;       /* 0 = each dispatcher calls cudaLaunchKernel itself; n > 0 =
                                    n helper threads per GPU perform the launches (stream s is
                                    owned by helper s % n, so per-stream order is kept); the
                                    decisions stay on the one dispatcher core */
  uint32_t no_proxy;             /* 0 (default): kernels write notification records to a
                                    device-memory ring and one persistent proxy warp forwards
                                    them to the pinned host ring (keeps the PCIe write off every
                                    kernel's exit path); 1: kernels write the host ring directly,
                                    as in the paper (P1104-1106) */
  uint32_t no_pdl;               /* 0 (default): kernels are launched with programmatic
                                    dependent launch (a kernel queued behind another on its
                                    stream starts ~0.6 us after it instead of on the next
                                    ~2 us front-end quantum); 1: plain launches.
                                    The naive baseline always uses plain launches. */
  uint32_t notify_mode;          /* PAELLA_NOTIFY_COUNTERS (0, default): blocks only bump their
                                    launch's {start, end} counters with fire-and-forget
                                    reductions; one resident warp mirrors the counter table to
                                    pinned host memory and the dispatcher turns counter
                                    progress into the same group-of-G records (no atomic
                                    round trip and no record write on any block's exit path,
                                    DESIGN.md §7).  PAELLA_NOTIFY_RING (1): blocks write 16 B
                                    records into a device ring that a resident warp forwards
                                    to the pinned host ring (records carry SM id and
                                    globaltimer; G = 1 debug mode).  no_proxy = 1 overrides
                                    both with the paper's direct ring writes. */
  uint32_t prio_classes;         /* 0/1 = one class (the paper).  K > 1: the stream pool is split
                                    into K classes of consecutive indices created with
                                    descending hardware stream priority; a job takes a stream
                                    of the class of its remaining work R_j (number of
                                    registered models whose whole-job T-bar sum is below R_j,
                                    clamped to K-1; deficit-override picks take class 0), so the
                                    blocks the +B slack keeps queued in hardware are also served
                                    shortest-remaining first (B200-Q2).  K <= P. */
  uint32_t online_tbar;           /* NEXT-4: 1 = refine T-bar online, as the running average of
                                    the profiling runs and every observed duration of that
                                    kernel (first placement -> final completion seen by the
                                    dispatcher, P1249-1266); 0 (default) = frozen profile */
  uint32_t decide_delay_ns;       /* NEXT-2 sensitivity (Fig. 9, P1215-1241): the dispatcher
                                    busy-waits this long before every decide() pass, an
                                    injected scheduler delay; 0 (default) = none */
  uint32_t naive_pdl;             /* naive baseline only: 1 = launch its kernels with programmatic
                                    dependent launch too (CUDA-MS + PDL: the same launch mechanics
                                    as the Paella path, so a comparison isolates the scheduler);
                                    0 (default) = plain launches */
  uint32_t watchdog_ms;           /* 0 = off.  A GPU whose in-flight launches report no record
                                    progress for this long is declared hung: its live jobs complete
                                    with -ETIMEDOUT, later requests are routed to the remaining GPUs
                                    (or complete with -EIO when none is left) */
  uint32_t fake_fault;            /* FAKE device fault injection (tests): PAELLA_FAULT_*, on GPU 0
                                    of the instance only */
  uint32_t fake_fault_arg;        /* ... the ordinal of the record / launch it applies to */
  uint32_t branches;              /* NEXT-4 intra-job concurrency (Fig. 7 waitlists, P906-951): 1 =
                                    a job's kernels form a DAG over up to 4 virtual streams
                                    (Inception / SqueezeNet / ResNet branches run concurrently on
                                    several CUDA streams; a kernel is issued once its cross-
                                    stream inputs have completed); 0 (default) = one chain per job */
  const char* route_log_path;     /* multi-GPU routing log (printf pattern, "%u" = client id), or
                                    NULL: every routing decision of that client with the W_g
                                    snapshot of ALL GPUs it was taken on (paella_route_rec_t
                                    records, written at shutdown / paella_flush_log), so the
                                    router replays against oracle/sim.py */
  uint32_t max_active_jobs;       /* K (reading B200-Q6): 0 = no cap (the paper).  K > 0:
                                    a ready job may issue only if it is among the K first jobs,
                                    in the policy's order (SRPT: remaining time R_j; FIFO: arrival),
                                    of the live jobs that still have kernels to issue (a deficit
                                    override is exempt).  Preemption stays kernel-granular: a
                                    job pushed out of the K first stops issuing, its in-flight
                                    kernels drain */
  uint32_t lookahead_unplaced;    /* NEXT-1 variant: 1 = launch-ahead queues the next kernel of a
                                    (virtual) stream as soon as <= D are in flight, without
                                    waiting for the oldest in-flight kernel's placement to be
                                    seen (the occupancy predicate's slack B still bounds the
                                    queued blocks).  Kernels shorter than the notification
                                    round trip otherwise complete before their placement is
                                    seen and launch-ahead degenerates to one kernel at a time */
  uint32_t cap_arrival_order;     /* with max_active_jobs = K: 0 = the K first live jobs in the
                                    policy's order (SRPT: remaining time) may issue; 1 = the K
                                    first in ARRIVAL order (the policy still orders the ready
                                    jobs among them): a long job cannot be kept out of the cap
                                    by a stream of shorter arrivals */
} paella_config_t;

/* One routing decision.  W_g = work[g] + pending[g] * tbar_model:
   work[g] = the outstanding work (sum of R_j, ns) GPU g's dispatcher last published,
   pending[g] = submissions routed to g that its dispatcher has not admitted yet, each
   estimated at the whole-job T-bar sum of the request's model.  alive = bit g set if
   GPU g had not failed. */
typedef struct {
  uint64_t req_id;
  uint32_t route;              /* PAELLA_ROUTE_* */
  uint32_t chosen;             /* GPU the request went to */
  uint32_t g0, g1;             /* power-of-two candidates (route 2), else = chosen */
  uint32_t num_gpus, model;
  uint32_t alive, pad;
  int64_t  tbar_model;
  int64_t  work[8];
  int64_t  pending[8];
} paella_route_rec_t;

/* fault injection of the FAKE device (paella_config_t.fake_fault); n = fake_fault_arg */
#define PAELLA_FAULT_NONE    0u
#define PAELLA_FAULT_DROP    1u   /* the n-th COMPLETION record is lost on its way to the ring */
#define PAELLA_FAULT_DUP     2u   /* the n-th record is written twice (two ring slots) */
#define PAELLA_FAULT_TORN    3u   /* every record's second half lands one poll iteration after
                                     its first half (n ignored): the reader must re-read, never
                                     consume a torn slot (P1107-1113) */
#define PAELLA_FAULT_HANG    4u   /* blocks of the n-th launch never complete (a hung kernel) */
#define PAELLA_FAULT_CORRUPT 5u   /* the n-th record carries an invalid record type */

/* ---- model description (input to paella_register_model) ---------------- */
#define PAELLA_OP_INPUT   0u
#define PAELLA_OP_CONV    1u
#define PAELLA_OP_MAXPOOL 2u
#define PAELLA_OP_AVGPOOL 3u   /* count_include_pad = True */
#define PAELLA_OP_GAP     4u   /* global average pool */
#define PAELLA_OP_FC      5u
#define PAELLA_OP_CONCAT  6u   /* channel concat, realised by channel-offset stores */
#define PAELLA_OP_SPIN    7u   /* synthetic kernel of the HoL microbenchmark (Fig. 2, P431-445):
                                  one block of 128 threads resident for kh microseconds that
                                  copies its input (c channels, 1 x 1) to its output */

#define PAELLA_ACT_NONE  0u
#define PAELLA_ACT_RELU  1u
#define PAELLA_ACT_RELU6 2u

#define PAELLA_NODE_PROLOGUE 1u  /* relu(pro_scale[c]*x + pro_shift[c]) on the input (DenseNet) */
#define PAELLA_NODE_CEIL     2u  /* maxpool ceil_mode */

typedef struct {
  uint32_t op;                 /* PAELLA_OP_* */
  uint32_t n_inputs;           /* 1, or the number of concat inputs; 0 for INPUT */
  const int32_t* inputs;       /* node ids (earlier nodes) */
  int32_t  residual;           /* conv: node id added before the activation, or -1 */
  uint32_t c, h, w;            /* output shape (C, H, W), batch 1 */
  uint32_t cout, kh, kw, sh, sw, ph, pw, groups;  /* conv; pools use kh=kw=k, sh=sw=s, ph=pw=p;
                                                     fc uses cout */
  uint32_t act;                /* PAELLA_ACT_* */
  uint32_t flags;              /* PAELLA_NODE_* */
  const float* weight;         /* conv [cout][cin/groups][kh][kw], fc [cout][cin]; fp32 host
                                  values (the bf16 path requires bf16-representable values
                                  and stores them as bf16 exactly) */
  const float* bias;           /* [cout] or NULL (zero) */
  const float* pro_scale;      /* [cin] if PROLOGUE */
  const float* pro_shift;      /* [cin] if PROLOGUE */
} paella_node_t;

typedef struct {
  const char* name;            /* unique */
  uint32_t dtype;              /* PAELLA_DTYPE_* */
  uint32_t n_nodes;
  const paella_node_t* nodes;  /* topologically ordered; node 0 is the INPUT; the last node
                                  produces the logits */
  uint32_t profile_runs;       /* isolated profiling runs for T-bar (0 = 20) */
} paella_model_desc_t;

/* ---- calls --------------------------------------------------------------- */

int paella_init(const paella_config_t* cfg, paella_t** out);
/* -EINVAL bad cfg; -ENODEV fewer than num_gpus sm_100 GPUs (CUDA backend);
   -ENOMEM.  Creates the client regions, rings, stream pools and starts one
   dispatcher thread per GPU. */

int paella_register_model(paella_t* p, const paella_model_desc_t* desc, uint32_t* model_id);
/* Copies the parameters (library owns the device copies on every GPU), builds the
   kernel chain (one kernel per non-concat node + ingest), queries each kernel's
   resource attributes (Table 1, P782-802; P814-830), profiles T-bar per kernel
   with isolated instrumented runs (P1249-1254) and freezes it.
   -EEXIST name taken; -EINVAL malformed graph or a kernel needing more records
   than the ring holds; -ENOMEM; -EIO CUDA failure. */

int64_t paella_submit(paella_t* p, uint32_t client_id, uint32_t model_id,
                      void* io, size_t len, uint32_t flags);
/* Zero-copy request: [io, io+len) must lie inside client_id's region
   (paella_client_region), else -EFAULT (P1060-1061).  -EINVAL unknown model or
   len < input_bytes + output_bytes; -EAGAIN ring full and PAELLA_NONBLOCK;
   -ESHUTDOWN.  Returns req_id = (client_id << 48) | seq. */

int64_t paella_submit_at(paella_t* p, uint32_t client_id, uint32_t model_id,
                         void* io, size_t len, uint32_t flags, int64_t t_sched_ns);
/* paella_submit with the request's scheduled arrival time (CLOCK_MONOTONIC ns),
   recorded in the event log; paella_submit uses "now". */

int64_t paella_poll_completion(paella_t* p, uint32_t client_id, uint32_t flags, int32_t* status);
/* Returns the req_id of the FIRST available completion of this client (completion
   order, not submission order, P1149).  PAELLA_NONBLOCK: -EAGAIN if none (P1155);
   PAELLA_HYBRID: spin, then futex sleep between the dispatcher's hints (above);
   otherwise spins until one is available.  *status (if non-NULL): 0 ok, -EIO CUDA
   error on that GPU, -ECANCELED shutdown. */

int paella_route_pair(uint64_t req_id, uint32_t num_gpus, uint32_t* g0, uint32_t* g1);
/* The two candidate GPUs of PAELLA_ROUTE_POWER_OF_TWO (SURVEY.md §8(e) "Variants:
   round-robin, power-of-two-choices"; the paper routes nothing, it serves one GPU,
   P1024-1033).  Pure and deterministic: h = splitmix64(req_id) (one output of the
   generator seeded with req_id), *g0 = h mod num_gpus, *g1 = (*g0 + 1 + (h >> 32)
   mod (num_gpus - 1)) mod num_gpus, so *g0 != *g1 when num_gpus > 1 (both 0 when
   num_gpus == 1).  paella_submit sends the request to the candidate with the lower
   published outstanding work W_g (+ unadmitted estimate), ties to the lower index.
   -EINVAL num_gpus == 0 or > PAELLA_MAX_GPUS or a NULL output. */

int paella_shutdown(paella_t* p);
/* Stop admitting; drain in-flight kernels; requests not yet admitted complete with
   -ECANCELED; join dispatchers; free everything. */

int paella_client_region(paella_t* p, uint32_t client_id, void** base, size_t* bytes);
/* The shared io region of a client (page-locked, device-mapped on every GPU). */

/* ---- client processes (P1030-1033: "each client obtains a shared memory region when
   setting up the connection") ---------------------------------------------------------
   All client channels -- the io regions, the submission / completion rings and the
   routing state the dispatchers publish -- live in one shared mapping created by
   paella_init.  Another process of the same user attaches to it by path and then
   submits and polls exactly as paella_submit / paella_poll_completion do (same code,
   same semantics and error codes, zero copy: its io buffers are in the mapped region).
   A client id may be held by one process at a time (the rings are single-producer). */
typedef struct paella_client_s paella_client_t;

int paella_channel_path(paella_t* p, char* buf, size_t n);
/* Path of the channel mapping ("/proc/<pid>/fd/<n>"), valid while the instance lives. */
int paella_client_attach(const char* path, uint32_t client_id, paella_client_t** out);
/* Map the channels and claim client_id.  -EINVAL bad path / layout / id; -EBUSY the id
   is attached by another process; -errno of open(2). */
int paella_client_region_of(paella_client_t* c, void** base, size_t* bytes);
/* The attached client's io region in this process. */
int paella_client_model_io(paella_client_t* c, uint32_t model_id, size_t* input_bytes, size_t* output_bytes);
/* io sizes of a registered model (-EINVAL if not registered). */
int64_t paella_client_submit(paella_client_t* c, uint32_t model_id, void* io, size_t len, uint32_t flags);
/* = paella_submit for the attached client id. */
int64_t paella_client_poll(paella_client_t* c, uint32_t flags, int32_t* status);
/* = paella_poll_completion for the attached client id. */
int paella_client_detach(paella_client_t* c);
/* Release the id and unmap. */

/* ---- introspection (tests, bench) ---------------------------------------- */

typedef struct {
  uint32_t n_kernels;          /* kernels per job (incl. ingest) */
  size_t   input_bytes, output_bytes;
  uint64_t weight_bytes;       /* device bytes of parameters */
  int64_t  total_tbar_ns;      /* sum of frozen T-bar */
} paella_model_info_t;

int paella_model_info(paella_t* p, uint32_t model_id, paella_model_info_t* info);

typedef struct {
  uint32_t grid, block, smem, regs, tmem_cols;
  uint32_t kind;               /* kernel kind id (paella_kernel_name) */
  int64_t  tbar_ns;            /* frozen profile */
  uint64_t flops, bytes;       /* algorithmic work per launch */
  uint32_t vs;                 /* virtual stream in the job's kernel DAG (NEXT-4) */
  uint32_t n_deps;             /* kernels whose outputs it reads (through concats / fused GAPs) */
  uint32_t deps[8];            /* the first 8 of them */
} paella_kernel_info_t;

int paella_kernel_info(paella_t* p, uint32_t model_id, uint32_t k, paella_kernel_info_t* info);
const char* paella_kernel_name(uint32_t kind);

typedef struct {
  uint64_t admitted, completed, launches, records, torn_retries, decide_calls;
  uint64_t loop_iters;
  int64_t  outstanding_work_ns;   /* W_g published for the router */
  uint64_t ev_launches, ev_ns, ev_bytes, ev_flops;   /* event-timed launches (event_time_kind) */
  uint64_t stop_reason[5];     /* why each decide() pass stopped: [0] no ready work left,
                                  [1] no free stream, [2] occupancy predicate (fits),
                                  [3] ring flow control, [4] ready jobs exist but all are
                                  outside the job cap K (B200-Q6) */
  uint64_t sum_ready, sum_live_jobs, sum_Q;   /* summed over decide() passes (averages) */
  uint64_t rel_events;         /* counter mode: stream-release events recorded (a job left idle) */
  uint64_t xstream_waits;      /* ... of which the job's next kernel went to another stream
                                  and waited for the event (relaxed exits) */
  uint64_t busy_ns;            /* time the dispatcher spent in loop iterations that did work
                                  (admitted, consumed records or issued): its core's useful
                                  load; the rest of the time it spins on empty rings */
} paella_stats_t;

int paella_stats(paella_t* p, uint32_t gpu, paella_stats_t* st);

/* globaltimer -> host clock of GPU `gpu` (SURVEY.md §8(c) C3 "Clocks"), calibrated at
   paella_init by a ping-pong with a probe kernel through mapped memory (the sample with
   the smallest round trip): a record's %globaltimer value t_dev corresponds to host
   CLOCK_MONOTONIC t_dev - *offset_ns, within +- *rtt_ns / 2; *resolution_ns = the
   smallest observed step of %globaltimer.  Also logged as a CLOCK event.  -ENODEV on
   the FAKE device, -ENOTSUP when not calibrated (under a profiler). */
int paella_clock_info(paella_t* p, uint32_t gpu, int64_t* offset_ns, int64_t* rtt_ns, int64_t* resolution_ns);

/* Re-calibrate GPU `gpu`'s clock now (the two clocks drift apart by ppm): a new CLOCK
   event is written to its event log at the dispatcher's current position, so records
   can be converted by interpolating between calibrations.  Blocks for ~100 us; do not
   call it with a profiler attached.  0, -ENODEV (FAKE device), -ENOTSUP, -EIO. */
int paella_clock_sync(paella_t* p, uint32_t gpu);

/* Counter mode, device side of the exactly-once invariant (S5 b, C3): with no job live,
   every counter slot's device {start, end} counts and their host mirror equal the sum of
   the grids of all launches counted on that slot (each block entered and exited once;
   nothing lost, nothing doubled).  Returns the number of mismatching slots (0 = all
   good), *slots_checked = slots used so far; -EBUSY jobs live, -ENOTSUP not counter
   mode, -ENODEV FAKE device. */
int paella_check_counters(paella_t* p, uint32_t gpu, uint32_t* slots_checked);

/* Flush and close the event logs (also done by shutdown). */
int paella_flush_log(paella_t* p);

/* Run one job of model_id synchronously on GPU `gpu`, outside the dispatcher
   (no other work must be in flight): every kernel in order on one stream, with
   instrumentation as configured.  Used by parity tests and the device-only
   roofline (summed isolated kernel time).  If kernel_ns is non-NULL it receives
   n_kernels per-kernel device times (CUDA events).  Returns 0 or -errno. */
int paella_run_isolated(paella_t* p, uint32_t gpu, uint32_t model_id, const void* input,
                        void* output, int64_t* kernel_ns);

/* Device-only kernel timing (the "summed isolated kernel time" roofline of the north
   star, and instrumentation overhead, config 5): kernel k of the model's chain is
   launched `reps` times back to back behind a gate on an otherwise idle GPU
   (instrumented if `instrumented`, else the uninstrumented twin); kernel_ns[k] =
   elapsed / reps.  Returns 0 or -errno. */
int paella_time_kernels(paella_t* p, uint32_t gpu, uint32_t model_id, uint32_t instrumented,
                        uint32_t reps, int64_t* kernel_ns);
#define PAELLA_TIME_L2_COLD 2u   /* `instrumented` bit: L2-cold timing -- before every launch a
                                    256 MiB buffer (2 x L2) is overwritten on the stream and each
                                    launch is timed alone (plain launch, median of reps); without
                                    it the launches run back to back (PDL chain, L2-warm) */

/* X_dev, the device-only saturation throughput: request i runs model
   models[seq[i]] as a CUDA graph of its uninstrumented kernel chain on stream i % streams
   (workspace slot = stream; needs max_jobs_per_model >= streams and no serving in
   progress); all n requests are enqueued at once and *req_per_s = n / device time.  No
   dispatcher, no notifications: the bound the served throughput is compared with. */
int paella_bench_xdev(paella_t* p, uint32_t gpu, const uint32_t* models, uint32_t n_models, const uint32_t* seq,
                      uint32_t n, uint32_t streams, double* req_per_s);

/* Notification microbenchmarks (config 5, P1881-1897 Fig. 15).
   paella_bench_empty: `iters` launches of an empty kernel with `grid` x `block`
   threads, back to back behind a gate; *ns_per_launch = elapsed / iters.
   paella_bench_roundtrip: `n` times, launch a 1-block instrumented empty kernel and
   spin on the ring until its PLACEMENT / COMPLETION records are visible to the host;
   place_ns[i] / complete_ns[i] = host time from before the launch call.  Both run
   on the isolated ring, outside the dispatcher. */
int paella_bench_empty(paella_t* p, uint32_t gpu, uint32_t grid, uint32_t block, uint32_t instrumented,
                       uint32_t group, uint32_t iters, double* ns_per_launch);
int paella_bench_roundtrip(paella_t* p, uint32_t gpu, uint32_t n, int64_t* place_ns, int64_t* complete_ns);

/* ---- open-loop load generator (benchmark harness; same front end for every system) ----
   Replays requests at their scheduled times from the calling thread: request i of
   client c uses io slot (i-th free slot of c) at offset slot*stride in c's region;
   a request waits for a free slot (that wait counts in its JCT).  With copy_inputs
   != NULL (end-to-end mode) the client copies the request's input from
   copy_inputs[model][input_idx] into its slot right before submitting and copies the
   logits out after completion (the host<->device traffic of the step); otherwise the
   slots must hold the inputs already.  jct_ns[i] = completion seen by the client -
   t_sched (scheduled arrival; no coordinated omission).  t0_ns = the monotonic time
   that request times are relative to (0 = now).  Returns completed count or -errno. */
typedef struct {
  int64_t t_ns;        /* scheduled arrival, relative to t0 */
  uint32_t client, model, input_idx, pad;
} paella_req_t;

int64_t paella_loadgen(paella_t* p, const paella_req_t* reqs, uint32_t n, size_t stride,
                       uint32_t slots_per_client, const void* const* const* copy_inputs,
                       int64_t t0_ns, int64_t* jct_ns, int64_t* elapsed_ns);

int paella_bench_wait(paella_t* p, uint32_t client_id, uint32_t model_id, uint32_t n, int64_t gap_ns,
                      uint32_t poll_flags, size_t stride, uint32_t slots, int64_t* jct_ns,
                      double* waiter_cpu_frac);
/* NEXT-3 measurement (P1157-1171, Fig. 14): the calling thread submits n requests of
   one model at a fixed gap (open loop, slots of `stride` bytes in the client's region,
   inputs pre-staged); a second thread waits for the completions with
   paella_poll_completion(poll_flags: 0 = spin, PAELLA_HYBRID).  jct_ns[n]: submit ->
   completion seen; *waiter_cpu_frac: the waiting thread's CPU time / wall time.
   Returns 0 or -errno. */

/* Debug: copy node `node`'s activation of the last isolated run to host as fp32
   NCHW (C*H*W floats).  Returns 0 or -errno. */
int paella_debug_node(paella_t* p, uint32_t gpu, uint32_t model_id, uint32_t node, float* out);

#ifdef __cplusplus
}
#endif
#endif /* PAELLA_H_ */
