// The dispatcher's scheduling state machine (Paella §6, PAPER.md P1222-1323).
//
//   (1) SRPT: remaining = sum_{i in K} max(0, C_i - c_i) * T_i  (P1257-1261).  Our jobs
//       are static kernel chains, so C_i is an exact count and R_j is the sum of the
//       frozen T-bar of the kernels not yet dispatched (readings C2-Q8, C2-Q9).
//   (2) Deficit fairness (P1287-1298): the scheduled client's deficit drops by
//       (1 - 1/N), every other client's rises by 1/N; if a client's deficit exceeds
//       theta, the oldest ready job of the highest-deficit client is chosen.  Kept in
//       integer units of 1/N with a global offset Omega -- the paper's O(1)
//       threshold-shift trick (P1316-1323) without its floating-point underflow.
//   (3) Slack B beyond full utilisation (P1300-1304) and the dispatch loop
//       (P1306-1314): issue while (unplaced blocks Q < B) or (every resource U_r <
//       C_r), and while the notification ring has room for the launch's records
//       (flow control, P1115-1119).
//
// Exactly the rules of oracle/sim.py::Policy; the replay test
// checks the issue sequence bit for bit.  Data structures are the fast ones
// (ordered sets instead of linear scans), the decisions are identical.
#pragma once
#include <cstdint>
#include <set>
#include <tuple>
#include <vector>

namespace paella {

constexpr int NRES = 5;   // blocks, warps, regs, smem, tmem (Table 1 + TMEM)

struct PolicyLayer {
  uint32_t grid;
  int64_t demand[NRES];
  int64_t tbar;
  // NEXT-4 intra-job concurrency (Fig. 7 waitlists, P906-951): virtual stream of the
  // kernel and the kernels of OTHER virtual streams it consumes (they must have
  // completed; predecessors on its own virtual stream are ordered by the stream)
  uint32_t vs = 0;
  std::vector<uint32_t> cross;
};

constexpr uint32_t MAX_VS = 4;   // virtual streams per job

struct PolicyJob {
  uint32_t id = 0;
  uint32_t client = 0, model = 0;
  uint64_t seq = 0;
  int64_t R = 0;
  uint32_t cursor = 0;       // kernels dispatched
  uint32_t done = 0;         // kernels completed
  uint32_t last_uid = 0;
  int64_t rr = -1;           // RR ablation: uid of the last issued kernel (-1 = never)
  uint32_t model_pos = 0;    // index in live_by_model_[model] (NEXT-4)
  bool live = false;
  bool in_ready = false;
  std::vector<uint8_t> state;   // per kernel: 0 waiting, 1 in flight, 2 completed
  // per virtual stream: next kernel (position in the stream), in-flight uids (FIFO),
  // the CUDA stream held while it has kernels in flight, the last one it held
  uint32_t nvs = 1;
  uint32_t vs_next[MAX_VS] = {0};
  uint32_t vs_uid[MAX_VS][8] = {{0}};   // in-flight uids in issue order (vs_infl of them)
  uint8_t vs_infl[MAX_VS] = {0};
  int32_t vs_stream[MAX_VS] = {-1, -1, -1, -1};
  int32_t vs_last[MAX_VS] = {-1, -1, -1, -1};
  uint32_t inflight() const { return cursor - done; }
};

struct PolicyLaunch {
  uint32_t uid = 0, job = 0, layer = 0, grid = 0, stream = 0;
  uint32_t p = 0, f = 0;
  bool live = false;
  bool has_obs = false;      // NEXT-4: an observed duration is pending for this launch
  int64_t obs = 0;
};

struct Issue {
  uint32_t uid, job, layer, stream;
};

enum : uint32_t { POL_SRPT_DEFICIT = 0, POL_FIFO = 1, POL_SJF = 2, POL_RR = 3 };   // SJF/RR: Table 3 ablations

class Policy {
 public:
  struct Cfg {
    uint32_t num_clients = 1, policy = POL_SRPT_DEFICIT;
    int64_t theta = 100;
    int64_t slack = 148;
    uint32_t group = 16;
    int64_t ring_capacity = 65536;
    uint32_t streams = 32;
    int64_t capacity[NRES] = {148 * 32, 148 * 64, 148 * 65536, 148 * 233472, 148 * 512};
    uint32_t lookahead = 0;   // NEXT-1 launch-ahead depth (0 = the paper's semantics)
    uint32_t prio_classes = 1;   // stream-priority classes (1 = the paper: one class)
    uint32_t online_tbar = 0;    // NEXT-4: refine T-bar online (running average, P1252-1254)
    uint32_t max_active = 0;     // K: only the K first jobs in the policy's order that still
                                 // have kernels to issue may issue (0 = no cap); B200-Q6
    uint32_t la_unplaced = 0;    // NEXT-1 variant: launch-ahead without the oldest-placed test
    uint32_t cap_fifo = 0;       // B200-Q6 variant: the job cap admits in arrival order
  };
  static constexpr int64_t kProfileRuns = 20;   // observations behind the profiled T-bar
  // class of stream s: consecutive index ranges, class 0 = highest hardware priority
  static uint32_t stream_class(uint32_t s, uint32_t K, uint32_t P) { return (uint32_t)((uint64_t)s * K / P); }

  explicit Policy(const Cfg& c);

  void add_model(uint32_t mid, const std::vector<PolicyLayer>& layers);
  const std::vector<PolicyLayer>& model(uint32_t m) const { return models_[m]; }

  // job ids are dense, assigned by the caller in admission order
  void arrival(uint32_t job_id, uint32_t client, uint32_t model);
  // returns true if the launch finished; *job_done set if its job completed
  bool record(uint32_t type, uint32_t uid, uint32_t n, int64_t* job_done);
  // NEXT-4: duration of launch uid (first PLACEMENT seen -> final COMPLETION seen),
  // consumed right before its final COMPLETION record (logged as an OBSERVE event)
  void observe(uint32_t uid, int64_t d);
  // dispatch loop; appends issues
  void decide(std::vector<Issue>* out);

  int64_t outstanding_work() const { return work_; }
  uint64_t live_jobs() const { return live_jobs_; }
  const PolicyJob& job(uint32_t id) const { return jobs_[id]; }
  const PolicyLaunch& launch(uint32_t uid) const { return launches_[uid % kLaunchSlots]; }
  int64_t deficit(uint32_t c) const { return Dt_[c] + Omega_; }
  int64_t Q() const { return Q_; }
  // why the last decide() stopped: 0 nothing ready, 1 no free stream, 2 fits, 3 ring,
  // 4 ready jobs all outside the job cap
  int last_stop() const { return last_stop_; }
  size_t ready_count() const { return srpt_.size(); }
  int64_t O() const { return O_; }

 private:
  static constexpr uint32_t kLaunchSlots = 8192;
  static constexpr uint32_t kMaxModels = 256;
  bool pick(uint32_t* job_id);
  bool pick_capped(uint32_t* job_id) const;
  uint32_t job_class(const PolicyJob& j) const;
  int lowest_free_in_class(uint32_t c) const;
  bool predicate(uint32_t grid) const;
  int64_t order_key(const PolicyJob& j) const;
  int64_t active_key(const PolicyJob& j) const;
  void active_erase(const PolicyJob& j);
  void active_insert(const PolicyJob& j);
  void refine(const PolicyLaunch& L);
  void make_ready(PolicyJob& j);
  void make_unready(PolicyJob& j);
  bool is_ready(const PolicyJob& j) const { return head(j) >= 0; }
  int64_t head(const PolicyJob& j) const;
  void refresh(PolicyJob& j);
  int lowest_free() const;

  Cfg cfg_;
  std::vector<std::vector<PolicyLayer>> models_;
  std::vector<std::vector<std::vector<uint32_t>>> vs_kernels_;   // per model, per virtual stream
  std::vector<PolicyJob> jobs_;
  std::vector<PolicyLaunch> launches_;
  int64_t U_[NRES] = {0, 0, 0, 0, 0};
  int64_t Q_ = 0, O_ = 0;
  int last_stop_ = 0;
  bool over_ = false;                  // the last pick was a deficit override
  std::vector<int64_t> totals_;        // sorted distinct whole-job T-bar sums of the models
  std::vector<int64_t> model_total_;   // whole-job T-bar sum per model (SJF key)
  std::vector<std::vector<int64_t>> tb_sum_, tb_cnt_;   // NEXT-4 running averages
  std::vector<std::vector<uint32_t>> live_by_model_;    // live job ids per model (NEXT-4)
  std::vector<uint64_t> free_;   // bitmap of free streams
  std::vector<int64_t> Dt_;
  int64_t Omega_ = 0;
  std::vector<uint32_t> unfinished_;
  uint32_t next_uid_ = 0;
  uint64_t next_seq_ = 0;
  int64_t work_ = 0;             // sum of R over live jobs (router's W_g)
  uint64_t live_jobs_ = 0;
  // ready structures
  std::set<std::tuple<int64_t, uint64_t, uint32_t>> srpt_;     // (R, seq, id)
  std::set<std::pair<uint64_t, uint32_t>> fifo_;               // (seq, id)
  std::vector<std::set<std::pair<uint64_t, uint32_t>>> per_client_;  // (seq, id)
  // B200-Q6: live jobs with kernels left to issue, in the policy's order (max_active > 0)
  std::set<std::tuple<int64_t, uint64_t, uint32_t>> active_;
};

}  // namespace paella
