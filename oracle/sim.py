"""ORACLE (test infrastructure) -- C2: scheduling-policy reference + discrete-event
simulator, step by step in the paper's order.

Paper: §6 "Scheduling Strategy" (PAPER.md P1222-1323): (1) SRPT on the remaining
time  remaining = sum_{i in K} max(0, C_i - c_i) * T_i  (P1257-1261), (2) deficit
counters -- the scheduled user's deficit drops by (1 - 1/#users), every other
user's rises by 1/#users; above a threshold the oldest job of the highest-deficit
client is chosen (P1287-1298), (3) B blocks of slack beyond full utilisation
(P1300-1304), and the dispatch loop (P1306-1314).  Notification semantics: Fig. 6
(P848-870), flow control (P1115-1119), block groups of <=16 (P1138-1142).  Resource
accounting: Table 1 (P782-802).  Every reading of a silent/garbled passage is
SURVEY.md §8(c) C2-Q1..Q20, restated in DESIGN.md §"Readings".

The state machine ``Policy`` is the reference for the C++ dispatcher: replaying the
dispatcher's event log through it (``replay``) must reproduce the dispatcher's issue
sequence (uid, job, layer, stream) bit-exactly (pin S6).  All quantities are
integers: times in ns, deficits in units of 1/N with a global offset Omega
(the paper's O(1) threshold-shift trick, P1316-1323, in integer form).

``SyntheticGPU`` + ``simulate`` model a GPU (S SMs with Table-1 resources, H FIFO
hardware queues, greedy placement, launch/notification delays) driving either the
Paella dispatcher (``Policy``) or the naive submit-everything-at-arrival baseline.
It backs the brute-force and closed-form pins (S1-S3), the invariants (S5) and
what-if sweeps; it is not expected to reproduce B200 timing.
"""
from __future__ import annotations

import heapq
import itertools
from dataclasses import dataclass, field

PLACEMENT, COMPLETION = 1, 2
SRPT_DEFICIT, FIFO, SJF, RR = 0, 1, 2, 3   # SJF / RR: Table 3 ablations (NEXT-2, P1341-1359)
RESOURCES = ("blocks", "warps", "regs", "smem", "tmem")
INF_THETA = (1 << 63) - 1


@dataclass
class Layer:
    grid: int
    demand: tuple          # per-block demand, one int per RESOURCES entry (blocks=1)
    tbar: int              # profiled mean kernel time, ns (frozen)
    dur: int = 0           # synthetic-mode block duration, ns
    # NEXT-4 intra-job concurrency (Fig. 7 waitlists, P918-951): the kernels this one
    # consumes (None = the previous kernel: a chain) and its virtual stream
    deps: tuple | None = None
    vs: int = 0


class Topo:
    """A model's kernel DAG as the dispatcher sees it (Fig. 7 waitlists, P906-951):
    per kernel its dependencies and virtual stream; per virtual stream its kernels in
    order.  A kernel is *active* (CUDA stream semantics, P943-947) when it is the next
    kernel of its virtual stream and every kernel it depends on in ANOTHER virtual stream
    has completed; its predecessors in its own virtual stream are ordered by the stream."""

    def __init__(self, layers):
        n = len(layers)
        self.deps = [tuple(range(k - 1, k)) if L.deps is None else tuple(L.deps) for k, L in enumerate(layers)]
        self.vs = [L.vs for L in layers]
        nv = 1 + max(self.vs, default=0)
        self.vs_kernels = [[k for k in range(n) if self.vs[k] == v] for v in range(nv)]
        self.pos = [self.vs_kernels[self.vs[k]].index(k) for k in range(n)]
        self.cross = [tuple(d for d in self.deps[k] if self.vs[d] != self.vs[k]) for k in range(n)]


@dataclass
class Config:
    num_clients: int
    policy: int = SRPT_DEFICIT
    theta: int = 100                  # fairness threshold in kernel dispatches
    slack: int = 148                  # B, in blocks
    group: int = 16                   # G
    ring_capacity: int = 65536
    streams: int = 32                 # P
    capacity: tuple = (148 * 32, 148 * 64, 148 * 65536, 148 * 233472, 148 * 512)
    lookahead: int = 0                # NEXT-1 launch-ahead depth (0 = the paper's semantics)
    prio_classes: int = 1             # stream-priority classes (1 = the paper: one class)
    online_tbar: int = 0              # NEXT-4: refine T-bar online (running average, P1252-1254)
    max_active: int = 0               # K: only the K first jobs in the policy's order that still
                                      # have kernels to issue may issue (0 = no cap); B200-Q6
    lookahead_unplaced: int = 0       # NEXT-1 variant: launch-ahead without the oldest-placed test
    cap_fifo: int = 0                 # B200-Q6 variant: the job cap admits in arrival order


# NEXT-4 (P1249-1266: "x-bar is the average of all previous observations of x"; "these
# profiles can be further refined online"): with online_tbar, T-bar of (model, layer)
# is the integer running average of the PROFILE_RUNS profiling observations plus every
# observed duration of that kernel (first PLACEMENT seen -> final COMPLETION seen by the
# dispatcher, logged as an OBSERVE event).  It is updated when the launch completes;
# every live job whose remaining kernels include that layer has R_j adjusted by the
# change.  SJF keys and stream-priority classes keep the frozen profile.
PROFILE_RUNS = 20


def groups(g, G):
    return -(-g // G)


@dataclass
class Job:
    id: int
    client: int
    model: int
    seq: int
    R: int
    cursor: int = 0          # kernels dispatched (c_i of P1265)
    done: int = 0            # kernels completed
    last_uid: int = -1
    rr: int = -1             # RR ablation: uid of the job's last issued kernel (-1 = never)
    # per kernel: 0 = waiting, 1 = in flight, 2 = completed
    state: list = field(default_factory=list)
    # per virtual stream: next kernel (position), in-flight uids (issue order), the CUDA
    # stream held while it has kernels in flight, the last stream it held
    vs_next: list = field(default_factory=list)
    vs_uids: list = field(default_factory=list)
    vs_stream: list = field(default_factory=list)
    vs_last: list = field(default_factory=list)

    @property
    def inflight(self):
        return self.cursor - self.done


@dataclass
class Launch:
    uid: int
    job: int
    layer: int
    grid: int
    demand: tuple
    stream: int
    p: int = 0
    f: int = 0


class Policy:
    """The dispatcher state machine of SURVEY.md §8(c) C2, integer-exact.

    Launch-ahead (NEXT-1; off by default): with lookahead = D > 0 a
    job whose OLDEST in-flight kernel is fully placed (p_eff = grid, i.e. running) and
    that has at most D kernels in flight may issue its next kernel onto the SAME stream
    (stream order carries the dependency, P947-951); the paper's semantics is D = 0."""

    def __init__(self, cfg: Config, models: list[list[Layer]]):
        self.cfg = cfg
        self.models = models
        self.jobs: dict[int, Job] = {}
        self.launches: dict[int, Launch] = {}
        self.U = [0] * len(RESOURCES)
        self.Q = 0
        self.O = 0
        self.free = set(range(cfg.streams))
        self.Dt = [0] * cfg.num_clients      # stored deficits D~_c
        self.Omega = 0                       # global offset
        self.unfinished = [0] * cfg.num_clients
        self.next_uid = 0
        self.next_seq = 0
        self.completed: list[int] = []
        self.issues: list[tuple] = []
        self.over = False                    # the last pick was a deficit override
        self.checks = True                   # assert invariants (c),(d),(g) as we go
        self.log: list[tuple] | None = None  # consumed-event log in replay format
        # current T-bar per (model, layer) and the running-average state (NEXT-4)
        self.tb = [[l.tbar for l in m] for m in models]
        self.tb_sum = [[l.tbar * PROFILE_RUNS for l in m] for m in models]
        self.tb_cnt = [[PROFILE_RUNS for _ in m] for m in models]
        self.obs: dict[int, int] = {}        # launch uid -> observed duration (pending)
        # models known to the dispatcher so far (a model registered while serving enters
        # the stream-priority class boundaries at its MODEL event; replay feeds them in
        # log order, a fresh Policy knows every model)
        self.registered = set(range(len(models)))
        self.topo = [Topo(m) for m in models]

    # effective deficit, units of 1/N
    def D(self, c):
        return self.Dt[c] + self.Omega

    def remaining(self, model, cursor):
        """R_j = sum of T-bar over kernels not yet dispatched (C2-Q8, C2-Q9)."""
        return sum(self.tb[model][cursor:])

    def observe(self, uid, d):
        """NEXT-4: the duration of launch uid, consumed before its final COMPLETION."""
        if self.log is not None:
            self.log.append((EV_OBSERVE, uid, d))
        self.obs[uid] = d

    def _refine(self, L):
        d = self.obs.pop(L.uid, None)
        if not self.cfg.online_tbar or d is None:
            return
        m, lay = self.jobs[L.job].model, L.layer
        self.tb_sum[m][lay] += d
        self.tb_cnt[m][lay] += 1
        new = self.tb_sum[m][lay] // self.tb_cnt[m][lay]
        delta = new - self.tb[m][lay]
        self.tb[m][lay] = new
        if delta:
            for j in self.jobs.values():
                if j.model == m and j.state[lay] == 0:      # not dispatched yet
                    j.R += delta

    # --- events -------------------------------------------------------------
    def arrival(self, job_id, client, model):
        if self.unfinished[client] == 0:          # C2-Q11: idle client restarts at 0
            self.Dt[client] = -self.Omega
        self.unfinished[client] += 1
        if self.log is not None:
            self.log.append((EV_ARRIVAL, job_id, client, model))
        j = Job(job_id, client, model, self.next_seq, self.remaining(model, 0))
        nv = len(self.topo[model].vs_kernels)
        j.state = [0] * len(self.models[model])
        j.vs_next, j.vs_uids = [0] * nv, [[] for _ in range(nv)]
        j.vs_stream, j.vs_last = [-1] * nv, [-1] * nv
        self.next_seq += 1
        self.jobs[job_id] = j
        return j

    def record(self, typ, uid, n):
        """Consume one notification record (type, launch uid, block count)."""
        L = self.launches[uid]
        self.O -= 1
        if self.log is not None:
            self.log.append((EV_RECORD, typ, uid, n))
        old = max(L.p, L.f)
        if typ == PLACEMENT:
            L.p += n
        elif typ == COMPLETION:
            L.f += n
            for r in range(len(RESOURCES)):
                self.U[r] -= n * L.demand[r]
        else:
            raise ValueError(typ)
        self.Q -= max(L.p, L.f) - old
        assert L.p <= L.grid and L.f <= L.grid
        done = None
        if L.f == L.grid:
            del self.launches[uid]
            self._refine(L)
            j = self.jobs[L.job]
            j.done += 1
            j.state[L.layer] = 2
            v = self.topo[j.model].vs[L.layer]
            j.vs_uids[v].remove(uid)
            if not j.vs_uids[v]:              # the virtual stream drained: its stream is free
                self.free.add(L.stream)
                j.vs_stream[v] = -1
                j.vs_last[v] = L.stream
            if j.done == len(self.models[j.model]):
                if self.checks:
                    assert j.R == 0
                del self.jobs[j.id]
                self.unfinished[j.client] -= 1
                self.completed.append(j.id)
                if self.log is not None:
                    self.log.append((EV_COMPLETE, j.id))
                done = j.id
        return done

    def head(self, j):
        """The job's lowest-index active kernel that may be dispatched now, or None:
        the next kernel of a virtual stream whose cross-stream dependencies have all
        completed, and whose stream is idle -- or, with launch-ahead D > 0, whose oldest
        in-flight kernel is fully placed (running) with at most D in flight (with
        lookahead_unplaced: at most D in flight, whether or not the oldest is placed)."""
        T = self.topo[j.model]
        best = None
        for v, ks in enumerate(T.vs_kernels):
            if j.vs_next[v] >= len(ks):
                continue
            k = ks[j.vs_next[v]]
            if any(j.state[d] != 2 for d in T.cross[k]):
                continue
            infl = len(j.vs_uids[v])
            if infl > 0:
                if self.cfg.lookahead <= 0 or infl > self.cfg.lookahead:
                    continue
                L = self.launches[j.vs_uids[v][0]]          # the oldest kernel in flight
                if not self.cfg.lookahead_unplaced and max(L.p, L.f) < L.grid:
                    continue
            if best is None or k < best:
                best = k
        return best

    def is_ready(self, j):
        return self.head(j) is not None

    def ready(self):
        return [j for j in self.jobs.values() if self.is_ready(j)]

    def order(self, j):
        """The policy's total order on jobs (ties: arrival seq, then job id)."""
        p = self.cfg.policy
        if p == FIFO:
            return (j.seq, j.id)
        if p == SJF:               # shortest (whole) job first: profiled T-bar sum of the model
            return (sum(l.tbar for l in self.models[j.model]), j.seq, j.id)
        if p == RR:                # kernel-granular round robin: least recently issued job
            return (j.rr, j.seq, j.id)
        return (j.R, j.seq, j.id)  # SRPT

    def eligible(self):
        """B200-Q6: with max_active = K > 0, the ids of the K first jobs, in the
        policy's order (cap_fifo: in arrival order), among the live jobs that still have
        kernels to issue; None = no cap."""
        K = self.cfg.max_active
        if K <= 0:
            return None
        left = [j for j in self.jobs.values() if j.cursor < len(self.models[j.model])]
        key = (lambda j: (j.seq, j.id)) if self.cfg.cap_fifo else self.order
        return {j.id for j in sorted(left, key=key)[:K]}

    def pick(self, rdy):
        cfg = self.cfg
        self.over = False
        top = self.eligible()
        ok = rdy if top is None else [j for j in rdy if j.id in top]
        if cfg.policy != SRPT_DEFICIT:
            return min(ok, key=self.order) if ok else None
        clients = sorted({j.client for j in rdy})
        cstar = max(clients, key=lambda c: (self.D(c), -c))
        self.over = cfg.theta != INF_THETA and self.D(cstar) > cfg.theta * cfg.num_clients
        if self.over:            # the deficit rule overrides the cap as it overrides SRPT
            return min((j for j in rdy if j.client == cstar), key=lambda j: j.seq)
        return min(ok, key=self.order) if ok else None

    # Stream-priority classes (B200 adaptation, reading B200-Q2).  The pool's
    # P streams are split into K classes of consecutive indices (class 0 = highest
    # hardware priority), so the blocks the +B slack leaves queued in hardware
    # (P1300-1304) are served in SRPT order too.  A job takes a stream of the class
    # of its remaining work: the number of registered models whose whole-job T-bar sum
    # is strictly below R_j (clamped to K-1); a deficit-override pick takes class 0.
    def stream_class(self, s):
        return s * self.cfg.prio_classes // self.cfg.streams

    def job_class(self, j):
        K = self.cfg.prio_classes
        if K <= 1 or self.over:
            return 0
        totals = sorted({sum(layer.tbar for layer in m) for i, m in enumerate(self.models)
                         if m and i in self.registered})
        return min(K - 1, sum(1 for t in totals if t < j.R))

    def predicate(self, grid):
        cfg = self.cfg
        fits = self.Q < cfg.slack or all(u < c for u, c in zip(self.U, cfg.capacity))
        ring_ok = self.O + 2 * groups(grid, cfg.group) <= cfg.ring_capacity
        return fits and ring_ok

    def decide(self):
        """Dispatch loop (P1306-1314). Returns the list of issues made."""
        cfg = self.cfg
        out = []
        if self.log is not None:
            self.log.append((EV_BATCH_END,))
        while True:
            rdy = self.ready()
            if not rdy:
                break
            j = self.pick(rdy)
            if j is None:
                break
            k = self.head(j)
            v = self.topo[j.model].vs[k]
            if not j.vs_uids[v] and not self.free:
                break
            layer = self.models[j.model][k]
            if not self.predicate(layer.grid):
                break
            uid = self.next_uid
            self.next_uid += 1
            if j.vs_uids[v]:
                stream = j.vs_stream[v]      # launch-ahead: behind its predecessor
            else:
                c = self.job_class(j)
                last = j.vs_last[v]
                if last in self.free and self.stream_class(last) == c:
                    stream = last
                else:
                    cand = [s for s in self.free if self.stream_class(s) == c]
                    stream = min(cand) if cand else min(self.free)
                self.free.remove(stream)
                j.vs_stream[v] = stream
            self.launches[uid] = Launch(uid, j.id, k, layer.grid, layer.demand, stream)
            for r in range(len(RESOURCES)):
                self.U[r] += layer.grid * layer.demand[r]
            self.Q += layer.grid
            self.O += 2 * groups(layer.grid, cfg.group)
            j.R -= self.tb[j.model][k]
            rec = (uid, j.id, k, stream)
            j.state[k] = 1
            j.vs_uids[v].append(uid)
            j.vs_next[v] += 1
            j.cursor += 1
            j.last_uid = uid
            j.rr = uid
            if self.checks:
                assert j.R >= 0
            self.Dt[j.client] -= cfg.num_clients
            self.Omega += 1
            if self.log is not None:
                self.log.append((EV_ISSUE,) + rec)
            out.append(rec)
            self.issues.append(rec)
        return out


# ---------------------------------------------------------------------------
# Replay mode (pin S6)
# ---------------------------------------------------------------------------

EV_ARRIVAL, EV_RECORD, EV_BATCH_END, EV_ISSUE, EV_COMPLETE, EV_OBSERVE = 1, 2, 3, 4, 5, 6
EV_MODEL = 110


def replay(cfg: Config, models, events, published=None):
    """Drive ``Policy`` with a recorded event sequence.

    events: iterable of tuples
      (EV_ARRIVAL, job_id, client, model) | (EV_RECORD, type, uid, n) |
      (EV_BATCH_END,) | (EV_ISSUE, uid, job, layer, stream) | (EV_COMPLETE, job_id)
    Inputs (arrivals, records, batch ends) are applied in order; the policy's own
    issues / completions are compared with the logged ones.  Returns
    (ok, first_divergence_message, n_issues_checked).

    published: optional list; receives the dispatcher's outstanding work W_g = sum of
    R_j over live jobs after every decide pass (the value it publishes to the router,
    SURVEY.md §8(e)), starting with 0.
    """
    pol = Policy(cfg, models)
    if published is not None:
        published.append(0)
    if any(ev[0] == EV_MODEL for ev in events):
        pol.registered = set()     # models enter at their MODEL events
    expect = []            # issues the policy produced, awaiting the logged ones
    expect_done = []
    n = 0
    for ev in events:
        k = ev[0]
        if k == EV_MODEL:
            pol.registered.add(ev[1])
        elif k == EV_ARRIVAL:
            pol.arrival(ev[1], ev[2], ev[3])
        elif k == EV_OBSERVE:
            pol.observe(ev[1], ev[2])
        elif k == EV_RECORD:
            d = pol.record(ev[1], ev[2], ev[3])
            if d is not None:
                expect_done.append(d)
        elif k == EV_BATCH_END:
            if expect:
                return False, f"dispatcher issued fewer kernels than the reference: missing {expect[0]}", n
            expect = list(pol.decide())
            if published is not None:
                published.append(sum(j.R for j in pol.jobs.values()))
        elif k == EV_ISSUE:
            got = tuple(ev[1:5])
            if not expect:
                return False, f"dispatcher issued {got} where the reference issues nothing", n
            want = expect.pop(0)
            if want != got:
                return False, f"issue #{n}: dispatcher {got} != reference {want}", n
            n += 1
        elif k == EV_COMPLETE:
            if not expect_done or expect_done[0] != ev[1]:
                return False, f"completion {ev[1]} != reference {expect_done[:1]}", n
            expect_done.pop(0)
    if expect:
        return False, f"log ends with reference issues pending: {expect[0]}", n
    return True, "", n


# ---------------------------------------------------------------------------
# Synthetic mode: a GPU model
# ---------------------------------------------------------------------------

@dataclass
class GPUModel:
    sms: int = 148
    per_sm: tuple = (32, 64, 65536, 233472, 512)   # Table 1 + TMEM, per SM
    hw_queues: int = 32                            # H
    launch_delay: int = 0                          # delta_l, ns
    notif_delay: int = 0                           # delta_n, ns
    decide_delay: int = 0                          # scheduler delay per decide pass, ns (Fig. 9):
                                                   # the dispatcher is busy that long after each
                                                   # pass; its issues launch after it


@dataclass
class SimResult:
    arrival: dict = field(default_factory=dict)
    finish: dict = field(default_factory=dict)
    issues: list = field(default_factory=list)
    records: list = field(default_factory=list)    # (t, type, uid, n, group)
    blocks: list = field(default_factory=list)     # (uid, sm, t_start, t_end)
    max_running_blocks: int = 0
    busy_block_time: int = 0
    violations: list = field(default_factory=list)
    policy: Policy | None = None

    def jct(self):
        return {j: self.finish[j] - self.arrival[j] for j in self.finish}


class _Kernel:
    __slots__ = ("uid", "job", "layer", "grid", "demand", "dur", "stream", "placed", "done",
                 "start_count", "end_count")

    def __init__(self, uid, job, layer, grid, demand, dur, stream):
        self.uid, self.job, self.layer = uid, job, layer
        self.grid, self.demand, self.dur, self.stream = grid, demand, dur, stream
        self.placed = self.done = 0
        self.start_count = self.end_count = 0


def simulate(cfg: Config, models, trace, gpu: GPUModel, system="paella", naive_streams=None,
             check=True, horizon=None):
    """Event-driven simulation.

    trace: list of (t_arrival_ns, client, model).  system: 'paella' (Policy drives
    issue) or 'naive' (every kernel of a job enters stream job % naive_streams at
    arrival; the hardware model decides everything).  Returns SimResult.
    """
    res = SimResult()
    S = gpu.sms
    free_sm = [list(gpu.per_sm) for _ in range(S)]
    hwq = [[] for _ in range(gpu.hw_queues)]       # FIFO of _Kernel per hardware queue
    stream_busy_until_done = {}                    # stream -> kernel currently ahead
    stream_fifo = {}                               # stream -> list of kernels (stream order)
    evq = []
    cnt = itertools.count()

    def push(t, kind, *a):
        heapq.heappush(evq, (t, next(cnt), kind, a))

    pol = Policy(cfg, models) if system == "paella" else None
    if pol is not None:
        pol.checks = check
    res.policy = pol
    naive_streams = naive_streams or cfg.streams
    running_blocks = 0
    uid_counter = itertools.count()

    for jid, (t, c, m) in enumerate(trace):
        push(t, "arrival", jid, c, m)

    def enqueue_kernel(k):
        # CUDA stream semantics: a kernel waits for its stream predecessor; the
        # stream is bound to hardware queue stream % H (FIFO, head-of-line).
        stream_fifo.setdefault(k.stream, []).append(k)
        hwq[k.stream % gpu.hw_queues].append(k)

    def try_place(t):
        nonlocal running_blocks
        progress = True
        while progress:
            progress = False
            for q in hwq:
                if not q:
                    continue
                k = q[0]
                # the head kernel must also be the head of its stream
                if stream_fifo[k.stream][0] is not k:
                    continue
                while k.placed < k.grid:
                    sm = next((i for i in range(S)
                               if all(free_sm[i][r] >= k.demand[r] for r in range(len(RESOURCES)))), None)
                    if sm is None:
                        break
                    for r in range(len(RESOURCES)):
                        free_sm[sm][r] -= k.demand[r]
                    k.placed += 1
                    running_blocks += 1
                    res.max_running_blocks = max(res.max_running_blocks, running_blocks)
                    progress = True
                    push(t, "block_start", k, sm)
                    push(t + k.dur, "block_end", k, sm, t)
                if k.placed == k.grid:
                    q.pop(0)
                    progress = True

    def emit(t, typ, k, count):
        G = cfg.group
        if count % G == 0 or count == k.grid:
            n = G if count % G == 0 else count % G
            grp = (count - 1) // G
            res.records.append((t, typ, k.uid, n, grp))
            if pol is not None:
                push(t + gpu.notif_delay, "record", typ, k.uid, n)

    busy = [0, False]       # dispatcher busy until busy[0]; a deferred pass is pending

    def dispatch(t):
        if gpu.decide_delay:
            if t < busy[0]:                 # still deciding: one more pass once it is free
                if not busy[1]:
                    busy[1] = True
                    push(busy[0], "decide")
                return
            busy[0] = t + gpu.decide_delay
        for (uid, jid, layer, stream) in pol.decide():
            m = pol.jobs[jid].model
            L = models[m][layer]
            res.issues.append((t, uid, jid, layer, stream))
            push(t + gpu.decide_delay + gpu.launch_delay, "launch",
                 _Kernel(uid, jid, layer, L.grid, L.demand, L.dur, stream))

    kernels_left = {}
    seen = False
    while evq:
        t, _, kind, a = heapq.heappop(evq)
        if horizon is not None and t > horizon:
            break
        if kind == "arrival":
            jid, c, m = a
            res.arrival[jid] = t
            if pol is not None:
                pol.arrival(jid, c, m)
            else:
                s = jid % naive_streams
                kernels_left[jid] = len(models[m])
                for li, L in enumerate(models[m]):
                    k = _Kernel(next(uid_counter), jid, li, L.grid, L.demand, L.dur, s)
                    res.issues.append((t, k.uid, jid, li, s))
                    enqueue_kernel(k)
                try_place(t)
        elif kind == "launch":
            enqueue_kernel(a[0])
            try_place(t)
        elif kind == "block_start":
            k, sm = a
            k.start_count += 1
            emit(t, PLACEMENT, k, k.start_count)
        elif kind == "block_end":
            k, sm, t0 = a
            for r in range(len(RESOURCES)):
                free_sm[sm][r] += k.demand[r]
            running_blocks -= 1
            res.busy_block_time += t - t0
            res.blocks.append((k.uid, sm, t0, t))
            k.end_count += 1
            emit(t, COMPLETION, k, k.end_count)
            if k.end_count == k.grid:
                fifo = stream_fifo[k.stream]
                assert fifo[0] is k
                fifo.pop(0)
                if pol is None:
                    kernels_left[k.job] -= 1
                    if kernels_left[k.job] == 0:
                        res.finish[k.job] = t
            try_place(t)
        elif kind == "record":
            typ, uid, n = a
            done = pol.record(typ, uid, n)
            if done is not None:
                res.finish[done] = t
        elif kind == "decide":
            busy[1] = False
        # the dispatcher decides once every event of this instant is consumed -- after the
        # events it observes (arrivals, records, its own deferred pass); launches and block
        # starts/ends inside the GPU change nothing the policy can see
        if kind in ("arrival", "record", "decide"):
            seen = True
        if pol is not None and seen and (not evq or evq[0][0] > t):
            seen = False
            dispatch(t)
        if check:
            for i in range(S):
                if any(v < 0 for v in free_sm[i]):
                    res.violations.append(("capacity", t, i))
    return res


# ---------------------------------------------------------------------------
# Invariants (pin S5), usable on simulator results and on GPU event logs
# ---------------------------------------------------------------------------

def check_exactly_once(records, grids, G):
    """(b): per uid, sum of PLACEMENT counts = sum of COMPLETION counts = grid,
    ceil(grid/G) records per type, group indices unique and covering [0, ceil)."""
    per = {}
    for rec in records:
        _, typ, uid, n, grp = rec[:5]
        per.setdefault((uid, typ), []).append((grp, n))
    bad = []
    for uid, g in grids.items():
        for typ in (PLACEMENT, COMPLETION):
            lst = per.get((uid, typ), [])
            ng = groups(g, G)
            gs = sorted(x[0] for x in lst)
            if gs != list(range(ng)) or sum(x[1] for x in lst) != g:
                bad.append((uid, typ, lst))
    return bad


def deficit_bound_holds(trace_of_D, N, theta):
    """(f): for a client continuously ready since s, D(t) <= max(D(s), theta*N) + N."""
    bad = []
    for c, series in trace_of_D.items():
        if not series:
            continue
        d0 = series[0]
        for d in series:
            if d > max(d0, theta * N) + N:
                bad.append((c, d0, d))
    return bad


# --- multi-GPU routing variant ---------------------------------

M64 = (1 << 64) - 1


def splitmix64(state):
    """One output of Vigna's SplitMix64 generator from ``state`` (the state is
    advanced by the golden gamma, then mixed)."""
    z = (state + 0x9E3779B97F4A7C15) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def route_pair(req_id, num_gpus):
    """Power-of-two-choices candidates of request ``req_id`` (SURVEY.md §8(e),
    ``include/paella.h`` paella_route_pair): two distinct GPUs drawn from one
    SplitMix64 output of the request id."""
    if num_gpus == 1:
        return 0, 0
    h = splitmix64(req_id)
    g0 = h % num_gpus
    g1 = (g0 + 1 + (h >> 32) % (num_gpus - 1)) % num_gpus
    return g0, g1


def route_pick(pair, W):
    """The candidate with the lower outstanding work W[g]; ties to the lower index."""
    lo, hi = min(pair), max(pair)
    return hi if W[hi] < W[lo] else lo


# --- least-outstanding-work routing -------------------------------

def route_least_work(work, pending, tbar_model, alive):
    """The GPU a request goes to under least outstanding work: W_g = work[g] (the sum of
    R_j its dispatcher last published) + pending[g] (submissions routed to g and not yet
    admitted) x the request model's whole-job T-bar sum; argmin over the GPUs that have
    not failed (bit g of ``alive``), ties to the lowest index."""
    best = None
    for g in range(len(work)):
        if not (alive >> g) & 1:
            continue
        w = work[g] + pending[g] * tbar_model
        if best is None or w < best[0]:
            best = (w, g)
    return None if best is None else best[1]


def check_inflight_bound(events, models, lookahead):
    """NEXT-1 invariant on a consumed-event log: a job never has more than lookahead + 1
    kernels of one virtual stream issued whose final COMPLETION has not been consumed
    (launch-ahead depth D), and each virtual stream issues its kernels in order (a chain
    job has one virtual stream: layer order).  Returns the violations."""
    topo = [Topo(m) for m in models]
    model_of, grid_of, done_of, infl, nxt = {}, {}, {}, {}, {}
    bad = []
    for ev in events:
        k = ev[0]
        if k == EV_ARRIVAL:
            model_of[ev[1]] = ev[3]
            nv = len(topo[ev[3]].vs_kernels)
            infl[ev[1]] = [0] * nv
            nxt[ev[1]] = [0] * nv
        elif k == EV_ISSUE:
            uid, job, layer = ev[1], ev[2], ev[3]
            T = topo[model_of[job]]
            v = T.vs[layer]
            if T.vs_kernels[v][nxt[job][v]] != layer:
                bad.append(("order", uid, job, layer))
            nxt[job][v] += 1
            grid_of[uid] = (job, v, models[model_of[job]][layer].grid)
            done_of[uid] = 0
            infl[job][v] += 1
            if infl[job][v] > lookahead + 1:
                bad.append(("depth", uid, job, infl[job][v]))
        elif k == EV_RECORD and ev[1] == COMPLETION and ev[2] in grid_of:
            uid = ev[2]
            done_of[uid] += ev[3]
            job, v, g = grid_of[uid]
            if done_of[uid] == g:
                infl[job][v] -= 1
    return bad
