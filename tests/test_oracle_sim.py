"""Pins for oracle C2 (policy reference + discrete-event simulator), SURVEY.md §8(c):

S1a  brute force: single server, all releases at 0 -> SRPT total JCT = exhaustive min
S1b  brute force: unit kernels, integer releases -> SRPT = exhaustive min incl. idling
S1c  SRPT is NOT optimal in general (counterexample kept as a regression guard)
S2   Fig. 1 setup (P214-219): 4 jobs x 3 unit kernels, 2 SMs -> mean JCT 4.5
S3   Fig. 2 closed form (P431-442): naive job-by-job submission caps running
     kernels at H = 32 of 176; the dispatcher reaches 176
S4   special cases: theta=inf / N=1 => SRPT; theta=0 => round-robin windows; FIFO order
S5   invariants: capacity, exactly-once records, dependency, predicate, deficit
     rule and bound, R_j >= 0
S6   replay of the policy's own consumed-event log reproduces its issue sequence
"""
import itertools
import random
from functools import lru_cache

import pytest

from oracle import sim
from oracle.sim import Config, GPUModel, Layer

UNIT = 1000  # ns per time unit


def whole_sm_models(job_lens_units):
    """Each kernel = 1 block that takes a whole SM (per-SM block capacity 1)."""
    return [[Layer(1, (1, 1, 1, 1, 0), d * UNIT, d * UNIT) for d in lens] for lens in job_lens_units]


def single_server_cfg(n_clients=1, sms=1):
    return Config(num_clients=n_clients, theta=sim.INF_THETA, slack=0, group=16,
                  capacity=(sms, 10**9, 10**12, 10**12, 10**9))


ONE_SM = GPUModel(sms=1, per_sm=(1, 64, 65536, 233472, 512), hw_queues=32)


def brute_min_total_completion(jobs):
    """All interleavings (each job's kernels in order), single server, no idling."""
    best = None
    n = len(jobs)
    seq = [i for i, lens in enumerate(jobs) for _ in lens]
    for perm in set(itertools.permutations(seq)):
        t, cur, fin = 0, [0] * n, [0] * n
        for i in perm:
            t += jobs[i][cur[i]]
            cur[i] += 1
            if cur[i] == len(jobs[i]):
                fin[i] = t
        tot = sum(fin)
        best = tot if best is None else min(best, tot)
    return best


@pytest.mark.parametrize("seed", range(60))
def test_S1a_srpt_optimal_all_released_at_zero(seed):
    r = random.Random(seed)
    jobs = [[r.randint(1, 9) for _ in range(r.randint(1, 3))] for _ in range(r.randint(2, 4))]
    models = whole_sm_models(jobs)
    trace = [(0, 0, m) for m in range(len(jobs))]
    res = sim.simulate(single_server_cfg(), models, trace, ONE_SM)
    assert sum(res.jct().values()) == brute_min_total_completion(jobs) * UNIT


def brute_unit_with_releases(lens, rel):
    """Exact min total JCT for unit kernels with integer releases, idling allowed."""
    n = len(lens)

    @lru_cache(None)
    def go(t, rem):
        if all(x == 0 for x in rem):
            return 0
        best = None
        opts = [i for i in range(n) if rem[i] > 0 and rel[i] <= t]
        choices = opts + [None]
        for c in choices:
            if c is None:
                if all(rel[i] <= t for i in range(n) if rem[i] > 0):
                    continue   # idling only helps while something is unreleased
                v = go(t + 1, rem)
            else:
                nr = list(rem)
                nr[c] -= 1
                v = go(t + 1, tuple(nr)) + ((t + 1 - rel[c]) if nr[c] == 0 else 0)
            best = v if best is None else min(best, v)
        return best

    return go(0, tuple(lens))


@pytest.mark.parametrize("seed", range(60))
def test_S1b_srpt_optimal_unit_kernels_with_releases(seed):
    r = random.Random(1000 + seed)
    n = r.randint(2, 4)
    lens = [r.randint(1, 3) for _ in range(n)]
    rel = [r.randint(0, 4) for _ in range(n)]
    models = whole_sm_models([[1] * k for k in lens])
    trace = sorted([(rel[i] * UNIT, 0, i) for i in range(n)], key=lambda x: x[0])
    res = sim.simulate(single_server_cfg(), models, trace, ONE_SM)
    assert sum(res.jct().values()) == brute_unit_with_releases(tuple(lens), tuple(rel)) * UNIT


def test_S1c_srpt_not_optimal_in_general():
    # jobs [[4],[3,7]] released at [6,5]: SRPT total 20 vs optimum 19 (optimum idles)
    models = whole_sm_models([[4], [3, 7]])
    trace = [(5 * UNIT, 0, 1), (6 * UNIT, 0, 0)]
    res = sim.simulate(single_server_cfg(), models, trace, ONE_SM)
    assert sum(res.jct().values()) == 20 * UNIT


def test_S2_fig1_setup():
    models = whole_sm_models([[1, 1, 1]] * 4)
    trace = [(0, 0, i) for i in range(4)]
    gpu = GPUModel(sms=2, per_sm=(1, 64, 65536, 233472, 512))
    res = sim.simulate(single_server_cfg(sms=2), models, trace, gpu)
    jct = sorted(res.jct().values())
    assert sum(jct) / 4 == 4.5 * UNIT
    assert jct == [3 * UNIT, 3 * UNIT, 6 * UNIT, 6 * UNIT]


def test_S3_fig2_hol_blocking_closed_form():
    # GTX 1660 SUPER: 22 SMs x 1024 threads, 32 HW queues; jobs of 8 kernels, each
    # 1 block x 128 threads (4 warps), 9 regs, no smem, ~300 us.  176 could run.
    per_sm = (32, 32, 65536, 100 * 1024, 512)
    gpu = GPUModel(sms=22, per_sm=per_sm, hw_queues=32)
    regs = -(-9 * 32 // 256) * 256 * 4
    layer = Layer(1, (1, 4, regs, 0, 0), 300_000, 300_000)
    models = [[layer] * 8]
    trace = [(0, 0, 0)] * 400
    naive = sim.simulate(Config(num_clients=1), models, trace, gpu, system="naive",
                         naive_streams=400, horizon=2_000_000)
    assert naive.max_running_blocks == 32          # 32/176 = 18%
    cap = tuple(22 * x for x in per_sm)
    cfg = Config(num_clients=1, slack=0, capacity=cap, streams=176)
    gpu176 = GPUModel(sms=22, per_sm=per_sm, hw_queues=176)
    paella = sim.simulate(cfg, models, trace, gpu176, horizon=2_000_000)
    assert paella.max_running_blocks == 176        # 176/176


def random_models(r, n_models=3):
    ms = []
    for _ in range(n_models):
        ms.append([Layer(r.randint(1, 40), (1, r.choice([4, 8]), 4096 * r.randint(1, 4),
                                            r.choice([0, 8192, 40960]), r.choice([0, 0, 32])),
                         tb, tb)
                   for tb in (r.randint(1, 20) * 500 for _ in range(r.randint(1, 6)))])
    return ms


def random_trace(r, n, n_clients, n_models, rate_ns=3000):
    t, out = 0, []
    for _ in range(n):
        t += int(r.expovariate(1.0 / rate_ns))
        out.append((t, r.randrange(n_clients), r.randrange(n_models)))
    return out


@pytest.mark.parametrize("lookahead", [0, 1])
@pytest.mark.parametrize("policy", [sim.SRPT_DEFICIT, sim.FIFO])
@pytest.mark.parametrize("seed", range(6))
def test_S5_invariants_and_S6_self_replay(seed, policy, lookahead):
    r = random.Random(seed)
    models = random_models(r)
    gpu = GPUModel(sms=8, per_sm=(32, 64, 65536, 233472, 512), launch_delay=700, notif_delay=900)
    N = 3
    cfg = Config(num_clients=N, policy=policy, theta=r.choice([0, 1, 5, 100]), slack=r.choice([0, 8, 16]),
                 group=r.choice([1, 4, 16]), ring_capacity=256, streams=r.choice([4, 32]),
                 capacity=tuple(8 * x for x in (32, 64, 65536, 233472, 512)), lookahead=lookahead)
    trace = random_trace(r, 150, N, len(models))
    res = sim.simulate(cfg, models, trace, gpu)
    assert not res.violations                                  # (a) per-SM capacity
    assert len(res.finish) == len(trace)                       # everything completes
    # (b) exactly once
    grids = {}
    for (t, uid, jid, layer, stream) in res.issues:
        grids[uid] = models[trace[jid][2]][layer].grid
    assert sim.check_exactly_once(res.records, grids, cfg.group) == []
    # (c) dependency: kernel k+1 of a job issued after kernel k's last completion
    last_done = {}
    placed = {}
    first_place_done = {}
    for (t, typ, uid, n, grp) in res.records:
        if typ == sim.COMPLETION:
            last_done[uid] = t
        else:
            placed[uid] = placed.get(uid, 0) + n
            if uid in grids and placed[uid] == grids[uid]:
                first_place_done[uid] = t
    by_job = {}
    for (t, uid, jid, layer, stream) in res.issues:
        by_job.setdefault(jid, []).append((layer, t, uid))
    for jid, lst in by_job.items():
        lst.sort()
        assert [x[0] for x in lst] == list(range(len(models[trace[jid][2]])))
        for (l0, t0, u0), (l1, t1, u1) in zip(lst, lst[1:]):
            if lookahead == 0:
                assert t1 >= last_done[u0]
            else:   # launch-ahead: issued behind a fully placed predecessor on its stream
                assert t1 >= first_place_done.get(u0, t1) or t1 >= last_done[u0]


def _run_policy_with_log(cfg, models, trace, gpu):
    """simulate() with the Policy event log switched on."""
    orig = sim.Policy.__init__

    def init(self, *a, **k):
        orig(self, *a, **k)
        self.log = []
    sim.Policy.__init__ = init
    try:
        return sim.simulate(cfg, models, trace, gpu)
    finally:
        sim.Policy.__init__ = orig


@pytest.mark.parametrize("lookahead", [0, 1, 2, -2])
@pytest.mark.parametrize("seed", range(8))
def test_S6_replay_reproduces_issue_order(seed, lookahead):
    """lookahead < 0: depth |lookahead| with lookahead_unplaced (NEXT-1 variant)."""
    unplaced, lookahead = lookahead < 0, abs(lookahead)
    r = random.Random(50 + seed)
    models = random_models(r)
    gpu = GPUModel(sms=4, per_sm=(32, 64, 65536, 233472, 512), launch_delay=300, notif_delay=1100)
    cfg = Config(num_clients=4, theta=r.choice([0, 3, 100]), slack=4, group=r.choice([1, 16]),
                 ring_capacity=128, streams=8, capacity=tuple(4 * x for x in (32, 64, 65536, 233472, 512)),
                 lookahead=lookahead, lookahead_unplaced=int(unplaced))
    trace = random_trace(r, 120, 4, len(models), rate_ns=2000)
    res = _run_policy_with_log(cfg, models, trace, gpu)
    log = res.policy.log
    ok, msg, n = sim.replay(cfg, models, log)
    assert ok, msg
    assert n == len(res.issues) > 0
    # a corrupted log (one record's count changed) must be detected as a divergence
    # or an inconsistency
    bad = list(log)
    idx = next(i for i, e in enumerate(bad) if e[0] == sim.EV_ISSUE and i > len(bad) // 2)
    e = bad[idx]
    bad[idx] = (e[0], e[1], e[2], e[3], (e[4] + 1) % cfg.streams)
    ok2, msg2, _ = sim.replay(cfg, models, bad)
    assert not ok2 and "issue" in msg2


def test_S4_theta_inf_and_single_client_are_srpt():
    r = random.Random(3)
    models = random_models(r)
    trace = random_trace(r, 100, 1, len(models))
    gpu = GPUModel(sms=2)
    base = Config(num_clients=1, theta=sim.INF_THETA, slack=0,
                  capacity=tuple(2 * x for x in (32, 64, 65536, 233472, 512)))
    a = sim.simulate(base, models, trace, gpu)
    for th in (0, 1, 7):
        b = sim.simulate(Config(num_clients=1, theta=th, slack=0, capacity=base.capacity), models, trace, gpu)
        assert [i[1:] for i in a.issues] == [i[1:] for i in b.issues]


@pytest.mark.parametrize("N", [2, 3, 4, 8])
def test_S4_theta_zero_round_robin_windows(N):
    """theta = 0, all clients always ready: every aligned window of N dispatches
    serves each client exactly once and deficits return to 0 at window ends."""
    r = random.Random(N)
    models = [[Layer(1, (1, 1, 1, 1, 0), 1000 * r.randint(1, 9), 1)] * 3 for _ in range(3)]
    cfg = Config(num_clients=N, theta=0, slack=10**9, streams=8,
                 capacity=(10**9,) * 5)
    pol = sim.Policy(cfg, models)
    jid = 0
    for c in range(N):
        for _ in range(400):
            pol.arrival(jid, c, r.randrange(3))
            jid += 1
    clients = []
    for w in range(200):
        for _ in range(N):
            # one dispatch at a time: issue, then complete it immediately
            (uid, job, layer, stream), = _issue_one(pol)
            clients.append(pol.jobs[job].client if job in pol.jobs else None)
            pol.record(sim.PLACEMENT, uid, 1)
            pol.record(sim.COMPLETION, uid, 1)
        assert all(pol.D(c) == 0 for c in range(N))
    for w in range(200):
        win = clients[w * N:(w + 1) * N]
        assert None not in win and sorted(win) == list(range(N))


def _issue_one(pol):
    saved = set(pol.free)
    pol.free = {min(saved)}
    out = pol.decide()
    pol.free = saved - {o[3] for o in out}
    return out


def test_S4_fifo_order():
    r = random.Random(9)
    models = random_models(r)
    trace = random_trace(r, 120, 3, len(models), rate_ns=500)
    cfg = Config(num_clients=3, policy=sim.FIFO, slack=0, streams=4,
                 capacity=tuple(2 * x for x in (32, 64, 65536, 233472, 512)))
    res = _run_policy_with_log(cfg, models, trace, GPUModel(sms=2))
    assert len(res.finish) == len(trace)
    # at each issue the chosen job is the oldest ready job: replay the log and check
    pol = sim.Policy(cfg, models)
    for ev in res.policy.log:
        if ev[0] == sim.EV_ARRIVAL:
            pol.arrival(*ev[1:])
        elif ev[0] == sim.EV_RECORD:
            pol.record(*ev[1:])
        elif ev[0] == sim.EV_ISSUE:
            rdy = pol.ready()
            assert ev[2] == min(rdy, key=lambda j: j.seq).id
            _force_issue(pol, ev[2], ev[4])


def _force_issue(pol, job_id, stream):
    saved = set(pol.free)
    pol.free = {stream}
    (out,) = pol.decide()
    assert out[1] == job_id
    pol.free = saved - {stream}


@pytest.mark.parametrize("N,theta", [(2, 0), (3, 1), (4, 5), (8, 20), (3, 0)])
def test_S5_deficit_rule_and_bound(N, theta):
    """(e) when some ready client has D > theta*N the pick is the oldest ready job of
    the max-D client; (f) a continuously-ready client never exceeds
    max(D(s), theta*N) + N."""
    r = random.Random(N * 100 + theta)
    models = [[Layer(1, (1, 1, 1, 1, 0), 100 * r.randint(1, 50), 1)] * r.randint(1, 5) for _ in range(4)]
    cfg = Config(num_clients=N, theta=theta, slack=10**9, streams=8, capacity=(10**9,) * 5)
    pol = sim.Policy(cfg, models)
    jid = 0
    for c in range(N):
        for _ in range(300):
            pol.arrival(jid, c, r.randrange(4))
            jid += 1
    series = {c: [] for c in range(N)}
    for step in range(280):  # every client stays ready (>= 300 kernels each)
        rdy = pol.ready()
        if not rdy:
            break
        ds = {c: pol.D(c) for c in {j.client for j in rdy}}
        cstar = max(sorted(ds), key=lambda c: (ds[c], -c))
        srpt = min(rdy, key=lambda j: (j.R, j.seq, j.id)).id
        (uid, job, layer, stream), = _issue_one(pol)
        picked = pol.jobs[job]
        if ds[cstar] > theta * N:
            assert picked.client == cstar
            assert picked.seq == min(j.seq for j in rdy if j.client == cstar)
        else:
            assert picked.id == srpt
        pol.record(sim.PLACEMENT, uid, 1)
        pol.record(sim.COMPLETION, uid, 1)
        for c in range(N):
            series[c].append(pol.D(c))
    assert sim.deficit_bound_holds(series, N, theta) == []
    assert max(max(s) for s in series.values()) <= max(0, theta * N) + N


@pytest.mark.parametrize("seed", range(4))
def test_prio_classes_stream_rule(seed):
    """Stream-priority classes (reading B200-Q2): with enough streams and no
    deficit override, every fresh stream acquisition lands in the class given by the
    rank of R_j (remaining T-bar before the kernel) among the models' whole-job sums;
    K = 1 reproduces the one-class issue sequence exactly."""
    r = random.Random(300 + seed)
    models = random_models(r)
    gpu = GPUModel(sms=8, per_sm=(32, 64, 65536, 233472, 512), launch_delay=500, notif_delay=700)
    base = dict(num_clients=3, theta=sim.INF_THETA, slack=8, group=4, ring_capacity=4096, streams=32,
                capacity=tuple(8 * x for x in (32, 64, 65536, 233472, 512)), lookahead=0)
    trace = random_trace(r, 60, 3, len(models), rate_ns=20000)
    one = sim.simulate(Config(**base), models, trace, gpu)
    one_k1 = sim.simulate(Config(**base, prio_classes=1), models, trace, gpu)
    assert one.issues == one_k1.issues
    K = 3
    res = sim.simulate(Config(**base, prio_classes=K), models, trace, gpu)
    assert len(res.finish) == len(trace)
    totals = sorted({sum(l.tbar for l in m) for m in models})
    checked = 0
    for (t, uid, jid, layer, stream) in res.issues:
        ls = models[trace[jid][2]]
        R = sum(l.tbar for l in ls[layer:])
        want = min(K - 1, sum(1 for x in totals if x < R))
        assert stream * K // 32 == want, (jid, layer, stream, R, totals)
        checked += 1
    assert checked == len(res.issues) > 0


# --- NEXT-2 ablations (Table 3, P1341-1359): SJF and RR orders ----------------------

@pytest.mark.parametrize("seed", range(40))
def test_sjf_optimal_all_released_at_zero(seed):
    """Single server, all jobs at t = 0: shortest-whole-job-first serves jobs one after
    another in SPT order, which is optimal (the same brute force as S1a)."""
    r = random.Random(500 + seed)
    jobs = [[r.randint(1, 9) for _ in range(r.randint(1, 3))] for _ in range(r.randint(2, 4))]
    models = whole_sm_models(jobs)
    trace = [(0, 0, m) for m in range(len(jobs))]
    cfg = single_server_cfg()
    cfg.policy = sim.SJF
    res = sim.simulate(cfg, models, trace, ONE_SM)
    assert sum(res.jct().values()) == brute_min_total_completion(jobs) * UNIT


@pytest.mark.parametrize("n,k", [(2, 3), (3, 2), (4, 4), (5, 1)])
def test_rr_closed_form(n, k):
    """n identical jobs of k unit kernels, single server, all at t = 0: kernel-granular
    round robin finishes job i (arrival order) at (k - 1) n + i + 1 units, so the total
    JCT is n^2 (k - 1) + n (n + 1) / 2 (SRPT would give k n (n + 1) / 2)."""
    models = whole_sm_models([[1] * k for _ in range(n)])
    trace = [(0, 0, m) for m in range(n)]
    cfg = single_server_cfg()
    cfg.policy = sim.RR
    res = sim.simulate(cfg, models, trace, ONE_SM)
    assert sum(res.jct().values()) == (n * n * (k - 1) + n * (n + 1) // 2) * UNIT
    cfg2 = single_server_cfg()
    res2 = sim.simulate(cfg2, models, trace, ONE_SM)
    assert sum(res2.jct().values()) == (k * n * (n + 1) // 2) * UNIT


# --- NEXT-4: online T-bar refinement (running average, P1249-1266) -------------------

def test_online_tbar_running_average_and_remaining_invariant():
    """T-bar of a layer = integer mean of the PROFILE_RUNS profiled observations and
    every observed duration; R_j of every live job stays the sum of the current T-bar
    over its undispatched kernels (so it reaches exactly 0 at its last issue)."""
    layers = [Layer(1, (1, 1, 1, 1, 0), t) for t in (1000, 3000, 5000)]
    cfg = Config(num_clients=1, theta=sim.INF_THETA, slack=0, streams=8, online_tbar=1)
    pol = sim.Policy(cfg, [layers])
    for jid in range(3):
        pol.arrival(jid, 0, 0)
    obs = {}
    for step in range(40):
        for (uid, job, layer, stream) in pol.decide():
            obs[uid] = (job, layer)
        if not pol.launches:
            break
        uid = min(pol.launches)
        job, layer = obs[uid]
        d = 2000 + 700 * layer + 13 * uid
        before_sum = pol.tb_sum[0][layer]
        pol.observe(uid, d)
        pol.record(sim.PLACEMENT, uid, 1)
        pol.record(sim.COMPLETION, uid, 1)
        assert pol.tb_sum[0][layer] == before_sum + d
        assert pol.tb[0][layer] == pol.tb_sum[0][layer] // pol.tb_cnt[0][layer]
        for j in pol.jobs.values():
            assert j.R == pol.remaining(0, j.cursor)
    assert pol.completed == [0, 1, 2] or sorted(pol.completed) == [0, 1, 2]
    # closed form for the first layer: 3 observations on top of 20 profiled runs
    ds = [2000 + 13 * u for u, (jb, ly) in obs.items() if ly == 0]
    assert pol.tb[0][0] == (1000 * sim.PROFILE_RUNS + sum(ds)) // (sim.PROFILE_RUNS + len(ds))


def test_online_tbar_off_keeps_profile():
    layers = [Layer(1, (1, 1, 1, 1, 0), 1000)]
    pol = sim.Policy(Config(num_clients=1, slack=0), [layers])
    pol.arrival(0, 0, 0)
    (uid, _, _, _), = pol.decide()
    pol.observe(uid, 99999)
    pol.record(sim.COMPLETION, uid, 1)
    assert pol.tb[0][0] == 1000


def test_splitmix64_published_outputs():
    """Pin of sim.splitmix64: the first outputs of Vigna's reference splitmix64.c
    seeded with 0 are 0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F
    (state advances by the gamma 0x9E3779B97F4A7C15 per output)."""
    g = 0x9E3779B97F4A7C15
    want = [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]
    assert [sim.splitmix64((k * g) & sim.M64) for k in range(3)] == want


def test_route_pair_candidates_valid_and_spread():
    """Power-of-two choices: two distinct in-range candidates; over
    many request ids every unordered pair of 8 GPUs is drawn about equally often;
    the pick is the lower-W candidate with ties to the lower index."""
    from collections import Counter
    for ng in range(2, 9):
        for rid in range(500):
            a, b = sim.route_pair(rid, ng)
            assert 0 <= a < ng and 0 <= b < ng and a != b
    assert sim.route_pair(123, 1) == (0, 0)
    cnt = Counter(frozenset(sim.route_pair(rid, 8)) for rid in range(28000))
    assert len(cnt) == 28
    assert all(700 <= v <= 1300 for v in cnt.values()), cnt
    assert sim.route_pick((5, 2), [0, 0, 7, 0, 0, 3, 0, 0]) == 5
    assert sim.route_pick((5, 2), [0, 0, 3, 0, 0, 3, 0, 0]) == 2
    assert sim.route_pick((2, 5), [0, 0, 1, 0, 0, 3, 0, 0]) == 2


# --- NEXT-1 launch-ahead: closed forms derived by hand (not the rule re-typed) -------

def _chain(L, d):
    return [[Layer(1, (1, 1, 1, 1, 0), d, d) for _ in range(L)]]


@pytest.mark.parametrize("D", [0, 1, 2, 3, 6, 7])
def test_launch_ahead_closed_form_zero_delay(D):
    """One job of L single-block kernels of duration d, zero launch/notification delay:
    at t = 0 kernels 0..D are issued (each new one is queued behind a fully placed
    predecessor); every time kernel m completes, kernel m+1 is placed and kernel m+D+1
    is issued.  So kernel k is issued at max(0, (k - D) d), and JCT = L d for every D.
    A rule that looked at the NEWEST in-flight kernel instead of the oldest would issue
    only one kernel ahead; one that ignored D would issue all L at t = 0."""
    Lk, d = 10, 1000   # longer than D + 1 for every D tested (the bench runs D = 6)
    cfg = Config(num_clients=1, theta=sim.INF_THETA, slack=10**6, lookahead=D,
                 capacity=(10**6, 10**9, 10**12, 10**12, 10**9))
    res = sim.simulate(cfg, _chain(Lk, d), [(0, 0, 0)], GPUModel(sms=1, per_sm=(1, 64, 65536, 233472, 512)))
    issue_t = [t for (t, uid, jid, layer, stream) in sorted(res.issues, key=lambda x: x[3])]
    assert issue_t == [max(0, (k - D) * d) for k in range(Lk)]
    assert res.jct()[0] == Lk * d
    assert len({s for (_, _, _, _, s) in res.issues}) == (1 if D > 0 else 1)


@pytest.mark.parametrize("D", [1, 2, 3, 6])
def test_launch_ahead_unplaced_closed_form_zero_delay(D):
    """The NEXT-1 variant without the placement test gives the same schedule as the
    original rule when placement is seen instantly: kernel k issued at max(0, (k - D) d),
    JCT = L d."""
    Lk, d = 10, 1000
    cfg = Config(num_clients=1, theta=sim.INF_THETA, slack=10**6, lookahead=D, lookahead_unplaced=1,
                 capacity=(10**6, 10**9, 10**12, 10**12, 10**9))
    res = sim.simulate(cfg, _chain(Lk, d), [(0, 0, 0)], GPUModel(sms=1, per_sm=(1, 64, 65536, 233472, 512)))
    issue_t = [t for (t, uid, jid, layer, stream) in sorted(res.issues, key=lambda x: x[3])]
    assert issue_t == [max(0, (k - D) * d) for k in range(Lk)]
    assert res.jct()[0] == Lk * d


def test_launch_ahead_unplaced_closed_form_with_delays():
    """Launch delay 2, notification delay 3 (units of 1 us), derived by hand.
    (a) d = 10, L = 4.  Original rule D = 1: issues 0, 5, 15, 25 (test below).  Without
        the placement test, D = 1: k0 and k1 are both issued at 0 (k1 queued behind k0);
        k0 ends 12, its completion is seen 15 -> k2 issued 15; k1 ends 22, seen 25 -> k3
        issued 25, runs 32..42, seen 45: issues 0, 0, 15, 25, JCT 45.  D = 2: k0..k2 at
        0, k3 when k0's completion is seen (15): issues 0, 0, 0, 15, JCT 45.
    (b) d = 2 (shorter than the notification round trip), L = 4, D = 3.  Original rule:
        k0 issued 0, launched 2, runs 2..4; its placement is seen 5 -> k1, k2, k3 issued
        5, launched 7, run 7..9, 9..11, 11..13; seen 16: JCT 16.  Without the placement
        test all four are issued at 0, launched 2, run 2..4, 4..6, 6..8, 8..10, the last
        completion is seen 13: JCT 13."""
    u = 1000
    gpu = GPUModel(sms=1, per_sm=(1, 64, 65536, 233472, 512), launch_delay=2 * u, notif_delay=3 * u)
    for d, L, D, unpl, want_issue, want_jct in ((10, 4, 1, 1, [0, 0, 15, 25], 45),
                                                (10, 4, 2, 1, [0, 0, 0, 15], 45),
                                                (2, 4, 3, 0, [0, 5, 5, 5], 16),
                                                (2, 4, 3, 1, [0, 0, 0, 0], 13)):
        cfg = Config(num_clients=1, theta=sim.INF_THETA, slack=10**6, lookahead=D, lookahead_unplaced=unpl,
                     capacity=(10**6, 10**9, 10**12, 10**12, 10**9))
        res = sim.simulate(cfg, _chain(L, d * u), [(0, 0, 0)], gpu)
        got = [t for (t, *_r) in sorted(res.issues, key=lambda x: x[3])]
        assert got == [x * u for x in want_issue], (d, D, unpl, got)
        assert res.jct()[0] == want_jct * u, (d, D, unpl, res.jct()[0])


def test_launch_ahead_closed_form_with_delays():
    """d = 10, launch delay 2, notification delay 3, L = 4 (times in units of 1 us),
    derived step by step in the test docstring's notation:
    D = 0: each kernel waits for its predecessor's completion record:
           issue at 0, 15, 30, 45; the last completion is seen at 60.
    D = 1: k0 issued 0, placed 2, PLACEMENT seen 5 -> k1 issued 5 (launched 7, queued);
           k0 ends 12, k1 placed 12, both records seen 15 -> k2 issued 15;
           k1 ends 22, k2 placed 22, seen 25 -> k3 issued 25; k3 runs 32..42, seen 45."""
    u = 1000
    gpu = GPUModel(sms=1, per_sm=(1, 64, 65536, 233472, 512), launch_delay=2 * u, notif_delay=3 * u)
    for D, want_issue, want_jct in ((0, [0, 15, 30, 45], 60), (1, [0, 5, 15, 25], 45)):
        cfg = Config(num_clients=1, theta=sim.INF_THETA, slack=10**6, lookahead=D,
                     capacity=(10**6, 10**9, 10**12, 10**12, 10**9))
        res = sim.simulate(cfg, _chain(4, 10 * u), [(0, 0, 0)], gpu)
        assert [t for (t, *_r) in sorted(res.issues, key=lambda x: x[3])] == [x * u for x in want_issue]
        assert res.jct()[0] == want_jct * u


@pytest.mark.parametrize("D", [0, 1, 3, 6, -3])
def test_inflight_bound_checker(D):
    """check_inflight_bound accepts every simulator log at its own depth; on the chain of
    test_launch_ahead_closed_form_zero_delay (depth D + 1 reached at t = 0) it rejects
    the log when checked against depth D - 1.  D < 0: depth |D| with lookahead_unplaced."""
    unpl, D = int(D < 0), abs(D)
    r = random.Random(900 + D)
    models = random_models(r)
    gpu = GPUModel(sms=4, per_sm=(32, 64, 65536, 233472, 512), launch_delay=300, notif_delay=400)
    cfg = Config(num_clients=2, slack=64, group=4, streams=8, lookahead=D, lookahead_unplaced=unpl,
                 capacity=tuple(4 * x for x in (32, 64, 65536, 233472, 512)))
    trace = random_trace(r, 30, 2, len(models), rate_ns=3000)
    res = _run_policy_with_log(cfg, models, trace, gpu)
    assert sim.check_inflight_bound(res.policy.log, models, D) == []
    chain = _chain(10, 1000)
    cfg1 = Config(num_clients=1, theta=sim.INF_THETA, slack=10**6, lookahead=D, lookahead_unplaced=unpl,
                  capacity=(10**6, 10**9, 10**12, 10**12, 10**9))
    res1 = _run_policy_with_log(cfg1, chain, [(0, 0, 0)], GPUModel(sms=1, per_sm=(1, 64, 65536, 233472, 512)))
    assert sim.check_inflight_bound(res1.policy.log, chain, D) == []
    if D > 0:
        assert sim.check_inflight_bound(res1.policy.log, chain, D - 1) != []


# --- stream-priority classes: worked example (B200-Q2) -------------------------------

def _one_layer_models(tbars):
    return [[Layer(1, (1, 1, 1, 1, 0), t, t)] for t in tbars]


def test_prio_classes_worked_example():
    """Models with whole-job T-bar 10, 20, 40; K = 3 classes over P = 6 streams
    (class of stream s = floor(3 s / 6): {0,1}, {2,3}, {4,5}); one client, theta = inf.
    Jobs A (40), B (10), C (20), D (40), E (40) arrive at once.  SRPT issues B, C, A, D, E.
    Class of a job = number of models whose sum is strictly below R_j:
    B -> 0 -> stream 0;  C -> 1 -> stream 2;  A -> 2 -> stream 4;  D -> 2 -> stream 5;
    E -> 2, class 2 full -> the lowest free stream overall, 1."""
    models = _one_layer_models([10, 20, 40])
    cfg = Config(num_clients=1, theta=sim.INF_THETA, slack=10**6, streams=6, prio_classes=3,
                 capacity=(10**6, 10**9, 10**12, 10**12, 10**9))
    pol = sim.Policy(cfg, models)
    for jid, m in enumerate([2, 0, 1, 2, 2]):     # A B C D E
        pol.arrival(jid, 0, m)
    got = [(job, stream) for (uid, job, layer, stream) in pol.decide()]
    assert got == [(1, 0), (2, 2), (0, 4), (3, 5), (4, 1)]


def test_prio_classes_deficit_override_takes_class0():
    """theta = 0, two clients.  Y (client 1, R = 10) is picked first by SRPT (both
    deficits 0, not > 0) -> class 0, stream 0; deficits become D0 = +1, D1 = -1 (units
    1/N).  X (client 0, R = 40) is then picked by the deficit override (1 > 0) and takes
    class 0 -> stream 1 (without the override it would be class 2, stream 4)."""
    models = _one_layer_models([10, 20, 40])
    cfg = Config(num_clients=2, theta=0, slack=10**6, streams=6, prio_classes=3,
                 capacity=(10**6, 10**9, 10**12, 10**12, 10**9))
    pol = sim.Policy(cfg, models)
    pol.arrival(0, 0, 2)    # X
    pol.arrival(1, 1, 0)    # Y
    got = [(job, stream) for (uid, job, layer, stream) in pol.decide()]
    assert got == [(1, 0), (0, 1)]
    assert (pol.D(0), pol.D(1)) == (0, 0)


# --- B200-Q6: the job cap K (max_active) ---------------------------------------------

def test_max_active_worked_example():
    """K = 2, SRPT, one client, theta = inf, single-kernel jobs with T-bar 30, 10, 20
    arriving together: only the two shortest (10, 20) may issue; the 30 waits until one
    of them has issued its last kernel (then it has no kernel left and leaves the set)."""
    models = _one_layer_models([30, 10, 20])
    cfg = Config(num_clients=1, theta=sim.INF_THETA, slack=10**6, streams=8, max_active=2,
                 capacity=(10**6, 10**9, 10**12, 10**12, 10**9))
    pol = sim.Policy(cfg, models)
    for jid, m in enumerate([0, 1, 2]):
        pol.arrival(jid, 0, m)
    first = [job for (uid, job, layer, stream) in pol.decide()]
    # both capped jobs issued their only kernel, so the set {1, 2} is exhausted and job 0
    # becomes one of the K first with kernels left: same pass
    assert first == [1, 2, 0]
    # two-kernel jobs: the set keeps them while they have kernels left
    models2 = [[Layer(1, (1, 1, 1, 1, 0), 15, 15)] * 2, _one_layer_models([10])[0], _one_layer_models([20])[0]]
    pol2 = sim.Policy(Config(num_clients=1, theta=sim.INF_THETA, slack=10**6, streams=8, max_active=2,
                             capacity=(10**6, 10**9, 10**12, 10**12, 10**9)), models2)
    for jid, m in enumerate([0, 1, 2]):      # R = 30, 10, 20
        pol2.arrival(jid, 0, m)
    iss = pol2.decide()
    # SRPT top-2 = {1 (10), 2 (20)}: both issue; then {0 (30)} is top -> issues layer 0;
    # job 0 is in flight (no launch-ahead) so the pass ends
    assert [job for (_, job, _, _) in iss] == [1, 2, 0]
    uid0 = iss[2][0]
    pol2.record(sim.PLACEMENT, uid0, 1)
    pol2.record(sim.COMPLETION, uid0, 1)
    pol2.arrival(3, 0, 1)                    # a short job arrives (R = 10) with job 0 at R = 15
    assert [job for (_, job, _, _) in pol2.decide()] == [3, 0]


def test_max_active_fifo_order_and_override():
    """FIFO, K = 1, launch-ahead 1, two 2-kernel jobs: job 1 may start only once job 0
    has issued its LAST kernel (it then has nothing left to issue and leaves the set).
    SRPT, K = 1, theta = 0, two clients: P (client 0, 2 x 5 ns) is the SRPT head and
    issues; Q (client 1, 40 ns) is outside the cap, but after P's dispatch client 1's
    deficit is +1 > theta N = 0, so the override issues Q in the same pass."""
    big = (10**6, 10**9, 10**12, 10**12, 10**9)
    models = [[Layer(1, (1, 1, 1, 1, 0), 10, 10)] * 2] * 2
    pol = sim.Policy(Config(num_clients=1, policy=sim.FIFO, slack=10**6, streams=8, max_active=1,
                            lookahead=1, capacity=big), models)
    pol.arrival(0, 0, 0)
    pol.arrival(1, 0, 1)
    iss = pol.decide()
    assert [(j, l) for (_, j, l, _) in iss] == [(0, 0)]
    pol.record(sim.PLACEMENT, iss[0][0], 1)
    assert [(j, l) for (_, j, l, _) in pol.decide()] == [(0, 1), (1, 0)]
    m2 = [[Layer(1, (1, 1, 1, 1, 0), 5, 5)] * 2, [Layer(1, (1, 1, 1, 1, 0), 40, 40)]]
    pol2 = sim.Policy(Config(num_clients=2, theta=0, slack=10**6, streams=8, max_active=1, capacity=big), m2)
    pol2.arrival(0, 0, 0)    # P
    pol2.arrival(1, 1, 1)    # Q
    assert [(j, l) for (_, j, l, _) in pol2.decide()] == [(0, 0), (1, 0)]
    assert pol2.over


def test_cap_arrival_order_worked_example():
    """K = 1, SRPT, theta = inf, no launch-ahead; A (2 kernels x 15 ns, R = 30) arrives
    before B (1 kernel, 10 ns).  Cap in SRPT order: B is the cap's job, issues, leaves the
    set (nothing left), then A issues its first kernel: [B, A.0]; after A.0 completes:
    [A.1].  Cap in arrival order (cap_fifo): A holds the cap until it has issued its LAST
    kernel: [A.0]; after A.0 completes: [A.1, B]."""
    big = (10**6, 10**9, 10**12, 10**12, 10**9)
    m = [[Layer(1, (1, 1, 1, 1, 0), 15, 15)] * 2, [Layer(1, (1, 1, 1, 1, 0), 10, 10)]]
    for cf, want1, want2 in ((0, [(1, 0), (0, 0)], [(0, 1)]), (1, [(0, 0)], [(0, 1), (1, 0)])):
        pol = sim.Policy(Config(num_clients=1, theta=sim.INF_THETA, slack=10**6, streams=8, max_active=1,
                                cap_fifo=cf, capacity=big), m)
        pol.arrival(0, 0, 0)
        pol.arrival(1, 0, 1)
        iss = pol.decide()
        assert [(j, l) for (_, j, l, _) in iss] == want1, cf
        ua = next(u for (u, j, l, _) in iss if j == 0)
        pol.record(sim.PLACEMENT, ua, 1)
        pol.record(sim.COMPLETION, ua, 1)
        assert [(j, l) for (_, j, l, _) in pol.decide()] == want2, cf


# --- S5 (b) exactly-once checker on bad logs ------------------------------------------

def test_exactly_once_checker_rejects_bad_logs():
    """grid 40, G 16 -> groups (0:16), (1:16), (2:8) per type.  Each corruption a device
    or a consumer could produce must be flagged."""
    good = []
    for typ in (sim.PLACEMENT, sim.COMPLETION):
        good += [(0, typ, 7, 16, 0), (0, typ, 7, 16, 1), (0, typ, 7, 8, 2)]
    assert sim.check_exactly_once(good, {7: 40}, 16) == []
    dropped = good[:-1]
    dup = good + [good[0]]
    wrong_count = good[:2] + [(0, sim.PLACEMENT, 7, 7, 2)] + good[3:]
    wrong_group = good[:2] + [(0, sim.PLACEMENT, 7, 8, 1)] + good[3:]
    other_uid = good[:5] + [(0, sim.COMPLETION, 8, 8, 2)]
    for bad in (dropped, dup, wrong_count, wrong_group, other_uid):
        assert sim.check_exactly_once(bad, {7: 40}, 16) != []


# --- Fig. 9: scheduler-delay injection in the simulator (NEXT-2) ---------------------

def test_decide_delay_closed_form():
    """One job of 3 kernels (d = 10), launch delay 2, notification delay 3, decide delay 5
    (units of 1 us), no launch-ahead: each decision takes 5 before its launch is sent,
    so decisions happen at 0, 20, 40 (= k (5 + 2 + 10 + 3)) and the job completes at 60."""
    u = 1000
    gpu = GPUModel(sms=1, per_sm=(1, 64, 65536, 233472, 512), launch_delay=2 * u, notif_delay=3 * u,
                   decide_delay=5 * u)
    cfg = Config(num_clients=1, theta=sim.INF_THETA, slack=10**6, capacity=(10**6, 10**9, 10**12, 10**12, 10**9))
    res = sim.simulate(cfg, _chain(3, 10 * u), [(0, 0, 0)], gpu)
    assert [t for (t, *_r) in sorted(res.issues, key=lambda x: x[3])] == [0, 20 * u, 40 * u]
    assert res.jct()[0] == 60 * u


def test_decide_delay_throughput_falls():
    """Fig. 9 (P1178-1241): a saturated stream of jobs is served at a rate that does not
    rise as the per-decision delay grows, and falls once the delay is comparable to a
    kernel (the dispatcher, not the GPU, becomes the bottleneck)."""
    models = [[Layer(4, (1, 4, 4096, 1024, 0), 2000, 2000)] * 6]
    trace = [(i * 500, 0, 0) for i in range(120)]
    cfg = Config(num_clients=1, slack=64, lookahead=0, streams=32,
                 capacity=tuple(8 * x for x in (32, 64, 65536, 233472, 512)))
    rates = []
    for dd in (0, 100, 1000, 10000):
        gpu = GPUModel(sms=8, launch_delay=500, notif_delay=500, decide_delay=dd)
        res = sim.simulate(cfg, models, trace, gpu, check=False)
        assert len(res.finish) == 120
        rates.append(120 / max(res.finish.values()))
    assert all(a >= b for a, b in zip(rates, rates[1:])), rates
    assert rates[-1] < 0.5 * rates[0], rates


# --- NEXT-4: intra-job branches (Fig. 7 waitlists, P906-951), hand-derived ----------

def _diamond(d):
    """k0 (vs 0) -> k1 (vs 0) and k2 (vs 1) -> k3 (vs 0, consumes k2 from vs 1)."""
    Ld = lambda deps, vs: Layer(1, (1, 1, 1, 1, 0), d, d, deps=deps, vs=vs)   # noqa: E731
    return [[Ld((), 0), Ld((), 0), Ld((0,), 1), Ld((2,), 0)]]


@pytest.mark.parametrize("D", [0, 1])
def test_branches_diamond_closed_form(D):
    """Zero delays, 2 SMs, d = 1 unit.  t = 0: k0 issued (with D = 1 also k1, queued
    behind it on stream 0); k2 waits for its cross-stream input k0.  t = 1: k0 completes;
    k2 is issued on a second stream (and k1 too when D = 0, lower index first); k1 and
    k2 run together 1..2.  k3 waits for k2 (another virtual stream) even with
    launch-ahead: issued at 2, done at 3.  JCT = 3 units (the chain takes 4)."""
    u = 1000
    cfg = Config(num_clients=1, theta=sim.INF_THETA, slack=10**6, lookahead=D, streams=4,
                 capacity=(10**6, 10**9, 10**12, 10**12, 10**9))
    gpu = GPUModel(sms=2, per_sm=(1, 64, 65536, 233472, 512))
    res = sim.simulate(cfg, _diamond(u), [(0, 0, 0)], gpu)
    t_issue = {layer: t for (t, uid, jid, layer, stream) in res.issues}
    stream = {layer: s for (t, uid, jid, layer, s) in res.issues}
    assert t_issue == ({0: 0, 1: u, 2: u, 3: 2 * u} if D == 0 else {0: 0, 1: 0, 2: u, 3: 2 * u})
    assert stream[2] != stream[1] and stream[0] == stream[1] == stream[3]
    assert res.jct()[0] == 3 * u
    chain = [[Layer(1, (1, 1, 1, 1, 0), u, u)] * 4]
    assert sim.simulate(cfg, chain, [(0, 0, 0)], gpu).jct()[0] == 4 * u


def test_branches_cross_dependency_blocks_until_completion():
    """k3 consumes k2 from another virtual stream: it is not active while k2 is merely
    placed, only once k2's final COMPLETION is consumed (policy-level trace)."""
    pol = sim.Policy(Config(num_clients=1, theta=sim.INF_THETA, slack=10**6, lookahead=3, streams=4,
                            capacity=(10**6, 10**9, 10**12, 10**12, 10**9)), _diamond(10))
    pol.arrival(0, 0, 0)
    (u0, _, l0, s0), = pol.decide()
    assert l0 == 0
    pol.record(sim.PLACEMENT, u0, 1)
    (u1, _, l1, _), = pol.decide()
    assert l1 == 1                                              # k1 behind k0; k2 not active
    pol.record(sim.COMPLETION, u0, 1)
    iss = pol.decide()
    assert [l for (_, _, l, _) in iss] == [2]
    u2 = iss[0][0]
    pol.record(sim.PLACEMENT, u2, 1)
    pol.record(sim.PLACEMENT, u1, 1)
    assert pol.head(pol.jobs[0]) is None      # k1 running (launch-ahead would allow k3) but k2 not done
    pol.record(sim.COMPLETION, u2, 1)
    assert pol.head(pol.jobs[0]) == 3
