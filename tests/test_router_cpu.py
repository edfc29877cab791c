"""Multi-GPU routing replayed against the oracle, on 8 FAKE GPUs.

The router runs inside paella_submit.  With route_log_path every decision is logged
with the snapshot of ALL GPUs it was taken on (paella_route_rec_t: published work,
unadmitted backlog, the model's whole-job T-bar, liveness).  The oracle recomputes
each decision from that snapshot:

* least work: argmin_g work[g] + pending[g] * tbar_model, ties to the lowest index
  (oracle.sim.route_least_work) -- catches a router that ignores the backlog term, a
  wrong tie-break, an off-by-one over the GPU range;
* round robin: the client's i-th request goes to GPU i mod 8;
* power of two: the candidates are oracle.sim.route_pair(req_id) (independent
  SplitMix64) and the lower W wins, ties to the lower index.

And the snapshot itself is pinned to the dispatchers: every work[g] the router read
must be a value GPU g's dispatcher actually published, i.e. the sum of R_j over its
live jobs after one of its decide passes, as recomputed by replaying GPU g's event
log through the oracle policy (a router reading a stale or wrong W_g fails).
"""
import time

import numpy as np
import pytest

from oracle import eventlog, sim
from workload import archs, rng

L = pytest.importorskip("paper_conf_sosp_ngd023_b200._lib")
NG = 8


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_sosp_ngd023_b200 import build
    build.build()
    L.load()


def test_route_least_work_worked_examples():
    """Hand-computed decisions (the definition, not a re-typed formula): the backlog
    term, ties, and failed GPUs."""
    # W = [5, 3, 3 + 1*10] -> GPU 1
    assert sim.route_least_work([5, 3, 3], [0, 0, 1], 10, 0b111) == 1
    # the backlog decides: W = [5 + 0, 3 + 2*10] -> GPU 0
    assert sim.route_least_work([5, 3], [0, 2], 10, 0b11) == 0
    # tie between GPUs 2 and 3 (W = 7) -> the lower index
    assert sim.route_least_work([9, 8, 7, 7], [0, 0, 0, 0], 10, 0b1111) == 2
    # GPU 1 failed: the best alive is GPU 2
    assert sim.route_least_work([5, 1, 3], [0, 0, 0], 10, 0b101) == 2
    assert sim.route_least_work([5, 1], [0, 0], 10, 0) is None


def _serve_bursts(e, mids, n, n_clients, seed, stride=16384):
    r = np.random.default_rng(seed)
    infos = {m: e.model_info(m) for m in mids}
    pending = set()
    for i in range(n):
        c = int(r.integers(n_clients))
        m = int(r.choice(mids))
        need = infos[m]["input_bytes"] + infos[m]["output_bytes"]
        rid = e.submit(c, m, (i % 256) * stride, need)
        assert rid >= 0
        pending.add(rid)
        if i % 40 == 39:
            time.sleep(0.002)     # bursts: work builds up, then drains
    t0 = time.time()
    while pending:
        assert time.time() - t0 < 60
        for c in range(n_clients):
            rid, st = e.poll(c)
            if rid >= 0:
                assert st == 0
                pending.remove(rid)


@pytest.mark.parametrize("route", [L.ROUTE_LEAST_WORK, L.ROUTE_ROUND_ROBIN, L.ROUTE_POWER_OF_TWO])
def test_router_replay_8_gpus(tmp_path, route):
    log = str(tmp_path / "ev_%u.log")
    rlog = str(tmp_path / "route_%u.log")
    models = [archs.toy(), archs.squeezenet1_1()]
    nclients = 3
    with L.Engine(device=L.DEVICE_FAKE, fake_sms=4, num_gpus=NG, num_clients=nclients, route=route,
                  event_log=log, route_log=rlog, streams=8, slack=8) as e:
        mids = [e.register_model(g, rng.model_params(g)) for g in models]
        _serve_bursts(e, mids, 600, nclients, seed=route + 3)
        per = [e.stats(i)["completed"] for i in range(NG)]
    assert sum(per) == 600
    # what each GPU's dispatcher published (W_g after every decide pass), and per-GPU replay
    published = {}
    for g in range(NG):
        cfg, ms, events, ex = eventlog.read(log % g)
        pub = []
        ok, msg, _ = sim.replay(cfg, ms, events, published=pub)
        assert ok, (g, msg)
        published[g] = set(pub)
    n = 0
    used = set()
    for c in range(nclients):
        recs = eventlog.read_routes(rlog % c)
        for i, r in enumerate(recs):
            assert r["route"] == route and r["num_gpus"] == NG and r["alive"] == (1 << NG) - 1
            W = [w + p * r["tbar_model"] for w, p in zip(r["work"], r["pending"])]
            if route == L.ROUTE_LEAST_WORK:
                want = sim.route_least_work(r["work"], r["pending"], r["tbar_model"], r["alive"])
            elif route == L.ROUTE_ROUND_ROBIN:
                want = i % NG
            else:
                g0, g1 = sim.route_pair(r["req_id"], NG)
                assert (r["g0"], r["g1"]) == (g0, g1)
                want = sim.route_pick((g0, g1), W)
            assert r["chosen"] == want, (c, i, r, want)
            for g in range(NG):
                assert r["pending"][g] >= 0
                assert r["work"][g] in published[g], (g, r["work"][g])
            used.add(r["chosen"])
            n += 1
    assert n == 600
    if route != L.ROUTE_POWER_OF_TWO:
        assert len(used) == NG      # bursts spread over all 8 GPUs
    if route == L.ROUTE_LEAST_WORK:
        # the decisions were not trivial: some snapshot had unequal W across GPUs
        assert any(len({w + p * r["tbar_model"] for w, p in zip(r["work"], r["pending"])}) > 1
                   for c in range(nclients) for r in eventlog.read_routes(rlog % c))
