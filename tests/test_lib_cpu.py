"""CPU tests of the C-ABI library (no GPU): exported symbols, argument checking,
and the dispatcher / router / replay path driven by the FAKE device backend (a CPU
model of a GPU that synthesises notification records in the same ring format).

Replay parity (pin S6): the C++ dispatcher's event log, replayed
through the oracle policy (oracle/sim.py), reproduces its issue sequence bit for bit.
"""
import errno
import os
import re
import subprocess
import time

import numpy as np
import pytest

from oracle import eventlog, sim
from workload import archs, rng

L = pytest.importorskip("paper_conf_sosp_ngd023_b200._lib")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_sosp_ngd023_b200 import build
    build.build()
    L.load()


def test_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "paella.h")).read()
    declared = set(re.findall(r"^\s*(?:int|int64_t|const char\*)\s+(paella_\w+)\s*\(", hdr, re.M))
    assert declared == set(L.SYMBOLS), declared ^ set(L.SYMBOLS)
    out = subprocess.run(["nm", "-D", "--defined-only", L.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (paella_\w+)", out))
    assert declared <= exported, declared - exported
    lib = L.load()
    for s in declared:
        assert hasattr(lib, s)


def _toy_engine(**kw):
    kw.setdefault("device", L.DEVICE_FAKE)
    kw.setdefault("fake_sms", 4)
    return L.Engine(**kw)


def test_init_rejects_bad_config():
    with pytest.raises(OSError) as ei:
        L.Engine(num_clients=0, device=L.DEVICE_FAKE)
    assert ei.value.errno == errno.EINVAL
    with pytest.raises(OSError):
        L.Engine(num_clients=1, device=L.DEVICE_FAKE, ring_capacity=1000)   # not a power of two
    with pytest.raises(OSError):
        L.Engine(num_clients=1, device=L.DEVICE_FAKE, group=17)


def test_submit_argument_errors_and_eagain():
    g = archs.toy()
    P = rng.model_params(g)
    with _toy_engine(num_clients=2) as e:
        mid = e.register_model(g, P)
        with pytest.raises(OSError) as ei:
            e.register_model(g, P)
        assert ei.value.errno == errno.EEXIST
        info = e.model_info(mid)
        need = info["input_bytes"] + info["output_bytes"]
        base, reg = e.region(0)
        lib = e.lib
        # outside the client's region -> EFAULT (P1060-1061)
        assert lib.paella_submit(e.h, 0, mid, base + len(reg) - 16, need, 0) == -errno.EFAULT
        base1, _ = e.region(1)
        assert lib.paella_submit(e.h, 0, mid, base1, need, 0) == -errno.EFAULT
        assert lib.paella_submit(e.h, 0, mid, base, need - 1, 0) == -errno.EINVAL
        assert lib.paella_submit(e.h, 0, 7, base, need, 0) == -errno.EINVAL
        assert lib.paella_submit(e.h, 5, mid, base, need, 0) == -errno.EINVAL
        rid, st = e.poll(0, L.NONBLOCK)
        assert rid == -errno.EAGAIN    # readResult NONBLOCK (P1150-1155)


def _serve(e, mids, n, n_clients, seed, stride=16384, timeout=60):
    r = np.random.default_rng(seed)
    infos = {m: e.model_info(m) for m in mids}
    out = {}
    pending = set()
    for i in range(n):
        c = int(r.integers(n_clients))
        m = int(r.choice(mids))
        need = infos[m]["input_bytes"] + infos[m]["output_bytes"]
        off = (i % 512) * stride
        rid = e.submit(c, m, off, need)
        assert rid >= 0, rid
        assert rid >> 48 == c
        pending.add(rid)
        if r.random() < 0.3:
            time.sleep(0.0002)
    t0 = time.time()
    while pending:
        assert time.time() - t0 < timeout, f"{len(pending)} requests never completed"
        for c in range(n_clients):
            rid, st = e.poll(c)
            if rid >= 0:
                assert st == 0
                pending.remove(rid)
                out[rid] = st
    return out


@pytest.mark.parametrize("policy,theta,group,streams,look,prio", [
    (L.POLICY_SRPT_DEFICIT, 100, 16, 8, 0, 1), (L.POLICY_SRPT_DEFICIT, 0, 1, 4, 0, 1),
    (L.POLICY_SRPT_DEFICIT, None, 4, 32, 0, 1), (L.POLICY_FIFO, 100, 16, 8, 0, 1),
    (L.POLICY_SRPT_DEFICIT, 3, 16, 2, 0, 1), (L.POLICY_SRPT_DEFICIT, 100, 16, 8, 1, 1),
    (L.POLICY_FIFO, 100, 4, 4, 1, 1), (L.POLICY_SRPT_DEFICIT, 0, 1, 16, 2, 1),
    (L.POLICY_SRPT_DEFICIT, 100, 16, 8, 1, 4), (L.POLICY_SRPT_DEFICIT, 3, 4, 12, 2, 3),
    (L.POLICY_SRPT_DEFICIT, None, 16, 32, 0, 2), (L.POLICY_FIFO, 100, 16, 8, 1, 2),
    (L.POLICY_SJF, 100, 16, 8, 0, 1), (L.POLICY_SJF, 100, 4, 4, 2, 2),
    (L.POLICY_RR, 100, 16, 8, 0, 1), (L.POLICY_RR, 100, 4, 12, 1, 3),
    (L.POLICY_SRPT_DEFICIT, 100, 16, 8, 0, -1), (L.POLICY_SRPT_DEFICIT, None, 4, 12, 2, -3),
    (L.POLICY_SJF, 3, 16, 8, 1, -1), (L.POLICY_SRPT_DEFICIT, 100, 16, 8, 6, 1),
    (L.POLICY_FIFO, 100, 1, 16, 7, 1)])
def test_fake_device_replay_parity(tmp_path, policy, theta, group, streams, look, prio):
    """prio < 0: |prio| classes with NEXT-4 online T-bar refinement (OBSERVE events)."""
    log = str(tmp_path / "ev_%u.log")
    models = [archs.toy(), archs.squeezenet1_1()]
    online, prio = prio < 0, abs(prio)
    with _toy_engine(num_clients=3, policy=policy, theta=theta, group=group, streams=streams,
                     event_log=log, ring_capacity=1024, slack=8, lookahead=look, prio_classes=prio,
                     online_tbar=online) as e:
        mids = [e.register_model(g, rng.model_params(g)) for g in models]
        _serve(e, mids, 300, 3, seed=policy * 10 + group)
    cfg, ms, events, ex = eventlog.read(log % 0)
    assert cfg.num_clients == 3 and cfg.policy == policy and cfg.group == group and cfg.lookahead == look
    assert cfg.prio_classes == prio and cfg.online_tbar == int(online)
    assert any(ev[0] == sim.EV_OBSERVE for ev in events) == online
    ok, msg, n = sim.replay(cfg, ms, events)
    assert ok, msg
    assert n == len(ex["issues"]) > 0 and ex["n_arrivals"] == 300 == len(ex["completes"])
    # S5 (b) exactly-once coverage of every launch's records
    grids = {uid: ms[model][layer].grid for (uid, job, layer, stream, model) in ex["issues"]}
    assert sim.check_exactly_once(ex["records"], grids, cfg.group) == []


def test_fake_replay_with_job_id_reuse(tmp_path):
    """Long run (job ids are recycled) still replays exactly."""
    log = str(tmp_path / "ev_%u.log")
    g = archs.toy()
    with _toy_engine(num_clients=2, event_log=log, max_jobs_per_model=8, streams=4) as e:
        mid = e.register_model(g, rng.model_params(g))
        _serve(e, [mid], 600, 2, seed=5)
        st = e.stats()
        assert st["completed"] == 600 and st["launches"] == 600 * 5
    cfg, ms, events, ex = eventlog.read(log % 0)
    ok, msg, n = sim.replay(cfg, ms, events)
    assert ok and n == 3000, msg


@pytest.mark.parametrize("route", [L.ROUTE_LEAST_WORK, L.ROUTE_ROUND_ROBIN, L.ROUTE_POWER_OF_TWO])
def test_router_multi_gpu_fake(tmp_path, route):
    log = str(tmp_path / "ev_%u.log")
    g = archs.toy()
    with _toy_engine(num_clients=2, num_gpus=4, route=route, event_log=log) as e:
        mid = e.register_model(g, rng.model_params(g))
        _serve(e, [mid], 400, 2, seed=11)
        per = [e.stats(i)["completed"] for i in range(4)]
    assert sum(per) == 400
    if route == L.ROUTE_ROUND_ROBIN:
        assert max(per) - min(per) <= 2 and min(per) > 0
    else:   # least outstanding work (of all GPUs or of two candidates): a burst spreads out
        assert sum(1 for x in per if x > 0) >= 2
    nroutes = 0
    for gi in range(4):   # every per-GPU dispatcher replays exactly
        cfg, ms, events, ex = eventlog.read(log % gi)
        ok, msg, n = sim.replay(cfg, ms, events)
        assert ok, (gi, msg)
        for g0, g1, r, rid, w0, w1 in ex["routes"]:   # the routing decisions replay too
            assert r == route
            if route == L.ROUTE_POWER_OF_TWO:
                assert (g0, g1) == sim.route_pair(rid, 4)
                assert sim.route_pick((g0, g1), {g0: w0, g1: w1}) == gi
            else:
                assert g0 == g1 == gi
        nroutes += len(ex["routes"])
    assert nroutes == 400


def test_shutdown_cancels_unadmitted():
    g = archs.toy()
    e = _toy_engine(num_clients=1, max_jobs_per_model=1, fake_time_scale_ns=1)
    mid = e.register_model(g, rng.model_params(g))
    info = e.model_info(mid)
    need = info["input_bytes"] + info["output_bytes"]
    for i in range(50):
        assert e.submit(0, mid, i * 16384, need) >= 0
    e.shutdown()


def test_hybrid_poll_sleeps_between_hints():
    """PAELLA_HYBRID (NEXT-3, P1157-1171): a client waiting for sparse completions
    spins briefly, then sleeps on the futex the dispatcher bumps on the "almost
    finished" hint and on completion -- every request completes, and the waiting thread
    uses a small fraction of one core (a spinning poll would use all of it)."""
    import threading
    e = _toy_engine(num_clients=1)
    mid = e.register_model(archs.toy(), rng.model_params(archs.toy()))
    info = e.model_info(mid)
    need = info["input_bytes"] + info["output_bytes"]
    n, gap = 20, 0.01
    got = []

    def waiter():
        t0 = time.thread_time()
        while len(got) < n:
            rid, st = e.poll(0, L.HYBRID)
            assert rid >= 0 and st == 0, (rid, st)
            got.append(rid)
        got.append(time.thread_time() - t0)

    th = threading.Thread(target=waiter)
    th.start()
    w0 = time.time()
    sent = []
    for i in range(n):
        sent.append(e.submit(0, mid, (i % 8) * 16384, need))
        time.sleep(gap)
    th.join(timeout=30)
    assert not th.is_alive()
    cpu, wall = got.pop(), time.time() - w0
    assert sorted(got) == sorted(sent)
    assert cpu < 0.5 * wall, (cpu, wall)
    e.shutdown()


def test_bench_wait_spin_vs_hybrid_fake():
    """paella_bench_wait (the NEXT-3 measurement): every request completes under both
    waiting modes; the hybrid waiter uses less CPU than the spinning one."""
    e = _toy_engine(num_clients=1)
    mid = e.register_model(archs.toy(), rng.model_params(archs.toy()))
    info = e.model_info(mid)
    stride = (info["input_bytes"] + info["output_bytes"] + 4095) // 4096 * 4096
    j0, spin = e.bench_wait(0, mid, 200, 500_000, 0, stride, 16)
    j1, hyb = e.bench_wait(0, mid, 200, 500_000, L.HYBRID, stride, 16)
    assert (j0 > 0).all() and (j1 > 0).all()
    assert hyb < 0.5 * spin, (hyb, spin)
    e.shutdown()


def test_route_pair_matches_oracle():
    """paella_route_pair (power-of-two choices) is bit-exact with the
    oracle's independent SplitMix64 derivation on every GPU count, and rejects bad
    arguments."""
    from oracle import sim
    r = np.random.default_rng(5)
    ids = [0, 1, (1 << 48) - 1, (63 << 48) | 12345] + [int(x) for x in r.integers(0, 1 << 62, 2000)]
    for ng in range(1, 9):
        for rid in ids:
            assert L.route_pair(rid, ng) == sim.route_pair(rid, ng), (rid, ng)
    for ng in (0, 9):
        with pytest.raises(OSError):
            L.route_pair(1, ng)


@pytest.mark.parametrize("policy,theta,K,look", [
    (L.POLICY_SRPT_DEFICIT, 100, 2, 0), (L.POLICY_SRPT_DEFICIT, None, 3, 2), (L.POLICY_SRPT_DEFICIT, 0, 1, 1),
    (L.POLICY_FIFO, 100, 2, 3), (L.POLICY_SJF, 100, 4, 1), (L.POLICY_RR, 100, 2, 0),
    (L.POLICY_SRPT_DEFICIT, 100, 3, 6), (L.POLICY_SRPT_DEFICIT, 100, 3, -6), (L.POLICY_FIFO, 100, 2, -2),
    (L.POLICY_SRPT_DEFICIT, None, 0, -3), (L.POLICY_SRPT_DEFICIT, 100, 103, -6), (L.POLICY_SRPT_DEFICIT, None, 101, 0)])
def test_fake_replay_max_active(tmp_path, policy, theta, K, look):
    """B200-Q6 (max_active = K): the C++ dispatcher's decisions with the job cap replay
    bit-exactly through the oracle policy; at most K capped jobs (plus deficit
    overrides) ever have kernels in flight.  look < 0: launch-ahead |look| without the
    placement test (lookahead_unplaced, the bench arms' NEXT-1 variant); K > 100: cap
    K - 100 admitting in arrival order (cap_fifo)."""
    log = str(tmp_path / "ev_%u.log")
    models = [archs.toy(), archs.squeezenet1_1()]
    unpl, look = look < 0, abs(look)
    cap_fifo, K = K > 100, K - 100 if K > 100 else K
    with _toy_engine(num_clients=3, policy=policy, theta=theta, streams=8, event_log=log, ring_capacity=1024,
                     slack=8, lookahead=look, max_active=K, lookahead_unplaced=unpl, cap_fifo=cap_fifo) as e:
        mids = [e.register_model(g, rng.model_params(g)) for g in models]
        _serve(e, mids, 200, 3, seed=K * 3 + policy)
    cfg, ms, events, ex = eventlog.read(log % 0)
    assert cfg.max_active == K and cfg.lookahead_unplaced == int(unpl) and cfg.cap_fifo == int(cap_fifo)
    assert sim.check_inflight_bound(events, ms, look) == []
    ok, msg, n = sim.replay(cfg, ms, events)
    assert ok, msg
    assert n == len(ex["issues"]) > 0 and len(ex["completes"]) == 200


# --- NEXT-4 intra-job branch concurrency (Fig. 7 waitlists, P906-951) ---------------

def _graph_kernel_deps(g):
    """Independent derivation of each kernel's inputs from the graph: kernel nodes are
    every node except concats and a GAP whose only consumer is an FC (fused); a node's
    tensor is written by its own kernel, else (concat / fused GAP) by the kernels of its
    inputs.  Returns {node: sorted producer nodes of the node's inputs + residual}."""
    nodes = g.nodes
    users = {}
    for i, n in enumerate(nodes):
        for s in n["inputs"]:
            users.setdefault(s, []).append(i)
        if n.get("residual") is not None:
            users.setdefault(n["residual"], []).append(i)
    fused = {i for i, n in enumerate(nodes) if n["op"] == "gap" and len(users.get(i, [])) == 1
             and nodes[users[i][0]]["op"] == "fc"}

    def writers(i):
        if i == 0 or (nodes[i]["op"] != "concat" and i not in fused):
            return {i}
        out = set()
        for s in nodes[i]["inputs"]:
            out |= writers(s)
        return out
    deps = {}
    for i, n in enumerate(nodes):
        if i == 0 or n["op"] == "concat" or i in fused:
            continue
        ws = set()
        for s in n["inputs"]:
            ws |= writers(s)
        if n.get("residual") is not None:
            ws |= writers(n["residual"])
        deps[i] = sorted(ws)
    return deps


@pytest.mark.parametrize("name", ["squeezenet1_1", "inception_v3", "resnet50", "densenet121"])
def test_planner_dag_matches_graph(name):
    """The planner's per-kernel dependencies equal an independent derivation from the
    graph; virtual streams number <= 4; every dependency on the SAME virtual stream is an
    earlier kernel of that stream (so stream order covers it)."""
    g = archs.build(name)
    with _toy_engine(num_clients=1, branches=True) as e:
        mid = e.register_model(g, rng.model_params(g))
        ks = e.kernels(mid)
    node_of = {}
    kidx = 1
    want = _graph_kernel_deps(g)
    kernel_nodes = [0] + sorted(want)
    assert len(kernel_nodes) == len(ks)
    node_of = {k: n for k, n in enumerate(kernel_nodes)}
    kof = {n: k for k, n in node_of.items()}
    for k, info in enumerate(ks):
        if k == 0:
            assert info["n_deps"] == 0
            continue
        exp = [kof[n] for n in want[node_of[k]]]
        assert info["n_deps"] == len(exp), (k, info["n_deps"], exp)
        assert info["deps"] == exp[:8], (k, info["deps"], exp)
        assert info["vs"] < 4
    nvs = len({k["vs"] for k in ks})
    if name in ("inception_v3", "squeezenet1_1", "resnet50"):
        assert nvs >= 2                   # branches exist
    if name == "densenet121":
        assert nvs == 1                   # every layer reads all earlier ones: one chain


@pytest.mark.parametrize("policy,look,K", [(L.POLICY_SRPT_DEFICIT, 0, 0), (L.POLICY_SRPT_DEFICIT, 2, 0),
                                           (L.POLICY_FIFO, 3, 2), (L.POLICY_SRPT_DEFICIT, 3, 3),
                                           (L.POLICY_SRPT_DEFICIT, -6, 3)])
def test_fake_replay_branches(tmp_path, policy, look, K):
    """NEXT-4: jobs whose kernels form a DAG over virtual streams (several CUDA streams
    per job) replay bit-exactly through the oracle policy (Topo / head).  look < 0:
    launch-ahead |look| without the placement test."""
    log = str(tmp_path / "ev_%u.log")
    models = [archs.squeezenet1_1(), archs.inception_v3()]
    unpl, look = look < 0, abs(look)
    with _toy_engine(num_clients=2, policy=policy, streams=12, event_log=log, ring_capacity=4096, slack=8,
                     lookahead=look, branches=True, max_active=K, fake_sms=8, lookahead_unplaced=unpl) as e:
        mids = [e.register_model(g, rng.model_params(g)) for g in models]
        _serve(e, mids, 60, 2, seed=17 + look)
    cfg, ms, events, ex = eventlog.read(log % 0)
    assert any(l.vs > 0 for m in ms for l in m)
    ok, msg, n = sim.replay(cfg, ms, events)
    assert ok, msg
    assert n == len(ex["issues"]) and len(ex["completes"]) == 60
    # two kernels of one job were in flight on different streams at the same time
    grid = {uid: ms[model][layer].grid for (uid, job, layer, stream, model) in ex["issues"]}
    done, live, conc = {}, {}, False
    for ev in events:
        if ev[0] == sim.EV_ISSUE:
            uid, job, layer, stream = ev[1:5]
            live[uid] = (job, stream)
            conc |= len({s for (j, s) in live.values() if j == job}) > 1
        elif ev[0] == sim.EV_RECORD and ev[1] == sim.COMPLETION:
            done[ev[2]] = done.get(ev[2], 0) + ev[3]
            if done[ev[2]] == grid[ev[2]]:
                live.pop(ev[2])
    assert conc


def test_hol_synthetic_model_plans_and_serves():
    """Fig. 2's synthetic job (8 one-block spin kernels + a 1-pixel GAP): planned as
    ingest + 8 spin kernels + GAP, each spin kernel 1 block x 128 threads; served on the
    fake device; the oracle's forward is the identity on the 8-channel input (closed form)."""
    from oracle import infer
    g = archs.hol_synthetic(8, 50)
    P = rng.model_params(g)
    assert P == {}
    x = rng.image(g, 3)
    assert np.array_equal(infer.forward(g, P, x, dtype="fp32"), x.reshape(-1).astype(np.float64))
    with _toy_engine(num_clients=1, max_jobs_per_model=64) as e:
        mid = e.register_model(g, P)
        ks = e.kernels(mid)
        assert [k["name"] for k in ks] == ["ingest"] + ["spin"] * 8 + ["gap"]
        assert all(k["grid"] == 1 and k["block"] == 128 for k in ks[1:9])
        _serve(e, [mid], 40, 1, seed=2, stride=256)


def test_struct_layout_matches_header(tmp_path):
    """The ctypes mirrors of paella_config_t / paella_stats_t / paella_kernel_info_t /
    paella_route_rec_t have exactly the C layout of include/paella.h (sizes and every
    field offset, compiled with gcc here): marshalling cannot silently shift a field."""
    import ctypes as C
    checks = [("paella_config_t", L.Config), ("paella_stats_t", L.Stats), ("paella_kernel_info_t", L.KernelInfo),
              ("paella_model_info_t", L.ModelInfo), ("paella_req_t", L.Req), ("paella_node_t", L.Node),
              ("paella_model_desc_t", L.ModelDesc)]
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "paella.h"', "int main(void){"]
    for cname, py in checks:
        lines.append(f'printf("{cname} %zu\\n", sizeof({cname}));')
        for f, _ in py._fields_:
            lines.append(f'printf("{cname}.{f} %zu\\n", offsetof({cname}, {f}));')
    lines.append("return 0;}")
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    subprocess.run(["gcc", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)], check=True)
    out = dict(l.rsplit(" ", 1) for l in subprocess.run([str(exe)], capture_output=True, text=True,
                                                         check=True).stdout.splitlines())
    for cname, py in checks:
        assert int(out[cname]) == C.sizeof(py), cname
        for f, _ in py._fields_:
            assert int(out[f"{cname}.{f}"]) == getattr(py, f).offset, (cname, f)
