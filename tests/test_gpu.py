"""GPU parity tests (need a B200 and the built libpaella.so; run with -m gpu).

* kernels: every model of the mix, run isolated through the C ABI, vs the float64
  oracle (oracle/infer.py) -- bf16 path within max-abs 2e-2 / rel 1e-2, fp32 path
  within 1e-4 (BASELINE.json north_star tolerances, reading C1-Q6: atol + rtol|ref|);
* serving: mixed concurrent requests through paella_submit / poll_completion on the
  real dispatcher; every output checked against the oracle; the GPU event log
  replayed through the oracle policy reproduces the issue order bit-exactly (S6);
  every launch's notification records tile its grid exactly once (S5 b);
* the naive baseline path produces the same outputs;
* ring wrap-around (small ring, many laps), G = 1, a single stream.
"""
import os
import time

import numpy as np
import pytest

from oracle import eventlog, infer, sim
from workload import archs, rng

pytestmark = pytest.mark.gpu

L = pytest.importorskip("paper_conf_sosp_ngd023_b200._lib")

BF16_TOL = (2e-2, 1e-2)
FP32_TOL = (1e-4, 1e-4)
_ORACLE = {}


def oracle_out(name, i, dtype):
    key = (name, i, dtype)
    if key not in _ORACLE:
        g = archs.build(name)
        _ORACLE[key] = infer.forward(g, rng.model_params(g), rng.image(g, i), dtype=dtype)
    return _ORACLE[key]


def within(out, ref, tol):
    atol, rtol = tol
    return np.abs(out - ref) <= atol + rtol * np.abs(ref)


@pytest.fixture(scope="module")
def engine():
    from paper_conf_sosp_ngd023_b200 import build
    build.build()
    e = L.Engine(num_clients=1)
    yield e
    e.shutdown()


MODELS = ["toy", "resnet18", "mobilenet_v2", "squeezenet1_1", "resnet50", "densenet121", "inception_v3"]


@pytest.mark.parametrize("name", MODELS)
def test_isolated_bf16_parity(engine, name):
    g = archs.build(name)
    mid = engine.register_model(g, rng.model_params(g), dtype=L.DTYPE_BF16, name=name + "-iso")
    for i in (0, 1):
        out = engine.run_isolated(mid, rng.image(g, i))
        ref = oracle_out(name, i, "bf16")
        ok = within(out, ref, BF16_TOL)
        assert ok.all(), f"{name} input {i}: {np.sum(~ok)} logits out of tolerance, max err {np.abs(out-ref).max()}"


@pytest.mark.parametrize("name", ["mobilenet_v2", "densenet121", "inception_v3"])
def test_isolated_bf16_parity_m64(engine, name, monkeypatch):
    """The opt-in UMMA M = 64 conv (PAELLA_M64, layers with <= 64 output channels),
    planned at registration, against the same float64 oracle as the default kernels."""
    monkeypatch.setenv("PAELLA_M64", "1")
    g = archs.build(name)
    mid = engine.register_model(g, rng.model_params(g), dtype=L.DTYPE_BF16, name=name + "-m64")
    assert any(k["name"].startswith("conv_tcgen05") for k in engine.kernels(mid))
    out = engine.run_isolated(mid, rng.image(g, 0))
    ref = oracle_out(name, 0, "bf16")
    ok = within(out, ref, BF16_TOL)
    assert ok.all(), f"{name}: {np.sum(~ok)} logits out of tolerance, max err {np.abs(out-ref).max()}"


@pytest.mark.parametrize("name", ["toy", "resnet18", "mobilenet_v2", "squeezenet1_1", "densenet121", "resnet50",
                                  "inception_v3"])
def test_isolated_fp32_parity(engine, name):
    g = archs.build(name)
    mid = engine.register_model(g, rng.model_params(g), dtype=L.DTYPE_FP32, name=name + "-f32")
    out = engine.run_isolated(mid, rng.image(g, 0))
    ref = oracle_out(name, 0, "fp32")
    assert within(out, ref, FP32_TOL).all(), np.abs(out - ref).max()


@pytest.mark.parametrize("name", ["resnet18", "densenet121"])
def test_forced_split_k_parity(engine, name, tmp_path, monkeypatch):
    """Every cluster split-K factor the autotuner may pick (1..16, including splits with
    empty k-ranges) with either split-K reduction (bulk fp32 adds in L2, or pushes over
    DSMEM), forced on every tcgen05 layer through the split cache (PAELLA_SPLITS_FILE),
    stays within the bf16 tolerance."""
    g = archs.build(name)
    P = rng.model_params(g)
    ref = oracle_out(name, 0, "bf16")
    for sp, dsm in ((1, 0), (2, 0), (4, 0), (8, 0), (16, 0), (2, 1), (4, 1), (8, 1), (16, 1)):
        mname = f"{name}-split{sp}-{dsm}"
        f = tmp_path / f"splits{sp}-{dsm}.txt"
        f.write_text("".join(f"{mname} {l} {sp} {dsm}\n" for l in range(len(g.nodes) + 2)))
        monkeypatch.setenv("PAELLA_SPLITS_FILE", str(f))
        mid = engine.register_model(g, P, dtype=L.DTYPE_BF16, name=mname)
        monkeypatch.delenv("PAELLA_SPLITS_FILE")
        ks = engine.kernels(mid)
        assert any(k["name"].startswith("conv_tcgen05") and k["grid"] % sp == 0 for k in ks)
        out = engine.run_isolated(mid, rng.image(g, 0))
        ok = within(out, ref, BF16_TOL)
        assert ok.all(), f"{name} split {sp} dsmem {dsm}: max err {np.abs(out - ref).max()}"
        out2 = engine.run_isolated(mid, rng.image(g, 0))   # the workspace is zero again
        assert within(out2, ref, BF16_TOL).all(), f"{name} split {sp} dsmem {dsm}: second run"


def _serve_and_check(e, specs, n, n_clients, seed, rate_us=30.0):
    """specs: list of (model id, model name, graph).  Submits n requests with Poisson
    gaps, distinct pooled inputs, checks all outputs against the oracle."""
    r = np.random.default_rng(seed)
    infos = {mid: e.model_info(mid) for mid, _, _ in specs}
    stride = max(i["input_bytes"] + i["output_bytes"] for i in infos.values())
    stride = (stride + 4095) // 4096 * 4096
    slots = 64
    free = {c: list(range(slots)) for c in range(n_clients)}
    pending = {}
    done = 0
    sent = 0
    t0 = time.time()
    while done < n:
        assert time.time() - t0 < 120, f"timeout: {done}/{n} completed"
        if sent < n:
            c = int(r.integers(n_clients))
            if free[c]:
                mid, name, g = specs[int(r.integers(len(specs)))]
                slot = free[c].pop()
                off = slot * stride
                idx = int(r.integers(4))
                x = rng.image(g, idx)
                _, reg = e.region(c)
                reg[off:off + x.nbytes] = np.frombuffer(x.tobytes(), np.uint8)
                rid = e.submit(c, mid, off, infos[mid]["input_bytes"] + infos[mid]["output_bytes"])
                assert rid >= 0
                pending[rid] = (c, slot, off, mid, name, idx)
                sent += 1
                time.sleep(r.exponential(rate_us) * 1e-6)
        for c in range(n_clients):
            while True:
                rid, st = e.poll(c)
                if rid < 0:
                    break
                assert st == 0
                c2, slot, off, mid, name, idx = pending.pop(rid)
                _, reg = e.region(c2)
                ib = infos[mid]["input_bytes"]
                out = np.frombuffer(reg[off + ib:off + ib + infos[mid]["output_bytes"]].tobytes(), np.float32)
                ref = oracle_out(name, idx, "bf16")
                assert within(out, ref, BF16_TOL).all(), (name, np.abs(out - ref).max())
                free[c2].append(slot)
                done += 1


@pytest.mark.parametrize("policy,group,streams,ring,look,lt,notify,prio", [
    (L.POLICY_SRPT_DEFICIT, 16, 32, 65536, 0, 0, "counters", 1),
    (L.POLICY_FIFO, 16, 32, 65536, 0, 0, "counters", 1),
    (L.POLICY_SRPT_DEFICIT, 1, 8, 1024, 0, 0, "ring", 1),     # G = 1 debug mode, ring wraps many laps
    (L.POLICY_SRPT_DEFICIT, 1, 8, 1024, 0, 0, "counters", 2),
    (L.POLICY_SRPT_DEFICIT, 16, 1, 1024, 0, 0, "counters", 1),    # a single stream
    (L.POLICY_SRPT_DEFICIT, 16, 32, 65536, 3, 4, "counters", 4),  # the bench arm
    (L.POLICY_SRPT_DEFICIT, 4, 16, 4096, 2, 3, "ring", 4),
    (L.POLICY_SRPT_DEFICIT, 16, 32, 2048, 1, 2, "direct", 1),  # direct record writes (the paper's path)
    (L.POLICY_SRPT_DEFICIT, 16, 32, 65536, 3, 4, "counters", -4),  # bench arm + online T-bar (NEXT-4)
    (L.POLICY_SJF, 16, 32, 65536, 3, 4, "counters", 1),
    (L.POLICY_SRPT_DEFICIT, 16, 32, 65536, -6, 8, "counters", 108),  # the bench arm: K = 8, launch-ahead 6 unplaced
    (L.POLICY_SRPT_DEFICIT, 16, 32, 65536, -6, 8, "counters", 208),  # ... with the cap admitting in arrival order
    (L.POLICY_SRPT_DEFICIT, 16, 32, 65536, 6, 4, "counters", 108),
    (L.POLICY_SRPT_DEFICIT, 16, 32, 65536, 3, 4, "counters", 108),
    (L.POLICY_FIFO, 16, 32, 65536, 3, 4, "counters", 104),           # FIFO arm, K = 4
    (L.POLICY_RR, 16, 8, 4096, 0, 0, "counters", 1),
])
def test_serving_parity_and_replay(tmp_path, policy, group, streams, ring, look, lt, notify, prio):
    log = str(tmp_path / "gpu_%u.log")
    names = ["toy", "resnet18", "mobilenet_v2", "squeezenet1_1"]
    online, prio = prio < 0, abs(prio)
    unpl, look = look < 0, abs(look)          # look < 0: launch-ahead without the placement test
    cap_fifo = prio > 200                     # 2xx: job cap K = xx admitting in arrival order
    K = prio % 100 if prio > 100 else 0       # 1xx: job cap K = xx (B200-Q6), one priority class
    prio = 1 if K else prio
    with L.Engine(num_clients=3, policy=policy, group=group, streams=streams, ring_capacity=ring,
                  event_log=log, max_jobs_per_model=32, lookahead=look, launch_threads=lt, notify=notify,
                  prio_classes=prio, slack=(3552 if K else 1184) if (prio > 1 or K) else 0, online_tbar=online,
                  max_active=K, lookahead_unplaced=unpl, cap_fifo=cap_fifo) as e:
        specs = []
        for nm in names:
            g = archs.build(nm)
            specs.append((e.register_model(g, rng.model_params(g)), nm, g))
        _serve_and_check(e, specs, 120, 3, seed=policy * 7 + group)
        st = e.stats()
        assert st["completed"] == 120
        if notify == "counters":
            # S5 (b) on the device: the blocks' own counts, not the records the dispatcher
            # synthesised from them -- every slot advanced by exactly its launches' grids
            time.sleep(0.01)
            bad, used = e.check_counters()
            assert bad == 0 and used > 0, (bad, used)
        if notify == "counters" and look == 0:
            # relaxed exits: jobs that went idle recorded a release event; moves to another
            # stream waited for it (the outputs above are checked either way; with
            # launch-ahead a job rarely goes idle between its kernels)
            assert st["rel_events"] > 0
            print("release events", st["rel_events"], "cross-stream waits", st["xstream_waits"])
    cfg, ms, events, ex = eventlog.read(log % 0)
    ok, msg, n = sim.replay(cfg, ms, events)
    assert ok, msg
    assert n == len(ex["issues"]) == st["launches"]
    grids = {uid: ms[model][layer].grid for (uid, job, layer, stream, model) in ex["issues"]}
    assert sim.check_exactly_once(ex["records"], grids, cfg.group) == []
    assert sim.check_inflight_bound(events, ms, look) == []


@pytest.mark.parametrize("lt", [0, 2])
def test_naive_baseline_outputs(lt):
    names = ["toy", "squeezenet1_1"]
    with L.Engine(num_clients=2, naive=True, instrument=False, launch_threads=lt) as e:
        specs = []
        for nm in names:
            g = archs.build(nm)
            specs.append((e.register_model(g, rng.model_params(g)), nm, g))
        _serve_and_check(e, specs, 60, 2, seed=3)


def test_ring_records_carry_sm_and_time(tmp_path):
    """G=1: one PLACEMENT and one COMPLETION per block, SM ids < 148, completion time
    of a block's group never before the first placement of its launch."""
    log = str(tmp_path / "g1_%u.log")
    g = archs.toy()
    with L.Engine(num_clients=1, group=1, event_log=log, notify="ring") as e:
        mid = e.register_model(g, rng.model_params(g))
        _serve_and_check(e, [(mid, "toy", g)], 10, 1, seed=1)
    cfg, ms, events, ex = eventlog.read(log % 0)
    recs = ex["records"]
    assert all(r[3] == 1 for r in recs)
    assert all(r[5] < 148 for r in recs)
    first_place = {}
    for (t, typ, uid, n, grp, sm) in recs:
        if typ == sim.PLACEMENT:
            first_place[uid] = min(first_place.get(uid, t), t)
    for (t, typ, uid, n, grp, sm) in recs:
        if typ == sim.COMPLETION:
            assert (t - first_place[uid]) % (1 << 40) < (1 << 39)


def test_per_sm_capacity_from_g1_records(tmp_path):
    """S5 (a) on the GPU: with G = 1 every block reports (SM id, globaltimer) at entry
    and exit; the blocks resident on any SM at any time never need more than one SM's
    Table-1 resources (+TMEM) according to the demands the dispatcher accounts."""
    log = str(tmp_path / "cap_%u.log")
    names = ["resnet18", "mobilenet_v2", "squeezenet1_1"]
    with L.Engine(num_clients=3, group=1, event_log=log, ring_capacity=4096, lookahead=1, launch_threads=2,
                  notify="ring") as e:
        specs = []
        for nm in names:
            g = archs.build(nm)
            specs.append((e.register_model(g, rng.model_params(g)), nm, g))
        _serve_and_check(e, specs, 60, 3, seed=11, rate_us=5.0)
    cfg, ms, events, ex = eventlog.read(log % 0)
    demand = {uid: ms[model][layer].demand for (uid, job, layer, stream, model) in ex["issues"]}
    opened = {}
    evs = []
    for (t, typ, uid, n, grp, sm) in ex["records"]:
        evs.append((t, 0 if typ == sim.COMPLETION else 1, uid, sm))   # exits before entries at equal t
    evs.sort()
    per_sm = (32, 64, 65536, 233472, 512)
    use = {}
    worst = [0] * 5
    for (t, kind, uid, sm) in evs:
        u = use.setdefault(sm, [0] * 5)
        d = demand[uid]
        if kind == 1:
            for r in range(5):
                u[r] += d[r]
                worst[r] = max(worst[r], u[r])
            opened[(uid, sm)] = opened.get((uid, sm), 0) + 1
        elif opened.get((uid, sm), 0) > 0:
            opened[(uid, sm)] -= 1
            for r in range(5):
                u[r] -= d[r]
    for r in range(5):
        assert worst[r] <= per_sm[r], (r, worst)


@pytest.mark.gpu
def test_serving_parity_c3_models_bench_arm(tmp_path):
    """C-3's models (ResNet-50, DenseNet-121, Inception-v3, MobileNetV2) served
    concurrently in the launch configuration bench.py times (launch-ahead 6 without the
    placement test, job cap 8, 8 launcher threads, counter notification, B = 24x148,
    dispatcher on its own core): every output
    within the bf16 tolerance of the float64 oracle and the issue order replayed."""
    log = str(tmp_path / "gpu_%u.log")
    names = ["resnet50", "densenet121", "inception_v3", "mobilenet_v2"]
    for nm in names:   # the float64 references first: the serving loop has a 120 s bound
        for i in range(4):
            oracle_out(nm, i, "bf16")
    cpus = sorted(os.sched_getaffinity(0))
    with L.Engine(num_clients=4, event_log=log, max_jobs_per_model=32, lookahead=6, launch_threads=8,
                  slack=3552, max_active=8, lookahead_unplaced=True,
                  region_bytes=96 << 20,   # 64 slots of Inception-v3's 1.08 MB io buffer
                  dispatcher_cpus=[cpus[min(2, len(cpus) - 1)]]) as e:
        specs = []
        for nm in names:
            g = archs.build(nm)
            specs.append((e.register_model(g, rng.model_params(g)), nm, g))
        _serve_and_check(e, specs, 80, 4, seed=21)
        st = e.stats()
        assert st["completed"] == 80
    cfg, ms, events, ex = eventlog.read(log % 0)
    ok, msg, n = sim.replay(cfg, ms, events)
    assert ok, msg
    assert n == len(ex["issues"]) == st["launches"]
    assert sim.check_inflight_bound(events, ms, 6) == []


@pytest.mark.parametrize("name", ["resnet18", "inception_v3"])
def test_ingest_rne_bit_exact(engine, name):
    """The ingest kernel's bf16 rounding (C3 / reading C1-Q7) is bit-exact with
    oracle.bf16.round_bf16 -- on the pooled inputs AND on an adversarial image: exact
    ties between neighbouring bf16 values (must round to even), one fp32 ulp either side
    of the tie, exact bf16 values, negatives, subnormals and finite values that round
    up to infinity.  224x224 takes the 4-pixel path (196 CTAs), 299x299 the 1-pixel one."""
    from oracle.bf16 import round_bf16
    g = archs.build(name)
    mid = engine.register_model(g, rng.model_params(g), dtype=L.DTYPE_BF16, name=name + "-rne")
    shape = tuple(g.nodes[0]["out"])
    n = int(np.prod(shape))
    r = np.random.default_rng(77)
    hi = r.integers(0, 0x7F80, n, dtype=np.uint32)                 # finite bf16 magnitudes
    sign = (r.integers(0, 2, n, dtype=np.uint32) << 31)
    low = r.choice(np.array([0x8000, 0x7FFF, 0x8001, 0x0000, 0x0001, 0xFFFF], dtype=np.uint32), n)
    bits = sign | (hi << 16) | low
    bits[:8] = [0x7F7FFFFF, 0xFF7FFFFF, 0x7F7F8000, 0x00008000, 0x80018000, 0x3F808000, 0x3F818000, 0]
    adversarial = bits.view(np.float32).reshape(shape)
    images = [rng.image(g, i) for i in range(4)] + [adversarial]
    for x in images:
        engine.run_isolated(mid, x)
        got = engine.debug_node(mid, 0, shape)
        want = round_bf16(x)
        diff = got.view(np.uint32) != want.view(np.uint32)
        assert not diff.any(), (int(diff.sum()), x[diff][:4], got[diff][:4], want[diff][:4])


def test_clock_calibration_and_record_times(tmp_path):
    """globaltimer -> host clock (C3): calibrated at init and again after serving
    (paella_clock_sync; the two oscillators drift by ppm, so records are converted with
    the offset interpolated between calibrations); the round trip and the timer
    resolution are measured.  Every G = 1 ring record, converted to host time, falls
    inside the life of its job: [scheduled arrival, completion seen by the dispatcher]
    (tolerance: the larger calibration round trip + 5 us)."""
    from oracle import ringcheck
    log = str(tmp_path / "clk_%u.log")
    names = ["toy", "resnet18"]
    with L.Engine(num_clients=2, group=1, event_log=log, notify="ring", ring_capacity=8192) as e:
        off0, rtt0, res = e.clock_info()
        assert 0 < rtt0 < 200_000 and 0 < res < 10_000, (off0, rtt0, res)
        specs = []
        for nm in names:
            g = archs.build(nm)
            specs.append((e.register_model(g, rng.model_params(g)), nm, g))
        e.clock_sync()
        _serve_and_check(e, specs, 40, 2, seed=4)
        e.clock_sync()
        off1, rtt1, _ = e.clock_info()
    cfg, ms, events, ex = eventlog.read(log % 0)
    cl = ex["clocks"]
    assert len(cl) == 3 and cl[0]["offset"] == off0 and cl[-1]["offset"] == off1
    span = (cl[-1]["at"] - cl[0]["at"]) / 1e9
    print(f"clock: resolution {res} ns, rtt {rtt0}/{rtt1} ns, offset drift {off1 - off0} ns over {span:.2f} s "
          f"({(off1 - off0) / max(span, 1e-9) / 1e3:.2f} ppm)")
    lives = ex["lives"]
    windows = {uid: (lives[li]["t_sched"], lives[li]["t_complete"]) for uid, li in ex["uid_life"].items()}
    recs = [r for r in ex["records"] if r[2] in windows]
    assert len(recs) == len(ex["records"]) > 0
    bad = ringcheck.check_record_times(recs, windows, cl[1:], max(c["rtt"] for c in cl) + 5000)
    assert bad == [], bad[:5]


def test_hybrid_completion_serving(tmp_path):
    """NEXT-3 on the GPU (P1157-1171): a client thread waits with PAELLA_HYBRID polls
    (spin, then futex sleep between the dispatcher's hints) while another submits; every
    output matches the oracle and the waiter uses well under a full core."""
    import threading
    names = ["resnet18", "squeezenet1_1"]
    with L.Engine(num_clients=1, lookahead=3, launch_threads=2, slack=1184) as e:
        specs = []
        for nm in names:
            g = archs.build(nm)
            specs.append((e.register_model(g, rng.model_params(g)), nm, g))
        infos = {mid: e.model_info(mid) for mid, _, _ in specs}
        stride = (max(i["input_bytes"] + i["output_bytes"] for i in infos.values()) + 4095) // 4096 * 4096
        n = 60
        sent = {}
        got = []
        slot_free = [threading.Event() for _ in range(16)]
        for ev in slot_free:
            ev.set()
        lock = threading.Lock()

        def waiter():
            t0 = time.thread_time()
            while len(got) < n:
                rid, st = e.poll(0, L.HYBRID)
                assert rid >= 0 and st == 0, (rid, st)
                with lock:
                    slot, mid, nm, idx = sent[rid]
                _, reg = e.region(0)
                ib = infos[mid]["input_bytes"]
                out = np.frombuffer(reg[slot * stride + ib:slot * stride + ib + infos[mid]["output_bytes"]].tobytes(),
                                    np.float32)
                got.append((nm, idx, out.copy()))
                slot_free[slot].set()
            got.append(time.thread_time() - t0)

        th = threading.Thread(target=waiter)
        w0 = time.time()
        th.start()
        r = np.random.default_rng(9)
        for i in range(n):
            slot = i % 16
            assert slot_free[slot].wait(30)
            slot_free[slot].clear()
            mid, nm, g = specs[i % 2]
            idx = int(r.integers(4))
            x = rng.image(g, idx)
            _, reg = e.region(0)
            reg[slot * stride:slot * stride + x.nbytes] = np.frombuffer(x.tobytes(), np.uint8)
            with lock:
                rid = e.submit(0, mid, slot * stride, infos[mid]["input_bytes"] + infos[mid]["output_bytes"])
                assert rid >= 0
                sent[rid] = (slot, mid, nm, idx)
            time.sleep(0.002)
        th.join(timeout=60)
        assert not th.is_alive()
        cpu, wall = got.pop(), time.time() - w0
    for nm, idx, out in got:
        assert within(out, oracle_out(nm, idx, "bf16"), BF16_TOL).all()
    assert cpu < 0.7 * wall, (cpu, wall)


@pytest.mark.parametrize("look,K", [(3, 8), (0, 0), (-6, 8)])
def test_serving_branches_c3_models(tmp_path, look, K):
    """NEXT-4 intra-job branch concurrency on the GPU: C-3's models served with their
    kernel DAGs over virtual streams (Inception / ResNet-50 branches on several CUDA
    streams at once; a consumer on another stream is issued after its inputs' final
    COMPLETION, whose exit count is a release): every output within the bf16 tolerance,
    the issue order replayed bit-exactly, launch-ahead depth respected per stream.
    look < 0: launch-ahead |look| without the placement test (the bench arms' rule)."""
    log = str(tmp_path / "br_%u.log")
    unpl, look = look < 0, abs(look)
    names = ["resnet50", "inception_v3", "mobilenet_v2", "squeezenet1_1"]
    for nm in names:
        for i in range(4):
            oracle_out(nm, i, "bf16")
    with L.Engine(num_clients=4, event_log=log, max_jobs_per_model=32, lookahead=look, launch_threads=4,
                  slack=1184, region_bytes=96 << 20, branches=True, max_active=K, lookahead_unplaced=unpl) as e:
        specs = []
        for nm in names:
            g = archs.build(nm)
            specs.append((e.register_model(g, rng.model_params(g)), nm, g))
        _serve_and_check(e, specs, 80, 4, seed=23 + look)
        st = e.stats()
        assert st["completed"] == 80
    cfg, ms, events, ex = eventlog.read(log % 0)
    assert any(l.vs > 0 for m in ms for l in m)
    ok, msg, n = sim.replay(cfg, ms, events)
    assert ok, msg
    assert n == len(ex["issues"]) == st["launches"]
    assert sim.check_inflight_bound(events, ms, look) == []


@pytest.mark.parametrize("dtype", ["bf16", "fp32"])
def test_c1_toy_config(tmp_path, dtype):
    """BASELINE configs[0] / SURVEY.md 8(d) C-1 as specified: 2 clients x 100 requests of
    the toy model, superposed Poisson arrivals at 5,000 req/s, every request with its own
    input (pool indices 0..199), theta = 100, B = 148, G = 16.  Every output is checked
    against the float64 oracle (bf16: 2e-2 / 1e-2, fp32: 1e-4), the issue order replays
    bit-exactly, records tile every launch exactly once, and the oracle simulator runs
    the same trace (synthetic mode, profiled T-bar) in seconds."""
    from workload import traces
    log = str(tmp_path / "c1_%u.log")
    g = archs.toy()
    P = rng.model_params(g)
    n = 200
    t = traces.arrivals(n, 5000.0, kind="poisson", seed=1)
    clients = np.arange(n) % 2
    tol = BF16_TOL if dtype == "bf16" else FP32_TOL
    with L.Engine(num_clients=2, event_log=log, slack=148) as e:
        mid = e.register_model(g, P, dtype=L.DTYPE_BF16 if dtype == "bf16" else L.DTYPE_FP32)
        info = e.model_info(mid)
        need = info["input_bytes"] + info["output_bytes"]
        stride = (need + 255) // 256 * 256
        offs = {}
        for i in range(n):                       # request i: its own slot and input
            c = int(clients[i])
            off = (i // 2) * stride
            x = rng.image(g, i)
            _, reg = e.region(c)
            reg[off:off + x.nbytes] = np.frombuffer(x.tobytes(), np.uint8)
            offs[i] = (c, off)
        t0 = time.monotonic_ns() + 2_000_000
        pending = set()
        i = 0
        while i < n or pending:
            now = time.monotonic_ns()
            while i < n and t0 + int(t[i]) <= now:
                c, off = offs[i]
                rid = e.submit(c, mid, off, need, t_sched_ns=t0 + int(t[i]))
                assert rid >= 0
                pending.add(rid)
                i += 1
            for c in (0, 1):
                rid, st = e.poll(c)
                if rid >= 0:
                    assert st == 0
                    pending.discard(rid)
            assert time.monotonic_ns() - t0 < 30e9
        ib = info["input_bytes"]
        for i in range(n):                       # every output, against the float64 oracle
            c, off = offs[i]
            _, reg = e.region(c)
            out = np.frombuffer(reg[off + ib:off + need].tobytes(), np.float32)
            ref = infer.forward(g, P, rng.image(g, i), dtype=dtype)
            assert within(out, ref, tol).all(), (i, np.abs(out - ref).max())
    cfg, ms, events, ex = eventlog.read(log % 0)
    ok, msg, nchk = sim.replay(cfg, ms, events)
    assert ok, msg
    grids = {uid: ms[model][layer].grid for (uid, job, layer, stream, model) in ex["issues"]}
    assert sim.check_exactly_once(ex["records"], grids, cfg.group) == []
    assert ex["n_arrivals"] == n == len(ex["completes"])
    # the simulator on the same trace: synthetic GPU, block durations = profiled T-bar
    models = [[sim.Layer(l.grid, l.demand, l.tbar, max(1, l.tbar)) for l in m] for m in ms]
    trace = [(int(t[k]), int(clients[k]), 0) for k in range(n)]
    ts = time.perf_counter()
    res = sim.simulate(sim.Config(num_clients=2, slack=148), models, trace, sim.GPUModel(), check=True)
    assert len(res.finish) == n and not res.violations
    assert time.perf_counter() - ts < 30


def test_hol_spin_kernels(engine):
    """The Fig. 2 synthetic job on the GPU: 8 one-block kernels, each resident >= its spin
    time (device time of the chain >= 8 x 20 us), output = the bf16-rounded input
    (identity copies; oracle closed form)."""
    from oracle.bf16 import round_bf16
    g = archs.hol_synthetic(8, 20)
    mid = engine.register_model(g, rng.model_params(g), name="hol-test")
    for i in range(3):
        x = rng.image(g, i)
        out, kt = engine.run_isolated(mid, x, timing=True)
        assert np.array_equal(out, round_bf16(x).reshape(-1)), (out, x)
        assert all(t >= 20_000 for t in kt[1:9]), kt


def test_bench_xdev_graph_replay():
    """X_dev: each model's uninstrumented chain captured as a CUDA graph
    (PDL edges) per stream and replayed at overload; the device-only rate of a 2-model
    mix exceeds what one stream achieves (concurrency pays) and is finite."""
    with L.Engine(num_clients=1, max_jobs_per_model=32) as e:
        mids = []
        for nm in ("resnet18", "squeezenet1_1"):
            g = archs.build(nm)
            mids.append(e.register_model(g, rng.model_params(g)))
        seq = np.arange(400) % 2
        r32 = e.bench_xdev(mids, seq, streams=32)
        r1 = e.bench_xdev(mids, seq, streams=1)
    assert 0 < r1 < r32 < 1e6, (r1, r32)


def test_wide_tile_conv_parity(engine):
    """KIND_CONV_TC128 (128-pixel tiles, chosen for saturating shapes: >= 2 waves of
    64-pixel tiles): a 3x3 64->64 conv over 200x200 pixels (625 tiles of 64) and the
    logits behind it match the float64 oracle -- the conv's own output element by
    element (bf16 tolerance), with the ragged last tile (40,000 = 312 x 128 + 64)."""
    from oracle.bf16 import round_bf16
    g = archs.Graph("wide200", (3, 200, 200), 10)
    x = g.conv(g.input, 64, 1, name="stem")
    y = g.conv(x, 64, 3, 1, 1, name="big")
    z = g.gap(y, name="gap")
    g.fc(z, 10, name="fc")
    r = np.random.default_rng(5)
    P = {}
    for nd in g.weight_nodes():
        shp = g.param_shapes()[nd["name"] + ".weight"]
        P[nd["name"] + ".weight"] = round_bf16((r.standard_normal(shp) / np.sqrt(np.prod(shp[1:]))).astype(np.float32))
        P[nd["name"] + ".bias"] = (0.01 * r.standard_normal(shp[0])).astype(np.float32)
    mid = engine.register_model(g, P, dtype=L.DTYPE_BF16, name="wide200")
    names = [k["name"] for k in engine.kernels(mid)]
    assert any(n.startswith("conv_tcgen05_n") for n in names), names   # n128 (or n256: PAELLA_WIDE=256)
    img = r.standard_normal((1, 3, 200, 200)).astype(np.float32)
    out = engine.run_isolated(mid, img)
    vals = infer.forward(g, P, img, dtype="bf16", return_all=True)
    big = next(nd["id"] for nd in g.nodes if nd["name"] == "big")
    got = engine.debug_node(mid, big, (64, 200, 200))
    want = vals[big]
    ok = within(got, want, BF16_TOL)
    assert ok.all(), (int((~ok).sum()), float(np.abs(got - want).max()))
    assert within(out, vals[g.output].reshape(-1), BF16_TOL).all()
