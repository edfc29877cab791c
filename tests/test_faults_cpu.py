"""Failure handling of the dispatcher, driven by the FAKE device's fault injection
(paella_config_t.fake_fault, no GPU needed).

The notification stream is the dispatcher's only view of the GPU (P1100-1113: records
are consumed once, the slot reset to INVALID; flow control P1115-1119).  A device or
transport fault shows up as a record that is lost, duplicated, torn or invalid, or as
a launch that never completes.  Required behaviour (include/paella.h):

* a torn record (second half not landed) is re-read, never consumed -- every request
  still completes with status 0 and the issue order still replays exactly;
* a duplicated or invalid record makes the state machine inconsistent: the GPU's live
  jobs complete with -EIO, the process does NOT terminate (it used to: the policy's
  std::runtime_error escaped the dispatcher thread);
* a lost record or a hung kernel: the -ETIMEDOUT watchdog fails the live jobs;
* after a failure, new requests go to the remaining GPUs, or complete with -EIO
  when none is left; a blocking poll returns -EIO instead of spinning forever;
* the consumed-event log of a faulty run FAILS the exactly-once check (S5 b), so the
  checker is not vacuous.
"""
import errno
import time

import numpy as np
import pytest

from oracle import eventlog, sim
from workload import archs, rng

L = pytest.importorskip("paper_conf_sosp_ngd023_b200._lib")


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_sosp_ngd023_b200 import build
    build.build()
    L.load()


def _engine(**kw):
    kw.setdefault("device", L.DEVICE_FAKE)
    kw.setdefault("fake_sms", 4)
    return L.Engine(**kw)


def _run(e, mid, n, n_clients=1, stride=16384, timeout=30):
    """Submit n requests, then collect every completion; returns {req_id: status}."""
    info = e.model_info(mid)
    need = info["input_bytes"] + info["output_bytes"]
    sent = []
    for i in range(n):
        c = i % n_clients
        rid = e.submit(c, mid, (i // n_clients % 64) * stride, need)
        if rid < 0:
            sent.append((c, rid))
            continue
        sent.append((c, rid))
    got = {}
    want = sum(1 for _, r in sent if r >= 0)
    t0 = time.time()
    while len(got) < want:
        assert time.time() - t0 < timeout, f"only {len(got)}/{want} completions"
        for c in range(n_clients):
            rid, st = e.poll(c)
            if rid >= 0:
                got[rid] = st
    return sent, got


def test_torn_records_are_reread_not_consumed(tmp_path):
    log = str(tmp_path / "ev_%u.log")
    g = archs.toy()
    with _engine(num_clients=2, event_log=log, fake_fault=L.FAULT_TORN, group=4) as e:
        mid = e.register_model(g, rng.model_params(g))
        sent, got = _run(e, mid, 40, n_clients=2)
        st = e.stats()
    assert all(s == 0 for s in got.values()) and len(got) == 40
    assert st["torn_retries"] > 0          # the reader saw torn slots and waited
    cfg, ms, events, ex = eventlog.read(log % 0)
    ok, msg, _ = sim.replay(cfg, ms, events)
    assert ok, msg
    grids = {uid: ms[model][layer].grid for (uid, job, layer, stream, model) in ex["issues"]}
    assert sim.check_exactly_once(ex["records"], grids, cfg.group) == []


@pytest.mark.parametrize("fault", [L.FAULT_DUP, L.FAULT_CORRUPT])
def test_inconsistent_record_fails_jobs_with_eio(tmp_path, fault):
    """A duplicated record (count beyond the grid / unknown launch) or an invalid record
    type fails the GPU's live jobs with -EIO; the process survives; afterwards submit
    returns -EIO (single GPU) and a blocking poll returns -EIO."""
    log = str(tmp_path / "ev_%u.log")
    g = archs.toy()
    with _engine(num_clients=1, event_log=log, fake_fault=fault, fake_fault_arg=7) as e:
        mid = e.register_model(g, rng.model_params(g))
        info = e.model_info(mid)
        need = info["input_bytes"] + info["output_bytes"]
        rids = [e.submit(0, mid, i * 16384, need) for i in range(6)]
        assert all(r >= 0 for r in rids)
        got = {}
        t0 = time.time()
        while len(got) < 6:
            assert time.time() - t0 < 20
            rid, st = e.poll(0)
            if rid >= 0:
                got[rid] = st
        assert -errno.EIO in got.values()
        # the GPU is dead: new work is refused, a blocking poll does not hang
        deadline = time.time() + 5
        while True:
            r = e.submit(0, mid, 0, need)
            if r == -errno.EIO or time.time() > deadline:
                break
            rid, st = e.poll(0, 0)
            assert st == -errno.EIO
        assert r == -errno.EIO
        rid, _ = e.poll(0, 0)
        assert rid == -errno.EIO
    if fault == L.FAULT_DUP:
        # the consumed log holds the duplicate: the exactly-once check must flag it
        cfg, ms, events, ex = eventlog.read(log % 0)
        grids = {uid: ms[model][layer].grid for (uid, job, layer, stream, model) in ex["issues"]}
        bad = sim.check_exactly_once(ex["records"], grids, cfg.group)
        assert bad, "a duplicated record passed the exactly-once check"


@pytest.mark.parametrize("fault", [L.FAULT_DROP, L.FAULT_HANG])
def test_lost_record_or_hung_kernel_trips_watchdog(tmp_path, fault):
    log = str(tmp_path / "ev_%u.log")
    g = archs.toy()
    with _engine(num_clients=1, event_log=log, fake_fault=fault, fake_fault_arg=5, watchdog_ms=200) as e:
        mid = e.register_model(g, rng.model_params(g))
        sent, got = _run(e, mid, 8, timeout=20)
        assert -errno.ETIMEDOUT in got.values()
        assert all(s in (0, -errno.ETIMEDOUT) for s in got.values())
    cfg, ms, events, ex = eventlog.read(log % 0)
    grids = {uid: ms[model][layer].grid for (uid, job, layer, stream, model) in ex["issues"]}
    if fault == L.FAULT_DROP:
        assert sim.check_exactly_once(ex["records"], grids, cfg.group), "a lost record passed the check"


def test_router_avoids_failed_gpu(tmp_path):
    """Fault on GPU 0 of a 3-GPU instance: its jobs fail, every later request is routed
    to GPUs 1-2 and completes with status 0."""
    g = archs.toy()
    with _engine(num_clients=1, num_gpus=3, fake_fault=L.FAULT_CORRUPT, fake_fault_arg=3,
                 route=L.ROUTE_ROUND_ROBIN) as e:
        mid = e.register_model(g, rng.model_params(g))
        sent, got = _run(e, mid, 12)
        time.sleep(0.05)
        sent2, got2 = _run(e, mid, 60)
        assert all(r >= 0 for _, r in sent2)
        assert all(s == 0 for s in got2.values()), got2
        per = [e.stats(i)["completed"] for i in range(3)]
    assert -errno.EIO in got.values()
    assert per[1] > 0 and per[2] > 0


def test_completion_overflow_does_not_block_other_clients():
    """Client 0 submits more requests than its completion ring holds and does not poll;
    client 1 must still be served (the dispatcher used to spin in push_completion),
    and client 0 later receives every completion, in completion order."""
    g = archs.toy()
    with _engine(num_clients=2, submit_slots=4) as e:
        mid = e.register_model(g, rng.model_params(g))
        info = e.model_info(mid)
        need = info["input_bytes"] + info["output_bytes"]
        r0 = [e.submit(0, mid, i * 16384, need) for i in range(24)]
        assert all(r >= 0 for r in r0)
        time.sleep(0.2)
        r1 = [e.submit(1, mid, i * 16384, need) for i in range(3)]
        got1 = []
        t0 = time.time()
        while len(got1) < 3:
            assert time.time() - t0 < 10, "client 1 starved behind client 0's full completion ring"
            rid, st = e.poll(1)
            if rid >= 0:
                got1.append(rid)
        assert sorted(got1) == sorted(r1)
        got0 = []
        t0 = time.time()
        while len(got0) < 24:
            assert time.time() - t0 < 10
            rid, st = e.poll(0)
            if rid >= 0:
                assert st == 0
                got0.append(rid)
        assert sorted(got0) == sorted(r0)


def test_register_while_serving_replays(tmp_path):
    """Models registered while requests are in flight are added by the dispatcher thread
    itself (ADVICE: the policy's class table used to be written from the registering
    thread); the MODEL events land in order in the log and the run replays exactly."""
    log = str(tmp_path / "ev_%u.log")
    with _engine(num_clients=2, event_log=log, prio_classes=2, streams=8, slack=8) as e:
        m0 = e.register_model(archs.toy(), rng.model_params(archs.toy()))
        info = e.model_info(m0)
        need = info["input_bytes"] + info["output_bytes"]
        rids = [e.submit(i % 2, m0, (i // 2) * 16384, need) for i in range(20)]
        g2 = archs.squeezenet1_1()
        m1 = e.register_model(g2, rng.model_params(g2))
        i1 = e.model_info(m1)
        need1 = i1["input_bytes"] + i1["output_bytes"]
        stride = (max(need, need1) + 4095) // 4096 * 4096
        rids += [e.submit(0, m1, (32 + i) * stride, need1) for i in range(6)]
        done = 0
        t0 = time.time()
        while done < len(rids):
            assert time.time() - t0 < 20
            for c in (0, 1):
                rid, st = e.poll(c)
                if rid >= 0:
                    assert st == 0
                    done += 1
    cfg, ms, events, ex = eventlog.read(log % 0)
    ok, msg, n = sim.replay(cfg, ms, events)
    assert ok, msg
    assert len(ms) == 2


def test_init_rejects_oversized_job_table():
    with pytest.raises(OSError):
        _engine(num_clients=1, max_jobs_per_model=5000)
