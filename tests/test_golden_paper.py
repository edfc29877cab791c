"""Pins against values the paper prints (tests/golden/paper_values.json, each with
its passage)."""
import json
import os

from oracle import sim
from oracle.sim import Config, GPUModel, Layer

G = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_values.json")))


def test_fig2_hol_bound_from_printed_setup():
    f = G["fig2_hol"]
    warps = f["block_threads"] // 32
    per_sm = (32, f["threads_per_sm"] // 32, 65536, 100 * 1024, 512)
    # potential concurrency printed as 176 = 22 SMs x (1024 / 128) blocks
    assert f["sms"] * (f["threads_per_sm"] // f["block_threads"]) == f["potential_concurrency"]
    regs = -(-f["regs_per_thread"] * 32 // 256) * 256 * warps
    layer = Layer(1, (1, warps, regs, f["smem"], 0), 300_000, 300_000)
    models = [[layer] * f["kernels_per_job"]]
    trace = [(0, 0, 0)] * 300
    naive = sim.simulate(Config(num_clients=1), models, trace,
                         GPUModel(sms=f["sms"], per_sm=per_sm, hw_queues=f["hw_queues"]),
                         system="naive", naive_streams=300, horizon=2_000_000)
    assert naive.max_running_blocks == f["naive_running"]
    assert round(naive.max_running_blocks / f["potential_concurrency"], 2) == f["naive_utilisation"]
    cap = tuple(f["sms"] * x for x in per_sm)
    paella = sim.simulate(Config(num_clients=1, slack=0, capacity=cap, streams=176), models, trace,
                          GPUModel(sms=f["sms"], per_sm=per_sm, hw_queues=176), horizon=2_000_000)
    assert paella.max_running_blocks == f["potential_concurrency"]


def test_fig1_setup_optimum():
    f = G["fig1_setup"]
    models = [[Layer(1, (1, 1, 1, 1, 0), 1000, 1000)] * f["kernels_per_task"]] * f["tasks"]
    cfg = Config(num_clients=1, theta=sim.INF_THETA, slack=0, capacity=(f["sms"], 10**9, 10**12, 10**12, 10**9))
    res = sim.simulate(cfg, models, [(0, 0, i) for i in range(f["tasks"])],
                       GPUModel(sms=f["sms"], per_sm=(1, 64, 65536, 233472, 512)))
    # two tasks finish at 3 kernel-times, two at 6: mean 4.5 (the optimum, by exhaustion)
    assert sum(res.jct().values()) / f["tasks"] == 4.5 * 1000


def test_deficit_deltas_printed_rule():
    N = 4
    pol = sim.Policy(Config(num_clients=N, theta=10**6, slack=10, streams=8, capacity=(10**9,) * 5),
                     [[Layer(1, (1, 1, 1, 1, 0), 5, 1)] * 3])
    for c in range(N):
        pol.arrival(c, c, 0)
    before = [pol.D(c) for c in range(N)]
    saved = set(pol.free)
    pol.free = {0}
    (uid, job, layer, stream), = pol.decide()
    after = [pol.D(c) for c in range(N)]
    chosen = pol.jobs[job].client
    for c in range(N):
        assert after[c] - before[c] == (-(N - 1) if c == chosen else 1)


def test_group_and_entry_fields():
    assert G["fig6_group"]["group"] == sim.Config(num_clients=1).group
    e = G["notification_entry"]
    assert e["type_bits"] + e["smid_bits"] + e["kernel_id_bits"] == 48   # 16 bits unspecified (C2-Q5)
