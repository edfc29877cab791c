"""The multi-rank path of bench.py on CPU: world_size 2 over gloo (torchrun, 127.0.0.1),
fake device backend.  Checks the contract keys, weak scaling, and that only rank 0
prints.  (The GPU numbers come from the real run; this covers the plumbing.)"""
import json
import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.timeout(600)
def test_bench_two_ranks_gloo_fake_device():
    from paper_conf_sosp_ngd023_b200 import build
    build.build()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), "bench.py", "--gpus", "2",
           "--fake", "--steps", "1", "--warmup", "1", "--reqs", "150", "--no-baselines", "--config", "c1_toy"]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=580)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "e2e", "gpu_launches", "clocks"):
        assert k in d, k
    assert d["n_gpus"] == 2 and d["scaling"] == "weak" and d["value"] > 0
    assert d["jct_mean_us"] > 0 and d["jct_p99_us"] >= d["jct_mean_us"] * 0.5
    assert "least-work router" in d["config"]["parallelism"] and len(d["dispatcher_busy_frac"]) == 2
    assert len(json.dumps(d)) < 2500, "the driver keeps only the tail of stdout"
    detail = json.load(open(os.path.join(ROOT, "gpurun_out", "bench_detail_c1_toy_n2.json")))
    assert detail["arms"]["paella"]["completed"] == 300   # --reqs 150 per GPU x 2 GPUs, one process
