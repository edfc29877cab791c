"""Out-of-process clients (P1030-1033: "each client obtains a shared memory region when
setting up the connection"): a second Python process attaches to the engine's channel
mapping by path (paella_client_attach) and drives predict / readResult through it,
zero-copy, while the engine (FAKE device) runs in this process.  Also: the client id is
exclusive, a bad path / id is refused, and the in-process client on another id keeps
working concurrently."""
import errno
import os
import subprocess
import sys
import textwrap
import time

import pytest

from workload import archs, rng

L = pytest.importorskip("paper_conf_sosp_ngd023_b200._lib")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = textwrap.dedent("""
    import sys, time
    import numpy as np
    sys.path.insert(0, sys.argv[1])
    from paper_conf_sosp_ngd023_b200 import _lib as L
    c = L.Client(sys.argv[2], int(sys.argv[3]))
    mid, n = int(sys.argv[4]), int(sys.argv[5])
    ib, ob = c.model_io(mid)
    stride = (ib + ob + 255) // 256 * 256
    x = np.arange(ib // 4, dtype=np.float32)
    sent, done = set(), 0
    for i in range(n):
        c.region[i * stride:i * stride + ib] = np.frombuffer(x.tobytes(), np.uint8)
        rid = c.submit(mid, i * stride, ib + ob)
        assert rid >= 0 and rid >> 48 == int(sys.argv[3]), rid
        sent.add(rid)
    t0 = time.time()
    while done < n:
        assert time.time() - t0 < 30, "child: completions missing"
        rid, st = c.poll()
        if rid >= 0:
            assert st == 0 and rid in sent
            sent.discard(rid)
            done += 1
    # a second attach of the same id from this process is refused
    try:
        L.Client(sys.argv[2], int(sys.argv[3]))
        raise SystemExit("double attach accepted")
    except OSError as e:
        assert e.errno == 16, e   # EBUSY
    c.close()
    print("child ok", n)
""")


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_sosp_ngd023_b200 import build
    build.build()
    L.load()


def test_client_in_another_process():
    g = archs.toy()
    with L.Engine(device=L.DEVICE_FAKE, fake_sms=4, num_clients=2) as e:
        mid = e.register_model(g, rng.model_params(g))
        path = e.channel_path()
        assert path.startswith("/proc/")
        child = subprocess.Popen([sys.executable, "-c", CHILD, ROOT, path, "1", str(mid), "60"],
                                 stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True)
        # meanwhile the in-process client 0 is served too
        info = e.model_info(mid)
        need = info["input_bytes"] + info["output_bytes"]
        rids = {e.submit(0, mid, i * 16384, need) for i in range(20)}
        got = 0
        t0 = time.time()
        while got < 20:
            assert time.time() - t0 < 30
            rid, st = e.poll(0)
            if rid >= 0:
                assert st == 0 and rid in rids
                got += 1
        out, err = child.communicate(timeout=60)
        assert child.returncode == 0, err[-2000:]
        assert "child ok 60" in out
        assert e.stats()["completed"] == 80


def test_attach_rejects_bad_arguments(tmp_path):
    g = archs.toy()
    with L.Engine(device=L.DEVICE_FAKE, fake_sms=4, num_clients=1) as e:
        e.register_model(g, rng.model_params(g))
        path = e.channel_path()
        with pytest.raises(OSError) as ei:
            L.Client(path, 5)                        # no such client id
        assert ei.value.errno == errno.EINVAL
        bogus = tmp_path / "x"
        bogus.write_bytes(b"\0" * 8192)
        with pytest.raises(OSError):
            L.Client(str(bogus), 0)                  # not a channel mapping
        c = L.Client(path, 0)
        with pytest.raises(OSError) as ei:
            L.Client(path, 0)
        assert ei.value.errno == errno.EBUSY
        c.close()
        L.Client(path, 0).close()                    # released by close()
