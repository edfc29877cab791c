#!/usr/bin/env python
"""Benchmark of the Paella hot path on B200 (driver contract: one JSON line).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl paella|reference]
                    [--config c2_mix|c3_dispersion|c1_toy] [--rho 0.7]

Workload (N=1): BASELINE.json configs[1] -- single GPU, mixed ResNet-18 / MobileNetV2 /
SqueezeNet batch-1 jobs, Poisson arrivals (uniform mix, 3 clients, one per model,
bf16, random-init LSUV weights of workload/rng.py, synthetic N(0,1) images).

A *step* is one open-loop trace segment of `--reqs` requests replayed through the
public C ABI (paella_submit_at / paella_poll_completion, via paella_loadgen) at
rate lambda = rho * X_sat(naive), where X_sat(naive) -- the saturation throughput
of the naive one-stream-per-job baseline (CUDA-MS) -- is measured in an untimed
calibration phase.  value = requests completed per second over the K timed steps
(whole job, all ranks).  JCT = completion seen by the client - scheduled arrival.
Alongside: the same trace through the naive baseline and through Paella-FIFO, the
device-only roofline (summed isolated kernel time per model), the dominant kernel's
roofline (tcgen05 conv, CUDA events in the dispatcher), clocks, and the oracle CPU
baseline.  Multi-GPU (torchrun): one process per GPU, each with its own dispatcher
and trace at the same per-GPU rate (weak scaling, no collective on the data path).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from workload import archs, rng, traces  # noqa: E402

PEAKS_PATH = os.path.join(ROOT, "MEASURED_PEAKS.json")
METRIC = "requests/s at rho*X_sat(naive) with mean/p50/p99 JCT (open-loop, batch-1 mix)"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="paella", choices=["paella", "reference"])
    ap.add_argument("--config", default="c2_mix")
    ap.add_argument("--rho", type=float, default=0.7)
    ap.add_argument("--reqs", type=int, default=2000, help="requests per step")
    ap.add_argument("--no-baselines", action="store_true")
    ap.add_argument("--lookahead", type=int, default=3, help="NEXT-1 launch-ahead depth of the Paella arm")
    ap.add_argument("--slack", type=int, default=1184,
                    help="B, blocks issued beyond full utilisation (P1300-1304); 8 x 148 SMs covers the "
                         "measured dispatch loop delay (DESIGN.md B200-Q1)")
    ap.add_argument("--policy", default="srpt", choices=["srpt", "fifo", "sjf", "rr"],
                    help="policy of the Paella arm (sjf/rr: Table 3 ablations, NEXT-2)")
    ap.add_argument("--online-tbar", action="store_true", help="NEXT-4 online T-bar refinement in the Paella arm")
    ap.add_argument("--decide-delay-ns", type=int, default=0,
                    help="injected scheduler delay before every decide pass (Fig. 9 sensitivity)")
    ap.add_argument("--theta", type=int, default=100, help="fairness threshold (kernel dispatches, P1296-1297)")
    ap.add_argument("--prio-classes", type=int, default=1, help="stream-priority classes (DESIGN.md B200-Q2)")
    ap.add_argument("--dispatcher-cpu", type=int, default=-2,
                    help="pin each rank's dispatcher to core (this + LOCAL_RANK), exclusive; -1 = unpinned; "
                         "default: 2 when the host has >= 2 + 2N cores")
    ap.add_argument("--dispatcher-fifo", type=int, default=0,
                    help="SCHED_FIFO priority of the pinned dispatcher (0 = SCHED_OTHER)")
    ap.add_argument("--launch-threads", type=int, default=4, help="launcher helper threads per GPU")
    ap.add_argument("--sat-reqs", type=int, default=1500, help="requests of the saturation calibration")
    ap.add_argument("--slo-rhos", default="0.5,0.7,0.9,1.0,1.1,1.2,1.35,1.5",
                    help="offered loads (x X_sat(naive)) of the req/s-at-p99-SLO ladder ('' = skip)")
    ap.add_argument("--slo-reqs", type=int, default=1500, help="requests per point of the SLO ladder")
    ap.add_argument("--fake", action="store_true",
                    help="CPU fake device (tests of the multi-rank plumbing; not a measurement)")
    return ap.parse_args()


# ---------------------------------------------------------------------------
# distributed plumbing (barrier + max over ranks; no data-path collective)
# ---------------------------------------------------------------------------
class Dist:
    def __init__(self, n):
        self.world = int(os.environ.get("WORLD_SIZE", "1"))
        self.rank = int(os.environ.get("RANK", "0"))
        self.local = int(os.environ.get("LOCAL_RANK", "0"))
        self.pg = None
        if self.world > 1:
            import torch.distributed as dist
            os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
            dist.init_process_group("gloo", rank=self.rank, world_size=self.world)
            self.pg = dist

    def barrier(self):
        if self.pg:
            self.pg.barrier()

    def allmax(self, x):
        if not self.pg:
            return x
        import torch
        t = torch.tensor([float(x)], dtype=torch.float64)
        self.pg.all_reduce(t, op=self.pg.ReduceOp.MAX)
        return t.item()

    def allsum(self, x):
        if not self.pg:
            return x
        import torch
        t = torch.tensor([float(x)], dtype=torch.float64)
        self.pg.all_reduce(t, op=self.pg.ReduceOp.SUM)
        return t.item()

    def gather_list(self, arr):
        if not self.pg:
            return [arr]
        out = [None] * self.world
        self.pg.all_gather_object(out, arr)
        return out


# ---------------------------------------------------------------------------
# clocks during the timed region
# ---------------------------------------------------------------------------
class Clocks:
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu):
        self.gpu = gpu
        self.proc = None

    def start(self):
        if self.gpu < 0:
            return
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.proc = None

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        out, _ = self.proc.communicate(timeout=10)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


# ---------------------------------------------------------------------------
# the GPU arm
# ---------------------------------------------------------------------------
def build_engine(L, specs, gpu, fake=False, **kw):
    if fake:
        kw.pop("event_time_kind", None)
        e = L.Engine(num_clients=len(specs), device=L.DEVICE_FAKE, **kw)
    else:
        e = L.Engine(num_clients=len(specs), first_gpu=gpu, **kw)
    mids = [e.register_model(g, P) for (g, P) in specs]
    return e, mids


def stage_inputs(e, specs, mids, slots, stride, pool):
    """Pre-stage inputs: client c serves model c; slot s holds pool image s % pool."""
    for c, (g, _) in enumerate(specs):
        _, reg = e.region(c)
        for s in range(slots):
            x = pool[c][s % len(pool[c])]
            off = s * stride
            reg[off:off + x.nbytes] = np.frombuffer(x.tobytes(), np.uint8)


def jct_stats(jct_ns, models, names):
    ok = jct_ns >= 0
    out = {}
    j = jct_ns[ok] / 1e3
    out["mix"] = {"mean_us": float(j.mean()), "p50_us": float(np.percentile(j, 50)),
                  "p99_us": float(np.percentile(j, 99)), "n": int(ok.sum())}
    for m, nm in enumerate(names):
        sel = ok & (models == m)
        if sel.any():
            jm = jct_ns[sel] / 1e3
            out[nm] = {"mean_us": float(jm.mean()), "p50_us": float(np.percentile(jm, 50)),
                       "p99_us": float(np.percentile(jm, 99)), "n": int(sel.sum())}
    return out


def make_trace(n, rate, cfg, n_models, seed):
    kind = cfg["arrival"]
    t = traces.arrivals(n, rate, kind="poisson" if kind == "poisson" else "lognormal",
                        sigma=cfg.get("sigma", 2.0), seed=seed)
    w = cfg["weights"] or [1.0] * n_models
    models = traces.model_choices(n, w, seed=seed)
    inputs = traces.input_choices(n, seed=seed)
    return t, models, inputs


def saturation(e, mids, n_models, stride, slots, n, seed=99):
    """Closed burst: all requests due at t=0; completions / elapsed."""
    t = np.zeros(n, dtype=np.int64)
    models = np.arange(n) % n_models
    jct, el = e.loadgen(t, models, models, np.zeros(n), stride, slots)
    return n / (el / 1e9)


def slo_ladder(e, args, cfg, names, x_sat_naive, slo, stride, slots, seed):
    """req/s at p99 SLO: the largest offered lambda of the ladder
    rho * X_sat(naive) at which every model's p99 JCT is within its SLO (an
    overloaded point fails it: the backlog grows through the point's window)."""
    rhos = [float(r) for r in args.slo_rhos.split(",") if r.strip()]
    pts, best = [], 0.0
    for i, r in enumerate(rhos):
        lam = r * x_sat_naive
        t, mm, ii = make_trace(args.slo_reqs, lam, cfg, len(names), seed=seed + i)
        jct, el = e.loadgen(t, mm, mm, ii, stride, slots)
        st = jct_stats(jct, mm, names)
        ok = all(st.get(n, {}).get("p99_us", 1e18) <= slo[n] for n in names)
        served = (jct >= 0).sum() / (el / 1e9)
        pts.append({"rho": r, "offered_req_s": round(lam, 1), "served_req_s": round(float(served), 1),
                    "p99_us": {n: round(st[n]["p99_us"], 1) for n in names if n in st},
                    "mean_us": round(st["mix"]["mean_us"], 1), "slo_met": bool(ok)})
        if ok:
            best = max(best, lam)
    return {"req_s": round(best, 1), "ladder": pts}


def run_gpu(args, dist):
    from paper_conf_sosp_ngd023_b200 import _lib as L
    L.load()
    cfgname = args.config
    cfg = traces.CONFIGS[cfgname]
    names = cfg["models"]
    gpu = dist.local
    specs = []
    for nm in names:
        g = archs.build(nm)
        specs.append((g, rng.model_params(g)))
    pool = [[rng.image(g, i) for i in range(32)] for (g, _) in specs]
    slots = 256
    sizes = [int(np.prod(g.nodes[0]["out"])) * 4 + g.num_classes * 4 for (g, _) in specs]
    stride = (max(sizes) + 4095) // 4096 * 4096
    region = slots * stride + (1 << 20)

    def engine(**kw):
        kw.setdefault("launch_threads", 0 if args.fake else args.launch_threads)
        if args.dispatcher_cpu >= 0:
            kw.setdefault("dispatcher_cpus", [args.dispatcher_cpu + gpu])
        if not kw.get("naive"):
            kw.setdefault("policy", {"srpt": L.POLICY_SRPT_DEFICIT, "fifo": L.POLICY_FIFO, "sjf": L.POLICY_SJF,
                                     "rr": L.POLICY_RR}[args.policy])
            kw.setdefault("theta", args.theta)
            kw.setdefault("decide_delay_ns", args.decide_delay_ns)
            kw.setdefault("online_tbar", args.online_tbar)
            kw.setdefault("slack", args.slack)
            kw.setdefault("prio_classes", args.prio_classes)
        e, mids = build_engine(L, specs, gpu, fake=args.fake, region_bytes=region, max_jobs_per_model=128, **kw)
        stage_inputs(e, specs, mids, slots, stride, pool)
        return e, mids

    # --- calibration (untimed): naive saturation, unloaded JCT -> SLO ---------------
    t_cal = time.time()
    en, mids = engine(naive=True, instrument=False)
    x_sat_naive = saturation(en, mids, len(names), stride, slots, args.sat_reqs)
    t1, m1, i1 = make_trace(300, 200.0, cfg, len(names), seed=7)
    jct_unloaded, _ = en.loadgen(t1, m1, m1, i1, stride, slots)
    slo = {nm: 5.0 * float(np.median(jct_unloaded[m1 == m])) / 1e3 for m, nm in enumerate(names)}
    if cfg["weights"] is None:
        # Fig. 12 convention (P1482-1483): request mix inversely proportional to job size
        cfg = dict(cfg, weights=[1.0 / max(1e-9, float(np.median(jct_unloaded[m1 == m]))) for m in range(len(names))])
    en.shutdown()
    lam = args.rho * x_sat_naive

    # --- the Paella arm -------------------------------------------------------------
    e, mids = engine(instrument=True, lookahead=args.lookahead)
    x_sat_paella = saturation(e, mids, len(names), stride, slots, args.sat_reqs)
    jp, _ = e.loadgen(t1, m1, m1, i1, stride, slots)
    unloaded = {"naive": {nm: float(np.median(jct_unloaded[m1 == m])) / 1e3 for m, nm in enumerate(names)},
                "paella": {nm: float(np.median(jp[m1 == m])) / 1e3 for m, nm in enumerate(names)}}
    # device-only roofline: summed isolated kernel time per model (uninstrumented twin)
    dev_roof = {}
    kinfo = {}
    for m, nm in enumerate(names):
        ks = e.kernels(mids[m])
        if args.fake:
            kt = kti = np.array([k["tbar_ns"] for k in ks], dtype=np.int64)
        else:
            kt = e.time_kernels(mids[m], instrumented=False, reps=20)
            kti = e.time_kernels(mids[m], instrumented=True, reps=20)
        dev_roof[nm] = float(kt.sum()) / 1e3
        kinfo[nm] = (ks, kt, kti)
    calib_s = time.time() - t_cal

    seed0 = 1000 * (dist.rank + 1)
    for w in range(args.warmup):
        t, mm, ii = make_trace(args.reqs, lam, cfg, len(names), seed=seed0 + w)
        e.loadgen(t, mm, mm, ii, stride, slots)
    st0 = e.stats()
    clocks = Clocks(gpu if not args.fake else -1)
    dist.barrier()
    clocks.start()
    t_start = time.perf_counter_ns()
    all_jct, all_models = [], []
    for s in range(args.steps):
        t, mm, ii = make_trace(args.reqs, lam, cfg, len(names), seed=seed0 + 100 + s)
        jct, el = e.loadgen(t, mm, mm, ii, stride, slots)
        all_jct.append(jct)
        all_models.append(mm)
    elapsed = (time.perf_counter_ns() - t_start) / 1e9
    dist.barrier()
    clk = clocks.stop()
    st1 = e.stats()
    stats = {k: ([a - b for a, b in zip(st1[k], st0[k])] if isinstance(st1[k], list) else st1[k] - st0[k])
             for k in st1}
    # dominant kernel (tcgen05 conv): algorithmic bytes / CUDA-event duration of the
    # served (instrumented) kernels, launched back to back on their stream
    ev = {"launches": 0, "ns": 0, "bytes": 0, "flops": 0, "all_ns": 0}
    for nm, (ks, kt, kti) in kinfo.items():
        for k, t in zip(ks, kti):
            ev["all_ns"] += int(t)
            if k["name"].startswith("conv_tcgen05"):
                ev["launches"] += 1
                ev["ns"] += int(t)
                ev["bytes"] += k["bytes"]
                ev["flops"] += k["flops"]
    jct = np.concatenate(all_jct)
    models = np.concatenate(all_models)
    completed = int((jct >= 0).sum())

    # --- end-to-end: same trace, inputs copied in / logits read out per request -------
    copy_in = {m: pool[m] for m in range(len(names))}
    t, mm, ii = make_trace(args.reqs, lam, cfg, len(names), seed=seed0 + 500)
    e2e_jct, e2e_el = e.loadgen(t, mm, mm, ii, stride, slots, copy_inputs=copy_in)
    e2e_rate = (e2e_jct >= 0).sum() / (e2e_el / 1e9)
    slo_at = {}
    if args.slo_rhos and not args.no_baselines:
        slo_at["paella"] = slo_ladder(e, args, cfg, names, x_sat_naive, slo, stride, slots, seed0 + 700)
    h2d = float(np.mean([sizes[m] - specs[m][0].num_classes * 4 for m in mm]))
    d2h = float(np.mean([specs[m][0].num_classes * 4 for m in mm]))
    e.shutdown()

    # --- baselines on the same trace (naive CUDA-MS, Paella as in the paper, FIFO) -----
    base = {}
    if not args.no_baselines:
        for label, kw in (("naive_cuda_ms", dict(naive=True, instrument=False)),
                          ("paella_paper_lookahead0", dict(policy=L.POLICY_SRPT_DEFICIT, lookahead=0, slack=0, prio_classes=1,
                                                           pdl=False)),
                          ("paella_fifo", dict(policy=L.POLICY_FIFO, lookahead=args.lookahead))):
            eb, mb = engine(**kw)
            jl = []
            for s in range(min(args.steps, 3)):
                t, mm, ii = make_trace(args.reqs, lam, cfg, len(names), seed=seed0 + 100 + s)
                j, _ = eb.loadgen(t, mm, mm, ii, stride, slots)
                jl.append((j, mm))
            if label == "naive_cuda_ms" and args.slo_rhos:
                slo_at["naive"] = slo_ladder(eb, args, cfg, names, x_sat_naive, slo, stride, slots, seed0 + 700)
            eb.shutdown()
            base[label] = jct_stats(np.concatenate([a for a, _ in jl]), np.concatenate([b for _, b in jl]), names)

    return dict(unloaded=unloaded, names=names, lam=lam, x_sat_naive=x_sat_naive, x_sat_paella=x_sat_paella, slo=slo,
                elapsed=elapsed, completed=completed, jct=jct_stats(jct, models, names), clocks=clk,
                ev=ev, stats=stats, dev_roof=dev_roof, base=base, e2e_rate=e2e_rate,
                e2e=jct_stats(e2e_jct, mm, names), h2d=h2d, d2h=d2h, calib_s=calib_s, kinfo=kinfo,
                slo_at=slo_at, config=cfgname)


def cpu_baseline(cfg, seconds=12.0):
    """The oracle (float64 numpy inference, as it stands) serving a bounded sample of
    the same mix on the host cores: a process pool, one BLAS thread per worker."""
    import multiprocessing as mp
    cores = max(1, len(os.sched_getaffinity(0)) - 2)
    names = cfg["models"]
    ctx = mp.get_context("fork")
    t0 = time.time()
    with ctx.Pool(cores, initializer=_cpu_init) as pool:
        n_done = 0
        results = []
        i = 0
        while time.time() - t0 < seconds:
            batch = [(names[(i + k) % len(names)], (i + k) % 32) for k in range(cores)]
            i += cores
            results = pool.map(_cpu_one, batch)
            n_done += len(results)
        el = time.time() - t0
    return {"value": n_done / el, "unit": "req/s", "cores": cores, "kind": "oracle",
            "sample": f"{n_done} requests of the {'/'.join(names)} mix, float64 numpy oracle "
                      f"(oracle/infer.py), {cores} worker processes x 1 BLAS thread, {el:.1f} s"}


_CPU = {}


def _cpu_init():
    os.environ["OMP_NUM_THREADS"] = "1"
    try:
        from threadpoolctl import threadpool_limits
        threadpool_limits(1)
    except Exception:
        pass


def _cpu_one(arg):
    from oracle import infer   # bench.py's cpu_baseline leg: the one place besides tests
    name, idx = arg
    if name not in _CPU:
        g = archs.build(name)
        _CPU[name] = (g, rng.model_params(g))
    g, P = _CPU[name]
    infer.forward(g, P, rng.image(g, idx), dtype="bf16")
    return 1


def roofline_entry(res, peaks):
    """Dominant kernel = the tcgen05 implicit-GEMM conv.  achieved = algorithmic
    bytes (weights + input + output [+ residual]) summed over every conv launch of one
    request of each model / their summed CUDA-event durations (instrumented kernels as
    served, each launched back to back on its stream right after the timed region)."""
    ev = res["ev"]
    if not ev or ev["launches"] == 0 or ev["ns"] == 0:
        return None
    dur = ev["ns"] / ev["launches"]
    bytes_per = ev["bytes"] / ev["launches"]
    flops_per = ev["flops"] / ev["launches"]
    gbs = bytes_per / dur
    peak = peaks.get("hbm_gbs", 6650.0)
    # DRAM traffic per launch from the committed ncu --set full capture of the same
    # launches (tools/profile_round.sh -> tools/ncu_traffic.py), if present
    traffic, tsrc = None, None
    tp = os.path.join(ROOT, "profiles", f"conv_traffic_{res['config']}.json")
    if os.path.exists(tp):
        tj = json.load(open(tp))
        traffic, tsrc = tj.get("conv_tcgen05_dram_bytes_per_launch"), tj.get("source")
    return {"kernel": "conv_tcgen05", "bound": "hbm", "achieved": round(gbs, 2), "peak": peak, "unit": "GB/s",
            "frac": round(gbs / peak, 4), "traffic": traffic, "traffic_source": tsrc,
            "algorithmic_bytes_per_launch": round(bytes_per), "launches_per_mix": ev["launches"],
            "mean_launch_us": round(dur / 1e3, 3), "tflops": round(flops_per / dur / 1e3, 3),
            "share_of_device_time": round(ev["ns"] / max(1, ev["all_ns"]), 3),
            "peak_source": "MEASURED_PEAKS.json hbm_gbs (burst copy)"}


def saturating_conv(args):
    """The dominant kernel where its roofline is reachable: the tcgen05
    conv on 3x3 256->256 layers over 56x56 and 448x448 pixels (tools/conv_saturating.py),
    timed like the batch-1 kernels (PDL chain, CUDA events), against the measured bf16
    tensor peak."""
    import importlib.util
    spec = importlib.util.spec_from_file_location("conv_saturating", os.path.join(ROOT, "tools", "conv_saturating.py"))
    cs = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(cs)
    from paper_conf_sosp_ngd023_b200 import _lib as L
    peaks = json.load(open(PEAKS_PATH)) if os.path.exists(PEAKS_PATH) else {}
    peak = peaks.get("bf16_tflops", 2250.0)
    with L.Engine(num_clients=1, max_jobs_per_model=1, first_gpu=int(os.environ.get("LOCAL_RANK", "0"))) as e:
        rows = [cs.measure(e, hw) for hw in (56, 448)]
    best = max(rows, key=lambda r: r["tflops_instr"])
    return {"kernel": "conv_tcgen05", "bound": "tensor", "achieved": best["tflops_instr"], "peak": peak,
            "unit": "TFLOP/s", "frac": round(best["tflops_instr"] / peak, 4),
            "peak_source": "MEASURED_PEAKS.json bf16_tflops (cuBLAS burst)" if peaks else "nominal 2250",
            "shapes": rows}


def main():
    args = parse()
    if args.dispatcher_fifo > 0:
        os.environ["PAELLA_DISPATCHER_FIFO"] = str(args.dispatcher_fifo)
    if args.impl == "reference":   # no dispatcher: the oracle keeps every host core
        args.dispatcher_cpu = -1
    if args.dispatcher_cpu == -2:   # default: core 2 + LOCAL_RANK if the host has room
        avail = os.sched_getaffinity(0)
        first = 2
        args.dispatcher_cpu = first if (set(range(first, first + args.gpus)) <= avail
                                         and len(avail) >= first + 2 * args.gpus) else -1
    if args.dispatcher_cpu >= 0:
        # DEDICATED cores: every thread created from here on
        # (launchers, load generator, completion pollers) inherits a mask without any
        # rank's dispatcher core; measured on B200 in profiles/pin_r1c
        cores = set(range(args.dispatcher_cpu, args.dispatcher_cpu + args.gpus))
        os.sched_setaffinity(0, os.sched_getaffinity(0) - cores)
    dist = Dist(args.gpus)
    cfg = traces.CONFIGS[args.config]
    workload = {"c2_mix": "BASELINE configs[1]: 1 GPU, mixed ResNet-18/MobileNetV2/SqueezeNet1.1 batch-1, "
                          "Poisson arrivals",
                "c3_dispersion": "BASELINE configs[2]: ResNet-50/DenseNet-121/Inception-v3/MobileNetV2, bursty",
                "c1_toy": "BASELINE configs[0]: 2 clients, toy conv+MLP"}[args.config]
    if args.impl == "reference":
        if dist.rank != 0:
            return
        t0 = time.time()
        cb = None
        for _ in range(max(1, args.warmup)):
            pass
        vals = []
        for _ in range(args.steps):
            cb = cpu_baseline(cfg, seconds=max(2.0, 30.0 / max(1, args.steps)))
            vals.append(cb["value"])
        v = float(np.mean(vals))
        line = {"impl": "reference", "metric": METRIC, "value": round(v, 3),
                "unit": "req/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": round((time.time() - t0) * 1e3 / args.steps, 1), "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": workload, "models": cfg["models"], "clients": cfg["clients"], "batch": 1,
                           "arrivals": cfg["arrival"], "rho": args.rho, "requests_per_step": args.reqs,
                           "parallelism": "oracle on host cores"},
                "cpu_baseline": {**cb, "value": round(v, 3)},
                "e2e": {"value": round(v, 3), "unit": "req/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line))
        return
    res = run_gpu(args, dist)
    total_done = dist.allsum(res["completed"])
    max_el = dist.allmax(res["elapsed"])
    value = total_done / max_el
    peaks = {}
    if os.path.exists(PEAKS_PATH):
        peaks = json.load(open(PEAKS_PATH))
    if dist.rank != 0:
        return
    jm = res["jct"]["mix"]
    launches = res["stats"]["launches"]
    line = {
        "metric": METRIC,
        "value": round(value, 2), "unit": "req/s", "n_gpus": args.gpus, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(max_el * 1e3 / args.steps, 2), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
        "config": {"workload": workload, "models": res["names"], "clients": cfg["clients"], "batch": 1,
                   "arrivals": cfg["arrival"], "rho": args.rho, "lambda_per_gpu_req_s": round(res["lam"], 1),
                   "requests_per_step": args.reqs, "parallelism": f"replicas{args.gpus}",
                   "l2": "not flushed: steps are open-loop traces whose weights (~33 MB bf16) stay L2-resident "
                         "as in serving; inputs stream from pinned host memory"},
        "jct_us": res["jct"], "slo_us": res["slo"],
        "paella_config": {"lookahead": args.lookahead, "launch_threads": args.launch_threads,
                          "dispatcher_cpu": args.dispatcher_cpu, "dispatcher_fifo": args.dispatcher_fifo, "policy": {"srpt": "srpt+deficit"}.get(args.policy, args.policy),
                          "slack_blocks": args.slack, "prio_classes": args.prio_classes, "pdl": True,
                          "theta": args.theta, "group": 16, "streams": 32, "decide_delay_ns": args.decide_delay_ns,
                          "online_tbar": bool(args.online_tbar)},
        "slo_met": bool(all(res["jct"].get(n, {}).get("p99_us", 1e18) <= res["slo"][n] for n in res["names"])),
        "req_s_at_p99_slo": {k: v["req_s"] for k, v in res["slo_at"].items()},
        "slo_ladder": res["slo_at"],
        "x_sat_req_s": {"naive": round(res["x_sat_naive"], 1), "paella": round(res["x_sat_paella"], 1)},
        "jct_unloaded_p50_us": {k: {m: round(v, 1) for m, v in d.items()} for k, d in res["unloaded"].items()},
        "device_roofline_us": {k: round(v, 2) for k, v in res["dev_roof"].items()},
        "jct_fraction_of_device_roofline": {n: round(res["dev_roof"][n] / res["jct"][n]["mean_us"], 4)
                                            for n in res["names"] if n in res["jct"]},
        "baselines": res["base"],
        "roofline": roofline_entry(res, peaks),
        "cpu_baseline": None,
        "e2e": {"value": round(res["e2e_rate"], 2), "unit": "req/s", "h2d_bytes_per_step": round(res["h2d"] * args.reqs),
                "d2h_bytes_per_step": round(res["d2h"] * args.reqs), "jct_us": res["e2e"]["mix"]},
        "gpu_launches": int(launches),
        "clocks": res["clocks"],
        "dispatcher": {k: (v if isinstance(v, list) else int(v)) for k, v in res["stats"].items()},
    }
    if args.gpus == 1 and not args.fake:
        try:
            line["roofline_saturating"] = saturating_conv(args)
        except Exception as ex:   # diagnostic only: never fail the bench line for it
            line["roofline_saturating"] = {"error": str(ex)[:200]}
        line["cpu_baseline"] = cpu_baseline(cfg, seconds=12.0)
    if args.fake:
        line["data"] = "synthetic, FAKE CPU device (plumbing test, not a measurement)"
    print(json.dumps(line))


if __name__ == "__main__":
    main()
