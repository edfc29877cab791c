"""Timeline of served jobs from a dispatcher event log (diagnosis tool, no oracle).

Serves a light trace of one config with per-block notification records (ring mode,
G = 1, records carry %globaltimer) and host-time events (PAELLA_TRACE_TIMES), then
reconstructs every launch's first-block start / last-block end on the device clock, the
host decision time of every launch (converted with the logged CLOCK calibration), and
per job the gap between consecutive kernels.  A gap is "host-late" when the successor
was decided only after its predecessor had ended (the dispatcher's notification loop
is the bubble), else "device" (launch path / PDL / placement).

Writes a Chrome trace (chrome://tracing, Perfetto: one process per job, one thread per
stream) and prints a JSON summary.

    python tools/timeline.py c3_dispersion 300 60 gpurun_out/tl '{"lookahead": 6, "slack": 2368, "max_active": 8}'
"""
import json
import os
import sys

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
os.environ["PAELLA_TRACE_TIMES"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

DT = np.dtype([("type", "<u4"), ("a", "<u4"), ("b", "<u8"), ("c", "<u8"), ("d", "<u8")])
EV_ARRIVAL, EV_RECORD, EV_ISSUE, EV_COMPLETE, EV_CLOCK, EV_TIME, EV_LAYER = 1, 2, 4, 5, 8, 9, 111


def parse(path):
    raw = np.fromfile(path, dtype=DT)
    offset = None
    launches = {}       # uid -> dict(job, layer, stream, t_issue_host, start, end)
    jobs = {}           # job life index -> dict(model, t_sched, uids, t_complete)
    cur = {}            # job id -> life index
    for r in raw:
        t, a, b, c, d = int(r["type"]), int(r["a"]), int(r["b"]), int(r["c"]), int(r["d"])
        if t == EV_CLOCK:   # the latest calibration before the traced jobs is used
            if not jobs:
                offset = b if b < (1 << 63) else b - (1 << 64)
        elif t == EV_ARRIVAL:
            cur[b] = len(jobs)
            jobs[len(jobs)] = dict(job=b, client=a, model=c, t_sched=d, uids=[], t_complete=None)
        elif t == EV_ISSUE:
            life = cur[c]
            launches[b] = dict(life=life, layer=d, stream=a, t_issue=None, start=None, end=None)
            jobs[life]["uids"].append(b)
        elif t == EV_TIME and a == 0:
            launches[b]["t_issue"] = c
        elif t == EV_TIME and a in (2, 3) and b in launches:   # counter mode: counts seen by the host
            L = launches[b]
            key = "seen_place" if a == 2 else "seen_done"
            if a == 2 and L.get("seen_place") is None:
                L["seen_place"] = c
            if a == 3:
                L["seen_done"] = c      # the last one is the final count
        elif t == EV_RECORD:
            L = launches.get(b)
            if L is None:
                continue
            g40 = d & ((1 << 40) - 1)
            if a == 1:
                L["start"] = g40 if L["start"] is None else min(L["start"], g40)
            elif a == 2:
                L["end"] = g40 if L["end"] is None else max(L["end"], g40)
        elif t == EV_COMPLETE:
            if b in cur:
                jobs[cur[b]]["t_complete"] = c
    if offset is None:   # fake device: no calibration, records carry virtual time
        offset = 0

    def full(g40, ref):   # unwrap a 40-bit globaltimer value near the reference (full ns)
        base = ref - (ref & ((1 << 40) - 1))
        cands = [base + g40 - (1 << 40), base + g40, base + g40 + (1 << 40)]
        return min(cands, key=lambda x: abs(x - ref))

    for L in launches.values():
        if L["t_issue"] is None:
            continue
        ref = L["t_issue"] + offset       # host -> device clock
        L["issue_dev"] = ref
        if L["start"] is not None:
            L["start"] = full(L["start"], ref)
        if L["end"] is not None:
            L["end"] = full(L["end"], ref)
    return jobs, launches, offset


def summarize(jobs, launches, names):
    gaps, late, dev_gaps, late_gaps, issue_lead = [], 0, [], [], []
    per_model = {}
    for jb in jobs.values():
        ks = [launches[u] for u in jb["uids"]]
        if any(k["start"] is None or k["end"] is None or k.get("issue_dev") is None for k in ks):
            continue
        ks.sort(key=lambda k: k["layer"])
        busy = sum(k["end"] - k["start"] for k in ks)
        span = ks[-1]["end"] - ks[0]["start"]
        pm = per_model.setdefault(names[jb["model"]], dict(n=0, busy=0.0, span=0.0, gap=0.0, late_gap=0.0))
        pm["n"] += 1
        pm["busy"] += busy
        pm["span"] += span
        for p, q in zip(ks, ks[1:]):
            g = q["start"] - p["end"]
            gaps.append(g)
            pm["gap"] += max(g, 0)
            issue_lead.append(p["end"] - q["issue_dev"])   # > 0: decided before the predecessor ended
            if q["issue_dev"] > p["end"]:
                late += 1
                late_gaps.append(g)
                pm["late_gap"] += max(g, 0)
            else:
                dev_gaps.append(g)
    pct = lambda v, p: round(float(np.percentile(v, p)) / 1e3, 3) if len(v) else None   # noqa: E731
    out = dict(kernel_pairs=len(gaps), host_late_pairs=late,
               gap_us=dict(p50=pct(gaps, 50), p90=pct(gaps, 90), mean=round(float(np.mean(gaps)) / 1e3, 3)),
               device_gap_us=dict(p50=pct(dev_gaps, 50), p90=pct(dev_gaps, 90)),
               host_late_gap_us=dict(p50=pct(late_gaps, 50), p90=pct(late_gaps, 90)),
               issue_lead_us=dict(p10=pct(issue_lead, 10), p50=pct(issue_lead, 50)),
               per_model={m: dict(jobs=v["n"], busy_us=round(v["busy"] / v["n"] / 1e3, 1),
                                  span_us=round(v["span"] / v["n"] / 1e3, 1),
                                  gaps_us=round(v["gap"] / v["n"] / 1e3, 1),
                                  host_late_gaps_us=round(v["late_gap"] / v["n"] / 1e3, 1))
                          for m, v in per_model.items()})
    return out


def summarize_seen(jobs, launches, names):
    """Counter mode (no device timestamps): host-observed times.  Per job: arrival ->
    first issue, and the completion-to-completion intervals of consecutive kernels as
    the host saw them (the notification latency cancels out in the differences), plus
    how far ahead each kernel was decided relative to its predecessor's completion seen."""
    per_model = {}
    lead = []
    for jb in jobs.values():
        ks = sorted((launches[u] for u in jb["uids"]), key=lambda k: k["layer"])
        if not ks or any(k.get("seen_done") is None or k.get("t_issue") is None for k in ks):
            continue
        pm = per_model.setdefault(names[jb["model"]], dict(n=0, admit=0.0, first_done=0.0, chain=0.0, tail=0.0,
                                                            late=0))
        pm["n"] += 1
        pm["admit"] += ks[0]["t_issue"] - jb["t_sched"]
        pm["first_done"] += ks[0]["seen_done"] - ks[0]["t_issue"]
        pm["chain"] += ks[-1]["seen_done"] - ks[0]["seen_done"]
        if jb["t_complete"] is not None:
            pm["tail"] += jb["t_complete"] - ks[-1]["seen_done"]
        for p, q in zip(ks, ks[1:]):
            lead.append(p["seen_done"] - q["t_issue"])
            if q["t_issue"] > p["seen_done"]:
                pm["late"] += 1
    pct = lambda v, p: round(float(np.percentile(v, p)) / 1e3, 2) if len(v) else None   # noqa: E731
    return dict(issue_lead_vs_pred_done_seen_us=dict(p10=pct(lead, 10), p50=pct(lead, 50)),
                per_model={m: dict(jobs=v["n"], admit_to_first_issue_us=round(v["admit"] / v["n"] / 1e3, 1),
                                   first_issue_to_first_done_seen_us=round(v["first_done"] / v["n"] / 1e3, 1),
                                   chain_done_seen_us=round(v["chain"] / v["n"] / 1e3, 1),
                                   last_done_seen_to_complete_us=round(v["tail"] / v["n"] / 1e3, 1),
                                   late_issues_per_job=round(v["late"] / v["n"], 2))
                           for m, v in per_model.items()})


def chrome(jobs, launches, names, path):
    ev = []
    t0 = min(L["start"] for L in launches.values() if L["start"] is not None)
    for life, jb in jobs.items():
        ev.append(dict(name="process_name", ph="M", pid=life, args=dict(name=f"job {life} {names[jb['model']]}")))
        for u in jb["uids"]:
            L = launches[u]
            if L["start"] is None or L["end"] is None:
                continue
            ev.append(dict(name=f"L{L['layer']}", ph="X", pid=life, tid=L["stream"], ts=(L["start"] - t0) / 1e3,
                           dur=max(L["end"] - L["start"], 1) / 1e3, args=dict(uid=u)))
            if L.get("issue_dev") is not None:
                ev.append(dict(name=f"issue L{L['layer']}", ph="i", s="t", pid=life, tid=L["stream"],
                               ts=(L["issue_dev"] - t0) / 1e3))
    with open(path, "w") as f:
        json.dump(dict(traceEvents=ev, displayTimeUnit="ns"), f)


def main():
    from paper_conf_sosp_ngd023_b200 import _lib as L
    from workload import archs, rng, traces
    import bench
    cfgname = sys.argv[1] if len(sys.argv) > 1 else "c3_dispersion"
    lam = float(sys.argv[2]) if len(sys.argv) > 2 else 300.0
    nreq = int(sys.argv[3]) if len(sys.argv) > 3 else 60
    out = sys.argv[4] if len(sys.argv) > 4 else "gpurun_out/timeline"
    variant = json.loads(sys.argv[5]) if len(sys.argv) > 5 else {}
    cfg = dict(traces.CONFIGS[cfgname])
    names = cfg["models"]
    if cfg["weights"] is None:
        est = {"resnet50": 640, "densenet121": 1840, "inception_v3": 1190, "mobilenet_v2": 450}
        cfg = dict(cfg, weights=[1.0 / est.get(n, 500) for n in names])
    specs = [(g, rng.model_params(g)) for g in (archs.build(n) for n in names)]
    slots, stride = 64, 1 << 21
    log = out + ".evlog"
    kw = dict(launch_threads=8, dispatcher_cpus=[2], notify="counters", group=16, slack=3552, lookahead=6,
              max_active=8, lookahead_unplaced=True)
    kw.update(variant)
    e = L.Engine(num_clients=len(specs), region_bytes=slots * stride + (1 << 20), max_jobs_per_model=64,
                 event_log=log, **kw)
    for c, (g, P) in enumerate(specs):
        e.register_model(g, P)
        _, reg = e.region(c)
        x = rng.image(g, 0)
        for s_ in range(slots):
            reg[s_ * stride:s_ * stride + x.nbytes] = np.frombuffer(x.tobytes(), np.uint8)
    e.clock_sync()   # calibrate after the profiling runs, right before the trace
    t, mm, ii = bench.make_trace(nreq, lam, cfg, len(names), seed=11)
    jct, _ = e.loadgen(t, mm, mm, ii, stride, slots)
    e.shutdown()
    jobs, launches, _ = parse(log)
    if kw.get("notify", "counters") == "counters":
        s = summarize_seen(jobs, launches, names)
    else:
        s = summarize(jobs, launches, names)
    s["variant"] = kw
    s["jct_mean_us"] = round(float(jct.mean()) / 1e3, 1)
    s["jct_per_model_us"] = {n: round(float(jct[mm == i].mean()) / 1e3, 1) for i, n in enumerate(names)
                             if (mm == i).any()}
    if kw.get("notify", "counters") != "counters":
        chrome(jobs, launches, names, out + ".trace.json")
    print(json.dumps(s))


if __name__ == "__main__":
    main()


def dump_jobs(path, names, n=5):
    """Print the first n jobs' launches: layer, issue / placement seen / completion seen
    (us after the job's scheduled arrival)."""
    jobs, launches, _ = parse(path)
    for li in list(jobs)[:n]:
        jb = jobs[li]
        t0 = jb["t_sched"]
        print(f"job {li} {names[jb['model']]}: complete {((jb['t_complete'] or t0) - t0) / 1e3:.1f}")
        for u in jb["uids"]:
            L = launches[u]
            f = lambda x: f"{(x - t0) / 1e3:7.1f}" if x is not None else "      -"   # noqa: E731
            print(f"   L{L['layer']:3d} issue {f(L['t_issue'])} placed {f(L.get('seen_place'))} done {f(L.get('seen_done'))}")
