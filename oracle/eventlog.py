"""ORACLE (test infrastructure): reader of the dispatcher's binary event log, for
replay parity (pin S6) and the GPU-log invariants (S5).

Format (DESIGN.md §"Event log"): a sequence of 32-byte little-endian records
``{u32 type, u32 a, u64 b, u64 c, u64 d}``:

  100 CONFIG    a=N clients, b=policy, c=theta, d=(B << 32) | G
  100 CONFIG    a=0xFFFFFFFF, b=ring capacity, c=stream pool P, d=(priority classes << 32) | launch-ahead depth
  100 CONFIG    a=0xFFFFFFFE, b=online T-bar refinement (NEXT-4), c=max_active K (B200-Q6),
                d=branches | lookahead_unplaced << 8 (NEXT-1 variant) | cap_fifo << 9 (B200-Q6 variant)
  101 CAPACITY  a=resource r, b=C_r
  110 MODEL     a=model, b=#kernels
  111 LAYER     a=model, b=layer, c=grid, d=T-bar ns
  112 DEMAND    a=model, b=layer, c=(warps << 32) | regs, d=(smem << 32) | tmem
  114 VS        a=model, b=layer, c=virtual stream            (NEXT-4 branches only)
  113 DEP       a=model, b=layer, c=a kernel of ANOTHER virtual stream it consumes
    1 ARRIVAL   a=client, b=job, c=model, d=t_sched ns
    2 RECORD    a=type, b=uid, c=count, d=globaltimer:40 | group:16 | smid:8
    3 BATCH_END
    4 ISSUE     a=stream, b=uid, c=job, d=layer
    5 COMPLETE  b=job, c=t ns
    6 OBSERVE   b=uid, c=observed duration ns (NEXT-4; precedes the final COMPLETION)
    9 TIME      (PAELLA_TRACE_TIMES only; ignored here) a=0 decision of launch b, 1 batch end,
                2/3 placement/completion count of launch b seen; c = host ns (tools/timeline.py)
    8 CLOCK     a=gpu | resolution ns << 8, b=offset (globaltimer - host CLOCK_MONOTONIC, ns),
                c=round trip ns, d=host time of the calibration sample (at init and at every
                paella_clock_sync)
    7 ROUTE     a=g0 | g1 << 8 | route << 16, b=req_id, c=W_g0, d=W_g1 (multi-GPU only;
                the router's decision inputs, logged by the GPU it chose, before ARRIVAL)
"""
import numpy as np

from . import sim

DT = np.dtype([("type", "<u4"), ("a", "<u4"), ("b", "<u8"), ("c", "<u8"), ("d", "<u8")])


def read(path):
    """Returns (Config, models, events, extras) where events are in sim.replay's format."""
    raw = np.fromfile(path, dtype=DT)
    cfg_kw = {}
    cap = [0] * 5
    layers = {}
    demands = {}
    nlayers = {}
    events = []
    arrivals = {}
    records = []
    issues = []
    completes = []
    routes = []
    clocks = []
    vss, xdeps = {}, {}   # NEXT-4 DAG: virtual stream and cross-stream dependencies per layer
    narrivals = 0
    lives = []          # one entry per admitted job occurrence (job ids are recycled)
    cur_life = {}       # job id -> index into lives of its current occurrence
    uid_life = {}       # launch uid -> index into lives
    for r in raw:
        t, a, b, c, d = int(r["type"]), int(r["a"]), int(r["b"]), int(r["c"]), int(r["d"])
        if t == 100:
            if a == 0xFFFFFFFE:
                cfg_kw["online_tbar"] = b
                cfg_kw["max_active"] = c
                cfg_kw["lookahead_unplaced"] = (d >> 8) & 1
                cfg_kw["cap_fifo"] = (d >> 9) & 1
            elif a == 0xFFFFFFFF:
                cfg_kw["ring_capacity"] = b
                cfg_kw["streams"] = c
                cfg_kw["lookahead"] = d & 0xFFFFFFFF
                cfg_kw["prio_classes"] = max(1, d >> 32)
            else:
                cfg_kw["num_clients"] = a
                cfg_kw["policy"] = b
                cfg_kw["theta"] = c if c < (1 << 63) else c - (1 << 64)
                cfg_kw["slack"] = d >> 32
                cfg_kw["group"] = d & 0xFFFFFFFF
        elif t == 101:
            cap[a] = b
        elif t == 110:
            nlayers[a] = b
            events.append((sim.EV_MODEL, a))
        elif t == 111:
            layers[(a, b)] = (c, d)
        elif t == 112:
            demands[(a, b)] = (c >> 32, c & 0xFFFFFFFF, d >> 32, d & 0xFFFFFFFF)
        elif t == 114:
            vss[(a, b)] = c
        elif t == 113:
            xdeps.setdefault((a, b), []).append(c)
        elif t == 1:
            events.append((sim.EV_ARRIVAL, b, a, c))
            arrivals[b] = (a, c, d)        # latest job with this id (ids are recycled)
            narrivals += 1
            cur_life[b] = len(lives)
            lives.append(dict(job=b, client=a, model=c, t_sched=d, t_complete=None, uids=[]))
        elif t == 2:
            events.append((sim.EV_RECORD, a, b, c))
            # (t, type, uid, n, group) as sim.check_exactly_once expects, + smid
            records.append((d & ((1 << 40) - 1), a, b, c, (d >> 40) & 0xFFFF, d >> 56))
        elif t == 3:
            events.append((sim.EV_BATCH_END,))
        elif t == 4:
            events.append((sim.EV_ISSUE, b, c, d, a))
            issues.append((b, c, d, a, arrivals[c][1]))   # (uid, job, layer, stream, model)
            uid_life[b] = cur_life[c]
            lives[cur_life[c]]["uids"].append(b)
        elif t == 7:
            routes.append((a & 0xFF, (a >> 8) & 0xFF, a >> 16, b,
                           c if c < (1 << 63) else c - (1 << 64), d if d < (1 << 63) else d - (1 << 64)))
        elif t == 6:
            events.append((sim.EV_OBSERVE, b, c))
        elif t == 8:
            clocks.append(dict(gpu=a & 0xFF, resolution=a >> 8, offset=b if b < (1 << 63) else b - (1 << 64),
                               rtt=c, at=d))
        elif t == 5:
            events.append((sim.EV_COMPLETE, b))
            completes.append((b, c))
            if b in cur_life:
                lives[cur_life[b]]["t_complete"] = c
    cfg = sim.Config(capacity=tuple(cap), **cfg_kw)
    models = []
    for m in range(len(nlayers)):
        ms = []
        for l in range(nlayers[m]):
            grid, tbar = layers[(m, l)]
            w, rg, sm, tm = demands[(m, l)]
            if (m, l) in vss:
                ms.append(sim.Layer(grid, (1, w, rg, sm, tm), tbar, deps=tuple(xdeps.get((m, l), ())),
                                    vs=vss[(m, l)]))
            else:
                ms.append(sim.Layer(grid, (1, w, rg, sm, tm), tbar))
        models.append(ms)
    extras = dict(records=records, issues=issues, completes=completes, arrivals=arrivals,
                  n_arrivals=narrivals, routes=routes, clocks=clocks, lives=lives, uid_life=uid_life)
    return cfg, models, events, extras


# routing log (paella_config_t.route_log_path): paella_route_rec_t, include/paella.h
ROUTE_DT = np.dtype([("req_id", "<u8"), ("route", "<u4"), ("chosen", "<u4"), ("g0", "<u4"), ("g1", "<u4"),
                     ("num_gpus", "<u4"), ("model", "<u4"), ("alive", "<u4"), ("pad", "<u4"),
                     ("tbar_model", "<i8"), ("work", "<i8", (8,)), ("pending", "<i8", (8,))])


def read_routes(path):
    """Every routing decision of one client, in submission order (dicts)."""
    raw = np.fromfile(path, dtype=ROUTE_DT)
    out = []
    for r in raw:
        ng = int(r["num_gpus"])
        out.append(dict(req_id=int(r["req_id"]), route=int(r["route"]), chosen=int(r["chosen"]),
                        g0=int(r["g0"]), g1=int(r["g1"]), num_gpus=ng, model=int(r["model"]),
                        alive=int(r["alive"]), tbar_model=int(r["tbar_model"]),
                        work=[int(x) for x in r["work"][:ng]], pending=[int(x) for x in r["pending"][:ng]]))
    return out
