"""Print the key numbers of a bench.py JSON line (diagnosis helper)."""
import json
import sys

d = json.loads([l for l in open(sys.argv[1]).read().splitlines() if l.startswith("{")][-1])
print("value", d["value"], d["unit"], "| mix", {k: round(v, 1) for k, v in d["jct_us"]["mix"].items()})
for k, v in d.get("baselines", {}).items():
    print(" ", k, {a: round(b, 1) for a, b in v["mix"].items()})
print("  req/s at SLO", d.get("req_s_at_p99_slo"), "x_sat", d.get("x_sat_req_s"))
print("  roofline", {k: d["roofline"][k] for k in ("achieved", "frac", "mean_launch_us", "share_of_device_time")})
print("  unloaded", d["jct_unloaded_p50_us"])
print("  device roofline", d["device_roofline_us"])
print("  e2e", d["e2e"]["value"], "clocks", d["clocks"], "launches", d.get("gpu_launches"))
for k, v in d.get("slo_ladder", {}).items():
    print("  ladder", k, [(p["rho"], p["mean_us"], max(p["p99_us"].values()), p["slo_met"]) for p in v["ladder"]])
