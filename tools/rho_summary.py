"""Summarise tools/rho_sweep.py output: per config and rho, the mix mean / p99 JCT of each
arm averaged over the seeds, and Paella's ratios vs naive and naive+PDL (markdown)."""
import json
import sys
from collections import defaultdict

rows = [json.loads(l) for l in open(sys.argv[1]) if '"arm"' in l]
acc = defaultdict(list)
for r in rows:
    acc[(r["config"], r["rho"], r["arm"])].append((r["jct"]["mix"]["mean_us"], r["jct"]["mix"]["p99_us"]))
arms = ["paella", "paella_fifo", "naive_pdl", "naive"]
for cfg in sorted({k[0] for k in acc}):
    print(f"\n### {cfg}\n")
    print("| rho | " + " | ".join(f"{a} mean / p99 (us)" for a in arms) + " | vs naive mean / p99 | vs naive+PDL mean / p99 |")
    print("|---" * (len(arms) + 3) + "|")
    for rho in sorted({k[1] for k in acc if k[0] == cfg}):
        m = {}
        for a in arms:
            v = acc.get((cfg, rho, a))
            if v:
                m[a] = (sum(x[0] for x in v) / len(v), sum(x[1] for x in v) / len(v))
        cells = [f"{m[a][0]:.0f} / {m[a][1]:.0f}" if a in m else "-" for a in arms]
        p = m.get("paella")
        r1 = f"{m['naive'][0] / p[0]:.2f} / {m['naive'][1] / p[1]:.2f}" if p and "naive" in m else "-"
        r2 = f"{m['naive_pdl'][0] / p[0]:.2f} / {m['naive_pdl'][1] / p[1]:.2f}" if p and "naive_pdl" in m else "-"
        print(f"| {rho} | " + " | ".join(cells) + f" | {r1} | {r2} |")
