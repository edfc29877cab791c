"""Print a load_exp JSONL sweep as a table (diagnosis helper)."""
import json
import sys

for path in sys.argv[1:]:
    print("==", path)
    for l in open(path):
        d = json.loads(l)
        v = d["variant"]
        if v.get("naive"):
            tag = "naive_pdl" if v.get("naive_pdl") else "naive"
        else:
            tag = f"B{v.get('slack')} la{v.get('lookahead')} {['srpt','fifo','sjf','rr'][v.get('policy',0)]}"
            if v.get("max_active"):
                tag += f" K{v['max_active']}"
            if "theta" in v:
                tag += f" th{v['theta']}"
            if v.get("branches"):
                tag += " br"
            if v.get("prio_classes", 1) > 1:
                tag += f" pc{v['prio_classes']}"
        pm = " ".join(f"{k[:5]}={x:.0f}" for k, x in d["per_model_mean_us"].items())
        print(f"{tag:28s} rate {d['rate']:6.0f} mean {d['mean_us']:6.0f} p50 {d['p50_us']:6.0f} "
              f"p99 {d['p99_us']:7.0f} | {pm} | stop {d['stop']} Q {d['avg_Q']} rdy {d['avg_ready']}")
