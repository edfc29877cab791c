"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) into per-kernel
shares of device time, and a --set full capture into the roofline fields."""
import csv
import sys
from collections import defaultdict


def launches(path):
    rows = list(csv.reader(open(path)))
    for i, r in enumerate(rows):
        if r and r[0] == "ID":
            hdr, start = r, i
            break
    iN, iV, iU = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    tot = defaultdict(float)
    cnt = defaultdict(int)
    for r in rows[start + 1:]:
        if len(r) <= iV:
            continue
        name = r[iN].split("(")[0].replace("void ", "").replace("paella::", "")
        v = float(r[iV].replace(",", ""))
        scale = {"ns": 1.0, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6, "nsecond": 1.0}.get(r[iU], 1.0)
        tot[name] += v * scale
        cnt[name] += 1
    T = sum(tot.values())
    out = []
    for k in sorted(tot, key=lambda k: -tot[k]):
        out.append((k, cnt[k], tot[k] / 1e3, tot[k] / T, tot[k] / cnt[k] / 1e3))
    return out, T


if __name__ == "__main__":
    res, T = launches(sys.argv[1])
    print(f"total device time {T/1e6:.3f} ms over {sum(r[1] for r in res)} launches")
    print(f"{'kernel':45s} {'launches':>8s} {'total_us':>10s} {'share':>7s} {'mean_us':>8s}")
    for k, n, t, sh, m in res:
        print(f"{k[:45]:45s} {n:8d} {t:10.1f} {sh:7.3f} {m:8.2f}")
