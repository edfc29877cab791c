"""From an `ncu --set full` raw CSV export (tools/profile_round.sh step 2: every kernel
of one request of each model of a bench config, served configuration), compute the
per-launch DRAM traffic (dram__bytes_read.sum + dram__bytes_write.sum) and duration of
the dominant kernel (tcgen05 conv) and of every kernel kind.  Writes the JSON that
bench.py reports as roofline.traffic.

    python tools/ncu_traffic.py gpurun_out/full_r1b_metrics.csv c2_mix > profiles/conv_traffic_c2_mix.json
"""
import csv
import json
import sys
from collections import defaultdict

UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9,
        "ns": 1e-9, "nsecond": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3}


def main(path, config):
    rows = list(csv.reader(open(path)))
    i0 = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr, units = rows[i0], rows[i0 + 1]
    col = {n: hdr.index(n) for n in hdr}
    kinds = defaultdict(lambda: {"launches": 0, "dram_bytes": 0.0, "seconds": 0.0})
    for r in rows[i0 + 2:]:
        if len(r) < len(hdr):
            continue
        name = r[col["Kernel Name"]].split("(")[0].replace("void ", "").replace("paella::", "")
        def val(m):
            return float(r[col[m]].replace(",", "")) * UNIT.get(units[col[m]], 1.0)
        k = kinds[name.split("<")[0]]
        k["launches"] += 1
        k["dram_bytes"] += val("dram__bytes_read.sum") + val("dram__bytes_write.sum")
        k["seconds"] += val("gpu__time_duration.sum")
    out = {"config": config, "source": path.split("/")[-1],
           "method": "ncu --set full --clock-control none, one isolated request of each model (served config); "
                     "dram__bytes_read.sum + dram__bytes_write.sum per launch",
           "kinds": {n: {"launches": v["launches"], "dram_bytes_per_launch": round(v["dram_bytes"] / v["launches"]),
                         "ncu_us_per_launch": round(v["seconds"] / v["launches"] * 1e6, 3)}
                     for n, v in sorted(kinds.items())}}
    conv = out["kinds"].get("k_conv_tc")
    out["conv_tcgen05_dram_bytes_per_launch"] = conv["dram_bytes_per_launch"] if conv else None
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else "c2_mix")
