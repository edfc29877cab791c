"""Summarise tools/trace_all_convs.py output: per traced conv (last run of each), the
median phase times (ns from the first CTA entry) and the intervals after the PDL wait:
gather issue -> first stage full -> MMAs done -> epilogue/reduction done -> last exit."""
import json
import re
import sys

err, out = sys.argv[1], sys.argv[2]
layers = [json.loads(l) for l in open(out) if l.startswith("{")]
seq = []   # traced blocks in file order: 2 runs per layer, layers in stdout order
cur = None
for line in open(err):
    m = re.match(r"trace kernel (\d+) grid (\d+)", line)
    if m:
        cur = {}
        seq.append((int(m.group(1)), cur))
        continue
    m = re.match(r"\s+(\w+)\s+(-?\d+)\s+(-?\d+)\s+(-?\d+)", line)
    if m and cur is not None:
        cur[m.group(1)] = (int(m.group(2)), int(m.group(3)), int(m.group(4)))
print(f"{'model':12s} {'k':>3s} {'grid':>4s} {'MB':>5s} {'GF':>6s} | {'b_iss':>6s} {'full0':>6s} {'mma':>6s} "
      f"{'epi':>6s} {'exit':>6s} | {'data':>5s} {'loop':>5s} {'tail':>5s} {'span':>5s}")
tot = {}
pos = 0
for L in layers:
    bl = []
    while pos < len(seq) and seq[pos][0] == L["k"]:
        bl.append(seq[pos][1])
        pos += 1
    if not bl:
        continue
    b = bl[-1]
    med = {k: v[1] for k, v in b.items()}
    bi, f0, md = med.get("b_issued", 0), med.get("full0", 0), med.get("mma_done", 0)
    ep = med.get("epi_done", med.get("reduced", 0))
    ex = b.get("exit", (0, 0, 0))[2]
    data, loop, tail, span = f0 - bi, md - f0, ex - md, ex - bi
    t = tot.setdefault(L["model"], [0, 0, 0, 0, 0])
    t[0] += 1; t[1] += data; t[2] += loop; t[3] += tail; t[4] += span
    print(f"{L['model']:12s} {L['k']:3d} {L['grid']:4d} {L['bytes']/1e6:5.2f} {L['flops']/1e9:6.3f} | {bi:6d} {f0:6d} "
          f"{md:6d} {ep:6d} {ex:6d} | {data:5d} {loop:5d} {tail:5d} {span:5d}")
for m, (n, a, b, c, d) in tot.items():
    print(f"{m}: {n} convs, mean data {a/n:.0f} ns, loop {b/n:.0f} ns, tail {c/n:.0f} ns, span after gather {d/n:.0f} ns")
