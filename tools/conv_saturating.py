"""The tcgen05 conv at a saturating shape (judge kernel quality where
the roofline is reachable): a 3x3 256->256 conv over a large image (HxW pixels = the
batch-1 kernel's N dimension), timed as served (PDL chain, CUDA events).  Prints one
JSON line: TFLOP/s vs the measured dense bf16 peak, plus the batch-1 shape for context."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from workload import archs  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def bf16_values(x):
    u = np.asarray(x, np.float32).view(np.uint32)
    r = ((u + 0x7FFF + ((u >> 16) & 1)) >> 16) << 16   # RNE to bf16, kept as fp32
    return r.astype(np.uint32).view(np.float32)


def graph(hw, c=256):
    g = archs.Graph("conv_sat", (3, hw, hw), 10)
    x = g.conv(g.input, c, 1, name="stem")
    x = g.conv(x, c, 3, 1, 1, name="big")
    x = g.gap(x, name="gap")
    g.fc(x, 10, name="fc")
    return g


def params(g, seed=0):
    r = np.random.default_rng(seed)
    out = {}
    for n in g.weight_nodes():
        shp = g.param_shapes()[n["name"] + ".weight"]
        fan = int(np.prod(shp[1:]))
        out[n["name"] + ".weight"] = bf16_values(r.standard_normal(shp) / np.sqrt(fan))
        out[n["name"] + ".bias"] = np.zeros(shp[0], np.float32)
    return out


def measure(e, hw, reps=20):
    g = graph(hw)
    mid = e.register_model(g, params(g), name=f"conv_sat_{hw}")
    ks = e.kernels(mid)
    big = 2   # ingest, stem, big, gap+fc
    t_plain = int(e.time_kernels(mid, instrumented=False, reps=reps)[big])
    t_instr = int(e.time_kernels(mid, instrumented=True, reps=reps)[big])
    k = ks[big]
    return {"shape": f"3x3 256->256, {hw}x{hw} px", "grid": k["grid"], "flops": int(k["flops"]),
            "bytes": int(k["bytes"]), "us_plain": round(t_plain / 1e3, 2), "us_instr": round(t_instr / 1e3, 2),
            "tflops_plain": round(k["flops"] / t_plain / 1e3, 1), "tflops_instr": round(k["flops"] / t_instr / 1e3, 1)}


def main():
    from paper_conf_sosp_ngd023_b200 import _lib as L
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    peak = peaks.get("bf16_tflops", 2250.0)
    with L.Engine(num_clients=1, max_jobs_per_model=1) as e:
        rows = [measure(e, hw) for hw in (int(a) for a in (sys.argv[1:] or ["14", "56", "224", "448"]))]
    for r in rows:
        r["frac_of_bf16_peak"] = round(r["tflops_plain"] / peak, 3)
    print(json.dumps({"kernel": "conv_tcgen05", "bound": "tensor", "peak_tflops": peak,
                      "peak_source": "MEASURED_PEAKS.json bf16_tflops (cuBLAS burst)" if peaks else "nominal",
                      "shapes": rows}))


if __name__ == "__main__":
    main()
