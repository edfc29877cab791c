"""Seeded synthetic inputs: weights, images and the calibration input.

NEUTRAL MODULE (serves both the oracle and the CUDA path; holds none of the
method's arithmetic).  Recipe: SURVEY.md §8(c) C1 "Weights: random init" and
DESIGN.md §"Input recipe".

* raw weights: conv/FC weight ~ N(0, 1/fan_in), bias ~ 0.01 N(0,1), drawn from a
  numpy PCG64 generator seeded by (model_seed, node_id).  BatchNorm is generated
  pre-folded (the folded conv weight/bias *is* the synthetic model), so there is no
  BN arithmetic anywhere.  DenseNet's unfoldable pre-activation BN is a
  per-channel prologue: scale ~ U(0.5, 1.5), shift ~ 0.1 N(0,1).
* LSUV scale: each conv/FC weight and bias is multiplied by a stored per-layer
  factor ``s`` so that, on the calibration input, every layer emits unit std.  The
  factors are *data*: ``workload/data/lsuv_scales.json``, written by the committed
  script ``oracle/make_lsuv_scales.py`` which calls only ``oracle/``.
* weights are then rounded to bfloat16 (round-to-nearest-even, torch's cast) and
  returned widened to float32: these bf16-representable values ARE the model on
  both sides, so weight quantisation is never counted as error.
* images: fp32 NCHW N(0,1), a pool of 32 per model, seeds 1000+i.
"""
from __future__ import annotations

import json
import os

import numpy as np

from . import archs

_DATA = os.path.join(os.path.dirname(__file__), "data")
SCALES_PATH = os.path.join(_DATA, "lsuv_scales.json")

MODEL_SEED = 0
CALIB_SEED = 123
INPUT_SEED_BASE = 1000
INPUT_POOL = 32


def _gen(*key):
    return np.random.Generator(np.random.PCG64(np.random.SeedSequence(list(key))))


def raw_params(g: archs.Graph, model_seed: int | None = None):
    """Unscaled float64 parameters {name: array} in canonical layouts."""
    if model_seed is None:
        model_seed = MODEL_SEED + archs.MODEL_INDEX.get(g.name, len(archs.MODEL_INDEX))
    shapes = g.param_shapes()
    out = {}
    for n in g.nodes:
        if n["op"] not in ("conv", "fc") and not n.get("prologue"):
            continue
        rng = _gen(model_seed, n["id"])
        if n["op"] in ("conv", "fc"):
            wshape = shapes[n["name"] + ".weight"]
            fan_in = int(np.prod(wshape[1:]))
            out[n["name"] + ".weight"] = rng.standard_normal(wshape) / np.sqrt(fan_in)
            b = 0.01 * rng.standard_normal(wshape[0])
            if n["op"] == "conv" and not n["bias"]:
                b = np.zeros_like(b)
            out[n["name"] + ".bias"] = b
        if n.get("prologue"):
            c = shapes[n["name"] + ".pro_scale"][0]
            out[n["name"] + ".pro_scale"] = rng.uniform(0.5, 1.5, c)
            out[n["name"] + ".pro_shift"] = 0.1 * rng.standard_normal(c)
    return out


def load_scales(name):
    with open(SCALES_PATH) as f:
        return json.load(f)[name]


def _to_bf16_values(a):
    import torch  # torch's fp32->bf16 cast is RNE
    t = torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32))
    return t.to(torch.bfloat16).to(torch.float32).numpy()


def model_params(g: archs.Graph, scales: dict | None = None):
    """Canonical synthetic parameters: {name: float32 array}.

    Weights are bf16-representable float32; biases and prologue affines are fp32.
    ``scales`` maps layer name -> LSUV factor (defaults to the stored table).
    """
    if scales is None:
        scales = load_scales(g.name) if g.weight_nodes() else {}
    raw = raw_params(g)
    out = {}
    for n in g.weight_nodes():
        s = scales[n["name"]]
        out[n["name"] + ".weight"] = _to_bf16_values(raw[n["name"] + ".weight"] * s)
        out[n["name"] + ".bias"] = (raw[n["name"] + ".bias"] * s).astype(np.float32)
    for n in g.prologue_nodes():
        out[n["name"] + ".pro_scale"] = raw[n["name"] + ".pro_scale"].astype(np.float32)
        out[n["name"] + ".pro_shift"] = raw[n["name"] + ".pro_shift"].astype(np.float32)
    return out


def image(g: archs.Graph, i: int):
    """Input i of the model's pool: fp32 NCHW (1, C, H, W), N(0,1)."""
    rng = _gen(INPUT_SEED_BASE + i, archs.MODEL_INDEX.get(g.name, len(archs.MODEL_INDEX)))
    return rng.standard_normal((1,) + g.nodes[0]["out"]).astype(np.float32)


def calibration_input(g: archs.Graph):
    rng = _gen(CALIB_SEED, archs.MODEL_INDEX[g.name])
    return rng.standard_normal((1,) + g.nodes[0]["out"])
