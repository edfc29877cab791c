"""Seeded request traces (NEUTRAL MODULE: input generation only).

Paper: "the request inter-arrival pattern follows a lognormal distribution with
either sigma = 2 (bursty) or sigma = 1.5 (less bursty) and varying mean" (PAPER.md
P1370-1372, §7); Fig. 11 uses a uniform mix of models (P1463-1464); Fig. 12 a ratio
of small to large jobs inversely proportional to their size (P1482-1483).
BASELINE.json configs use Poisson arrivals (configs 0-1) and bursty arrivals
(configs 2-3).  Reading: the lognormal's *arithmetic*
mean is 1/lambda, so mu_ln = ln(1/lambda) - sigma^2/2.  Arrival times are integer
ns; the model-choice generator is independent of the arrival generator.
"""
from __future__ import annotations

import numpy as np


def arrivals(n, rate_per_s, kind="poisson", sigma=2.0, seed=1):
    """n integer arrival times (ns, starting near 0) with mean rate `rate_per_s`."""
    r = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0xA221])))
    mean_ns = 1e9 / rate_per_s
    if kind == "poisson":
        gaps = r.exponential(mean_ns, n)
    elif kind == "lognormal":
        mu = np.log(mean_ns) - sigma * sigma / 2.0
        gaps = r.lognormal(mu, sigma, n)
    elif kind == "burst":
        gaps = np.zeros(n)
    else:
        raise ValueError(kind)
    return np.cumsum(gaps).astype(np.int64)


def model_choices(n, weights, seed=1):
    """n model indices drawn with probabilities proportional to `weights`."""
    r = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0x30DE])))
    w = np.asarray(weights, dtype=np.float64)
    return r.choice(len(w), size=n, p=w / w.sum())


def input_choices(n, pool=32, seed=1):
    r = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0x1A9])))
    return r.integers(0, pool, n)


#: BASELINE.json configs
CONFIGS = {
    "c1_toy": dict(models=["toy"], weights=[1.0], clients=2, arrival="poisson"),
    "c2_mix": dict(models=["resnet18", "mobilenet_v2", "squeezenet1_1"], weights=[1, 1, 1], clients=3,
                   arrival="poisson"),
    "c3_dispersion": dict(models=["resnet50", "densenet121", "inception_v3", "mobilenet_v2"], weights=None,
                          clients=4, arrival="lognormal", sigma=2.0),
    # C-3 variants: the less bursty arrivals (sigma = 1.5, P1370-1372) and
    # a uniform model mix (Fig. 11 convention, P1463-1464)
    "c3_sigma15": dict(models=["resnet50", "densenet121", "inception_v3", "mobilenet_v2"], weights=None,
                       clients=4, arrival="lognormal", sigma=1.5),
    "c3_uniform": dict(models=["resnet50", "densenet121", "inception_v3", "mobilenet_v2"], weights=[1, 1, 1, 1],
                       clients=4, arrival="lognormal", sigma=2.0),
}
