"""Capture target for ncu: the 3x3 256->256 conv of tools/conv_saturating.py at 448x448
(128-pixel tiles) run once in an isolated chain.  Diagnosis tool (no oracle).

    ncu --set full -k regex:k_conv_tc -o /tmp/sat python tools/ncu_saturating.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import conv_saturating  # noqa: E402
from paper_conf_sosp_ngd023_b200 import _lib as L  # noqa: E402

hw = int(sys.argv[1]) if len(sys.argv) > 1 else 448
with L.Engine(num_clients=1) as e:
    g = conv_saturating.graph(hw)
    mid = e.register_model(g, conv_saturating.params(g), name=f"sat{hw}")
    e.run_isolated(mid, np.zeros((1, 3, hw, hw), np.float32))
