#!/bin/bash
# Final validation of the round's last configuration (split gain 65 %, TMA im2col
# activations, M = 64 opt-in): GPU tests, smoke, smoke under ncu, bench line; then the
# ncu launch list of the served mix and the full conv capture.
bash tools/gpu_r2final.sh
bash tools/profile_r2.sh r2final
