"""ORACLE (test infrastructure). float32 -> bfloat16 round-to-nearest-even.

Reading C1-Q7: the bf16 path rounds the client's fp32 input with RNE
before any compute, so the oracle applies the same rounding to the input and then
computes in float64.  Pinned in tests/test_oracle_bf16.py against torch's own cast
(library special case) over every bf16 neighbourhood incl. exact ties.
"""
import numpy as np


def round_bf16(x):
    """RNE-round float32 values to the nearest bfloat16; returns float32 values.

    bf16 keeps the top 16 bits of the IEEE binary32 pattern.  Round half to even on
    the 16 dropped bits; NaN stays NaN (quietened), inf stays inf.
    """
    a = np.ascontiguousarray(x, dtype=np.float32)
    u = a.view(np.uint32).astype(np.uint64)
    lsb = (u >> 16) & 1
    r = ((u + 0x7FFF + lsb) >> 16) << 16
    nan = np.isnan(a)
    r = np.where(nan, (u | 0x00400000) & 0xFFFF0000, r)
    return r.astype(np.uint32).view(np.float32).reshape(a.shape)
