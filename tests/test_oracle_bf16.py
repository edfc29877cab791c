"""Pin for oracle.bf16.round_bf16 (C3 "RNE ingest"): torch's fp32->bf16 cast is the
library special case; checked over all 65,536 bf16 patterns +/- half-ulp ties and
their neighbours, plus 10^6 random fp32 values."""
import numpy as np
import torch

from oracle.bf16 import round_bf16


def _torch_bf16(a):
    return torch.from_numpy(a).to(torch.bfloat16).to(torch.float32).numpy()


def test_all_bf16_neighbourhoods():
    hi = np.arange(65536, dtype=np.uint32) << 16
    cands = [hi, hi | 0x8000, hi | 0x7FFF, hi | 0x8001, hi | 0x0001, hi | 0xFFFF]
    u = np.concatenate(cands)
    a = u.view(np.float32)
    a = a[~np.isnan(a)]
    np.testing.assert_array_equal(round_bf16(a).view(np.uint32), _torch_bf16(a).view(np.uint32))


def test_random_fp32():
    r = np.random.default_rng(0)
    a = r.integers(0, 2**32, size=1_000_000, dtype=np.uint64).astype(np.uint32).view(np.float32)
    a = a[np.isfinite(a)]
    np.testing.assert_array_equal(round_bf16(a).view(np.uint32), _torch_bf16(a).view(np.uint32))


def test_ties_to_even():
    # 1 + 2^-8 is exactly halfway between bf16 1.0 and 1.0078125 -> even (1.0)
    assert round_bf16(np.float32(1 + 2**-8)) == 1.0
    assert round_bf16(np.float32(1 + 3 * 2**-8)) == np.float32(1 + 2**-6)
