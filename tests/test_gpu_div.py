"""Device check of the split IEEE divisions every GETRF / GETRS / GETRI
quotient goes through (common.cuh, R3): bit-identical to __ddiv_rn /
__fdiv_rn on 10^8 pairs across all exponents and the specials, and a sample
against the host's IEEE division (numpy)."""
import numpy as np
import pytest
import torch

from paper_conf_icpp_anztdfq17_b200 import bj

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_split_division_is_ieee(dtype):
    n = 100_000_000
    counts, sample = bj.selftest_div(dtype, n, seed=2026, nsample=200_000)
    assert int(counts[5]) == n
    assert int(counts[0]) == 0, "div_pre differs from the IEEE quotient"
    assert int(counts[1]) == 0, "div_pre_flag unflagged quotient differs"
    assert int(counts[3]) == 0, "div_nz_flag unflagged quotient differs (domain: b normal, a finite, a != -0)"
    # the flag-only paths take the fast path for operands of ordinary size
    assert int(counts[2]) < n and int(counts[4]) < n
    a, b, q = sample[:, 0], sample[:, 1], sample[:, 2]
    with np.errstate(all="ignore"):
        ref = a / b
    nan = np.isnan(ref)
    assert np.array_equal(np.isnan(q), nan)
    iv = np.uint64 if dtype == torch.float64 else np.uint32
    assert np.array_equal(q[~nan].view(iv), ref[~nan].view(iv))
