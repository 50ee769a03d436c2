"""Properties the exact stage-0 SLO bound of the KS = 3 / 4 pre-filter relies on
(DESIGN.md §4.3): rounded addition is monotone in each operand (f16 and f32, +INF
included), so a sum of lower bounds never exceeds the sum it bounds, and the guarded
integer SLO test (bit pattern of slack - v3 with a guard bit, minus the bits of S3) is
monotone in S3 on non-negative f16.  CPU only; numpy's IEEE arithmetic is the ground truth.
"""
import numpy as np
import pytest


def _nonneg_f16(rng, n):
    # every finite non-negative f16 bit pattern is 0x0000..0x7bff; +INF = 0x7c00
    bits = rng.integers(0, 0x7c01, size=n, dtype=np.uint32).astype(np.uint16)
    return bits.view(np.float16)


@pytest.mark.parametrize("dtype", [np.float16, np.float32])
def test_rounded_addition_is_monotone(dtype):
    rng = np.random.default_rng(7)
    n = 200_000
    if dtype == np.float16:
        a, b = _nonneg_f16(rng, n), _nonneg_f16(rng, n)
        da, db = _nonneg_f16(rng, n), _nonneg_f16(rng, n)
    else:
        a = rng.uniform(0, 2 ** 25, n).astype(np.float32)
        b = rng.uniform(0, 2 ** 25, n).astype(np.float32)
        da = rng.uniform(0, 2 ** 10, n).astype(np.float32)
        db = rng.uniform(0, 2 ** 10, n).astype(np.float32)
    with np.errstate(over="ignore", invalid="ignore"):
        lo = (a + b).astype(dtype)
        hi = ((a + da).astype(dtype) + (b + db).astype(dtype)).astype(dtype)
    assert not np.isnan(lo).any() and not np.isnan(hi).any()
    assert (lo <= hi).all()
    # a chain of two additions (the S1 + v1min + v2min lower bound against S1 + w1 + w2)
    with np.errstate(over="ignore"):
        c = (_nonneg_f16(rng, n) if dtype == np.float16 else rng.uniform(0, 2 ** 25, n).astype(np.float32))
        lb = ((a + b).astype(dtype) + c).astype(dtype)
        full = (((a + da).astype(dtype) + b).astype(dtype) + c).astype(dtype)
    assert (lb <= full).all()


def _guard(w_bits):
    """h2guard for one half: guard bit | magnitude when the sign is clear, guard alone else."""
    w = np.asarray(w_bits, dtype=np.uint32)
    neg = (w & 0x8000) != 0
    return np.where(neg, 0x8000, (w & 0x7fff) | 0x8000).astype(np.uint32)


def test_guarded_slo_test_matches_f16_compare_and_is_monotone():
    rng = np.random.default_rng(11)
    n = 200_000
    slack = rng.uniform(-40, 40, n).astype(np.float16)
    s3 = _nonneg_f16(rng, n)
    s3[:64] = 0.0  # S3 = +0 against negative slacks: the one place the test is looser
    slack[:32] = -np.abs(slack[:32]) - np.float16(1)
    ok_int = ((_guard(slack.view(np.uint16)) - s3.view(np.uint16).astype(np.uint32)) & 0x8000) != 0
    # reference: the f16 comparison S3 <= slack.  The guarded test equals it except that
    # S3 = +0 always passes (a negative slack is the guard alone, 0x8000 - 0 keeps bit 15):
    # looser, so the pre-filter stays conservative (it may flag more, never fewer)
    ok_ref = s3.astype(np.float64) <= slack.astype(np.float64)
    assert (ok_int | ~ok_ref).all()
    assert (ok_int == ok_ref)[s3.view(np.uint16) != 0].all()
    # monotone: a larger S3 never passes where a smaller one fails
    s3b = np.maximum(s3, _nonneg_f16(rng, n))
    ok_b = ((_guard(slack.view(np.uint16)) - s3b.view(np.uint16).astype(np.uint32)) & 0x8000) != 0
    assert not (ok_b & ~ok_int).any()
