"""Pins for the per-level precision cast (L266; readings R16-R18): FP64 -> FP16 must
round to nearest even DIRECTLY from FP64 (no double rounding through FP32)."""
import numpy as np

import oracle


def test_direct_rounding_no_double_rounding():
    # x = 1 + 2^-11 + 2^-40: direct RN to FP16 (ulp 2^-10 at 1) -> 1 + 2^-10;
    # via FP32 it would first become 1 + 2^-11 (a tie) and then round to even = 1.0.
    x = 1.0 + 2.0 ** -11 + 2.0 ** -40
    assert oracle.cast_values(np.array([x]), "f16")[0] == np.float16(1.0 + 2.0 ** -10)
    assert np.float16(np.float32(x)) == np.float16(1.0)


def test_ties_to_even_and_overflow():
    v = np.array([1.0 + 2.0 ** -11, 1.0 + 3 * 2.0 ** -11, 65504.0, 65519.0, 65520.0, -70000.0, 2.0 ** -25,
                  2.0 ** -24 * 1.5])
    h = oracle.cast_values(v, "f16").astype(np.float64)
    assert h[0] == 1.0 and h[1] == 1.0 + 2.0 ** -9
    assert h[2] == 65504.0 and h[3] == 65504.0 and np.isinf(h[4]) and np.isinf(h[5]) and h[5] < 0
    assert h[6] == 0.0 and h[7] == 2.0 ** -23  # subnormal ties-to-even


def test_fp32_exact_for_small_integers():
    v = np.arange(-2048, 2049, dtype=np.float64)
    assert np.array_equal(oracle.cast_values(v, "f32").astype(np.float64), v)
    assert np.array_equal(oracle.cast_values(v, "f16").astype(np.float64), v)
