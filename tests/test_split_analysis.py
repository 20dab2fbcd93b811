"""CPU pins of the SGEMM split error analysis (R19) on the bit-level emulation in
split_emulation.py: the truncated TF32 head can exceed the 1e-5 componentwise contract
(worst case 2^-16 + 2^-20 ~ 1.6e-5), the rounded head cannot (2^-17 + 2^-22 ~ 7.9e-6)."""
import numpy as np

from split_emulation import ADVERSARIAL_RN, ADVERSARIAL_TRUNC, bf16_rn, split_rel_error, tf32_head

RN_BOUND = 2.0 ** -17 + 2.0 ** -22
TRUNC_BOUND = 2.0 ** -16 + 2.0 ** -20


def test_bf16_and_tf32_rounding_helpers():
    x = np.array([1.0, 1.0 + 2.0 ** -8, 1.0 + 3 * 2.0 ** -8, 1.0 + 2.0 ** -7], dtype=np.float32)
    # ties to even at the bf16 half-ulp (2^-8), exact otherwise
    assert list(bf16_rn(x)) == [1.0, 1.0, 1.0 + 2.0 ** -6, 1.0 + 2.0 ** -7]
    y = np.array([1.0 + 2.0 ** -11, 1.0 + 2.0 ** -12], dtype=np.float32)
    assert list(tf32_head(y, False)) == [1.0, 1.0]
    assert list(tf32_head(y, True)) == [1.0 + 2.0 ** -10, 1.0]  # ties away / below half


def test_integer_inputs_are_exact_in_both_splits():
    v = np.arange(-1024, 1025, dtype=np.float32)
    for rn in (False, True):
        assert split_rel_error(v[v != 0], v[v != 0][::-1], rn).max() == 0.0


def test_rounded_head_within_contract_on_random_and_adversarial_inputs():
    g = np.random.default_rng(3)
    a = (1 + g.integers(0, 2 ** 23, 1_000_000) / 2 ** 23).astype(np.float32)
    b = (1 + g.integers(0, 2 ** 23, 1_000_000) / 2 ** 23).astype(np.float32)
    e = split_rel_error(a, b, True)
    assert e.max() <= RN_BOUND < 1e-5
    for x in (ADVERSARIAL_RN, ADVERSARIAL_TRUNC):
        assert split_rel_error(x, x, True) <= RN_BOUND


def test_truncated_head_can_break_contract():
    e = float(split_rel_error(ADVERSARIAL_TRUNC, ADVERSARIAL_TRUNC, False))
    assert 1e-5 < e <= TRUNC_BOUND
