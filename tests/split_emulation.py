"""Bit-level emulation of the per-product arithmetic of the TF32+2xBF16 SGEMM split
(R19), used only to pick adversarial test inputs and to pin the error analysis.

x = h + l with h the TF32 head of x (11 significant bits) and l = x - h (exact in fp32);
the kernel computes h_a h_b (TF32 MMA, exact product) + bf16(h_a) bf16(l_b) + bf16(l_a)
bf16(h_b) (BF16 MMAs, exact products), all accumulated in fp32; l_a l_b is dropped.
``rn_head`` selects h = x rounded to nearest (ties away) instead of truncated."""
import numpy as np


def bf16_rn(x):
    u = np.asarray(x, dtype=np.float32).view(np.uint32).astype(np.uint64)
    r = (u + 0x7FFF + ((u >> 16) & 1)) & 0xFFFF0000
    return r.astype(np.uint32).view(np.float32)


def tf32_head(x, rn_head):
    u = np.asarray(x, dtype=np.float32).view(np.uint32).astype(np.uint64)
    u = ((u + 0x1000) if rn_head else u) & 0xFFFFE000
    return u.astype(np.uint32).view(np.float32)


def split_product(a, b, rn_head):
    """The split's value of a*b (float64, exact: every term has <= 22 significant bits)."""
    a = np.asarray(a, dtype=np.float32)
    b = np.asarray(b, dtype=np.float32)
    ha, hb = tf32_head(a, rn_head), tf32_head(b, rn_head)
    la, lb = (a - ha).astype(np.float32), (b - hb).astype(np.float32)
    return (ha.astype(np.float64) * hb + bf16_rn(ha).astype(np.float64) * bf16_rn(lb)
            + bf16_rn(la).astype(np.float64) * bf16_rn(hb))


def split_rel_error(a, b, rn_head):
    ab = np.asarray(a, dtype=np.float64) * np.asarray(b, dtype=np.float64)
    return np.abs(split_product(a, b, rn_head) - ab) / np.abs(ab)


# Found by hill-climbing single mantissa-bit flips of (a, b) from random starts (30
# restarts, both = the same value at the optimum): the truncated head's worst case and
# the rounded head's worst case.
ADVERSARIAL_TRUNC = np.uint32(0x3F809FEF).view(np.float32)  # 1.0048808: trunc split error 1.20e-5
ADVERSARIAL_RN = np.uint32(0x3F807018).view(np.float32)     # 1.0034208: rn split error 5.43e-6
