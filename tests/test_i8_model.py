"""CPU check of the digit scheme the int8 tensor-core GEMMs use (csrc/nl_i8.cu; numerical model in
tools/i8_model.py): 6 balanced base-128 digits per operand, digit pairs with i + j <= 7, exact integer
products, FP64 recombination. The product error must stay far inside what the FP64 parity contract allows
(the update B C'' is O(1e-3) of Psi, so a ~1e-11 product error is ~1e-14 of Psi per factor),
and the balanced digits must beat unsigned ones of similar width (the design reason for them)."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
from i8_model import digits, emulate  # noqa: E402


def _case(seed=0, R=1500):
    rng = np.random.default_rng(seed)
    B = rng.standard_normal((R, 128)) * rng.uniform(0.1, 10, size=(R, 1))
    W = rng.standard_normal((128, 128)) * 1e-3
    return B, W, B @ W


def test_six_balanced_digits_product_error():
    B, W, ex = _case()
    e = emulate(B, W, 6, bits8=False)
    assert np.linalg.norm(e - ex) / np.linalg.norm(ex) < 1e-11
    assert np.abs(e - ex).max() / np.abs(ex).max() < 2e-11


def test_digits_exact_and_in_int8_range():
    B, _, _ = _case(1, 300)
    ds, w, sc = digits(B, 6, bits8=False)
    assert np.abs(ds).max() <= 64
    rec = sum(ds[i] * w[i] for i in range(6)) * sc[:, None]
    # |rest| <= 2^-42 of the row's power-of-two scale (max_k |B[r][k]| < scale <= 2 max_k |B[r][k]|)
    assert (np.abs(rec - B) / sc[:, None]).max() <= 2.0 ** -42
    assert np.all(np.abs(B).max(axis=1) < sc) and np.all(sc <= 2 * np.abs(B).max(axis=1))


def test_balanced_beats_unsigned_digits():
    B, W, ex = _case(2)
    bal = np.linalg.norm(emulate(B, W, 5, bits8=False) - ex)
    uns = np.linalg.norm(emulate(B, W, 5, bits8=True) - ex)
    assert bal < uns
