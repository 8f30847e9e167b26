"""Host model of the int8-digit arithmetic behind the tcgen05 projector GEMMs (csrc/nl_i8.cu, lfd_tc.cuh), in
exact integer arithmetic (no GPU): the digit extraction from one floating-point add against 1.5 2^52, the
offset-binary / balanced digit algebra and its correction term, and the truncation error bound the headers
state. A wrong offset, digit weight, byte order or correction sign fails the exact identities below; the
GPU kernels are compared with the oracle in tests/test_gpu_i8.py."""
import numpy as np
import pytest

M52 = 6755399441055744.0  # 1.5 2^52


def low_bits(x, sc, madd, nbits):
    """the low nbits of the float64 bits of x*sc + madd (x*sc exact: sc is a power of two), as the kernels read
    them after one DFMA"""
    v = np.asarray(x, dtype=np.float64) * sc + madd
    return (v.view(np.int64) & ((1 << nbits) - 1)).astype(np.int64)


def g1_a_digits(x, S, e):
    """GEMM-1's Psi digits: X = rint(x 2^(8S-2-e)), the bytes u_k of X + 2^(8S-1) (offset binary, unsigned)"""
    sc = 2.0 ** (8 * S - 2 - e)
    Z = low_bits(x, sc, M52 + float(1 << (8 * S - 1)), 8 * S)
    X = np.rint(np.asarray(x) * sc).astype(np.int64)
    assert np.array_equal(Z, X + (1 << (8 * S - 1)))  # the DFMA trick gives exactly the offset integer
    return X, [(Z >> (8 * k)) & 255 for k in range(S)]


def g1_b_digits(b, S, e):
    """GEMM-1's B digits: Y = rint(b 2^(8S-2-e)), balanced base-256 digits d_i = byte_i(Y + C) - 128"""
    sc = 2.0 ** (8 * S - 2 - e)
    C = sum(128 << (8 * k) for k in range(S))
    Z = low_bits(b, sc, M52 + float(C), 8 * S)
    Y = np.rint(np.asarray(b) * sc).astype(np.int64)
    assert np.array_equal(Z, Y + C)
    return Y, [((Z >> (8 * k)) & 255) - 128 for k in range(S)]


def g2_digits(x, S, e):
    """GEMM-2's digits (both operands): balanced base-128, X = rint(x 2^(7S-1-e)) = sum d_i 128^(S-1-i),
    i = 0..S-1 most significant first, d in [-64, 64]"""
    sc = 2.0 ** (7 * S - 1 - e)
    C = sum(64 << (7 * k) for k in range(S))
    Z = low_bits(x, sc, M52 + float(C), 7 * S + 1)
    X = np.rint(np.asarray(x) * sc).astype(np.int64)
    assert np.array_equal(Z, X + C)
    d = [((Z >> (7 * k)) & 127) - 64 for k in range(S - 1)]
    d.append((Z >> (7 * (S - 1))) - 64)  # the top field may reach 128: digit 64
    return X, d[::-1]


def rnd(shape, rng):
    return rng.standard_normal(shape) * np.exp2(rng.integers(-6, 3, size=shape[-1:]))


def exps(a):
    """per column power-of-two scale exponent e: |a| < 2^e (as the kernels take it from the exponent field)"""
    return np.floor(np.log2(np.abs(a).max(axis=0))).astype(int) + 1


@pytest.mark.parametrize("S", [5, 3])
def test_gemm1_offset_digit_algebra_is_exact(S):
    """sum_K X Y = sum_{k,i} 256^(k+i) sum_K u_k d_i - 128 sum_i 256^(S-1+i) sum_K d_i, exactly (all pairs)"""
    rng = np.random.default_rng(S)
    K = 48
    x = rnd((K, 3), rng)
    b = rnd((K, 4), rng)
    ex, eb = exps(x), exps(b)
    for s in range(3):
        X, u = g1_a_digits(x[:, s], S, ex[s])
        for c in range(4):
            Y, d = g1_b_digits(b[:, c], S, eb[c])
            exact = sum(int(p) * int(q) for p, q in zip(X, Y))
            pairs = sum(256 ** (k + i) * int(np.dot(u[k].astype(object), d[i].astype(object)))
                        for k in range(S) for i in range(S))
            corr = 128 * sum(256 ** (S - 1 + i) * int(d[i].sum()) for i in range(S))
            assert pairs - corr == exact
            assert all(0 <= int(v.min()) and int(v.max()) <= 255 for v in u)
            assert all(-128 <= int(v.min()) and int(v.max()) <= 127 for v in d)


@pytest.mark.parametrize("S,bound", [(5, 2.0 ** -37), (3, 2.0 ** -21)])
def test_gemm1_truncated_product_error(S, bound):
    """the kept pairs k + i >= S - 2 (with the offset correction) give sum x b to within ~bound of the scales
    per term (nl_i8.cu: ~2^-38 for S = 5)"""
    rng = np.random.default_rng(10 + S)
    K = 256
    x = rnd((K, 1), rng)[:, 0]
    b = rnd((K, 1), rng)[:, 0]
    ex, eb = exps(x[:, None])[0], exps(b[:, None])[0]
    X, u = g1_a_digits(x, S, ex)
    Y, d = g1_b_digits(b, S, eb)
    acc = 0
    for k in range(S):
        for i in range(S):
            if k + i >= S - 2:
                acc += 256 ** (k + i) * int(np.dot(u[k].astype(object), d[i].astype(object)))
    acc -= 128 * sum(256 ** (S - 1 + i) * int(d[i].sum()) for i in range(S))
    got = acc * 2.0 ** (ex + eb - (16 * S - 4))
    want = float(np.dot(x, b))
    assert abs(got - want) <= K * bound * 2.0 ** (ex + eb)
    assert abs(got - want) > 0  # the truncation is real (the test would not notice a no-op)


def test_gemm2_balanced_digits_and_error():
    """GEMM-2: X = sum_i d_i 128^(S-1-i) exactly; the 21 kept pairs i + j <= S - 1 (0-based) give the product to
    ~2^-40 of the scales per term (nl_i8.cu header)"""
    S = 6
    rng = np.random.default_rng(7)
    K = 128
    x = rnd((K, 1), rng)[:, 0]
    w = rnd((K, 1), rng)[:, 0]
    ex, ew = exps(x[:, None])[0], exps(w[:, None])[0]
    X, dx = g2_digits(x, S, ex)
    W, dw = g2_digits(w, S, ew)
    assert np.array_equal(sum(dx[i] * 128 ** (S - 1 - i) for i in range(S)), X)
    assert all(np.abs(v).max() <= 64 for v in dx + dw)
    acc = sum(128 ** (2 * S - 2 - i - j) * int(np.dot(dx[i].astype(object), dw[j].astype(object)))
              for i in range(S) for j in range(S) if i + j <= S - 1)
    assert sum(1 for i in range(S) for j in range(S) if i + j <= S - 1) == 21
    got = acc * 2.0 ** (ex + ew - 2 * (7 * S - 1))
    want = float(np.dot(x, w))
    assert abs(got - want) <= K * 2.0 ** -39 * 2.0 ** (ex + ew)


def test_gemm1_sp_fp32_digit_trick():
    """The SP GEMM-1's digits from FP32 values (g1_bytes3f): the float bits of v*sc + 1.5 2^23, plus 2^22, hold
    the offset-binary X + 2^23 (X = rint(v sc), |X| <= 2^22) in their low 24 bits -- the same bytes as the
    FP64 form with g1_madd_a<3> -- including both ends X = -2^22 and X = +2^22 (where the float reaches 2^24 and
    its exponent's low bit becomes the 2^23 bit)."""
    rng = np.random.default_rng(7)
    e = -3  # tau = 2^e > max |v|
    sc = np.float32(2.0 ** (22 - e))
    v = rng.uniform(-1, 1, 200000).astype(np.float32) * np.float32(2.0 ** e)
    edge = (np.array([-2.0 ** 22, 2.0 ** 22, -2.0 ** 22 + 1, 2.0 ** 22 - 1, 0.5, -0.5, 1.5, -1.5, 0.0]) /
            float(sc)).astype(np.float32)
    v = np.concatenate([v, edge])
    f = v * sc + np.float32(12582912.0)  # v*sc exact (power of two); the add rounds to nearest even = rint
    assert f.dtype == np.float32
    low = (f.view(np.uint32).astype(np.int64) + (1 << 22)) & ((1 << 24) - 1)
    X = np.rint(v.astype(np.float64) * float(sc)).astype(np.int64)
    assert np.abs(X).max() <= 1 << 22
    assert np.array_equal(low, X + (1 << 23))
    # the same three bytes as the FP64 route of the 3-digit scheme
    Xd, bytes_d = g1_a_digits(v.astype(np.float64), 3, e)
    assert np.array_equal(Xd, X)
    for k in range(3):
        assert np.array_equal((low >> (8 * k)) & 255, bytes_d[k])
