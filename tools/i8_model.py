"""Numerical model of the int8-digit (Ozaki-type) GEMM-2 of nl_i8.cu, in numpy (exact integer digit
products, FP64 recombination), against the FP64 product: prints the relative error of B @ W for the
digit schemes considered.  python tools/i8_model.py"""
import numpy as np


def digits(M, S, bits8):
    """per-row power-of-two scale (max|M_row| < 2^e) and S digits of M / 2^e along axis 1"""
    mx = np.abs(M).max(axis=1)
    e = np.where(mx > 0, np.frexp(mx)[1], 0)
    x = M / np.ldexp(1.0, e)[:, None]
    ds = []
    if bits8:  # first digit signed floor(128 x) in [-128, 127], then unsigned floor(256 r) in [0, 255]
        d = np.floor(x * 128); r = x * 128 - d; ds.append(d)
        for _ in range(1, S):
            d = np.floor(r * 256); r = r * 256 - d; ds.append(d)
        w = [2.0 ** (-7 - 8 * i) for i in range(S)]
    else:  # rint(64 x) in [-64, 64], then rint(128 r)
        d = np.rint(x * 64); r = x * 64 - d; ds.append(d)
        for _ in range(1, S):
            d = np.rint(r * 128); r = r * 128 - d; ds.append(d)
        w = [2.0 ** (-6 - 7 * i) for i in range(S)]
    return np.array(ds), w, np.ldexp(1.0, e)


def emulate(B, W, S, bits8):
    bd, bw, sb = digits(B, S, bits8)
    wd, ww, sw = digits(W.T, S, bits8)
    out = np.zeros((B.shape[0], W.shape[1]))
    for i in range(S):
        for j in range(S):
            if i + j > S - 1:  # keep pairs with i + j <= S + 1 (1-based)
                continue
            P = bd[i].astype(np.int64) @ wd[j].T.astype(np.int64)
            assert np.abs(P).max() < 2 ** 31 / S
            out += P.astype(np.float64) * (bw[i] * ww[j])
    return out * sb[:, None] * sw[None, :]


if __name__ == "__main__":
    rng = np.random.default_rng(0)
    R, K, N = 4000, 128, 128
    B = rng.standard_normal((R, K)) * rng.uniform(0.1, 10, size=(R, 1))
    W = rng.standard_normal((K, N)) * 1e-3
    ex = B @ W
    for S, b8 in ((5, False), (6, False), (4, True), (5, True)):
        e = emulate(B, W, S, b8)
        print(f"S={S} {'8-bit' if b8 else '7-bit'} digits ({S * (S + 1) // 2} digit-pair GEMMs): "
              f"max rel {np.abs(e - ex).max() / np.abs(ex).max():.2e}  fro rel "
              f"{np.linalg.norm(e - ex) / np.linalg.norm(ex):.2e}")
