"""Bit-faithful numpy emulation of the int8 tensor-core apply (apply_tci) for
one fused gate, to dissect its error against the exact product: row scaling
2^(22-e), round-to-nearest-even slicing, balanced base-256 digits, the six
kept digit products in exact integers, and the fp32 epilogue.  The W slices
come from the library's own host packer semantics (re-derived here).

usage: python tools/tci_emulate.py            (CPU only; prints the norm change
                                               of the emulation and of each
                                               dropped / rounded component)
"""
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

from workloads import rqc as W


def digits(v):
    v = v.astype(np.int64)
    d2 = ((v + 128) & 255) - 128
    r1 = (v - d2) >> 8
    d1 = ((r1 + 128) & 255) - 128
    d0 = (r1 - d1) >> 8
    return d0, d1, d2


def pack_w(m, fix=True):
    """As pack_wi8: per-column power-of-two scale 2^(22-f), round to nearest,
    then (fix) flip rounding directions, largest entries first, to match the
    column's exact squared norm."""
    D = m.shape[0]
    Wm = np.zeros((2 * D, 2 * D))
    for r in range(D):
        for c in range(D):
            Wm[2 * c, 2 * r] = m[r, c].real
            Wm[2 * c + 1, 2 * r] = -m[r, c].imag
            Wm[2 * c, 2 * r + 1] = m[r, c].imag
            Wm[2 * c + 1, 2 * r + 1] = m[r, c].real
    wi = np.zeros_like(Wm, dtype=np.int64)
    fc = np.zeros(2 * D, dtype=np.float32)
    for n in range(2 * D):
        mx = np.abs(Wm[:, n]).max()
        f = max(math.frexp(mx)[1] if mx > 0 else 0, -100)
        sx = np.ldexp(Wm[:, n], 22 - f)
        col = np.rint(sx).astype(np.int64)
        if fix:
            target = float(sx @ sx)
            cur = float(col.astype(np.float64) @ col)
            for kk in sorted(range(2 * D), key=lambda i: -abs(int(col[i]))):
                s = 1 if sx[kk] > col[kk] else -1
                if abs(sx[kk] - (col[kk] + s)) >= 1.0:
                    continue
                change = float(2 * col[kk] * s + 1)
                if abs(target - cur - change) < abs(target - cur):
                    col[kk] += s
                    cur += change
        wi[:, n] = col
        fc[n] = np.float32(math.ldexp(1.0, f - 14))
    return Wm, wi, fc


def apply_rows(X, wi, fc):
    """X: (groups, 2D) float32 real-expanded rows.  Returns fp32 outputs and parts."""
    mx = np.abs(X).max(axis=1).astype(np.float32)
    E = (mx.view(np.uint32) >> 23).astype(np.int64) & 0xFF
    e = np.maximum(E - 126, -100)
    scale = np.ldexp(np.float32(1.0), (22 - e)).astype(np.float32)
    v = (X.astype(np.float32) * scale[:, None]).astype(np.float64)  # exact (power of two)
    xi = np.rint(v).astype(np.int64)                                   # RNE like the FFMA magic
    a0, a1, a2 = digits(xi)
    b0, b1, b2 = digits(wi)
    S32 = a0 @ b0
    S24 = a0 @ b1 + a1 @ b0
    S16 = a0 @ b2 + a1 @ b1 + a2 @ b0
    tt = S32 * 65536 + S24 * 256 + S16
    srow = np.ldexp(np.float32(1.0), (e - 14)).astype(np.float32)
    y = (tt.astype(np.float32) * srow[:, None]).astype(np.float32) * fc[None, :]
    return y.astype(np.float32), dict(xi=xi, e=e, dropped=(a1 @ b2 + a2 @ b1) * 256 + a2 @ b2)


def main():
    rs = np.random.default_rng(7)
    k = 5
    D = 1 << k
    M = W.haar_unitary(D, rs)
    X = (rs.standard_normal((1 << 15, 2 * D)) / np.sqrt(2 * D * (1 << 15))).astype(np.float32)
    for fix in (False, True):
        Wm, wi, fc = pack_w(M, fix)
        y, parts = apply_rows(X, wi, fc)
        x64 = X.astype(np.float64)
        yex = x64 @ Wm
        n_in = float((x64 ** 2).sum())
        print(f"fix={fix}: norm change / apply (emulated) {float((y.astype(np.float64) ** 2).sum()) / n_in - 1:+.3e}; "
              f"exact-W product {float((yex ** 2).sum()) / n_in - 1:+.3e}")
        # components: slicing of x only (exact W), W quantisation only (exact x)
        e = parts["e"]
        xs = parts["xi"].astype(np.float64) * np.ldexp(1.0, e - 22)[:, None]
        print(f"    x slicing only {float(((xs @ Wm) ** 2).sum()) / n_in - 1:+.3e}; dropped terms mean "
              f"{float(parts['dropped'].mean()):+.3f} (units of 2^(e+f-44))")


if __name__ == "__main__":
    main()


def decompose():
    rs = np.random.default_rng(7)
    D = 32
    M = W.haar_unitary(D, rs)
    X = (rs.standard_normal((1 << 15, 2 * D)) / np.sqrt(2 * D * (1 << 15))).astype(np.float32)
    x64 = X.astype(np.float64)
    n_in = float((x64 ** 2).sum())
    for fix in (False, True):
        Wm, wi, fc = pack_w(M, fix)
        y, parts = apply_rows(X, wi, fc)
        e = parts["e"]
        f = np.array([max(math.frexp(np.abs(Wm[:, n]).max())[1], -100) for n in range(2 * D)])
        colfix = np.ones(2 * D)
        Wq = wi.astype(np.float64) * np.ldexp(1.0, f - 22)[None, :] * colfix[None, :]
        xs = parts["xi"].astype(np.float64) * np.ldexp(1.0, e - 22)[:, None]
        full = xs @ Wq                          # no dropped terms, no final rounding
        dropped = parts["dropped"].astype(np.float64) * np.ldexp(1.0, e - 22)[:, None] * np.ldexp(1.0, f - 22)[None, :]
        kept = full - dropped
        nc = lambda z: float((z ** 2).sum()) / n_in - 1
        print(f"fix={fix}: W quantised only {nc(x64 @ Wq):+.3e}; x sliced + W quantised {nc(full):+.3e}; "
              f"minus dropped terms {nc(kept):+.3e}; + fp32 epilogue {nc(y.astype(np.float64)):+.3e}")


if __name__ == "__main__" and len(sys.argv) > 1 and sys.argv[1] == "decompose":
    decompose()
