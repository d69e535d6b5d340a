"""S5 reference sampler (TEST INFRASTRUCTURE ONLY -- see oracle/__init__.py).

PAPER.md L131-132 (§3, state_space files): the state space offers "measuring
quantum states" and "sampling from a quantum state to generate measurement
outcomes"; L69: |c_i|^2 is the probability of |i>.  The paper gives no
procedure; the integer fixed-point reading of SURVEY.md §8c-S5 (DESIGN.md,
Readings) makes the result independent of any reduction order:

  p_i = (double)re^2 + (double)im^2       (both products exact in fp64)
  w_i = floor(p_i * 2^62)                 (uint64)
  C_i = inclusive prefix of w over logical index order, T = C_last
  r_s = splitmix64 output #(s+1) from state = seed
  t_s = (r_s * T) >> 64                   (128-bit product)
  out[s] = min{ i : C_i > t_s }
"""
from __future__ import annotations

import numpy as np

from workloads.rqc import splitmix64_nth

TWO62 = float(2 ** 62)


def weights(psi: np.ndarray) -> np.ndarray:
    """w_i = floor(p_i * 2^62) with p_i computed in fp64.

    complex64 input: both products are exact in fp64, one rounding in the sum
    (S5).  complex128 input (NEXT-1, reading R5): p = fl(fl(re^2) + fl(im^2)),
    three separately rounded operations (numpy ufuncs do not contract)."""
    psi = np.asarray(psi)
    if psi.dtype != np.complex128:
        psi = psi.astype(np.complex64)
    re = psi.real.astype(np.float64)
    im = psi.imag.astype(np.float64)
    p = re * re + im * im
    return np.floor(p * TWO62).astype(np.uint64)


def sample(psi_in: np.ndarray, seed: int, n_samples: int):
    """S5 on a complex64 (or complex128) state in logical order.
    Returns (indices uint64, T)."""
    w = weights(psi_in)
    psi = np.asarray(psi_in)
    psum = float(np.sum(psi.real.astype(np.float64) ** 2 + psi.imag.astype(np.float64) ** 2))
    T = int(w.sum(dtype=np.uint64)) if w.size else 0
    if T == 0 or psum >= 3.99:
        raise ValueError("state has zero or excessive total weight (uint64 overflow risk)")
    C = np.cumsum(w, dtype=np.uint64)
    assert int(C[-1]) == T
    t = np.array([(splitmix64_nth(seed, s) * T) >> 64 for s in range(n_samples)], dtype=np.uint64)
    out = np.searchsorted(C, t, side="right").astype(np.uint64)
    return out, T


def exact_probabilities(psi: np.ndarray) -> np.ndarray:
    """|c_i|^2 in fp64 (for statistical checks)."""
    psi = np.asarray(psi, dtype=np.complex128)
    return (psi.real ** 2 + psi.imag ** 2)
