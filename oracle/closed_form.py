"""Matrix-free fp64 scores after a given selected set -- TEST INFRASTRUCTURE ONLY.

For full-size runs (N = 65536: the dense fp64 K would be 34 GB and two sweeps
per step) the tests check SAMPLED outputs one by one.  After the picks
S = (s_1 .. s_t) of Algorithm 1, the deflated matrix is
the Schur complement

    K^(S) = K - K_:S (K_SS + mu I)^-1 K_S:

(pin C2: tests/test_oracle_pins.py checks the literal Alg. 1 deflation
against exactly this formula), so the l.3 score of any candidate v,

    score_v = ||K^(S)_:v||^2 / (K^(S)_vv + mu),

needs only the columns K_:S and K_:v of the RBF Gram matrix, computed here
directly from the features in fp64 (reading A1), plus one t x t solve.
`tests/test_oracle_pins.py::test_closed_form_scores_match_literal` pins this
module against the literal oracle at small N.
"""
from __future__ import annotations

import numpy as np
import scipy.linalg as sla


def gram_columns(X: np.ndarray, cols, gamma: float) -> np.ndarray:
    """K_{:, cols} of the RBF kernel, fp64, direct-difference form (N x len(cols))."""
    X = np.asarray(X, dtype=np.float64)
    cols = np.asarray(cols, dtype=np.int64)
    out = np.empty((X.shape[0], len(cols)))
    for a, c in enumerate(cols):
        diff = X - X[c]
        out[:, a] = np.exp(-float(gamma) * np.einsum("ij,ij->i", diff, diff))
    return out


class ClosedForm:
    """fp64 scores of candidates after a growing selected set S."""

    def __init__(self, X: np.ndarray, gamma: float, mu: float):
        self.X = np.asarray(X, dtype=np.float64)
        self.gamma, self.mu = float(gamma), float(mu)
        self.S: list = []
        self.KS = np.zeros((self.X.shape[0], 0))

    def add(self, s: int):
        """X = X u s (Alg. 1 l.4)."""
        self.S.append(int(s))
        self.KS = np.concatenate([self.KS, gram_columns(self.X, [s], self.gamma)], axis=1)

    def scores(self, cand) -> np.ndarray:
        """score_v for v in cand, given the current S (Alg. 1 l.3 on K^(S))."""
        cand = np.asarray(cand, dtype=np.int64)
        Kv = gram_columns(self.X, cand, self.gamma)              # N x c
        if self.S:
            A = self.KS[self.S, :] + self.mu * np.eye(len(self.S))   # K_SS + mu I
            W = sla.solve(A, self.KS[cand, :].T, assume_a="pos")     # (K_SS + mu I)^-1 K_Sv
            col = Kv - self.KS @ W                                   # K^(S)_:v
        else:
            col = Kv
        diag = col[cand, np.arange(len(cand))]
        return np.einsum("ij,ij->j", col, col) / (diag + self.mu)
