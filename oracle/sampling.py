"""Batch sampler of Algorithm 2 line 2 -- TEST INFRASTRUCTURE ONLY.

PAPER.md:156 (Alg. 2 l.2): "Randomly sample a set V_b from V, with |V_b| = M".
The paper fixes neither the distribution's generator nor its seed (reading
A10): uniform without replacement inside a batch, independent
across batches.  Both sides implement the SAME counter-based definition
independently (this file for the oracle, csrc/sample.cu for the CUDA path);
tests/test_sampling*.py check them against each other bit for bit and check
this file against the splitmix64 reference vectors and against the
statistics of uniform sampling without replacement.

Definition:
  splitmix64(z):  z += 0x9E3779B97F4A7C15
                  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9
                  z = (z ^ (z >> 27)) * 0x94D049BB133111EB
                  return z ^ (z >> 31)                 (all mod 2^64)
  h_b       = splitmix64(seed + b * 0xD1B54A32D192ED03)
  key_b(i)  = (splitmix64(h_b + i) & 0xFFFFFFFF00000000) | i,   0 <= i < P < 2^32
  V_b       = the M indices i with the smallest key_b(i), in ascending order of i.
Keys are distinct (their low half is i), so V_b is well defined; choosing the
M smallest of exchangeable random keys is a uniform M-subset.
"""
from __future__ import annotations

import numpy as np

_G = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_BATCH = 0xD1B54A32D192ED03
_HI = np.uint64(0xFFFFFFFF00000000)


def splitmix64(z):
    """splitmix64 output function applied to state z (uint64, wraps mod 2^64)."""
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z + _G
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def batch_keys(P: int, b: int, seed: int) -> np.ndarray:
    hb = splitmix64(np.uint64((int(seed) + int(b) * _BATCH) % (1 << 64)))
    i = np.arange(P, dtype=np.uint64)
    with np.errstate(over="ignore"):
        r = splitmix64(hb + i)
    return (r & _HI) | i


def sample_batches(P: int, M: int, B: int, seed: int) -> np.ndarray:
    """int64 [B][M]: row b = sorted V_b (Alg. 2 l.2)."""
    if not (1 <= M <= P < (1 << 32)) or B < 1:
        raise ValueError("need 1 <= M <= P < 2^32 and B >= 1")
    out = np.empty((B, M), dtype=np.int64)
    for b in range(B):
        keys = batch_keys(P, b, seed)
        part = np.argpartition(keys, M - 1)[:M] if M < P else np.arange(P)
        out[b] = np.sort(part.astype(np.int64))
    return out
