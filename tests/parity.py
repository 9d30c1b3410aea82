"""Parity protocol between the CUDA path and the fp64 oracle (DESIGN.md
"Parity protocol"; the rule is BASELINE.json north_star's):

  P1  at every step the GPU's fp32 score of its pick s_t is within 1e-5
      relative of the oracle's fp64 score of s_t, given the same history;
  P2  where the oracle's top-two gap over unselected points exceeds 1e-6
      relative, s_t is exactly the oracle's argmax; otherwise s_t must be a
      near-tie: score64(s_t) >= (1 - 1e-5) * max64;
  P3  the oracle follows the GPU's history (teacher forcing), so a legitimate
      near-tie choice does not cascade.
"""
import numpy as np

SCORE_RTOL = 1e-5
GAP_EXACT = 1e-6
GAP_K4 = 1e-9       # with K4 every decision within 2e-5 is taken in fp64
REPORT = []          # per-call summaries; written by tests/conftest.py when BTED_PARITY_REPORT is set


def check_ted(gpu_idx, gpu_score, trace, label="", gap_exact=GAP_EXACT):
    """trace: oracle TedTrace run with forced = gpu_idx.  Returns #near-tie steps.
    gap_exact: P2 threshold; 1e-6 is the north_star rule, K4-refined engines
    (packed / implicit) are held to GAP_K4 (the fp64 decision itself)."""
    gpu_idx = np.asarray(gpu_idx, dtype=np.int64)
    gpu_score = np.asarray(gpu_score, dtype=np.float64)
    o_idx, o_score, o_arg, o_max, o_gap = trace.as_arrays() if hasattr(trace, "as_arrays") else trace
    assert np.array_equal(o_idx, gpu_idx), f"{label}: oracle was not forced along the GPU history"
    assert len(set(gpu_idx.tolist())) == len(gpu_idx), f"{label}: a point was selected twice"
    near = 0
    max_rel = 0.0
    for t in range(len(gpu_idx)):
        if gpu_score is not None and len(gpu_score):
            rel = abs(gpu_score[t] - o_score[t]) / max(abs(o_score[t]), 1e-300)
            max_rel = max(max_rel, rel)
            assert rel <= SCORE_RTOL, f"{label} P1 step {t}: gpu {gpu_score[t]!r} vs fp64 {o_score[t]!r} rel {rel:.3e}"
        if o_gap[t] > gap_exact:
            assert gpu_idx[t] == o_arg[t], (f"{label} P2 step {t}: gpu picked {gpu_idx[t]}, oracle argmax {o_arg[t]}"
                                           f" (gap {o_gap[t]:.3e})")
        else:
            near += 1
            assert o_score[t] >= (1 - SCORE_RTOL) * o_max[t], f"{label} P2 near-tie step {t}"
    gaps = np.asarray(o_gap, dtype=np.float64)
    REPORT.append({"label": label, "steps": int(len(gpu_idx)), "max_rel_score_err": float(max_rel),
                   "near_ties": int(near), "min_gap": float(gaps[np.isfinite(gaps)].min()) if np.isfinite(gaps).any() else None,
                   "steps_gap_below_1e-5": int((gaps <= 1e-5).sum())})
    return near


def ulp32(x):
    """Spacing of fp32 numbers at |x| (ulp), elementwise."""
    x = np.abs(np.asarray(x, dtype=np.float64)).astype(np.float32)
    return np.spacing(x).astype(np.float64)
