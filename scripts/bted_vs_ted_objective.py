"""how much of TED's objective does batching (Alg. 2) give up?

On one knob pool of P points, compare the selected sets S of
  * TED on the whole pool (Alg. 1, un-batched),
  * BTED with B batches of M = P / B points (Alg. 2),
  * uniform random sampling (the AutoTVM default initialisation),
by the objective TED minimises, Tr K^(S) = Tr K - Tr(K_:S (K_SS + mu I)^-1 K_S:)
over the WHOLE pool (fp64, closed form from the features), and time each.
Usage (GPU): python scripts/bted_vs_ted_objective.py [P] [B] [m]
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import scipy.linalg as sla

import paper_conf_date_sunbg021_b200 as bt
from oracle.closed_form import gram_columns
from synth import KnobSpace, WORKLOADS, make_pool, median_gamma

P = int(sys.argv[1]) if len(sys.argv) > 1 else 65536
B = int(sys.argv[2]) if len(sys.argv) > 2 else 4
m = int(sys.argv[3]) if len(sys.argv) > 3 else 64
MU = float(np.float32(0.1))
_, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), P, 7)
g = median_gamma(X, 7)


def objective(S):
    KS = gram_columns(X, S, g)                       # P x |S| fp64
    A = KS[S, :] + MU * np.eye(len(S))
    Wt = sla.solve(A, KS.T, assume_a="pos")           # |S| x P
    return float(P - np.einsum("ij,ji->", KS, Wt))    # Tr K = P (RBF: k(v,v) = 1)


out = {"P": P, "B": B, "M": P // B, "m": m, "mu": MU, "gamma": g, "objective": "Tr K^(S) over the whole pool"}
with bt.CandidateSet(X, g, num_batches=B, seed=3) as cs:
    cs.select(m, MU)                                    # warm-up (graph capture)
    t0 = time.perf_counter(); S_ted, _ = cs.select(m, MU); t_ted = time.perf_counter() - t0
    cs.run_batches(P // B, m, MU)
    t0 = time.perf_counter(); S_bted, _ = cs.run_batches(P // B, m, MU); t_bted = time.perf_counter() - t0
rng = np.random.default_rng(0)
S_rand = np.sort(rng.choice(P, m, replace=False))
out["TED_full"] = {"objective": objective(S_ted), "seconds": t_ted}
out["BTED"] = {"objective": objective(S_bted), "seconds": t_bted}
out["random"] = {"objective": objective(S_rand)}
out["trace_K"] = float(P)
print(json.dumps(out, indent=1))
