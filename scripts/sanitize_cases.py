"""Small runs of every engine for compute-sanitizer.
Usage: python scripts/sanitize_cases.py <case>   (see CASES)"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import paper_conf_date_sunbg021_b200 as bt  # noqa: E402
from paper_conf_date_sunbg021_b200 import _lib as L  # noqa: E402
from synth import KnobSpace, WORKLOADS, make_pool, median_gamma, config_pool  # noqa: E402

MU = float(np.float32(0.1))
NS = L.BTED_FLAG_NO_SMALL


def knob(N, seed=3):
    _, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), N, seed)
    return X, median_gamma(X, seed)


def sel(N, m, flags=0, **kw):
    X, g = knob(N, N)
    with bt.CandidateSet(X, g, flags=flags, **kw) as cs:
        return cs.select(m, MU)


CASES = {
    "toy": lambda: sel(256, 16),                                        # cluster kernel, C = 1
    "tiny64": lambda: sel(64, 64),                                      # ted_tiny_kernel (N <= 64)
    "tiny33": lambda: sel(33, 20),
    "cluster500": lambda: sel(500, 16),
    "cluster940": lambda: sel(940, 16),
    "implicit4096": lambda: sel(4096, 8, NS),
    "persistent4096": lambda: sel(4096, 8, NS | L.BTED_FLAG_PERSISTENT_LOOP),
    "packed4096": lambda: sel(4096, 8, NS | L.BTED_FLAG_LITERAL),
    "packedtma4096": lambda: sel(4096, 8, NS | L.BTED_FLAG_LITERAL | L.BTED_FLAG_TMA),
    "dense4096": lambda: sel(4096, 8, NS | L.BTED_FLAG_DENSE),
    "k4full2048": lambda: bt.CandidateSet((np.arange(2048, dtype=np.float32) * 100)[:, None], 1.0,
                                          flags=NS).select(4, MU),
    "recompute4096": lambda: sel(4096, 8, NS | L.BTED_FLAG_RECOMPUTE),       # rc_pass.cuh (TMEM, tcgen05)
    "recompute_guard": lambda: bt.CandidateSet((np.arange(2048, dtype=np.float32) * 100)[:, None], 1.0,
                                               flags=NS | L.BTED_FLAG_RECOMPUTE).select(4, MU),
    "tileshard3": lambda: sel(3001, 8, L.BTED_FLAG_LOOPBACK, num_devices=3),
    "rowbands2": lambda: sel(3001, 8, L.BTED_FLAG_LOOPBACK | L.BTED_FLAG_DENSE, num_devices=2),
    "bands_literal2": lambda: sel(3001, 8, L.BTED_FLAG_LOOPBACK | L.BTED_FLAG_DENSE, num_devices=2, norm_mode=1),
}


def run_batches():
    X, g = knob(20000, 5)
    with bt.CandidateSet(X, g, num_batches=3, seed=1, flags=NS) as pool:
        pool.run_batches(1024, 8, MU)
    with bt.CandidateSet(X, g, num_batches=3, seed=1) as pool:            # small batches: cluster kernels
        pool.run_batches(300, 16, MU)


CASES["batches"] = run_batches


def run_tiny_batches():
    X, g = knob(5000, 7)
    with bt.CandidateSet(X, g, num_batches=5, seed=2) as pool:            # 5 tiny batch TEDs, merge of <= 100
        pool.run_batches(50, 20, MU)


CASES["tinybatches"] = run_tiny_batches

if __name__ == "__main__":
    for name in sys.argv[1:]:
        CASES[name]()
        print(f"{name} ok")
