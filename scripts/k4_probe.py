import os, sys, time
sys.path.insert(0, os.getcwd())
import numpy as np
import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
from synth import config_pool
X, g, cfg = config_pool("paper")
mu = float(np.float32(cfg["mu"]))
for flags, lab in [(0, "k4"), (L.BTED_FLAG_NO_REFINE, "no-k4")]:
    with bt.CandidateSet(X, g, num_batches=cfg["B"], seed=cfg["seed"], flags=flags) as cs:
        cs.run_batches(cfg["M"], cfg["m"], mu)
        L.bted_reset_stats(cs.ctx)
        t0 = time.perf_counter()
        for _ in range(20):
            cs.run_batches(cfg["M"], cfg["m"], mu)
        dt = (time.perf_counter() - t0) / 20
        print(lab, "ms per call", round(dt * 1e3, 3), L.bted_get_stats(cs.ctx))
