"""K4 cost on the paper config: kernel list under ncu (5 calls, K4 on)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import paper_conf_date_sunbg021_b200 as bt
from synth import config_pool
X, g, cfg = config_pool("paper")
mu = float(np.float32(cfg["mu"]))
with bt.CandidateSet(X, g, num_batches=cfg["B"], seed=cfg["seed"]) as cs:
    for _ in range(5):
        cs.run_batches(cfg["M"], cfg["m"], mu)
