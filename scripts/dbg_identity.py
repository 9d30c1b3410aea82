import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
N = int(sys.argv[1]); flags = int(sys.argv[2])
X = (np.arange(N, dtype=np.float32) * 100.0)[:, None]
with bt.CandidateSet(X, 1.0, flags=flags) as cs:
    L.bted_reset_stats(cs.ctx)
    idx, sc = cs.select(64, float(np.float32(0.1)))
    print(idx[:10], sc[:3], L.bted_get_stats(cs.ctx))
