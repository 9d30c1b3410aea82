"""Run-to-run determinism of every engine: the same select repeated on fresh contexts must give
bitwise the same picks and fp32 scores.  The steps are PDL-chained kernels whose early parts read
the previous kernels' outputs before their programmatic waits, so an ordering mistake (a kernel
letting its dependent launch before its own inputs are complete) shows up as run-to-run
differences -- this caught one in the recomputing pass (a worker group without a tile triggered
the dependent launch at once)."""
import numpy as np
import pytest

import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
from synth import KnobSpace, WORKLOADS, make_pool, median_gamma

pytestmark = pytest.mark.gpu
MU = float(np.float32(0.1))
NS = L.BTED_FLAG_NO_SMALL
ENGINES = [("implicit", NS), ("recompute", NS | L.BTED_FLAG_RECOMPUTE), ("packed", NS | L.BTED_FLAG_LITERAL),
           ("dense", NS | L.BTED_FLAG_DENSE), ("persistent", NS | L.BTED_FLAG_PERSISTENT_LOOP), ("auto", 0)]


@pytest.fixture(scope="module", autouse=True)
def _gpu(need_gpu):
    yield


@pytest.mark.parametrize("name,flags", ENGINES, ids=[e[0] for e in ENGINES])
@pytest.mark.parametrize("N,m", [(64, 64), (128, 64), (500, 32), (1000, 24), (4099, 40)])
def test_repeated_selects_are_bitwise_identical(name, flags, N, m):
    _, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), N, 3)
    g = median_gamma(X, 2)
    ref = None
    for _ in range(6):
        with bt.CandidateSet(X, g, flags=flags) as cs:
            idx, sc = cs.select(m, MU)
        cur = (idx.tolist(), sc.view(np.uint32).tolist())
        if ref is None:
            ref = cur
        assert cur == ref, f"{name} N={N}: a repeated select differs"
