"""Full-protocol parity at the BASELINE.json batch sizes:
every step of every TED checked (P1 + P2 with teacher forcing, tests/parity.py)
against an fp64 oracle that scores ALL points at every step.

  * N = 32768  vgg16 batch 0 (dense C oracle, 8.6 GB of host RAM)
  * N = 32768  one ResNet-50 1x1 node and one MobileNet-v2 depthwise node of the
               wholemodel config (some knob features are identically 0 there)
  * N = 65536  the oversized batch (O2 matrix-free oracle; marked slow)
  * N = 16384  the resnet18 bench batch with exact and 1e-4-perturbed twins of
               its 256 best points written over random rows: near ties between
               CTAs on most steps, so K4 must fire at the bench size.
The GPU side runs the launch configuration bench.py times (the default
implicit engine, CUDA graphs, K4 on); the packed literal engine is checked
at N = 32768 as well.
"""
import numpy as np
import pytest

import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
from oracle import dense, matfree
from oracle.sampling import sample_batches as oracle_sample_batches
from synth import config_pool, whole_model_nodes, whole_model_pools
from tests.parity import check_ted, GAP_K4

pytestmark = pytest.mark.gpu
MU = float(np.float32(0.1))
PACKED = L.BTED_FLAG_NO_SMALL | L.BTED_FLAG_LITERAL


@pytest.fixture(scope="module", autouse=True)
def _gpu(need_gpu):
    yield


def _select(X, g, m, flags=0):
    with bt.CandidateSet(X, g, flags=flags) as cs:
        L.bted_reset_stats(cs.ctx)
        idx, sc = cs.select(m, MU)
        st = L.bted_get_stats(cs.ctx)
    return idx, sc, st


def test_vgg16_batch0_n32768_full_protocol():
    X, g, cfg = config_pool("vgg16")
    M, m, B, seed = cfg["M"], cfg["m"], cfg["B"], cfg["seed"]
    V = oracle_sample_batches(X.shape[0], M, B, seed)[0]
    Xb = X[V]
    idx, sc, _ = _select(Xb, g, m)
    check_ted(idx, sc, dense.ted(Xb, g, MU, m, forced=idx), "vgg16-b0-32768-implicit", gap_exact=GAP_K4)
    # the batch TED inside Alg. 2 (batch 0 of 8, round-robin stride 8) is that same TED
    with bt.CandidateSet(X, g, num_batches=B, seed=seed) as pool:
        w = np.empty(m, np.int64)
        pool.batch_teds(M, m, MU, 0, B, w)
    assert np.array_equal(w, V[idx])
    idx2, sc2, _ = _select(Xb, g, m, PACKED)
    tr2 = dense.ted(Xb, g, MU, m, forced=idx2) if not np.array_equal(idx2, idx) else None
    if tr2 is not None:
        check_ted(idx2, sc2, tr2, "vgg16-b0-32768-packed", gap_exact=GAP_K4)
    else:
        np.testing.assert_allclose(sc2, sc, rtol=1e-5)


@pytest.mark.parametrize("node", [1, 21], ids=["resnet50_n1_1x1", "mobilenetv2_n1_depthwise"])
def test_wholemodel_nodes_n32768_full_protocol(node):
    wl = whole_model_nodes()[node]
    assert (wl.kh, wl.kw) == (1, 1) or wl.depthwise
    (_, X, g), = whole_model_pools(which=[node])
    assert np.any(np.all(X == 0.0, axis=0))                  # knob features that are identically 0
    M, m, seed = 32768, 64, 5000 + node                      # bench.py: seed = cfg seed + node
    V = oracle_sample_batches(X.shape[0], M, 4, seed)[0]
    Xb = X[V]
    idx, sc, st = _select(Xb, g, m)
    check_ted(idx, sc, dense.ted(Xb, g, MU, m, forced=idx), f"{wl.name}-32768", gap_exact=GAP_K4)
    print(f"{wl.name}: K4 refined {st['refined_steps']} (full {st['full_refined_steps']}), "
          f"corrected {st['corrected_steps']}")


@pytest.mark.slow
def test_oversized_n65536_full_protocol_o2():
    X, g, cfg = config_pool("oversized")
    V = oracle_sample_batches(X.shape[0], cfg["M"], 1, cfg["seed"])[0]
    Xb = X[V]
    m = cfg["m"]
    idx, sc, _ = _select(Xb, g, m)
    tr = matfree.ted(Xb, g, MU, m, forced=idx)
    check_ted(idx, sc, tr, "oversized-65536-o2", gap_exact=GAP_K4)


def test_resnet18_bench_batch_with_near_ties():
    """The bench batch (N = 16384) rebuilt so that near ties are everywhere:
    the 256 points the TED would pick first get an exact twin and a twin
    perturbed by 1e-4 in one feature, written over random rows (3 % of the
    batch), so that almost every step ties exactly (twins) and nearly (the
    perturbed copies) between candidates in different CTAs.  K4 must fire
    on most steps and P2 hold at the fp64 gap."""
    X, g, cfg = config_pool("resnet18")
    V = oracle_sample_batches(X.shape[0], cfg["M"], 1, cfg["seed"])[0]
    Xb = X[V].copy()
    N, m = Xb.shape[0], cfg["m"]
    top, _, _ = _select(Xb, g, 256)                           # the points that matter
    rng = np.random.default_rng(1818)
    free_rows = np.setdiff1d(np.arange(N), top)
    rows = rng.choice(free_rows, 2 * len(top), replace=False)
    Xb[rows[: len(top)]] = Xb[top]                           # exact twins
    Xb[rows[len(top):]] = Xb[top]
    Xb[rows[len(top):], rng.integers(0, Xb.shape[1], len(top))] += np.float32(1e-4)   # near twins
    for flags, name in ((0, "implicit"), (PACKED, "packed")):
        idx, sc, st = _select(Xb, g, m, flags)
        tr = dense.ted(Xb, g, MU, m, forced=idx)
        check_ted(idx, sc, tr, f"resnet18-neartie-{name}", gap_exact=GAP_K4)
        near = int(np.sum(np.array(tr.gap) <= 1e-5))
        print(f"near-tie resnet18 {name}: K4 refined {st['refined_steps']} (full {st['full_refined_steps']}), "
              f"corrected {st['corrected_steps']}, oracle gaps <= 1e-5: {near} of {m}")
        assert st["refined_steps"] >= m // 2, "K4 did not fire on most steps"


@pytest.mark.slow
def test_large_n131072_tile_sharded_4_devices_full_protocol_o2():
    """the un-batched TED on N = 131072,
    tile-sharded over P = 4 devices through the C ABI (num_devices = 4, logical
    devices on the one GPU: the same kernels and peer exchange), P1 on every
    pick and P2 at every step against the O2 oracle (upper-triangle cache,
    68.7 GB of host RAM)."""
    X, g, cfg = config_pool("large")
    V = oracle_sample_batches(X.shape[0], cfg["M"], 1, cfg["seed"])[0]
    Xb = X[V]
    m = cfg["m"]
    with bt.CandidateSet(Xb, g, num_devices=4, flags=L.BTED_FLAG_LOOPBACK) as cs:
        idx, sc = cs.select(m, MU)
    tr = matfree.ted(Xb, g, MU, m, forced=idx)
    check_ted(idx, sc, tr, "large-131072-4shards-o2", gap_exact=GAP_K4)
