"""The multi-GPU half of the C-ABI boundary: one ctx
with params.num_devices = G drives G devices from one process.

  * bted_run_batches: batch b on device b mod G (Alg. 2 l.1-4 are independent,
    PAPER.md:150, 156), winners gathered to device 0 for the merge (l.5-6);
  * bted_select: one candidate set tile-sharded over P devices, the per-step
    sum of the partial q = K l exchanged through peer memory (fused into the
    score kernel) or NCCL (BTED_FLAG_NCCL).

The test box has one GPU, so the multi-device paths run with
BTED_FLAG_LOOPBACK (P logical devices on one GPU, one stream: the same kernels
and exchange protocol), and NCCL with a one-device communicator.  Results must
be bitwise those of the existing drivers and pass P1/P2 against the oracle.
"""
import os

import numpy as np
import pytest

import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
from oracle import dense
from synth import KnobSpace, WORKLOADS, make_pool, median_gamma
from tests.parity import check_ted, GAP_K4

pytestmark = pytest.mark.gpu
MU = float(np.float32(0.1))
LOOP = L.BTED_FLAG_LOOPBACK


@pytest.fixture(scope="module", autouse=True)
def _gpu(need_gpu):
    yield


def knob(N, d=16, seed=3):
    _, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], d), N, seed)
    return X


@pytest.mark.parametrize("N,P,d", [(3001, 2, 16), (4096, 3, 16), (2500, 4, 12), (1100, 5, 16)])
def test_select_tile_sharded_over_devices_equals_driver(N, P, d):
    import torch
    from paper_conf_date_sunbg021_b200.dist import isharded_select_loopback
    X = knob(N, d=d, seed=N + P)
    g = median_gamma(X, P)
    m = 40
    with bt.CandidateSet(X, g, num_devices=P, flags=LOOP) as cs:
        idx, sc = cs.select(m, MU)
        idx2, sc2 = cs.select(m, MU)                         # idempotent, deterministic
    assert np.array_equal(idx, idx2) and np.array_equal(sc.view(np.uint32), sc2.view(np.uint32))
    dev = torch.device("cuda", 0)
    ref_idx, ref_sc = isharded_select_loopback(X, g, P, m, MU, dev, torch.cuda.Stream(dev))
    assert np.array_equal(idx, ref_idx)                      # rank-order sums on both sides: bitwise
    assert np.array_equal(sc.view(np.uint32), ref_sc.view(np.uint32))
    check_ted(idx, sc, dense.ted(X, g, MU, m, forced=idx), f"multidev-select N={N} P={P}", gap_exact=GAP_K4)


def test_select_multidev_k4_exact_ties():
    X = knob(2500, seed=43)
    X = np.concatenate([X, X[::5]], axis=0)                  # exact duplicate pairs
    g = median_gamma(X, 43)
    with bt.CandidateSet(X, g, num_devices=3, flags=LOOP) as cs:
        L.bted_reset_stats(cs.ctx)
        idx, sc = cs.select(64, MU)
        st = L.bted_get_stats(cs.ctx)
    assert st["refined_steps"] > 0
    check_ted(idx, sc, dense.ted(X, g, MU, 64, forced=idx), "multidev-k4", gap_exact=GAP_K4)


@pytest.mark.parametrize("G", [2, 3])
def test_run_batches_round_robin_over_devices_equals_one_device(G):
    P, M, B, m, seed = 30000, 1024, 5, 16, 11
    X = knob(P, seed=4)
    g = median_gamma(X, 4)
    with bt.CandidateSet(X, g, num_batches=B, seed=seed) as one:
        sel1, bidx1 = one.run_batches(M, m, MU)
    with bt.CandidateSet(X, g, num_batches=B, seed=seed, num_devices=G, flags=LOOP) as many:
        selG, bidxG = many.run_batches(M, m, MU)
        selG2, _ = many.run_batches(M, m, MU)
    assert np.array_equal(bidxG, bidx1)
    assert np.array_equal(selG, sel1) and np.array_equal(selG2, sel1)


def test_run_batches_over_devices_paper_scale_cluster_kernel():
    """M = 500 batches (the cluster kernel) with their K4 resolved per device."""
    X = knob(20000, seed=21)
    g = median_gamma(X, 21)
    with bt.CandidateSet(X, g, num_batches=10, seed=2021) as one:
        sel1, b1 = one.run_batches(500, 64, MU)
    with bt.CandidateSet(X, g, num_batches=10, seed=2021, num_devices=4, flags=LOOP) as many:
        selG, bG = many.run_batches(500, 64, MU)
    assert np.array_equal(b1, bG) and np.array_equal(sel1, selG)


def test_nccl_exchange_single_device_communicator():
    """BTED_FLAG_NCCL with a one-device communicator (the box has one GPU): the
    q all-reduce runs through ncclAllReduce; with one rank it is the identity,
    so the result is bitwise the peer-exchange engine's at P = 1."""
    import torch
    from paper_conf_date_sunbg021_b200.dist import isharded_select_loopback
    X = knob(3001, seed=9)
    g = median_gamma(X, 9)
    with bt.CandidateSet(X, g, num_devices=1, flags=L.BTED_FLAG_NCCL) as cs:
        idx, sc = cs.select(32, MU)
    dev = torch.device("cuda", 0)
    ridx, rsc = isharded_select_loopback(X, g, 1, 32, MU, dev, torch.cuda.Stream(dev))
    assert np.array_equal(idx, ridx) and np.array_equal(sc.view(np.uint32), rsc.view(np.uint32))


def test_stalled_peer_fails_with_enccl_then_estate(monkeypatch):
    """A device that never publishes its step (BTED_DEBUG_DROP_PUBLISH): the
    other devices' flag waits time out (BTED_PEER_TIMEOUT_MS) and the call fails
    with BTED_ENCCL instead of hanging; the ctx is then poisoned (ESTATE)."""
    monkeypatch.setenv("BTED_PEER_TIMEOUT_MS", "200")
    monkeypatch.setenv("BTED_DEBUG_DROP_PUBLISH", "1")
    X = knob(1500, seed=5)
    with bt.CandidateSet(X, median_gamma(X, 5), num_devices=2, flags=LOOP) as cs:
        with pytest.raises(bt.BtedError) as e:
            cs.select(16, MU)
        assert e.value.status == 4, str(e.value)             # BTED_ENCCL
        with pytest.raises(bt.BtedError) as e2:
            cs.select(16, MU)
        assert e2.value.status == 6                          # BTED_ESTATE


def test_multidev_arguments_and_update():
    X = knob(2000, seed=6)
    g = median_gamma(X, 6)
    import torch
    ndev = torch.cuda.device_count()
    with pytest.raises(bt.BtedError) as e:
        bt.CandidateSet(X, g, num_devices=ndev + 1)          # more devices than visible
    assert e.value.status == 1
    with pytest.raises(bt.BtedError) as e:
        bt.CandidateSet(X, g, num_devices=2, flags=LOOP | L.BTED_FLAG_NCCL)
    assert e.value.status == 1
    X2 = knob(2000, seed=7)
    with bt.CandidateSet(X, g, num_devices=2, flags=LOOP) as cs, bt.CandidateSet(X2, g) as ref:
        a, _ = cs.select(24, MU)
        cs.update(X2)                                        # replicas rebuilt from the new features
        b, _ = cs.select(24, MU)
        r, _ = ref.select(24, MU)
    check_ted(b, [], dense.ted(X2, g, MU, 24, forced=b), "multidev-update", gap_exact=GAP_K4)
    assert not np.array_equal(a, b)
    k = int(np.argmax(b != r)) if not np.array_equal(b, r) else 24
    assert k == 24 or dense.ted(X2, g, MU, 24, forced=b).gap[k] <= 1e-5


@pytest.mark.parametrize("N,P", [(3000, 2), (3001, 3), (1024, 4)])
def test_select_row_bands_over_devices_bit_identical_to_dense(N, P):
    """BTED_FLAG_DENSE with P devices: row bands, pivot slices gathered and band
    maxima max-reduced through peer memory; bitwise the dense single-GPU select."""
    DENSE = L.BTED_FLAG_DENSE | L.BTED_FLAG_NO_SMALL
    X = knob(N, seed=N + P)
    g = median_gamma(X, P)
    with bt.CandidateSet(X, g, flags=DENSE) as one:
        idx, sc = one.select(24, MU)
    with bt.CandidateSet(X, g, flags=DENSE | LOOP, num_devices=P) as many:
        i2, s2 = many.select(24, MU)
    assert np.array_equal(i2, idx) and np.array_equal(s2.view(np.uint32), sc.view(np.uint32))


@pytest.mark.parametrize("P", [2, 3])
def test_select_row_bands_literal_column_norms_equal_driver(P):
    """norm_mode = 1: the bands' partial column norms summed (rank order) every
    step -- bitwise dist.ShardedTed's literal mode on the loopback driver, and
    P1/P2 against the oracle."""
    import torch
    from paper_conf_date_sunbg021_b200.dist import sharded_select_loopback
    X = knob(3001, seed=3001 + 7 * P)
    g = median_gamma(X, P)
    num = P
    with bt.CandidateSet(X, g, flags=L.BTED_FLAG_DENSE | LOOP, num_devices=num, norm_mode=1) as many:
        idx, sc = many.select(24, MU)
    dev = torch.device("cuda", 0)
    ridx, rsc = sharded_select_loopback(X, g, num, 24, MU, dev, torch.cuda.Stream(dev), norm_mode="literal")
    assert np.array_equal(idx, ridx) and np.array_equal(sc.view(np.uint32), rsc.view(np.uint32))
    check_ted(idx, sc, dense.ted(X, g, MU, 24, forced=idx), f"bands-literal P={num}", gap_exact=GAP_K4)


def test_select_row_bands_k4_near_ties():
    X = knob(1800, d=12, seed=53)                            # d = 12: exact duplicates
    X = np.concatenate([X, X[::4]], axis=0)
    g = median_gamma(X, 53)
    with bt.CandidateSet(X, g, flags=L.BTED_FLAG_DENSE | LOOP, num_devices=3) as many:
        L.bted_reset_stats(many.ctx)
        idx, sc = many.select(120, MU)
        st = L.bted_get_stats(many.ctx)
    check_ted(idx, sc, dense.ted(X, g, MU, 120, forced=idx), "bands-k4", gap_exact=GAP_K4)


def test_small_candidate_sets_are_not_sharded():
    """A candidate set the one-kernel cluster TED handles (N <= ~940), or one with
    fewer Gram tiles than devices, runs on the first device alone: bitwise the
    single-device selection."""
    for N in (300, 900):
        X = knob(N, seed=N)
        g = median_gamma(X, N)
        with bt.CandidateSet(X, g) as one, bt.CandidateSet(X, g, num_devices=4, flags=LOOP) as many:
            a, sa = one.select(32, MU)
            b, sb = many.select(32, MU)
        assert np.array_equal(a, b) and np.array_equal(sa.view(np.uint32), sb.view(np.uint32))
