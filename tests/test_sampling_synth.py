"""CPU pins of the oracle-side batch sampler (Alg. 2 l.2) and of
the synthetic pool generator (Def. 1; space sizes PAPER.md:44)."""
import numpy as np
import pytest
from scipy import stats

from oracle.sampling import splitmix64, sample_batches, batch_keys
from synth import KnobSpace, WORKLOADS, make_pool, config_pool, whole_model_nodes
from synth.knob_pools import ordered_factorizations


def test_splitmix64_reference_vectors():
    # canonical splitmix64 seeded with 0: state advances by the golden gamma,
    # outputs 0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F
    G = 0x9E3779B97F4A7C15
    outs = [int(splitmix64(np.uint64((k * G) % (1 << 64)))) for k in range(3)]
    assert outs == [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]


def test_sample_batches_shape_sorted_distinct_in_range():
    P, M, B = 5000, 700, 6
    out = sample_batches(P, M, B, seed=123)
    assert out.shape == (B, M) and out.dtype == np.int64
    for r in out:
        assert np.all(np.diff(r) > 0) and r[0] >= 0 and r[-1] < P
    assert not np.array_equal(out[0], out[1])          # independent across batches
    assert np.array_equal(out, sample_batches(P, M, B, seed=123))   # deterministic
    assert not np.array_equal(out, sample_batches(P, M, B, seed=124))


def test_sample_batches_matches_key_definition():
    P, M = 3000, 100
    keys = batch_keys(P, 2, 99)
    ref = np.sort(np.argsort(keys, kind="stable")[:M])
    assert np.array_equal(sample_batches(P, M, 3, 99)[2], ref)
    assert np.all((keys & np.uint64(0xFFFFFFFF)) == np.arange(P, dtype=np.uint64))


def test_sample_batches_uniform_inclusion():
    # each index is included with probability M/P; chi-square over 20 bins of
    # counts from 400 batches, and batch-overlap mean = M^2/P
    P, M, B = 2000, 200, 400
    out = sample_batches(P, M, B, seed=7)
    counts = np.bincount(out.ravel(), minlength=P)
    binned = counts.reshape(20, -1).sum(1)
    chi = stats.chisquare(binned)
    assert chi.pvalue > 1e-4
    assert abs(counts.mean() - B * M / P) < 1e-9
    ov = np.mean([len(np.intersect1d(out[i], out[i + 1])) for i in range(0, B - 1, 2)])
    assert abs(ov - M * M / P) < 3.0


def test_sample_all_when_M_equals_P():
    assert np.array_equal(sample_batches(50, 50, 2, 1), np.tile(np.arange(50), (2, 1)))
    with pytest.raises(ValueError):
        sample_batches(10, 11, 1, 0)


def test_space_sizes_match_paper_anchor():
    # PAPER.md:44 "the first optimization node in VGG-16 has approximately
    # 0.2 billion configuration points"
    assert KnobSpace(WORKLOADS["vgg16_conv1_1"]).size == 202_309_632
    assert KnobSpace(WORKLOADS["resnet18_layer1"]).size == 90_316_800
    # PAPER.md:364 "> 50 million configuration points" per node on average
    sizes = [KnobSpace(n).size for n in whole_model_nodes()]
    assert len(sizes) == 40 and np.mean(sizes) > 1e7


def test_factorizations():
    assert len(ordered_factorizations(64, 4)) == 84
    assert len(ordered_factorizations(224, 4)) == 224
    assert all(np.prod(f) == 224 for f in ordered_factorizations(224, 4))


def test_encoding_range_and_injective_d16():
    space = KnobSpace(WORKLOADS["resnet18_layer1"], 16)
    idx, X = make_pool(space, 20000, 5)
    assert X.shape == (20000, 16) and X.dtype == np.float32
    assert X.min() >= 0.0 and X.max() <= 1.0
    assert len(np.unique(X, axis=0)) == 20000            # d = 16 encoding is injective
    assert np.all(np.diff(idx) > 0)
    s12 = KnobSpace(WORKLOADS["resnet18_layer1"], 12)
    assert s12.size == space.size


def test_config_pool_gamma_positive():
    X, g, cfg = config_pool("toy")
    assert X.shape == (256, 12) and g > 0 and cfg["m"] == 16 and cfg["mu"] == 0.1
