"""Alg. 2 l.2 draws (reading A10) on pools far larger than the
bench's 2^20 rows: the device sampler's two-level radix select must agree bit
for bit with the oracle's sampler (oracle/sampling.py) at P = 2^25, and at the
full VGG-16 conv1_1 space (202,309,632 configurations) its draw
must be exactly the M smallest keys (checked by counting all P keys in chunks)."""
import numpy as np
import pytest

import paper_conf_date_sunbg021_b200 as bt
from oracle.sampling import batch_keys, sample_batches as oracle_sample_batches, splitmix64

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _gpu(need_gpu):
    yield


@pytest.mark.parametrize("P,M,B,seed", [(1 << 25, 32768, 2, 16), ((1 << 25) + 12345, 1000, 1, 3)])
def test_sampler_bit_exact_at_2pow25(P, M, B, seed):
    gpu = bt.bted_sample_batches(P, M, B, seed)
    ref = oracle_sample_batches(P, M, B, seed)
    assert np.array_equal(gpu, ref)


def _keys_chunk(hb, lo, hi):
    i = np.arange(lo, hi, dtype=np.uint64)
    with np.errstate(over="ignore"):
        r = splitmix64(hb + i)
    return (r & np.uint64(0xFFFFFFFF00000000)) | i


def test_sampler_full_vgg16_space_is_the_m_smallest_keys():
    P, M, seed = 202_309_632, 32768, 16                    # VGG-16 conv1_1 knob space
    V = bt.bted_sample_batches(P, M, 1, seed)[0]
    assert len(V) == M and np.all(np.diff(V) > 0) and V[0] >= 0 and V[-1] < P
    hb = splitmix64(np.uint64(seed % (1 << 64)))           # h_b for b = 0
    # the largest selected key k*: exactly M keys of the whole space are <= k*
    with np.errstate(over="ignore"):
        r = splitmix64(hb + V.astype(np.uint64))
    kall = (r & np.uint64(0xFFFFFFFF00000000)) | V.astype(np.uint64)
    kstar = kall.max()
    below = 0
    step = 1 << 24
    for lo in range(0, P, step):
        below += int(np.count_nonzero(_keys_chunk(hb, lo, min(P, lo + step)) <= kstar))
    assert below == M
    assert np.array_equal(batch_keys(1000, 0, seed)[:10], _keys_chunk(hb, 0, 10))
