"""Device generators against the oracle's (-m gpu): the Philox4x32-10 stream behind
lowrank_approx's sketch Omega and the orthogonality probes (reading #17).

Integer work is compared bit-exactly: the raw Philox words of the device kernel equal the
oracle's (itself pinned by the Random123 known-answer vectors, tests/golden/philox_kat.txt).
The Gaussians are the Box-Muller map of those words in fp64; CUDA's log / cos are within 1-2
ulp of glibc's correctly rounded ones, so they are compared to a few ulp, and the rounding to
fp32 (the sketch's operand precision) must then agree except at round-to-nearest ties.
"""
import numpy as np
import pytest

import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def rg():
    import paper_conf_hpdc_zhangbw20_b200 as rg
    return rg


@pytest.mark.parametrize("seed", [0, 99, 1234, 0xDEADBEEF_0BADF00D])
def test_device_philox_words_bit_exact(rg, seed):
    nc = 3000
    W = rg.debug_philox(nc, seed)
    for c in list(range(0, nc, 7)) + [nc - 1]:
        ref = oracle.philox4x32_10([c, 0, 0, 0], [seed & 0xFFFFFFFF, seed >> 32])
        assert list(W[c]) == ref, (c, list(W[c]), ref)


@pytest.mark.parametrize("seed", [99, 1234, 0xDEADBEEF_0BADF00D])
def test_device_gaussians_match_oracle(rg, seed):
    n = 20001                                   # odd: the last element uses words (0, 1) of its call
    z = rg.debug_gaussian(n, seed).cpu().numpy()
    zo = oracle.gaussian_philox(n, 1, seed)[:, 0]
    err = np.abs(z - zo)
    assert np.all(err <= 8 * np.finfo(np.float64).eps * np.maximum(1.0, np.abs(zo))), err.max()
    assert np.mean(z.astype(np.float32) == zo.astype(np.float32)) > 0.9999
