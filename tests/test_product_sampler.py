"""Distribution pins of the PRODUCT's binomial sampler (the merged walks of §IV-B draw B ~ Bin(n, p)).

The oracle estimates access frequencies by plain walks (§IV-A) and has no binomial sampler; the product's
merged form needs one (BINV for n p < 10, BTRD otherwise; reading R20). These tests check the product's
host sampler (gcsm_binomial_samples, pure host) against scipy's exact pmf (chi-square) and known moments;
the device walker draws the same values (bit-exact host-walker == GPU-walker test in test_gpu_parity.py).
"""
import numpy as np
import pytest

from paper_conf_ipps_wei024_b200 import binomial_samples


@pytest.mark.parametrize("n,p", [(20, 0.3), (200, 0.02), (1000, 0.3), (5000, 0.01), (40, 0.5), (10**6, 1e-4),
                                 (10**4, 0.7)])
def test_binomial_chi_square(n, p):
    scipy_stats = pytest.importorskip("scipy.stats")
    N = 40000
    x = binomial_samples(0xC0FFEE + n, n, p, N)
    assert x.min() >= 0 and x.max() <= n
    pmf = scipy_stats.binom.pmf(np.arange(n + 1), n, p)
    # bins with expected count >= 20, the rest pooled into the two tails
    lo = int(np.argmax(pmf * N >= 20))
    hi = int(len(pmf) - np.argmax(pmf[::-1] * N >= 20) - 1)
    obs = np.bincount(np.clip(x, lo - 1, hi + 1) - (lo - 1), minlength=hi - lo + 3).astype(float)
    exp = np.concatenate([[pmf[:lo].sum()], pmf[lo:hi + 1], [pmf[hi + 1:].sum()]]) * N
    keep = exp > 0
    stat = ((obs[keep] - exp[keep]) ** 2 / exp[keep]).sum()
    dof = keep.sum() - 1
    assert stat < scipy_stats.chi2.ppf(1 - 1e-4, dof), (stat, dof)


def test_binomial_huge_n_moments_and_edges():
    n, p = 10**12, 1e-9  # mean 1000 (BTRD)
    x = binomial_samples(77, n, p, 20000).astype(float)
    assert abs(x.mean() - 1000) < 5 * np.sqrt(1000 / 20000)
    assert abs(x.var() / (n * p * (1 - p)) - 1) < 0.05
    assert (binomial_samples(78, 5, 1.0, 10) == 5).all()
    assert (binomial_samples(78, 5, 0.0, 10) == 0).all()
    assert (binomial_samples(78, 0, 0.5, 10) == 0).all()
    z = binomial_samples(79, 100, 0.9, 20000).astype(float)  # p > 1/2 branch
    assert abs(z.mean() - 90) < 5 * np.sqrt(9 / 20000)
    # counter-based (R22): the same key gives the same draws
    assert np.array_equal(binomial_samples(5, 1000, 0.1, 100), binomial_samples(5, 1000, 0.1, 100))
