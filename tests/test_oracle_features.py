"""Pins of oracle/features.py (§I ¶1) against library routines and
closed forms — never against itself:
  * summary: numpy mean / std / min / max / percentile('lower') over the expanded cell values;
    closed form for v = c mod 7 over whole periods (mean 3, variance 4);
  * L1: scipy.spatial.distance.cityblock of the normalised histograms;
  * EMD: scipy.stats.wasserstein_distance with the bins as support and the counts as weights;
    deltas at bins i and j are |i - j| apart;
  * chi^2: closed forms (identical 0, disjoint supports 1, two-bin family), symmetry and the
    bound chi^2 <= L1 / 2."""
from fractions import Fraction

import numpy as np
import pytest
from scipy.spatial.distance import cityblock
from scipy.stats import wasserstein_distance

from oracle import features as F


def _hists(seed, P=6, B=40):
    rng = np.random.default_rng(seed)
    H = rng.integers(0, 9, size=(P, B)) * (rng.random((P, B)) < 0.4)
    H[0, :] = 0          # an empty row
    H[1, :] = 0
    H[1, 7] = 5          # a single-bin row
    return H.astype(np.uint64)


@pytest.mark.parametrize("lo,width", [(0, 1), (-40, 3), (100, 1)])
def test_summary_matches_numpy_on_expanded_values(lo, width):
    H = _hists(1)
    S = F.summary_exact(H, lo, width)
    for k in range(H.shape[0]):
        vals = np.repeat(lo + np.arange(H.shape[1]) * width, H[k].astype(np.int64))
        n, mn, mx, med, mean, var = S[k]
        assert n == vals.size
        if n == 0:
            assert mn is None and mean is None
            continue
        assert (mn, mx) == (vals.min(), vals.max())
        assert med == np.percentile(vals, 50, method="lower")
        assert float(mean) == pytest.approx(vals.mean(), rel=1e-13, abs=1e-13)
        assert float(var) == pytest.approx(vals.var(), rel=1e-12, abs=1e-12)
        assert float(F.sqrt_fraction(var)) == pytest.approx(vals.std(), rel=1e-12, abs=1e-12)


def test_summary_closed_form_mod7():
    # v = c mod 7 over 10 whole periods: uniform on 0..6, mean 3, population variance (7^2-1)/12 = 4
    H = np.zeros((1, 8), np.uint64)
    H[0, :7] = 10
    n, mn, mx, med, mean, var = F.summary_exact(H)[0]
    assert (n, mn, mx, med, mean, var) == (70, 0, 6, 3, 3, 4)


def test_l1_matches_cityblock():
    H = _hists(2)
    for a in range(1, H.shape[0]):
        for b in range(1, H.shape[0]):
            p = H[a] / H[a].sum()
            q = H[b] / H[b].sum()
            assert float(F.distance_exact(H, "l1", a, b)) == pytest.approx(cityblock(p, q), rel=1e-12, abs=1e-15)
    assert F.distance_exact(H, "l1", 0, 2) is None


def test_emd_matches_wasserstein():
    H = _hists(3)
    bins = np.arange(H.shape[1])
    for a in range(1, H.shape[0]):
        for b in range(1, H.shape[0]):
            want = wasserstein_distance(bins, bins, H[a].astype(float), H[b].astype(float))
            assert float(F.distance_exact(H, "emd", a, b)) == pytest.approx(want, rel=1e-12, abs=1e-12)


def test_emd_of_deltas():
    H = np.zeros((2, 50), np.uint64)
    H[0, 4] = 3
    H[1, 41] = 11
    assert F.distance_exact(H, "emd", 0, 1) == 37
    assert F.distance_exact(H, "l1", 0, 1) == 2


def test_chi2_closed_forms():
    H = np.zeros((4, 6), np.uint64)
    H[0, :3] = [1, 2, 3]
    H[1, :3] = [2, 4, 6]          # the same distribution
    H[2, 3:] = [5, 5, 1]          # disjoint support
    assert F.distance_exact(H, "chi2", 0, 1) == 0
    assert F.distance_exact(H, "chi2", 0, 2) == 1
    # p = (1, 0), q = (t, 1 - t): chi2 = ((1-t)^2/(1+t) + (1-t)) / 2
    for num, den in ((1, 3), (2, 5), (7, 8)):
        t = Fraction(num, den)
        T = np.zeros((2, 2), np.uint64)
        T[0] = [1, 0]
        T[1] = [num, den - num]
        want = ((1 - t) ** 2 / (1 + t) + (1 - t)) / 2
        assert F.distance_exact(T, "chi2", 0, 1) == want


def test_chi2_symmetric_and_bounded_by_half_l1():
    H = _hists(4)
    for a in range(1, H.shape[0]):
        for b in range(1, H.shape[0]):
            c = F.distance_exact(H, "chi2", a, b)
            assert c == F.distance_exact(H, "chi2", b, a)
            assert 0 <= c <= F.distance_exact(H, "l1", a, b) / 2


def test_sqrt_fraction():
    for q in (Fraction(2), Fraction(1, 3), Fraction(10 ** 30 + 7, 9)):
        assert float(F.sqrt_fraction(q)) == pytest.approx(float(q) ** 0.5, rel=1e-15)
