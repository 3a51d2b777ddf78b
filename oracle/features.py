"""Oracle for what the histograms are used for — TEST INFRASTRUCTURE ONLY.

PAPER.md:10 §I ¶1: zonal histogramming extends classic Zonal Statistics, "where only major
statistics, such as min, max, average, count and standard deviation, are reported", and the
histograms "can further be used as feature vectors for more sophisticated analysis, such as
computing various distance measurements which can be used for subsequent clustering".

Everything here is the plain definition in EXACT rational arithmetic (Python ints and
fractions.Fraction) over the multiset of bin values a histogram row describes, with the value of
bin b read as lo + b*width (R16).  No rounding happens before the final float().
Pinned in tests/test_oracle_features.py against library routines (numpy mean/std over the
expanded values, scipy's cityblock and wasserstein_distance) and closed forms.
"""
from __future__ import annotations

from fractions import Fraction
from math import isqrt

import numpy as np


def _row(H, k):
    return [int(v) for v in np.asarray(H[k]).tolist()]


def summary_exact(H, lo: int = 0, width: int = 1):
    """Per row: (count, min, max, lower median, mean, variance) of the values lo + b*width, each
    b repeated H[k][b] times; mean and variance as exact Fractions (population variance); None for
    the order statistics / moments of an empty row."""
    out = []
    for k in range(np.asarray(H).shape[0]):
        row = _row(H, k)
        n = sum(row)
        if n == 0:
            out.append((0, None, None, None, None, None))
            continue
        val = lambda b: lo + b * width
        nz = [b for b, v in enumerate(row) if v]
        target, run, med = (n + 1) // 2, 0, None
        for b, v in enumerate(row):
            run += v
            if run >= target:
                med = b
                break
        mean = Fraction(sum(val(b) * v for b, v in enumerate(row)), n)
        var = sum((val(b) - mean) ** 2 * v for b, v in enumerate(row)) / n
        out.append((n, val(nz[0]), val(nz[-1]), val(med), mean, var))
    return out


def sqrt_fraction(q: Fraction, digits: int = 40) -> Fraction:
    """sqrt of a non-negative Fraction to within 10^-digits relative (for comparing floats)."""
    if q == 0:
        return Fraction(0)
    scale = 10 ** (2 * digits)
    num = q.numerator * scale
    r = isqrt(num // q.denominator)
    return Fraction(r, 10 ** digits)


def _cum(row):
    out, run = [], 0
    for v in row:
        run += v
        out.append(run)
    return out


def distance_exact(H, kind: str, a: int, b: int):
    """Distance between the normalised histograms p = H[a]/n_a, q = H[b]/n_b as an exact Fraction
    (None if a row is empty):
      'l1'   sum |p - q|
      'emd'  sum |P - Q| over the cumulative distributions (1-D earth mover's distance in bins)
      'chi2' 1/2 sum_{p+q>0} (p - q)^2 / (p + q)"""
    ra, rb = _row(H, a), _row(H, b)
    na, nb = sum(ra), sum(rb)
    if na == 0 or nb == 0:
        return None
    if kind == "emd":
        ra, rb = _cum(ra), _cum(rb)
        kind = "l1"
    if kind == "l1":
        return sum((abs(Fraction(x, na) - Fraction(y, nb)) for x, y in zip(ra, rb)), Fraction(0))
    if kind == "chi2":
        s = Fraction(0)
        for x, y in zip(ra, rb):
            p, q = Fraction(x, na), Fraction(y, nb)
            if p + q:
                s += (p - q) ** 2 / (p + q)
        return s / 2
    raise ValueError(kind)
