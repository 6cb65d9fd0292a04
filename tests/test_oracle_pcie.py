"""Oracle pins: the PCIe model, §III-C of the paper.

Eq. (1) T(d) = alpha + beta*d; fit alpha = t_S, beta = t_L / s_L with
s_L = 512 MB (read as 2^29 bytes: DESIGN.md reading 2); magnitudes
alpha ~ 10 us, 1/beta ~ 2.5 GB/s, alpha dominates below 1 KB and beta*d above
1 MB; Table I measured transfer times.
"""
import math

import pytest


def test_fit_closed_form(O):
    # t_S = 1e-5 s, t_L = 0.2147483648 s for 2^29 B  ->  alpha = 1e-5, beta = 4e-10.
    # 0.2147483648 = 4e-10 * 2^29 exactly; dividing by a power of two is exact,
    # so beta is bitwise the double nearest 4e-10.
    rc, l = O.fit_pcie(1e-5, 0.2147483648, 1 << 29)
    assert rc == 0
    assert l.alpha == 1e-5
    assert l.beta == 4e-10


def test_fit_reproduces_its_two_points(O):
    # The fit is built from two measurements: the model returns
    # t_S + beta at 1 byte, and t_S + t_L at s_L (beta*s_L == t_L exactly
    # when s_L is a power of two).
    tS, tL, sL = 7.25e-6, 0.0123, 1 << 29
    rc, l = O.fit_pcie(tS, tL, sL)
    assert rc == 0
    assert O.pcie_time(l, sL) == tS + tL
    assert O.pcie_time(l, 1) == tS + tL / sL


def test_zero_bytes_is_no_transfer(O, paper_link):
    assert O.pcie_time(paper_link, 0) == 0.0


@pytest.mark.parametrize("args", [(-1e-6, 1.0, 10), (1e-6, 0.0, 10), (1e-6, 1.0, 0),
                                  (math.nan, 1.0, 10), (1e-6, math.inf, 10)])
def test_fit_rejects_invalid(O, args):
    rc, _ = O.fit_pcie(*args)
    assert rc != 0


# Eq. (1) itself is pinned against exact rational arithmetic in
# tests/test_oracle_golden.py::test_pcie_time_exact_rational.


def test_regimes_match_paper_magnitudes(O, paper_link):
    # "For small transfers (<1KB), the alpha term dominates ...
    # for large transfers (>1MB), the beta*d term dominates."
    for d in (1, 16, 256, 1023):
        assert O.pcie_time(paper_link, d) < 1.05 * paper_link.alpha
    for d in (1 << 21, 1 << 25, 1 << 29):
        t = O.pcie_time(paper_link, d)
        assert (t - paper_link.alpha) / t > 0.95
    # alpha on the order of 10 us; bandwidth ~2.5 GB/s
    assert 1e-6 < paper_link.alpha < 1e-4
    assert 2.0e9 < 1.0 / paper_link.beta < 3.0e9
