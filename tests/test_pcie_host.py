"""Host bookkeeping of the PCIe validation subsystem (no GPU): fit from a
sweep, per-size error magnitude, means and the noise floor."""
import pytest


@pytest.fixture(scope="module")
def P():
    from paper_conf_ipps_boyermk13_b200 import build
    build.build()
    from paper_conf_ipps_boyermk13_b200 import pcie
    return pcie


def _sweep(alpha, beta, sizes, jitter=None):
    jitter = jitter or {}
    return {d: [(s, (alpha + beta * s) * (1 + jitter.get(s, 0.0)), 0.0) for s in sizes]
            for d in ("h2d", "d2h")}


def test_exactly_linear_system_has_zero_error(P):
    sizes = P.default_sizes()
    sw = _sweep(1e-5, 4e-10, sorted(set(sizes) | {1 << 29}))
    links = P.fit_from_sweep(sw)
    rep = P.score(sw, links)
    for d in ("h2d", "d2h"):
        # beta is fitted as t_L / s_L, so T(d) = alpha + d*(alpha + beta s_L)/s_L:
        # the only model error is alpha*d/s_L (+ beta), < 0.01% of every measured time
        assert rep[d]["max_error"] < 1e-4
        assert links[d].alpha_s == 1e-5 + 4e-10


def test_error_of_a_perturbed_point(P):
    sizes = [1, 1024, 1 << 20, 1 << 29]
    sw = _sweep(1e-5, 4e-10, sizes, jitter={1024: 0.10})
    rep = P.score(sw, P.fit_from_sweep(sw))
    row = [r for r in rep["h2d"]["sizes"] if r["bytes"] == 1024][0]
    # predicted ~ unperturbed time t; measured 1.1 t -> |t - 1.1t| / 1.1t = 0.0909
    assert abs(row["error"] - 0.1 / 1.1) < 1e-4
    assert rep["h2d"]["max_error"] == row["error"]


def test_noise_floor(P):
    sizes = [1, 1024, 1 << 20]
    a = _sweep(1e-5, 4e-10, sizes)
    b = _sweep(1e-5, 4e-10, sizes, jitter={1: 0.02, 1024: -0.01})
    nf = P.noise_floor(a, b)
    e1 = abs(1 - 1 / 1.02)
    e2 = abs(1 - 1 / 0.99)
    assert abs(nf["h2d"]["mean_error"] - (e1 + e2) / 3) < 1e-12
