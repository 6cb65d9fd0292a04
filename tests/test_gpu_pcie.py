"""PCIe calibration subsystem on a real device (config 5, reduced sizes)."""
import pytest

from synth import skeletons as S

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def G():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_boyermk13_b200 import build
    build.build()
    from paper_conf_ipps_boyermk13_b200 import grophecy
    return grophecy


def test_calibrate_magnitudes(G):
    pc = G.calibrate(0, reps=5, large_bytes=1 << 26)
    for l in (pc.h2d, pc.d2h):
        assert 1e-7 < l.alpha_s < 1e-3          # microseconds of fixed cost
        bw = 1.0 / l.beta_s_per_byte
        assert 1e9 < bw < 1e12                  # a PCIe / C2C class link


def test_fit_reproduces_measured_large_point(G):
    """The model built from (t(1 B), t(L)) predicts t(L) to within alpha, and
    large transfers within 15% (error ~0 above 1 MB)."""
    from paper_conf_ipps_boyermk13_b200 import pcie
    sw = pcie.sweep(0, [1, 1 << 20, 1 << 24, 1 << 26], reps=5, warmup=2)
    links = pcie.fit_from_sweep(sw, 1 << 26)
    rep = pcie.score(sw, links)
    for d in ("h2d", "d2h"):
        rows = {r["bytes"]: r for r in rep[d]["sizes"]}
        assert rows[1 << 26]["error"] < 0.03   # overshoot by alpha / t_L (fit reading 1)
        assert rows[1 << 24]["error"] < 0.15


def test_measure_rejects_bad_args(G):
    with pytest.raises(G.GrophecyError):
        G.measure_transfer(0, 5, 1024)
    with pytest.raises(G.GrophecyError):
        G.measure_transfer(0, 0, 0)
