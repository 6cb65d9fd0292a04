"""Oracle pins: validation helpers (error magnitude P:L183, arithmetic means
P:L185, speedup P:L147) against the paper's printed arithmetic: Table II
(P:L261-280), the Stassuij example and the vector-add example
(P:L57-59)."""
import os

import pytest

HERE = os.path.dirname(os.path.abspath(__file__))


def table2():
    rows = []
    for line in open(os.path.join(HERE, "golden", "table2.txt")):
        line = line.strip()
        if line and not line.startswith("#"):
            f = line.split()
            rows.append((f[0], f[1], float(f[2]), float(f[3]), float(f[4]), f[5]))
    return rows


def test_stassuij_kernel_only_error(O):
    """kernel-only predicted speedup 1.10x vs measured 0.39x ->
    Table II prints 182%."""
    e = O.speedup_error(1.10, 0.39)
    assert round(100 * e) == 182


def test_table2_averages(O):
    """The printed averages are arithmetic means of the printed rows
    (±1 point: the rows themselves are rounded)."""
    rows = table2()
    data = [r for r in rows if not r[0].startswith("avg")]
    avg = {(r[0], r[1]): r[2:5] for r in rows if r[0].startswith("avg")}
    for col in range(3):
        per_ds = O.mean([r[2 + col] for r in data])
        assert abs(per_ds - avg[("avg_datasets", "-")][col]) <= 1.0
        apps = {}
        for r in data:
            apps.setdefault(r[0], []).append(r[2 + col])
        app_means = []
        for app, v in apps.items():
            m = O.mean(v)
            if len(v) > 1:
                assert abs(m - avg[("avg_app", app)][col]) <= 1.0, (app, col, m)
            app_means.append(m)
        assert abs(O.mean(app_means) - avg[("avg_apps", "-")][col]) <= 1.0


def test_srad_4096_from_component_errors(O):
    """kernel error 0.7%, transfer error 1.9% at SRAD 4096^2; Table I
    times 28.1 / 49.0 ms.  Under-predicting both, the speedup errors
    are ~176% (kernel only), ~60% (transfer only), ~1% (both) — Table II row
    P:L276 prints 176 / 61 / 1."""
    tk, tx = 28.1e-3, 49.0e-3
    t_cpu = 1.0  # cancels
    s_meas = O.speedup(t_cpu, tk + tx)
    pk, px = tk * (1 - 0.007), tx * (1 - 0.019)
    e_k = O.speedup_error(O.speedup(t_cpu, pk), s_meas)
    e_x = O.speedup_error(O.speedup(t_cpu, px), s_meas)
    e_b = O.speedup_error(O.speedup(t_cpu, pk + px), s_meas)
    assert abs(100 * e_k - 176) < 1.0
    assert abs(100 * e_x - 61) < 1.5
    assert round(100 * e_b) == 1


def test_vector_add_example(O):
    """bandwidth-bound vector add on a 77 GB/s GPU vs a 32 GB/s CPU:
    2.4x kernel-only; over a ~3 GB/s PCIe bus the CPU is ~10x faster."""
    n_bytes = 3 * 4 * (1 << 24)
    t_cpu = n_bytes / 32e9
    t_kern = n_bytes / 77e9
    assert round(O.speedup(t_cpu, t_kern), 1) == 2.4
    t_xfer = n_bytes / 3e9
    s = O.speedup(t_cpu, t_kern + t_xfer)
    assert 8.0 < 1.0 / s < 12.0


def test_error_magnitude_definition(O):
    assert O.error_magnitude(1.064, 1.0) == pytest.approx(0.064, rel=1e-12)
    assert O.error_magnitude(0.9, 1.0) == pytest.approx(0.1, rel=1e-12)
    assert O.error_magnitude(2.0, 2.0) == 0.0
