"""PCIe calibration / validation subsystem (§III-C and §V-A).

* calibrate(): the paper's automatic two-measurement fit,
  per direction, through grophecy_calibrate.
* validate(): the paper's validation protocol: transfer every
  size of a sweep (powers of two) with pinned memory, mean of `reps` runs
  after warm-ups, predict each with the two-point model, report the error
  magnitude |pred - meas| / meas per size, its mean and max per direction,
  and the run-to-run noise floor (a second sweep predicted from the first).
  Modes: "single" (one GPU at a time) and "concurrent" (all GPUs at once,
  barrier-aligned), the latter also scored against the single-mode fit.

Every transfer is measured by the CUDA library (grophecy_measure_transfer);
this module only orchestrates and does the bookkeeping arithmetic.
"""
import threading

from . import grophecy as G

DIRS = (("h2d", G.DIR_H2D), ("d2h", G.DIR_D2H))


def error_magnitude(pred, meas):
    """|pred - meas| / meas (as a fraction)."""
    return abs(pred - meas) / meas


def mean(v):
    v = list(v)
    return sum(v) / len(v)


def default_sizes(lo_exp=10, hi_exp=30, include_one=True):
    """2^0 and 2^10 ... 2^30 (BASELINE.json config 5: 1 KB - 1 GB)."""
    return ([1] if include_one else []) + [1 << e for e in range(lo_exp, hi_exp + 1)]


def sweep(device, sizes, reps=10, warmup=2):
    """{direction: [(bytes, mean_wall_s, mean_event_s)]} for one device."""
    out = {}
    for name, d in DIRS:
        out[name] = [(s, *G.measure_transfer(device, d, s, reps, warmup)) for s in sizes]
    return out


def fit_from_sweep(sw, large=1 << 29):
    """Two-point fit from a sweep containing 1 B and `large`."""
    links = {}
    for name, _ in DIRS:
        t = {s: w for s, w, _ in sw[name]}
        links[name] = G.fit_pcie(t[1], t[large], large)
    return links


def score(sw, links):
    """Per-size error magnitudes and their mean / max per direction."""
    rep = {}
    for name, _ in DIRS:
        rows = []
        for s, w, ev in sw[name]:
            pred = G.pcie_time(links[name], s)
            rows.append({"bytes": s, "measured_s": w, "event_s": ev, "predicted_s": pred,
                         "error": error_magnitude(pred, w)})
        errs = [r["error"] for r in rows]
        rep[name] = {"mean_error": mean(errs), "max_error": max(errs), "sizes": rows}
    return rep


def noise_floor(sw1, sw2):
    """Sweep 2 predicted by sweep 1, size by size."""
    out = {}
    for name, _ in DIRS:
        e = [error_magnitude(a[1], b[1]) for a, b in zip(sw1[name], sw2[name])]
        out[name] = {"mean_error": mean(e), "max_error": max(e)}
    return out


def _link_dict(l):
    return {"alpha_s": l.alpha_s, "beta_s_per_byte": l.beta_s_per_byte,
            "bandwidth_GBps": 1e-9 / l.beta_s_per_byte}


def validate_device(device, sizes, reps=10, warmup=2, large=1 << 29):
    if large not in sizes:
        sizes = sorted(set(sizes) | {large})
    s1 = sweep(device, sizes, reps, warmup)
    s2 = sweep(device, sizes, reps, warmup)
    links = fit_from_sweep(s1, large)
    return {"device": device, "fit": {k: _link_dict(v) for k, v in links.items()},
            "errors": score(s1, links), "noise_floor": noise_floor(s1, s2),
            "_links": links}


def validate(devices, sizes=None, reps=10, warmup=2, large=1 << 29, concurrent=True):
    """Config 5: single mode per device, then all devices concurrently."""
    sizes = sizes or default_sizes()
    single = [validate_device(d, sizes, reps, warmup, large) for d in devices]
    report = {"protocol": {"sizes": sizes, "reps": reps, "warmup": warmup, "fit_points": [1, large],
                           "memory": "pinned (cudaHostAlloc)",
                           "timer": "host steady_clock per transfer (cudaMemcpyAsync + sync)"},
              "single": [{k: v for k, v in r.items() if k != "_links"} for r in single]}
    if concurrent and len(devices) > 1:
        barrier = threading.Barrier(len(devices))
        results = {}

        def run(d):
            barrier.wait()
            results[d] = sweep(d, sizes, reps, warmup)

        th = [threading.Thread(target=run, args=(d,)) for d in devices]
        for t in th:
            t.start()
        for t in th:
            t.join()
        conc = []
        for r in single:
            d = r["device"]
            conc.append({"device": d, "errors_vs_single_fit": score(results[d], r["_links"]),
                         "fit": {k: _link_dict(v) for k, v in fit_from_sweep(results[d], large).items()}})
        report["concurrent"] = conc
    return report


def calibrate(device=0, reps=10, large=1 << 29):
    return G.calibrate(device, reps, large)
