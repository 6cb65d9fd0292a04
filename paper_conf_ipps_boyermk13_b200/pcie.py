"""PCIe calibration / validation subsystem (§III-C and §V-A).

* calibrate(): the paper's automatic two-measurement fit,
  per direction, through grophecy_calibrate.
* validate(): the paper's validation protocol: transfer every
  size of a sweep (powers of two) with pinned memory, mean of `reps` runs
  after warm-ups, predict each with the two-point model, report the error
  magnitude |pred - meas| / meas per size, its mean and max per direction,
  and the run-to-run noise floor (a second sweep predicted from the first).
  Modes: "single" (one GPU at a time) and "concurrent" (all GPUs at once,
  a barrier before every size and direction), the latter also scored
  against the single-mode fit.

Every transfer is measured by the CUDA library (grophecy_measure_transfer)
and every error magnitude and mean is computed by the library's helpers
(grophecy_error_magnitude, grophecy_mean); this module only orchestrates.
"""
import threading

from . import grophecy as G

DIRS = (("h2d", G.DIR_H2D), ("d2h", G.DIR_D2H))

error_magnitude = G.error_magnitude   # |pred - meas| / meas
mean = G.mean                         # arithmetic mean


def default_sizes(lo_exp=10, hi_exp=30, include_one=True):
    """2^0 and 2^10 ... 2^30 (BASELINE.json config 5: 1 KB - 1 GB)."""
    return ([1] if include_one else []) + [1 << e for e in range(lo_exp, hi_exp + 1)]


def sweep(device, sizes, reps=10, warmup=2, memory=G.MEM_PINNED, barrier=None):
    """{direction: [(bytes, mean_wall_s, mean_event_s)]} for one device.
    With a barrier (concurrent mode) every (direction, size) measurement
    starts together on all devices, so each size is measured under the
    contention of all of them."""
    out = {}
    for name, d in DIRS:
        rows = []
        for s in sizes:
            if barrier is not None:
                barrier.wait()
            rows.append((s, *G.measure_transfer_mem(device, d, memory, s, reps, warmup)))
        out[name] = rows
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

        def run(d):   # one host thread per GPU, aligned at every size
            results[d] = sweep(d, sizes, reps, warmup, barrier=barrier)

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


def memory_tradeoff(device, sizes=None, reps=10, warmup=2, large=1 << 29,
                    alloc_sizes=None):
    """NEXT-4 (reading 17): the pageable sweep with
    its own two-point fit and validation errors, the speedup of pinned over
    pageable per size and direction (the paper's Fig. 3), the pinned
    allocation overhead line A(F) = alpha + beta F (fit at 4 KiB and `large`,
    checked on a size sweep), and where the per-array choice flips for an
    array whose footprint equals its transfer size."""
    sizes = sizes or default_sizes()
    if large not in sizes:
        sizes = sorted(set(sizes) | {large})
    pin = sweep(device, sizes, reps, warmup, G.MEM_PINNED)
    page = sweep(device, sizes, reps, warmup, G.MEM_PAGEABLE)
    pin_links, page_links = fit_from_sweep(pin, large), fit_from_sweep(page, large)
    speed = {}
    for name, _ in DIRS:
        speed[name] = [{"bytes": a[0], "pinned_s": a[1], "pageable_s": b[1],
                        "pinned_speedup": b[1] / a[1]} for a, b in zip(pin[name], page[name])]
    # piecewise-linear alternative for the pageable links (footnote 4: pageable
    # transfers are "slightly more non-linear"): knots at 2^0, 2^12, 2^16,
    # 2^20, 2^24 and `large`, linear in d between knots, the last slope beyond
    knots = [k for k in (1, 1 << 12, 1 << 16, 1 << 20, 1 << 24, large) if k in sizes]
    piecewise = {}
    for name, _ in DIRS:
        t = {s_: w for s_, w, _ in page[name]}
        kt = [(k, t[k]) for k in knots]

        def pred(d, kt=kt):
            for (x0, y0), (x1, y1) in zip(kt, kt[1:]):
                if d <= x1 or (x1, y1) == kt[-1]:
                    return y0 + (y1 - y0) * (d - x0) / (x1 - x0)
            return kt[-1][1]
        errs = [error_magnitude(pred(s_), w) for s_, w, _ in page[name]]
        piecewise[name] = {"knots": knots, "mean_error": mean(errs), "max_error": max(errs)}
    alloc_sizes = alloc_sizes or [1 << e for e in range(12, 31, 2)]
    if 4096 not in alloc_sizes or large not in alloc_sizes:
        alloc_sizes = sorted(set(alloc_sizes) | {4096, large})
    at = {s: sum(G.measure_pin_alloc(device, s, reps)) for s in alloc_sizes}
    alloc_link = G.fit_pcie(at[4096], at[large], large)
    alloc_rows = [{"bytes": s, "measured_s": t, "predicted_s": G.pcie_time(alloc_link, s),
                   "error": error_magnitude(G.pcie_time(alloc_link, s), t)} for s, t in at.items()]
    model = G.MemoryModel()
    model.pinned.h2d, model.pinned.d2h = pin_links["h2d"], pin_links["d2h"]
    model.pageable.h2d, model.pageable.d2h = page_links["h2d"], page_links["d2h"]
    model.pin_alloc = alloc_link
    choice = {}
    for name, _ in DIRS:
        rows = []
        for s in sizes:
            c = G.choose_memory(model, s if name == "h2d" else 0, s if name == "d2h" else 0, s)
            rows.append({"bytes": s, "t_pinned_s": c.t_pinned_s, "t_pageable_s": c.t_pageable_s,
                         "memory": "pinned" if c.memory == G.MEM_PINNED else "pageable"})
        choice[name] = rows
    return {"device": device, "sizes": sizes, "reps": reps,
            "pageable_fit": {k: _link_dict(v) for k, v in page_links.items()},
            "pinned_fit": {k: _link_dict(v) for k, v in pin_links.items()},
            "pageable_errors": score(page, page_links),
            "pageable_piecewise": piecewise,
            "pinned_speedup": speed,
            "pin_alloc_fit": {"alpha_s": alloc_link.alpha_s,
                              "beta_s_per_byte": alloc_link.beta_s_per_byte},
            "pin_alloc": alloc_rows,
            "choice_single_transfer_arrays": choice}
