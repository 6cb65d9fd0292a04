"""BASELINE.json config 5: PCIe model calibration and validation on every
visible GPU, single and concurrent.  Writes JSON (argv[1], default
gpurun_out/pcie.json) and prints a one-line summary per device/direction."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_ipps_boyermk13_b200 import build  # noqa: E402

build.build()
from paper_conf_ipps_boyermk13_b200 import pcie  # noqa: E402


def main():
    out = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/pcie.json"
    reps = int(os.environ.get("PCIE_REPS", 10))
    devs = list(range(torch.cuda.device_count()))
    rep = pcie.validate(devs, reps=reps)
    rep["gpus"] = [torch.cuda.get_device_name(d) for d in devs]
    if not os.environ.get("NO_MEMORY_TRADEOFF"):
        rep["memory_tradeoff"] = [pcie.memory_tradeoff(d, reps=reps) for d in devs[:1]]
    os.makedirs(os.path.dirname(out) or ".", exist_ok=True)
    json.dump(rep, open(out, "w"), indent=1)
    for r in rep["single"]:
        for d in ("h2d", "d2h"):
            f, e, nf = r["fit"][d], r["errors"][d], r["noise_floor"][d]
            print(f"gpu{r['device']} {d}: alpha={f['alpha_s']*1e6:.2f}us "
                  f"1/beta={f['bandwidth_GBps']:.2f}GB/s mean_err={100*e['mean_error']:.2f}% "
                  f"max_err={100*e['max_error']:.2f}% noise_floor={100*nf['mean_error']:.2f}%")
    for r in rep.get("memory_tradeoff", []):
        for d in ("h2d", "d2h"):
            f, e = r["pageable_fit"][d], r["pageable_errors"][d]
            sp = r["pinned_speedup"][d]
            flips = [x["bytes"] for x in r["choice_single_transfer_arrays"][d]
                     if x["memory"] == "pageable"]
            print(f"gpu{r['device']} pageable {d}: alpha={f['alpha_s']*1e6:.2f}us "
                  f"1/beta={f['bandwidth_GBps']:.2f}GB/s mean_err={100*e['mean_error']:.2f}% "
                  f"pinned speedup {min(x['pinned_speedup'] for x in sp):.2f}-"
                  f"{max(x['pinned_speedup'] for x in sp):.2f}x; pageable chosen at {flips[:6]}; "
                  f"piecewise mean_err={100*r['pageable_piecewise'][d]['mean_error']:.2f}%")
        a = r["pin_alloc_fit"]
        print(f"gpu{r['device']} pinned alloc: alpha={a['alpha_s']*1e6:.1f}us "
              f"beta={a['beta_s_per_byte']*1e12:.2f}ps/B")


if __name__ == "__main__":
    main()
