"""Turn gpurun_out/ captures into committed summaries under profiles/.

    python scripts/make_profiles.py r01
Writes profiles/<tag>_bench.json, <tag>_launches.csv (+ share summary),
<tag>_ncu_best.txt, ncu_best_summary.json (read by bench.py for `traffic`),
<tag>_pcie.json (if present).
"""
import csv
import io
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")


def ncu_raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return [dict(zip(rows[0], r)) for r in rows[2:]], dict(zip(rows[0], rows[1]))


def num(v):
    try:
        return float(str(v).replace(",", ""))
    except ValueError:
        return None


def main(tag):
    os.makedirs(PROF, exist_ok=True)
    bench = os.path.join(OUT, "bench.log")
    line = None
    if os.path.exists(bench):
        for ln in open(bench):
            if ln.startswith("{"):
                line = json.loads(ln)
        if line:
            json.dump(line, open(os.path.join(PROF, f"{tag}_bench.json"), "w"), indent=1)
    lc = os.path.join(OUT, "launches.csv")
    if os.path.exists(lc):
        txt = open(lc).read()
        start = txt.index('"ID"')
        rows = list(csv.DictReader(io.StringIO(txt[start:])))
        shutil.copy(lc, os.path.join(PROF, f"{tag}_launches.csv"))
        tot = {}
        for r in rows:
            k = r["Kernel Name"].split("(")[0]
            tot.setdefault(k, []).append(num(r["Metric Value"]))
        all_ns = sum(sum(v) for v in tot.values())
        with open(os.path.join(PROF, f"{tag}_launches_summary.txt"), "w") as f:
            f.write("ncu --metrics gpu__time_duration.sum --clock-control none (cold, serialised)\n")
            f.write("command: python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline\n")
            for k, v in sorted(tot.items(), key=lambda kv: -sum(kv[1])):
                f.write(f"{k:40s} launches={len(v):3d} avg_ms={sum(v)/len(v)/1e6:9.3f} "
                        f"share={100*sum(v)/all_ns:5.1f}%\n")
    rep = os.path.join(OUT, "best_full.ncu-rep")
    if os.path.exists(rep):
        rows, units = ncu_raw(rep)
        r = rows[0]
        want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
                "sm__throughput.avg.pct_of_peak_sustained_elapsed",
                "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
                "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
                "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
                "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
                "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
                "sm__warps_active.avg.pct_of_peak_sustained_active",
                "smsp__issue_active.avg.pct_of_peak_sustained_active",
                "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
                "smsp__inst_executed.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed"]
        summ = {}
        with open(os.path.join(PROF, f"{tag}_ncu_best.txt"), "w") as f:
            f.write("ncu --set full --clock-control none -k regex:sweep_kernel (bench config, "
                    "the fused best projection of 10^9 candidates)\n")
            for k in want:
                if k in r:
                    f.write(f"{k:70s} {r[k]} {units.get(k, '')}\n")
                    summ[k] = num(r[k])
        def to_bytes(k):
            u = units.get(k, "")
            mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
            return summ.get(k, 0) * mult
        traffic = to_bytes("dram__bytes_read.sum") + to_bytes("dram__bytes_write.sum")
        n = (line or {}).get("config", {}).get("per_gpu", 10**9)
        winst = summ.get("smsp__inst_executed.sum")
        json.dump({"dram_bytes_per_launch": traffic, "n_candidates": n, "tag": tag,
                   "warp_inst_per_launch": winst,
                   "source": f"profiles/{tag}_ncu_best.txt"},
                  open(os.path.join(PROF, "ncu_best_summary.json"), "w"), indent=1)
    # stall / pipe breakdown and the hottest source lines of the same capture
    for src, dst in (("best_summary.txt", f"{tag}_ncu_best_stalls.txt"),
                     ("best_lines.txt", f"{tag}_ncu_best_lines.txt"),
                     ("best_groups.txt", f"{tag}_ncu_best_phases.txt")):
        p = os.path.join(OUT, src)
        if os.path.exists(p) and os.path.getsize(p) > 0:
            shutil.copy(p, os.path.join(PROF, dst))
    pj = os.path.join(OUT, "pcie.json")
    if os.path.exists(pj):
        shutil.copy(pj, os.path.join(PROF, f"{tag}_pcie.json"))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "r01")
