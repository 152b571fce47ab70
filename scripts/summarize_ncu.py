"""Summarise ncu captures (gpurun_out/prof_<wl>.ncu-rep, launches_<wl>.csv) into profiles/.

    python scripts/summarize_ncu.py <round-tag> [workloads...]

Writes profiles/<tag>/ncu_summary.md, copies the launch lists, and updates
profiles/ncu_traffic.json (dram bytes read+write per launch of the dominant kernel, which
bench.py reports as roofline.traffic).
"""
from __future__ import annotations

import csv
import io
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NCU = "/usr/local/cuda/bin/ncu"
METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % peak"),
    ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "ALU pipe % peak"),
    ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "FMA pipe % peak"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "LSU pipe % peak"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active % (achieved occupancy)"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput % peak"),
]
MAPPINGS = {"cfg1": 81, "cfg2": 10_000 * 4**8, "cfg3": 10**6 * 9, "cfg4": 4**16, "cfg5": 8**12}
# cfg5c (3 pinned + 3 masked queues, NEXT-3): thread instructions per FEASIBLE mapping
MAPPINGS["cfg5c"] = 9_437_184


def raw(rep):
    out = subprocess.run([NCU, "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[h.index("Kernel Name")]}
        for m, _ in METRICS:
            if m in h:
                d[m] = (r[h.index(m)], units[h.index(m)])
        res.append(d)
    return res


def to_bytes(v, unit):
    x = float(v.replace(",", ""))
    return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)


def main(tag, workloads):
    outdir = os.path.join(ROOT, "profiles", tag)
    os.makedirs(outdir, exist_ok=True)
    tpath = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    traffic = json.load(open(tpath)) if os.path.exists(tpath) else {}
    lines = [f"# ncu summary ({tag})", "",
             "`ncu --set full --clock-control none --import-source on` of one launch of the search kernel "
             "(`scripts/ncu_captures.sh`), read back with `ncu -i ... --page raw --csv`. Cold-cache, serialised: "
             "use shares and pipe utilisation, not absolute times.", ""]
    for wl in workloads:
        rep = os.path.join(ROOT, "gpurun_out", f"prof_{wl}.ncu-rep")
        if not os.path.exists(rep):
            continue
        for d in raw(rep):
            lines += [f"## {wl}: `{d['kernel']}`", "", "| metric | value |", "|---|---|"]
            for m, label in METRICS:
                if m in d:
                    lines.append(f"| {label} (`{m}`) | {d[m][0]} {d[m][1]} |")
            rd = to_bytes(*d["dram__bytes_read.sum"])
            wr = to_bytes(*d["dram__bytes_write.sum"])
            wi = float(d["smsp__inst_executed.sum"][0].replace(",", ""))
            if wl in MAPPINGS:
                lines += ["", f"thread instructions per mapping (warp instructions x 32 / mappings): "
                              f"{wi * 32 / MAPPINGS[wl]:.3f}", ""]
            else:
                lines += [""]
            traffic[wl] = {"dram_bytes_per_launch": rd + wr, "kernel": d["kernel"], "source": f"profiles/{tag}"}
        lp = os.path.join(ROOT, "gpurun_out", f"launches_{wl}.csv")
        if os.path.exists(lp):
            shutil.copy(lp, os.path.join(outdir, f"launches_{wl}.csv"))
    open(os.path.join(outdir, "ncu_summary.md"), "w").write("\n".join(lines) + "\n")
    json.dump(traffic, open(tpath, "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2:] or ["cfg5", "cfg4", "cfg2", "cfg3", "costs", "cfg5c"])
