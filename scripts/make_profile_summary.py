"""Write the committed profiling evidence for a round from ncu captures (run here, no GPU).

  python scripts/make_profile_summary.py TAG launches.csv prof_a.ncu-rep [prof_b.ncu-rep ...]

Produces profiles/<TAG>_launches.md (per-kernel share of one bench step, from the
`--metrics gpu__time_duration.sum --clock-control none` launch list — cold-cache and
serialised: compare shares, not absolutes), profiles/<TAG>_ncu.md (selected raw metrics
of one `--set full` launch per kernel), profiles/ncu_traffic.json (DRAM bytes per launch,
read by bench.py's roofline.traffic) and profiles/ncu_inst.json (warp instructions per launch,
read by bench.py's roofline.issue).
"""
from __future__ import annotations

import collections
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
    "launch__grid_size", "launch__block_size", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "smsp__pcsamp_warps_issue_stalled_barrier", "smsp__pcsamp_warps_issue_stalled_long_scoreboard",
    "smsp__pcsamp_warps_issue_stalled_short_scoreboard", "smsp__pcsamp_warps_issue_stalled_wait",
    "smsp__pcsamp_sample_count",
]
# bench.py's kernel names
NAMES = {"scatter_table_kernel": "scatter_table_kernel", "refine_kernel": "refine_kernel",
         "bucket_join_kernel": "bucket_join_kernel", "onesweep_kernel": "onesweep_kernel",
         "join_kernel": "join_kernel", "table_kernel": "table_kernel"}


def launch_table(path: str) -> str:
    rows = list(csv.reader(open(path)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    iN, iV, iM = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Name")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows[start + 1:]:
        if len(r) <= iV or r[iM] != "gpu__time_duration.sum":
            continue
        name = r[iN].split("(")[0].replace("void ", "")
        agg[name][0] += 1
        agg[name][1] += float(r[iV].replace(",", ""))
    tot = sum(v[1] for v in agg.values())
    out = ["| kernel | launches | total ms | avg us | share |", "|---|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        out.append(f"| `{k}` | {v[0]} | {v[1] / 1e6:.3f} | {v[1] / v[0] / 1e3:.2f} | {v[1] / tot:.3f} |")
    out.append(f"| total | {sum(v[0] for v in agg.values())} | {tot / 1e6:.3f} | | |")
    return "\n".join(out)


def raw(path: str) -> dict:
    """One launch's raw page: an .ncu-rep, or its `--page raw --csv` export (.csv)."""
    if path.endswith(".csv"):
        txt = open(path).read()
        txt = txt[txt.index('"ID"'):] if '"ID"' in txt else txt
    else:
        txt = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                             text=True).stdout
    rows = list(csv.reader(txt.splitlines()))
    hdr, units, vals = rows[0], rows[1], rows[2]
    d = {"Kernel Name": vals[hdr.index("Kernel Name")]}
    for m in METRICS:
        if m in hdr:
            i = hdr.index(m)
            d[m] = (vals[i], units[i])
    return d


def to_bytes(v: str, unit: str) -> float:
    x = float(v.replace(",", ""))
    return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)


def main() -> None:
    # python scripts/make_profile_summary.py TAG CFG launches.csv|- prof...
    tag, cfg, launches, reps = sys.argv[1], sys.argv[2], sys.argv[3], sys.argv[4:]
    prof = os.path.join(ROOT, "profiles")
    os.makedirs(prof, exist_ok=True)
    if launches != "-":
      with open(os.path.join(prof, f"{tag}_launches.md"), "w") as f:
        f.write(f"# {tag}: kernel launch list of one bench step ({cfg})\n\n")
        f.write("`ncu --metrics gpu__time_duration.sum --clock-control none` over "
                "`bench.py --steps 1 --warmup 1` (every step the bench runs: warm-up, timed, "
                "the serial and pipelined e2e legs). Cold-cache, "
                "serialised: compare shares, not absolute times.\n\n")
        f.write(launch_table(launches) + "\n")
    traffic_path = os.path.join(prof, "ncu_traffic.json")
    traffic_all = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    traffic = traffic_all.setdefault(cfg, {})  # per config: bytes depend on the workload
    inst_path = os.path.join(prof, "ncu_inst.json")
    inst_all = json.load(open(inst_path)) if os.path.exists(inst_path) else {}
    inst = inst_all.setdefault(cfg, {})
    lines = [f"# {tag}: one `ncu --set full --clock-control none` launch per kernel ({cfg})\n"]
    for rp in reps:
        d = raw(rp)
        name = d["Kernel Name"].split("(")[0].replace("void ", "").split("<")[0]
        lines.append(f"## `{d['Kernel Name']}`  ({os.path.basename(rp)})\n")
        lines.append("| metric | value |\n|---|---|")
        for m in METRICS:
            if m in d:
                lines.append(f"| {m} | {d[m][0]} {d[m][1]} |")
        rb = to_bytes(*d["dram__bytes_read.sum"])
        wb = to_bytes(*d["dram__bytes_write.sum"])
        lines.append(f"| DRAM bytes per launch | {rb + wb:.4g} |\n")
        if name in NAMES:
            traffic[NAMES[name]] = rb + wb
            if "smsp__inst_executed.sum" in d: # warp instructions per launch (issue view)
                inst[NAMES[name]] = float(d["smsp__inst_executed.sum"][0].replace(",", ""))
    with open(os.path.join(prof, f"{tag}_ncu.md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    with open(traffic_path, "w") as f:
        json.dump(traffic_all, f, indent=1)
    with open(inst_path, "w") as f:
        json.dump(inst_all, f, indent=1)
    print("wrote", tag)


if __name__ == "__main__":
    main()
