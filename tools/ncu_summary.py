#!/usr/bin/env python
"""Summarise ncu evidence for profiles/: key counters of --set full captures
and the kernel-time shares of a --metrics gpu__time_duration.sum launch list.

    python tools/ncu_summary.py full  REPORT.ncu-rep [label]
    python tools/ncu_summary.py launches LAUNCHES.csv
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("smsp__inst_executed.sum", "warp instructions executed"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue slots busy %"),
    ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "ALU pipe %"),
    ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "FMA pipe %"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "shared wavefronts"),
    ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "shared bank conflicts"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "active threads / warp instr"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__shared_mem_per_block_dynamic", "dynamic smem/CTA"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
]


def raw(report):
    out = subprocess.run(["ncu", "-i", report, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def full(report, label=""):
    hdr, units, rows = raw(report)
    for r in rows:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        print(f"### {label or report}: `{d.get('Kernel Name', '?')[:90]}`\n")
        print("| counter | value |\n|---|---|")
        for k, name in KEYS:
            if k in d:
                print(f"| {name} (`{k}`) | {d[k]} {u.get(k, '')} |")
        stalls = []
        for k, v in d.items():
            if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("_per_issue_active.ratio"):
                try:
                    stalls.append((float(v), k[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
                except ValueError:
                    pass
        stalls.sort(reverse=True)
        print("\nTop warp stall reasons (warps stalled per issued instruction): " +
              ", ".join(f"{n} {v:.2f}" for v, n in stalls[:6]) + "\n")


def launches(path):
    txt = open(path).read()
    start = txt.find('"ID"')
    rows = list(csv.DictReader(io.StringIO(txt[start:])))
    tot = defaultdict(float)
    cnt = defaultdict(int)
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = r["Kernel Name"].split("(")[0].replace("void ", "")
        if name.startswith("k_int"):  # bench.py's integer-peak microbenchmark (a child process), not the step
            continue
        v = float(r["Metric Value"].replace(",", ""))
        unit = r.get("Metric Unit", "")
        scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3,
                 "ms": 1e3}.get(unit, 1.0)
        tot[name] += v * scale
        cnt[name] += 1
    allt = sum(tot.values())
    print("| kernel | launches | total us | share |\n|---|---|---|---|")
    for k in sorted(tot, key=tot.get, reverse=True):
        print(f"| `{k[:70]}` | {cnt[k]} | {tot[k]:.1f} | {100 * tot[k] / allt:.1f}% |")


if __name__ == "__main__":
    if sys.argv[1] == "full":
        full(sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else "")
    else:
        launches(sys.argv[2])
