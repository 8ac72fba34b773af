#!/usr/bin/env python
"""Per-source-line warp instructions and stall samples of one ncu report
(needs a -lineinfo build and --import-source on), grouped into the kernel's
phases by line ranges.

    python tools/ncu_lines.py REPORT.ncu-rep [FILE_SUBSTR] [START:END:NAME ...] [--top N]
"""
import csv
import io
import subprocess
import sys


def per_line(report, file_sub):
    out = subprocess.run(["ncu", "-i", report, "--page", "source", "--csv", "--print-source",
                          "cuda,sass"], capture_output=True, text=True).stdout
    cur_file, hdr, res = None, None, {}
    for row in csv.reader(io.StringIO(out)):
        if not row:
            continue
        if row[0] == "File Path":
            cur_file = row[1]
            continue
        if row[0] == "Line No":
            hdr = row
            continue
        if row[0] in ("Function Name",) or hdr is None or not row[0]:
            continue
        if file_sub not in (cur_file or ""):
            continue
        d = dict(zip(hdr[4:], row[4:]))
        try:
            ins = float(d["Instructions Executed"])
            smp = float(d["Warp Stall Sampling (All Samples)"])
        except (KeyError, ValueError):
            continue
        res[int(row[0])] = (ins, smp, row[1].strip())
    return res


def main():
    args = [a for a in sys.argv[1:]]
    top = 25
    if "--top" in args:
        i = args.index("--top")
        top = int(args[i + 1])
        del args[i:i + 2]
    report = args[0]
    file_sub = args[1] if len(args) > 1 else "lzss_chunk.cu"
    ranges = [a.split(":") for a in args[2:]]
    res = per_line(report, file_sub)
    tot_i = sum(v[0] for v in res.values()) or 1
    tot_s = sum(v[1] for v in res.values()) or 1
    print(f"total warp instr {tot_i:.4g}, samples {tot_s:.0f}")
    for r in ranges:
        a, b, name = int(r[0]), int(r[1]), r[2]
        i = sum(v[0] for k, v in res.items() if a <= k <= b)
        s = sum(v[1] for k, v in res.items() if a <= k <= b)
        print(f"{name:>16s} lines {a}-{b}: instr {100 * i / tot_i:5.1f}%  samples {100 * s / tot_s:5.1f}%")
    print("\ntop lines by stall samples:")
    for k, v in sorted(res.items(), key=lambda kv: -kv[1][1])[:top]:
        print(f"{k:5d} instr {100 * v[0] / tot_i:5.1f}% samples {100 * v[1] / tot_s:5.1f}%  {v[2][:90]}")


if __name__ == "__main__":
    main()
