#!/bin/bash
# Write profiles/<TAG>_ncu_summary.md and profiles/traffic.json from gpurun_out/*_<TAG>* (the outputs of
# tools/profile_round2.sh TAG).  Usage: tools/write_summary2.sh TAG
TAG=$1
cd "$(dirname "$0")/.."
python - "$TAG" > profiles/${TAG}_ncu_summary.md <<'PY'
import json, subprocess, sys
t = sys.argv[1]
def line(f):
    return json.loads(open(f).read().strip().splitlines()[-1])
d = line(f"gpurun_out/bench_default_{t}.json")
print(f"# Round 2 evidence, capture {t} (B200)\n")
print(f"Captured with `tools/profile_round2.sh {t}`: bench lines without a profiler, launch lists "
      "(`ncu --metrics gpu__time_duration.sum --clock-control none`: per-launch, cold-cache, serialised -- compare "
      "shares, not absolute times) and `ncu --set full --clock-control none --import-source on` of one launch after "
      "warm-up.  Integer-pipe peak measured on the same box: `" + open(f"gpurun_out/int_peak_{t}.json").read().strip() + "`.\n")
print("## Bench lines (no profiler)\n")
print("| config | compress GB/s | ratio | chunk kernel ms | roofline frac (ALU-pipe peak) | decompress GB/s | e2e GB/s | SM MHz / throttle |")
print("|---|---|---|---|---|---|---|---|")
rows = [("default (" + d["config"]["workload"].split(":")[0] + ")", d)]
for cfg in ("c2_csource_128m", "c4_random_1g", "c5_tarmix_64g"):
    try:
        rows.append((cfg, line(f"gpurun_out/bench_{cfg}_{t}.json")))
    except Exception:
        pass
for name, x in rows:
    print("| %s | %.1f | %.4f | %.3f | %.3f | %.1f | %.1f | %s %s |" % (
        name, x["value"], x["ratio"], x["kernels_ms"]["chunk"], x["roofline"]["frac"], x["decompress"]["value"],
        x["e2e"]["value"], x["clocks"]["sm_mhz"], x["clocks"]["reasons"] or "none"))
c = d["cpu_baseline"]
print(f"\nCPU oracle beside the default line: {c['value']:.3f} GB/s on {c['cores']} threads ({c['sample']}); "
      f"single core {c['single_core']['value']:.4f} GB/s; parity with the GPU stream: {c['parity_with_gpu_stream']}.")
r = line(f"gpurun_out/bench_ref_{t}.json")
print(f"Reference arm (`--impl reference`, the oracle): {r['value']:.3f} GB/s on {r['cpu_baseline']['cores']} threads.")
n = line(f"gpurun_out/bench_n2gloo_{t}.json")
print(f"N=2 code path (gloo, two ranks sharing the one GPU; strong scaling of c3): {n['value']:.1f} GB/s aggregate, "
      f"exchange {n['exchange']['ms_per_step']:.3f} ms/step ({100 * n['exchange']['share_of_step']:.1f}% of a step, host-timed "
      f"gloo), sharded decompression {n['decompress']['value']:.1f} GB/s, assembly round trip exact: "
      f"{n.get('assembly', {}).get('roundtrip_exact')}.")
print("\n`configs` block of the default line (N = 1):\n")
for k, v in d.get("configs", {}).items():
    print(f"* {k}: " + ", ".join(f"{a} = {b:.4g}" if isinstance(b, float) else f"{a} = {b}" for a, b in v.items()
                                  if a not in ("workload", "what", "unit")))
sys.stdout.flush()
def run(*a):
    print(subprocess.run(["python", *a], capture_output=True, text=True).stdout)
print("\n## Launch list, compress only (default config, --steps 2 --warmup 3; torch L2-flush fill kernels included)\n")
run("tools/ncu_summary.py", "launches", f"gpurun_out/launches_{t}.csv")
print("## Launch list with the decompress leg\n")
run("tools/ncu_summary.py", "launches", f"gpurun_out/launches_dec_{t}.csv")
print("## Fused chunk kernel (rows a1-a4), --set full\n")
for cfg in ("c3_runs20_1g", "c2_csource_128m", "c4_random_1g", "c5_tarmix_64g"):
    run("tools/ncu_summary.py", "full", f"gpurun_out/full_{cfg}_{t}.ncu-rep", cfg)
print("### Per-phase split (tools/ncu_lines.py: warp instructions / stall samples by source line range)\n")
# phase line ranges from markers in the source (so they follow edits)
src = open("paper_conf_cluster_ozsoys11_b200/csrc/lzss_chunk.cu").read().split("\n")
def at(marker):
    return next(i + 1 for i, l in enumerate(src) if marker in l)
marks = [("// skewed byte index", "helpers"), ("__device__ uint32_t eval_pos", "evalpos"),
         ("// Run-boundary mask of a warp", "bndbuild"), ("// Speculative greedy walk", "machine1"),
         ("// ---- machine 2", "machine2"), ("// Re-walk from a corrected", "walkfix"),
         ("// Version 2: the paper", "version2"), ("void pair_sync(int id)", "kernelhead"),
         ("---------------- a1: stage", "stage"), ("---------------- a2 part 1", "build"),
         ("---------------- a3: lazy", "mask"), ("const int spec_exit =", "fixup"),
         ("---------------- a4: bit-pack", "emit"), ("exclusive scan of bit counts over the 64", "scan+write")]
starts = [(at(m), name) for m, name in marks]
rng = [f"{a}:{(starts[i + 1][0] - 1) if i + 1 < len(starts) else len(src)}:{name}" for i, (a, name) in enumerate(starts)]
for cfg in ("c3_runs20_1g", "c2_csource_128m", "c5_tarmix_64g"):
    print(f"{cfg}:\n```")
    print(subprocess.run(["python", "tools/ncu_lines.py", f"gpurun_out/full_{cfg}_{t}.ncu-rep", "lzss_chunk.cu", *rng,
                          "--top", "10"], capture_output=True, text=True).stdout + "```\n")
print("## Decoder (row a6), --set full\n")
for k in ("walk_kernel", "decode_kernel"):
    run("tools/ncu_summary.py", "full", f"gpurun_out/full_{k}_c2_{t}.ncu-rep", k + " (c2 stream)")
run("tools/ncu_summary.py", "full", f"gpurun_out/full_decode_kernel_c3_{t}.ncu-rep", "decode_kernel (c3 stream)")
run("tools/ncu_summary.py", "full", f"gpurun_out/full_literal_kernel_c4_{t}.ncu-rep", "literal_kernel (c4 stream)")
print("### Decoder launch lists per config (classify / literal / walk / decode, cold and serialised)\n")
for cfg in ("c2_csource_128m", "c3_runs20_1g", "c4_random_1g"):
    try:
        print(f"{cfg}:\n```\n" + open(f"gpurun_out/declaunch_{cfg}_{t}.txt").read() + "```\n")
    except Exception:
        pass
print("## Version 2 (the paper's all-position search), --set full, c2\n")
run("tools/ncu_summary.py", "full", f"gpurun_out/full_v2_c2_{t}.ncu-rep", "chunk_kernel, params.version = 2")
PY
python - "$TAG" <<'PY'
import csv, io, json, subprocess, sys
t = sys.argv[1]
per = {}
for cfg in ("c3_runs20_1g", "c2_csource_128m", "c4_random_1g", "c5_tarmix_64g"):
    out = subprocess.run(["ncu", "-i", f"gpurun_out/full_{cfg}_{t}.ncu-rep", "--page", "raw", "--csv"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u, r = rows[0], rows[1], rows[2]
    d, un = dict(zip(h, r)), dict(zip(h, u))
    def b(k):
        s = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(un[k], 1)
        return float(d[k].replace(",", "")) * s
    per[cfg] = int(b("dram__bytes_read.sum") + b("dram__bytes_write.sum"))
json.dump({"source": f"dram__bytes_read.sum + dram__bytes_write.sum of one chunk_kernel launch from ncu --set full "
                     f"(capture {t}, profiles/{t}_ncu_summary.md); bucket writes still in the 126 MB L2 at kernel end "
                     "are not counted by the DRAM counters",
           "per_launch_bytes": per}, open("profiles/traffic.json", "w"), indent=1)
print(per)
PY
cp gpurun_out/launches_$TAG.csv profiles/${TAG}_launches.csv
cp gpurun_out/launches_dec_$TAG.csv profiles/${TAG}_launches_dec.csv
for f in bench_default bench_ref bench_n2gloo bench_c2_csource_128m bench_c4_random_1g bench_c5_tarmix_64g int_peak; do
  cp gpurun_out/${f}_$TAG.json profiles/${TAG}_${f}.json 2>/dev/null
done
