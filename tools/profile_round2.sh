#!/bin/bash
# Round-2 evidence on one B200: the default bench line (c3 headline + configs block), the reference arm,
# the N=2 code path over gloo, launch lists, ncu --set full of the chunk kernel on c3/c2/c4/c5 and of the
# decoder kernels on c2, the int-pipe microbenchmark.  Usage: tools/profile_round2.sh TAG
TAG=${1:-r2}
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1 || tail -20 gpurun_out/build_$TAG.log
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu_$TAG.txt
./tools/micro/int_peak > gpurun_out/int_peak_$TAG.json
python bench.py > gpurun_out/bench_default_$TAG.json 2> gpurun_out/bench_default_$TAG.err
python bench.py --impl reference > gpurun_out/bench_ref_$TAG.json 2>&1
BENCH_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
   --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline --assemble \
   > gpurun_out/bench_n2gloo_$TAG.json 2> gpurun_out/bench_n2gloo_$TAG.err
for cfg in c2_csource_128m c4_random_1g c5_tarmix_64g; do
  python bench.py --config $cfg --steps 5 --warmup 3 --no-other-configs > gpurun_out/bench_${cfg}_$TAG.json 2>&1
done
CULZSS_BENCH_NO_LIVE_PEAK=1 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e \
    --no-decompress --no-versions --no-other-configs > /dev/null 2>&1
CULZSS_BENCH_NO_LIVE_PEAK=1 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches_dec_$TAG.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e \
    --no-versions --no-other-configs > /dev/null 2>&1
for cfg in c3_runs20_1g c2_csource_128m c4_random_1g c5_tarmix_64g; do
  CULZSS_BENCH_NO_LIVE_PEAK=1 ncu --set full --clock-control none --import-source on -k regex:chunk_kernel -s 1 -c 1 \
      -o gpurun_out/full_${cfg}_$TAG python bench.py --config $cfg --steps 1 --warmup 1 --no-cpu-baseline --no-e2e \
      --no-versions --no-decompress --no-other-configs > /dev/null 2>&1
done
for cfg in c2_csource_128m c3_runs20_1g c4_random_1g; do bash tools/dec_launch.sh $TAG $cfg > gpurun_out/declaunch_${cfg}_$TAG.txt 2>&1; done
CULZSS_BENCH_NO_LIVE_PEAK=1 ncu --set full --clock-control none --import-source on -k regex:decode_kernel -s 1 -c 1 \
    -o gpurun_out/full_decode_kernel_c3_$TAG python bench.py --config c3_runs20_1g --steps 1 --warmup 1 --no-cpu-baseline \
    --no-e2e --no-versions --no-other-configs > /dev/null 2>&1
CULZSS_BENCH_NO_LIVE_PEAK=1 ncu --set full --clock-control none --import-source on -k regex:literal_kernel -s 1 -c 1 \
    -o gpurun_out/full_literal_kernel_c4_$TAG python bench.py --config c4_random_1g --steps 1 --warmup 1 --no-cpu-baseline \
    --no-e2e --no-versions --no-other-configs > /dev/null 2>&1
# version 2: the bench's versions leg launches the V2 instantiation (-s 1 skips its warm-up launch;
# the filter matches the mangled name of the V2 instantiation only)
CULZSS_BENCH_NO_LIVE_PEAK=1 ncu --set full --clock-control none --import-source on \
    --kernel-name-base mangled -k 'regex:chunk_kernelILi0ELb0ELb1ELb0ELb0E' -s 1 -c 1 \
    -o gpurun_out/full_v2_c2_$TAG python bench.py --config c2_csource_128m --steps 1 --warmup 1 --no-cpu-baseline \
    --no-e2e --no-decompress --no-other-configs > /dev/null 2>&1
for k in walk_kernel decode_kernel; do
  CULZSS_BENCH_NO_LIVE_PEAK=1 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 \
      -o gpurun_out/full_${k}_c2_$TAG python bench.py --config c2_csource_128m --steps 1 --warmup 1 --no-cpu-baseline \
      --no-e2e --no-versions --no-other-configs > /dev/null 2>&1
done
ls gpurun_out/*_$TAG* | head -40
python - "$TAG" <<'PY'
import json, sys
t = sys.argv[1]
for f in (f"gpurun_out/bench_default_{t}.json", f"gpurun_out/bench_n2gloo_{t}.json", f"gpurun_out/bench_ref_{t}.json"):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, round(d["value"], 1), d.get("roofline", {}).get("frac"), (d.get("decompress") or {}).get("value"),
              (d.get("e2e") or {}).get("value"), d.get("clocks"))
    except Exception as e:
        print(f, "unreadable", e)
PY
