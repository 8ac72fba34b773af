#!/bin/bash
# Round-end evidence on one B200: bench lines, launch list, ncu --set full of
# the chunk kernel on three configs.  Usage: tools/profile_round.sh TAG
TAG=${1:-r1}
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu_$TAG.txt
python bench.py --steps 10 --warmup 3 > gpurun_out/bench_full_$TAG.json 2> gpurun_out/bench_full_$TAG.err
python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$TAG.json 2>&1
BENCH_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
   --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline \
   > gpurun_out/bench_n2gloo_$TAG.json 2> gpurun_out/bench_n2gloo_$TAG.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
    --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e \
    --no-decompress --no-versions > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
    --log-file gpurun_out/launches_dec_$TAG.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e \
    --no-versions > /dev/null 2>&1
for cfg in c2_csource_128m c4_random_1g c3_runs20_1g; do
  ncu --set full --clock-control none --import-source on -k regex:chunk_kernel -s 1 -c 1 \
      -o gpurun_out/full_${cfg}_$TAG python bench.py --config $cfg --steps 1 --warmup 1 --no-cpu-baseline --no-e2e \
      --no-versions > /dev/null 2>&1
done
for k in walk_kernel decode_kernel; do
  ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 \
      -o gpurun_out/full_${k}_c2_$TAG python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e \
      --no-versions > /dev/null 2>&1
done
python bench.py --config c5_tarmix_64g --steps 3 --warmup 3 > gpurun_out/bench_c5_$TAG.json 2>&1
python bench.py --config c3_runs20_1g --steps 5 --warmup 3 > gpurun_out/bench_c3_$TAG.json 2>&1
python bench.py --config c4_random_1g --steps 5 --warmup 3 > gpurun_out/bench_c4_$TAG.json 2>&1
tail -c 3000 gpurun_out/bench_full_$TAG.json; echo; tail -3 gpurun_out/bench_n2gloo_$TAG.json; tail -c 600 gpurun_out/bench_ref_$TAG.json
