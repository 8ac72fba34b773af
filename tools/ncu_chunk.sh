#!/bin/bash
# ncu --set full of the fused chunk kernel on the given configs.  Usage: tools/ncu_chunk.sh TAG cfg...
TAG=$1; shift
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
for cfg in "$@"; do
  ncu --set full --clock-control none --import-source on -k regex:chunk_kernel -s 1 -c 1 \
      -o gpurun_out/full_${cfg}_$TAG python bench.py --config $cfg --steps 1 --warmup 1 --no-cpu-baseline --no-e2e \
      --no-versions --no-decompress --no-other-configs > gpurun_out/ncu_${cfg}_$TAG.log 2>&1
  ls -la gpurun_out/full_${cfg}_$TAG.ncu-rep
done
