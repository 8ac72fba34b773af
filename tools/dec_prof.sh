#!/bin/bash
# Decoder evidence on the GPU box: launch list per config + ncu --set full of
# walk_kernel and decode_kernel on c2.  Usage: tools/dec_prof.sh TAG
TAG=${1:-x}
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
for cfg in c2_csource_128m c4_random_1g c3_runs20_1g; do
  ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"walk|decode" -c 8 --csv \
      --log-file gpurun_out/ll_${cfg}_$TAG.csv python bench.py --config $cfg --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
done
if [ -z "$NO_FULL" ]; then
for k in ${KERS:-walk_kernel decode_kernel}; do
  ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 -o gpurun_out/prof_${k}_$TAG \
      python bench.py --config ${CFG:-c2_csource_128m} --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
done
fi
