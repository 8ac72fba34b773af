#!/bin/bash
# Sweep the walk's switch thresholds over configs.  Usage: tools/sw_sweep.sh TAG "sw:tx ..." cfg...
TAG=$1; SWS=$2; shift 2
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
for cfg in "$@"; do
  for st in $SWS; do
    sw=${st%%:*}; tx=${st##*:}
    CULZSS_WALK_SWITCH=$sw CULZSS_WALK_TOKEN_SWITCH=$tx python bench.py --config $cfg --steps 5 --warmup 2 --no-cpu-baseline --no-e2e --no-versions \
      --no-decompress --no-other-configs > gpurun_out/sw_${TAG}_${cfg}_${sw}_$tx.json 2>&1
    python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(sys.argv[2], sys.argv[3], round(d['value'],1), round(d['kernels_ms']['chunk'],3))" gpurun_out/sw_${TAG}_${cfg}_${sw}_$tx.json $cfg $st || tail -3 gpurun_out/sw_${TAG}_${cfg}_${sw}_$tx.json
  done
done
