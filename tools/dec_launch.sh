#!/bin/bash
# Launch list (cold, serialised) of the decoder kernels on one config.  Usage: tools/dec_launch.sh TAG cfg
TAG=$1; cfg=${2:-c4_random_1g}
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"classify_kernel|walk_kernel|decode_kernel|literal_kernel" -c 12 --csv \
    --log-file gpurun_out/declaunch_${cfg}_$TAG.csv python bench.py --config $cfg --steps 2 --warmup 1 --no-cpu-baseline \
    --no-e2e --no-versions --no-other-configs > /dev/null 2>&1
python - gpurun_out/declaunch_${cfg}_$TAG.csv <<'PY'
import csv, sys, collections
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]; ki = h.index("Kernel Name"); vi = h.index("Metric Value")
d = collections.defaultdict(list)
for r in rows[1:]:
    d[r[ki].split("(")[0]].append(float(r[vi].replace(",", "")))
for k, v in d.items(): print(k, [round(x / 1000, 1) for x in v], "us")
PY
