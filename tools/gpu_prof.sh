#!/bin/bash
# Build here, then one ncu --set full capture of the chunk kernel (c2 csource) on the GPU box.
cd /root/repo
if python -m paper_conf_cluster_ozsoys11_b200.build --force 2>&1 | grep -E " error" ; then echo BUILD FAILED; exit 1; fi
CFG=${CFG:-c2_csource_128m}
timeout 1500 /usr/local/graft/bin/gpurun --timeout 600 -- "ncu --set full --clock-control none --import-source on -k regex:${KER:-chunk_kernel} -s 1 -c 1 -o gpurun_out/prof_$1 python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu-baseline --no-e2e ${NODEC---no-decompress} > gpurun_out/prof_$1.log 2>&1" 2>&1 | tail -1
python tools/ncu_summary.py full gpurun_out/prof_$1.ncu-rep $1 | sed -n 5,16p
