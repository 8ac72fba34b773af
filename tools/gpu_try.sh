#!/bin/bash
# Build here, refuse to ship a failed build, then run tools/gpu_round.sh TAG on the GPU box (retrying busy slots).
cd /root/repo
if python -m paper_conf_cluster_ozsoys11_b200.build --force 2>&1 | grep -E " error" ; then echo BUILD FAILED; exit 1; fi
NCU=${NCU:-0}
if [ "$NCU" = 1 ]; then CMD="$ENVV bash tools/gpu_round.sh $1"; else CMD="$ENVV NO_NCU=1 bash tools/gpu_round.sh $1"; fi
tools/gpu.sh 1200 "$CMD"
