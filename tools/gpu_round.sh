#!/bin/bash
# Dev loop on the GPU box: parity tests, benches on the 1-GPU configs,
# optionally one ncu --set full capture of the fused chunk kernel.  Usage: tools/gpu_round.sh TAG
TAG=${1:-x}
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
if [ -z "$NO_TESTS" ]; then timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -8; fi
python bench.py --config c2_csource_128m --steps 10 --warmup 3 --no-cpu-baseline --no-versions > gpurun_out/bench_c2_$TAG.json 2>&1
python bench.py --config c4_random_1g --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-versions > gpurun_out/bench_c4_$TAG.json 2>&1
python bench.py --config c3_runs20_1g --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-versions > gpurun_out/bench_c3_$TAG.json 2>&1
if [ -n "$C5" ]; then python bench.py --config c5_tarmix_64g --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-versions > gpurun_out/bench_c5_$TAG.json 2>&1; fi
if [ -z "$NO_NCU" ]; then
  ncu --set full --clock-control none --import-source on -k regex:chunk_kernel -s 1 -c 1 \
      -o gpurun_out/prof_chunk_$TAG python bench.py --config ${NCU_CFG:-c2_csource_128m} --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-versions \
      > gpurun_out/prof_$TAG.log 2>&1
fi
for f in gpurun_out/bench_c*_$TAG.json; do
  python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(sys.argv[1], round(d['value'],1), {k: round(v,3) for k,v in d['kernels_ms'].items()}, round(d['ratio'],4), 'dec', round(d.get('decompress',{}).get('value',0),1), round(d.get('decompress',{}).get('decode_kernel_ms',0),3))" $f || tail -5 $f
done
