#!/bin/bash
# Full check on one B200: GPU tests, smoke, the default bench line, the reference arm, the N=2 path over
# gloo (two ranks on the one GPU), the int-pipe microbenchmark.  Usage: tools/gpu_check.sh TAG
TAG=${1:-x}
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1 || tail -20 gpurun_out/build_$TAG.log
./tools/micro/int_peak > gpurun_out/int_peak_$TAG.json; cat gpurun_out/int_peak_$TAG.json
if [ -z "$NO_TESTS" ]; then timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4; fi
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
python bench.py > gpurun_out/bench_default_$TAG.json 2> gpurun_out/bench_default_$TAG.err; tail -c 400 gpurun_out/bench_default_$TAG.err
python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$TAG.json 2>&1
BENCH_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
   --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline --assemble \
   > gpurun_out/bench_n2gloo_$TAG.json 2> gpurun_out/bench_n2gloo_$TAG.err; tail -c 300 gpurun_out/bench_n2gloo_$TAG.err
python - "$TAG" <<'PY'
import json, sys
t = sys.argv[1]
for f in (f"gpurun_out/bench_default_{t}.json", f"gpurun_out/bench_n2gloo_{t}.json", f"gpurun_out/bench_ref_{t}.json"):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "unreadable", e); continue
    brief = {k: d.get(k) for k in ("value", "ms_per_step", "ratio", "scaling", "n_gpus", "gpu_launches")}
    brief["roofline"] = {k: d.get("roofline", {}).get(k) for k in ("frac", "peak", "bound")}
    brief["dec"] = (d.get("decompress") or {}).get("value")
    brief["e2e"] = (d.get("e2e") or {}).get("value")
    brief["exchange"] = d.get("exchange")
    brief["configs"] = {k: (round(v.get("value", 0), 1), v.get("us_per_call_device"), v.get("roofline_frac")) for k, v in (d.get("configs") or {}).items()}
    print(f, json.dumps(brief))
PY
