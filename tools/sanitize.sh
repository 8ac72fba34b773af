#!/bin/bash
# compute-sanitizer over tools/sanitize_run.py, one tool at a time.  Usage: tools/sanitize.sh TAG
TAG=${1:-x}
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  extra=""
  [ $tool = memcheck ] && extra="--leak-check no"
  [ $tool = racecheck ] && extra="--racecheck-report all --print-limit 3000"
  timeout 1500 compute-sanitizer --tool $tool $extra --error-exitcode 9 \
      python tools/sanitize_run.py > gpurun_out/sanitize_${tool}_$TAG.txt 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|sanitize workload ok' gpurun_out/sanitize_${tool}_$TAG.txt | tr '\n' ' ')"
done
