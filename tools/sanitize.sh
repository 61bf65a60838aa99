#!/bin/bash
# compute-sanitizer over tools/sanitize_cases.py (every kernel family, small n), one tool per pass
# (TOOLS="... initcheck" adds initcheck, which misreads TMA bulk stores as uninitialised output);
# logs under gpurun_out/sanitize_<tool>.log.  usage: bash tools/sanitize.sh [n]
set -u
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
N=${1:-}
for tool in ${TOOLS:-memcheck racecheck synccheck}; do
  timeout 1500 /usr/local/cuda/bin/compute-sanitizer --tool $tool --error-exitcode 99 \
    $( [ $tool = racecheck ] && echo --racecheck-report all ) \
    python tools/sanitize_cases.py $N > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?" | tee -a gpurun_out/sanitize_summary.txt
  tail -3 gpurun_out/sanitize_$tool.log
done
