#!/usr/bin/env bash
# Run on the GPU box (via gpurun): launch list of the default bench command + full ncu
# captures of the hot kernels for the headline config.  Output: gpurun_out/prof_<tag>_*.
set -u
TAG=${1:-r01}
CFG=${2:-C2}
mkdir -p gpurun_out
# (1) every launch with its device time (cold-cache, serialised: compare SHARES, not absolutes)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/prof_${TAG}_launches.csv python bench.py --steps 3 --warmup 3 --no-extra --no-cpu \
  > gpurun_out/prof_${TAG}_launches_bench.log 2>&1
# (2) one full capture per hot kernel (K1, K2, K3) on the headline config
for k in k1_prescan k2_scan k3p_postscan; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 \
    -o gpurun_out/prof_${TAG}_${CFG}_$k python tools/run_case.py $CFG 2 > /dev/null 2>&1
done
for c in NSko NSkv; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k3p_postscan -s 1 -c 1 \
    -o gpurun_out/prof_${TAG}_${c}_k3p_postscan python tools/run_case.py $c 2 > /dev/null 2>&1
done
ls gpurun_out | grep prof_${TAG}
