#!/usr/bin/env bash
# Run on the GPU box (via gpurun): launch list of the default bench command + full ncu
# captures of the hot kernels for the headline config and the north-star configs.
# Output: gpurun_out/prof_<tag>_*.  Summarise here with: python tools/summarize_profiles.py <tag>
set -u
TAG=${1:-r01}
CFG=${2:-C2}
mkdir -p gpurun_out
# (1) every launch with its device time (cold-cache, serialised: compare SHARES, not absolutes)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/prof_${TAG}_launches.csv python bench.py --steps 3 --warmup 3 --no-extra --no-cpu \
  > gpurun_out/prof_${TAG}_launches_bench.log 2>&1
# (2) one full capture per hot kernel (K1, K2, K3) on the headline config
for k in k1r_prescan k3v_postscan; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 \
    -o gpurun_out/prof_${TAG}_${CFG}_$k python tools/run_case.py $CFG 2 > /dev/null 2>&1
done
# (3) K3 (and K1) on the north-star and BJ configs
for c in NSko NSkv C3; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k3v_postscan -s 1 -c 1 \
    -o gpurun_out/prof_${TAG}_${c}_k3v_postscan python tools/run_case.py $c 2 > /dev/null 2>&1
done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k1_prescan -s 1 -c 1 \
  -o gpurun_out/prof_${TAG}_NSko_k1_prescan python tools/run_case.py NSko 2 > /dev/null 2>&1
for c in C4ko; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k3_postscan -s 1 -c 1 \
    -o gpurun_out/prof_${TAG}_${c}_k3_postscan python tools/run_case.py $c 2 > /dev/null 2>&1
done
ls gpurun_out | grep prof_${TAG}
