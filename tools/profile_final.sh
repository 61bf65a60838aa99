#!/usr/bin/env bash
# GPU box: launch list of the default bench + full captures of the headline kernel (C2) and of the
# m=256 post-scan (C4ko), summarised ON the box (only text comes back).  usage: bash tools/profile_final.sh TAG
set -u
TAG=${1:-r01e}
bash tools/profile_c2.sh $TAG C2 > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k3_postscan -s 1 -c 1 \
  -o gpurun_out/prof_${TAG}_C4ko_k3_postscan python tools/run_case.py C4ko 2 > /dev/null 2>&1
python tools/ncu_summary.py gpurun_out/prof_${TAG}_C4ko_k3_postscan.ncu-rep > gpurun_out/prof_${TAG}_C4ko_k3_postscan.txt 2>&1
python tools/ncu_stalls.py gpurun_out/prof_${TAG}_C4ko_k3_postscan.ncu-rep 25 >> gpurun_out/prof_${TAG}_C4ko_k3_postscan.txt 2>&1
rm -f gpurun_out/*.ncu-rep
ls gpurun_out | grep $TAG
