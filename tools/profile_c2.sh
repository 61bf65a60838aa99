#!/usr/bin/env bash
# GPU box: launch list of the default bench command + full ncu captures of the headline config's
# kernels, summarised ON the box (only text comes back: .ncu-rep files exceed gpurun's 64 MiB cap).
# usage: bash tools/profile_c2.sh TAG [CFG]
set -u
TAG=${1:-r01c}
CFG=${2:-C2}
mkdir -p gpurun_out profiles
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/prof_${TAG}_launches.csv python bench.py --steps 3 --warmup 3 --no-extra --no-cpu \
  > gpurun_out/prof_${TAG}_launches_bench.log 2>&1
for k in k1r_prescan k3v_postscan; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 \
    -o gpurun_out/prof_${TAG}_${CFG}_$k python tools/run_case.py $CFG 2 > /dev/null 2>&1
done
python tools/summarize_profiles.py $TAG > gpurun_out/prof_${TAG}_summarize.log 2>&1
cp profiles/${TAG}_summary.md profiles/ncu_traffic.json gpurun_out/ 2>/dev/null
for r in gpurun_out/prof_${TAG}_*.ncu-rep; do
  python tools/ncu_stalls.py $r 30 > ${r%.ncu-rep}_lines.txt 2>&1
done
rm -f gpurun_out/*.ncu-rep
ls gpurun_out
