#!/usr/bin/env bash
# Run on the GPU box (via gpurun): the launch list of the default bench command + one full ncu
# capture of each hot kernel on the headline / north-star / BJ configs.
# Output: gpurun_out/prof_<tag>_*.  Summarise here with: python tools/summarize_profiles.py <tag>
set -u
TAG=${1:-r02}
mkdir -p gpurun_out
# (1) every launch with its device time (cold-cache, serialised: compare SHARES, not absolutes)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/prof_${TAG}_launches.csv python bench.py --steps 3 --warmup 3 --no-extra --no-cpu \
  > gpurun_out/prof_${TAG}_launches_bench.log 2>&1
cap() {  # cap CONFIG KERNEL_REGEX
  timeout 400 ncu --set full --clock-control none --import-source on -k regex:$2 -s 1 -c 1 \
    -o gpurun_out/prof_${TAG}_$1_$2 python tools/run_one.py $1 2 > /dev/null 2>&1
}
cap NSko k3v_postscan
cap NSkv k3v_postscan
cap NSkv k1r_prescan
cap C4ko k3_postscan
cap C4ko k1a_prescan
cap C4ko k2w_rowscan
cap C3 k3v_postscan
cap IDSko k3v_postscan
cap sweep_m64_ko k3v_postscan
ls gpurun_out | grep prof_${TAG}
# summarise on the box (the .ncu-rep files are too large to bring back): text summaries only
PROF_OUT=gpurun_out python tools/summarize_profiles.py ${TAG} > /dev/null 2>&1
for f in gpurun_out/prof_${TAG}_*.ncu-rep; do
  b=$(basename $f .ncu-rep)
  python tools/ncu_summary.py $f > gpurun_out/${b}_metrics.txt 2>&1
  python tools/ncu_lines.py $f 40 > gpurun_out/${b}_lines.txt 2>&1
done
mkdir -p /tmp/ncu_reps && mv gpurun_out/prof_${TAG}_*.ncu-rep /tmp/ncu_reps/ 2>/dev/null
ls gpurun_out | grep ${TAG}
