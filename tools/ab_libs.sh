#!/usr/bin/env bash
# A/B timing of alternative libms builds on one GPU: for every ab/libms_<tag>.so, install it as the
# package's libms.so and run tools/quick_bench.py on the given configs (twice, interleaved).
# usage: bash tools/ab_libs.sh CONFIGS [steps]
set -u
CF=${1:-C4ko,C4kv}; ST=${2:-20}
LIB=paper_conf_ppopp_ashkianidmo16_b200/libms.so
for pass in 1 2; do
  for f in ab/libms_*.so; do
    t=$(basename $f .so); t=${t#libms_}
    cp $f $LIB; touch $LIB
    TAG="$t.$pass" timeout 900 python tools/quick_bench.py $CF $ST
  done
done
