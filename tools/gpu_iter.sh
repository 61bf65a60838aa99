#!/usr/bin/env bash
# One GPU iteration: parity tests, quick bench (new K3 vs old), optional ncu of one config.
# usage: bash tools/gpu_iter.sh TAG "C2,NSko" [ncu_cfg] [ncu_kernel_regex]
TAG=$1; CFGS=${2:-C1,C2,C3,C3bin,NSko,NSkv}; NCFG=${3:-}; NK=${4:-k3v_postscan}
mkdir -p gpurun_out
(timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -4) > gpurun_out/${TAG}_pytest.log
timeout 300 python tools/quick_bench.py $CFGS 10 > gpurun_out/${TAG}_qb.log 2>&1
if [ -n "$OLD" ]; then MS_K3V=0 TAG=old timeout 300 python tools/quick_bench.py $OLD 10 >> gpurun_out/${TAG}_qb.log 2>&1; fi
if [ -n "$NCFG" ]; then
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$NK -s 1 -c 1 \
    -o gpurun_out/${TAG}_${NCFG}_ncu python tools/run_case.py $NCFG 2 > /dev/null 2>&1
fi
cat gpurun_out/${TAG}_pytest.log gpurun_out/${TAG}_qb.log
