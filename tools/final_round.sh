#!/usr/bin/env bash
# End-of-round evidence on one B200 (via gpurun): full GPU tests, smoke, the default bench line,
# the reference arm, the Table-4 ablation, and ncu traffic for every bench workload.
# Output: gpurun_out/final_<tag>_*.  usage: bash tools/final_round.sh TAG
set -u
TAG=${1:-r02}
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/final_${TAG}_pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/final_${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_${TAG}_smoke.log 2>&1
timeout 1500 python bench.py > gpurun_out/final_${TAG}_bench.json 2> gpurun_out/final_${TAG}_bench.err
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/final_${TAG}_reference.json 2>&1
timeout 900 python tools/ablation.py 10 25 > gpurun_out/final_${TAG}_ablation.md 2> gpurun_out/final_${TAG}_ablation.err
CFGS=$(python -c "import bench; print(','.join(['NSko'] + bench.EXTRA_DEFAULT.split(',')))")
timeout 2400 python tools/ncu_traffic.py $CFGS > gpurun_out/final_${TAG}_ncu_traffic.log 2>&1
tail -2 gpurun_out/final_${TAG}_pytest_gpu.log; tail -1 gpurun_out/final_${TAG}_smoke.log
tail -c 300 gpurun_out/final_${TAG}_bench.json; tail -1 gpurun_out/final_${TAG}_ncu_traffic.log
