set -u
mkdir -p gpurun_out
for c in NSko NSkv; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k3p_postscan -s 1 -c 1 \
    -o gpurun_out/p1_${c}_k3 python tools/run_case.py $c 2 > /dev/null 2>&1
done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k1_prescan -s 1 -c 1 \
    -o gpurun_out/p1_C3_k1 python tools/run_case.py C3 2 > /dev/null 2>&1
ls -la gpurun_out
