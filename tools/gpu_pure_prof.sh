set -x
mkdir -p gpurun_out
R=r2
NCU="ncu --set full --clock-control none --import-source on -s 3 -c 1"
timeout 900 $NCU -k regex:select_kernel -o gpurun_out/prof_pure_k32_$R -f python tools/prof_any.py pure 32 > gpurun_out/ncu_pure32.log 2>&1
timeout 900 $NCU -k regex:select_kernel -o gpurun_out/prof_pure_k256_$R -f python tools/prof_any.py pure 256 > gpurun_out/ncu_pure256.log 2>&1
echo done
