mkdir -p gpurun_out
NCU="ncu --set full --clock-control none --import-source on -s 2 -c 1"
timeout 600 $NCU -k regex:pure_kernel -o gpurun_out/prof_purenew_k32_${1:-r2} -f python tools/prof_any.py pure 32 > gpurun_out/ncu_pn32.log 2>&1
timeout 600 $NCU -k regex:pure_kernel -o gpurun_out/prof_purenew_k1_${1:-r2} -f python tools/prof_any.py pure 1 > gpurun_out/ncu_pn1.log 2>&1
echo done
