set -x
mkdir -p gpurun_out
R=r1s3
NCU="ncu --set full --clock-control none --import-source on -s 3 -c 1"
timeout 600 $NCU -k regex:select_kernel -o gpurun_out/prof_select_k256_$R -f python tools/prof_any.py select 256 > gpurun_out/ncu_sel.log 2>&1
timeout 600 $NCU -k regex:select_kernel -o gpurun_out/prof_select_k1024_$R -f python tools/prof_any.py select 1024 > gpurun_out/ncu_sel1024.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'select_kernel|merge_kernel' -c 60 --csv --log-file gpurun_out/launches_$R.csv python bench.py --steps 20 --warmup 3 --no-sweep --no-cpu-baseline --no-big > gpurun_out/ncu_bench.log 2>&1; echo ncu rc=$?
