# ncu captures of the hot-path kernels (one GPU, one launch each after warm-ups)
set -x
mkdir -p gpurun_out
R=${R:-r1s3}
NCU="ncu --set full --clock-control none --import-source on -s 3 -c 1"
timeout 600 $NCU -k regex:select_kernel -o gpurun_out/prof_select_k256_$R -f python tools/prof_any.py select 256 > gpurun_out/ncu_sel.log 2>&1
timeout 600 $NCU -k regex:select_kernel -o gpurun_out/prof_query1_$R -f python tools/prof_any.py query1 50 > gpurun_out/ncu_q1.log 2>&1
timeout 600 $NCU -k regex:select_kernel -o gpurun_out/prof_query2_$R -f python tools/prof_any.py query2 50 > gpurun_out/ncu_q2.log 2>&1
timeout 600 $NCU -k regex:select_kernel -o gpurun_out/prof_kk_$R -f python tools/prof_any.py kk 64 > gpurun_out/ncu_kk.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:radix_hist -s 4 -c 1 -o gpurun_out/prof_radix_hist_$R -f python tools/prof_any.py radix 256 > gpurun_out/ncu_rh.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'select_kernel|merge_kernel' -c 60 --csv --log-file gpurun_out/launches_$R.csv python bench.py --steps 20 --warmup 3 --no-sweep --no-cpu-baseline --no-big > gpurun_out/ncu_bench.log 2>&1; echo ncu rc=$?
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/radix_launches.csv python tools/prof_any.py radix 256 > /dev/null 2>&1
ls -la gpurun_out
