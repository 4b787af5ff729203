set -x
mkdir -p gpurun_out
R=${R:-r1s3}
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo tests rc=$?
tail -3 gpurun_out/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 1200 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
tail -3 gpurun_out/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo ref rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'select_kernel|merge_kernel' -c 60 --csv --log-file gpurun_out/launches_$R.csv python bench.py --steps 20 --warmup 3 --no-sweep --no-cpu-baseline --no-big > gpurun_out/ncu_bench.log 2>&1; echo ncu rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:select_kernel -s 3 -c 1 -o gpurun_out/prof_kkk_$R -f python tools/prof_any.py kkk 64 > gpurun_out/ncu_kkk.log 2>&1
