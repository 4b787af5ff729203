set -x
mkdir -p gpurun_out
timeout 200 python tools/quick_time.py $((1<<29)) uniform filter 1,32,256,1024 > gpurun_out/qt_new.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo tests rc=$?
tail -3 gpurun_out/gpu_tests.log
timeout 900 python bench.py --no-big --no-cpu-baseline --steps 50 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
tail -3 gpurun_out/bench.err
