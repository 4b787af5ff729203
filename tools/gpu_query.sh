set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_query.py -x -q > gpurun_out/q_tests.log 2>&1; echo qtests rc=$?
tail -15 gpurun_out/q_tests.log
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo tests rc=$?
tail -3 gpurun_out/gpu_tests.log
timeout 900 python bench.py --no-big --no-cpu-baseline --steps 50 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
tail -3 gpurun_out/bench.err
