set -x
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k code_network > gpurun_out/t_cnet.log 2>&1; echo cnet rc=$?
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo tests rc=$?
tail -5 gpurun_out/gpu_tests.log
timeout 120 python tools/netbench.py > gpurun_out/netbench2.log 2>&1
timeout 300 bash tools/trace_run.sh
timeout 600 python bench.py --no-cpu-baseline --no-big --steps 50 > gpurun_out/bench.log 2>&1; echo bench rc=$?
