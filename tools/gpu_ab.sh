set -x
mkdir -p gpurun_out
nvidia-smi -q -d CLOCK,PERFORMANCE > gpurun_out/smi_q.txt 2>&1
timeout 200 python tools/probe_bw.py > gpurun_out/probe.log 2>&1
for i in 1 2; do
TOPK_LIB=tools/old_libtopk.so timeout 200 python tools/quick_time.py $((1<<29)) uniform filter 1,256 > gpurun_out/qt_old_$i.log 2>&1
timeout 200 python tools/quick_time.py $((1<<29)) uniform filter 1,256 > gpurun_out/qt_new_$i.log 2>&1
done
timeout 900 python -m pytest tests/test_gpu_query.py -x -q > gpurun_out/q_tests.log 2>&1; echo qtests rc=$?
tail -15 gpurun_out/q_tests.log
