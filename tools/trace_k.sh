for k in 256 512 1024 2048; do timeout 120 python tools/trace.py 536870912 uniform $k; done > gpurun_out/trace.log 2>&1
cat gpurun_out/trace.log
