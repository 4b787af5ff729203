for k in 1 32 128 256 1024; do python tools/trace.py 536870912 uniform $k; done > gpurun_out/trace.log 2>&1
python tools/trace.py 536870912 increasing 256 >> gpurun_out/trace.log 2>&1
python tools/trace.py 536870912 fewdistinct 256 >> gpurun_out/trace.log 2>&1
