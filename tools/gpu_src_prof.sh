# source-level stall attribution of one kernel (ncu --page source), exported on the box
mkdir -p gpurun_out
OP=$1; K=$2; KR=$3; TAG=$4
timeout 600 ncu --set full --clock-control none --import-source on -s 3 -c 1 -k regex:$KR -o /tmp/src_$TAG -f python tools/prof_any.py $OP $K > /dev/null 2>&1
ncu -i /tmp/src_$TAG.ncu-rep --page source --csv --print-source sass > gpurun_out/src_$TAG.csv 2>/dev/null
ncu -i /tmp/src_$TAG.ncu-rep --page source --csv > gpurun_out/srcline_$TAG.csv 2>/dev/null
ls -la gpurun_out/src_$TAG.csv gpurun_out/srcline_$TAG.csv
