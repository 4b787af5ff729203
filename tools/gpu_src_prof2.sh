# source-level stalls of the N-th launch of a kernel (ncu -s N -c 1)
mkdir -p gpurun_out
OP=$1; K=$2; KR=$3; TAG=$4; SKIP=$5
timeout 600 ncu --set full --clock-control none --import-source on -s $SKIP -c 1 -k regex:$KR -o /tmp/src_$TAG -f python tools/prof_any.py $OP $K > /dev/null 2>&1
ncu -i /tmp/src_$TAG.ncu-rep --page source --csv > gpurun_out/srcline_$TAG.csv 2>/dev/null
ncu -i /tmp/src_$TAG.ncu-rep --page raw --csv > gpurun_out/raw_$TAG.csv 2>/dev/null
