# per-CTA timelines with -DTOPK_DEBUG variants: bash tools/gpu_trace.sh TAG [dbg ...]
TAG=${1:-r2}; shift
mkdir -p gpurun_out
for V in ${@:-dbg}; do
  export TOPK_LIB=paper_conf_sigmod_shanbhagpm18_b200/variants/libtopk_$V.so
  ( for k in 32 256 1024; do python tools/trace.py 536870912 uniform $k; done
    python tools/trace.py 536870912 fewdistinct 256
    python tools/trace.py 1048576 uniform 32
    python tools/trace.py 33554432 uniform 64 ) > gpurun_out/trace_${TAG}_$V.log 2>&1
  echo trace $V rc=$?
done
