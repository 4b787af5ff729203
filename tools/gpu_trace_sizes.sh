# per-CTA timelines at several sizes (needs variants/libtopk_dbg.so): bash tools/gpu_trace_sizes.sh TAG
TAG=${1:-r2}
mkdir -p gpurun_out
export TOPK_LIB=paper_conf_sigmod_shanbhagpm18_b200/variants/libtopk_dbg.so
export TOPK_PURE_SMALL_N=0
( python tools/trace.py 2097152 uniform 64
  python tools/trace.py 536870912 uniform 1
  python tools/trace.py 536870912 uniform 256
  TOPK_END_ZONE=0 python tools/trace.py 536870912 uniform 256
  python tools/trace.py 536870912 uniform 1024 ) > gpurun_out/trace_$TAG.log 2>&1
echo rc=$?
