# A/B + traces of variant libraries (dev): bash tools/gpu_ab.sh TAG lib1 lib2 ...
TAG=$1; shift
mkdir -p gpurun_out
V=paper_conf_sigmod_shanbhagpm18_b200/variants
timeout 900 python tools/ab_check.py "$@" > gpurun_out/ab_$TAG.log 2>&1; echo ab rc=$?
if [ -f $V/libtopk_dbg.so ]; then bash tools/gpu_trace.sh $TAG; fi
