#!/bin/bash
# build_variant.sh NAME "-DMACRO=.. ..."  -> paper_conf_sigmod_shanbhagpm18_b200/variants/libtopk_NAME.so
set -e
cd "$(dirname "$0")/.."
mkdir -p paper_conf_sigmod_shanbhagpm18_b200/variants
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 --shared -Xcompiler -fPIC -diag-suppress 177 $2 -I include -o paper_conf_sigmod_shanbhagpm18_b200/variants/libtopk_$1.so paper_conf_sigmod_shanbhagpm18_b200/csrc/topk_api.cu
