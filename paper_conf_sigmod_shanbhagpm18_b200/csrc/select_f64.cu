// select_f64.cu -- select_kernel instantiations for double keys (see select_tu.cuh).
#define TOPK_TU_KEY double
#define TOPK_TU_NAME f64
#include "select_tu.cuh"
