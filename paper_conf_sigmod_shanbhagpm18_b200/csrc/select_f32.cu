// select_f32.cu -- select_kernel instantiations for float keys (see select_tu.cuh).
#define TOPK_TU_KEY float
#define TOPK_TU_NAME f32
#include "select_tu.cuh"
