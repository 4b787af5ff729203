// select_u32.cu -- select_kernel instantiations for uint32_t keys (see select_tu.cuh).
#define TOPK_TU_KEY uint32_t
#define TOPK_TU_NAME u32
#include "select_tu.cuh"
