// query_u32.cu -- select_kernel query-form instantiations for uint32_t keys (WHERE predicate
// and, for f32, the ranking function; see select_tu.cuh, select.cuh QCfg).
#define TOPK_TU_KEY uint32_t
#define TOPK_TU_NAME u32
#define TOPK_TU_QUERY 1
#include "select_tu.cuh"
