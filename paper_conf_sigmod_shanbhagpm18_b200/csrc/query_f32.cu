// query_f32.cu -- select_kernel query-form instantiations for float keys (WHERE predicate
// and, for f32, the ranking function; see select_tu.cuh, select.cuh QCfg).
#define TOPK_TU_KEY float
#define TOPK_TU_NAME f32
#define TOPK_TU_QUERY 1
#include "select_tu.cuh"
