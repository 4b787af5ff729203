// query_f64.cu -- select_kernel query-form instantiations for double keys (WHERE predicate
// and, for f32, the ranking function; see select_tu.cuh, select.cuh QCfg).
#define TOPK_TU_KEY double
#define TOPK_TU_NAME f64
#define TOPK_TU_QUERY 1
#include "select_tu.cuh"
