// query_kk.cu -- select_kernel instantiations for compound keys (two f32 columns,
// ORDER BY a, b; optional WHERE) -- KKV, P:274-278 (see select_tu.cuh, keys.cuh KK32).
#define TOPK_TU_KEY KK32
#define TOPK_TU_NAME kk
#define TOPK_TU_QUERY 1
#include "select_tu.cuh"
