// tlp_k_mh.cu -- one family of aggregation kernel specialisations (see
// tlp_agg_kernels.cuh); a separate translation unit so the library builds in
// parallel.
#include "tlp_agg_kernels.cuh"

namespace tlp {

// multi-head GAT: full-warp register path or cp.async ring
KernelFn pick_mh(int vec, bool async_path) {
    if (async_path)
        return vec == 4 ? k_agg<4, OP_GATH, COEF_NONE, kU, true, 1>
                        : vec == 2 ? k_agg<2, OP_GATH, COEF_NONE, kU, true, 1>
                                   : k_agg<1, OP_GATH, COEF_NONE, kU, true, 1>;
    return vec == 4 ? k_agg<4, OP_GATH, COEF_NONE, kU, false, 1>
                    : vec == 2 ? k_agg<2, OP_GATH, COEF_NONE, kU, false, 1>
                               : k_agg<1, OP_GATH, COEF_NONE, kU, false, 1>;
}

}  // namespace tlp
