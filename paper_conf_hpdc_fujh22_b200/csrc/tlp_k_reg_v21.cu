// tlp_k_reg_v21.cu -- one family of aggregation kernel specialisations (see
// tlp_agg_kernels.cuh); a separate translation unit so the library builds in
// parallel.
#include "tlp_agg_kernels.cuh"

namespace tlp {

KernelFn pick_reg_v21(int vec, int op, int coef) {
    return vec == 2 ? pick<2, false, 1>(op, coef) : pick<1, false, 1>(op, coef);
}

}  // namespace tlp
