// tlp_k_reg_v4.cu -- one family of aggregation kernel specialisations (see
// tlp_agg_kernels.cuh); a separate translation unit so the library builds in
// parallel.
#include "tlp_agg_kernels.cuh"

namespace tlp {

KernelFn pick_reg_v4(int op, int coef) { return pick<4, false, 1>(op, coef); }

}  // namespace tlp
