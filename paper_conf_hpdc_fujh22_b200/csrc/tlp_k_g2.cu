// tlp_k_g2.cu -- one family of aggregation kernel specialisations (see
// tlp_agg_kernels.cuh); a separate translation unit so the library builds in
// parallel.
#include "tlp_agg_kernels.cuh"

namespace tlp {

KernelFn pick_g2(int op, int coef) { return pick<4, false, 2>(op, coef); }

}  // namespace tlp
