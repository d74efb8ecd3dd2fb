// frontier_cc.cu -- the frontier relax kernels of CC (instantiations of frontier_kernel.cuh).
#include "frontier_kernel.cuh"

namespace tigr {

FqFn relax_fq_kernel_cc(int layout, bool bsp, bool stats) {
    return layout == TIGR_LAYOUT_STRIDED ? pick_fq<TIGR_CC, TIGR_LAYOUT_STRIDED>(bsp, stats)
                                         : pick_fq<TIGR_CC, TIGR_LAYOUT_CONSECUTIVE>(bsp, stats);
}

}  // namespace tigr
