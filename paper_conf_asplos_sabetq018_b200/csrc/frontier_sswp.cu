// frontier_sswp.cu -- the frontier relax kernels of SSWP (instantiations of frontier_kernel.cuh).
#include "frontier_kernel.cuh"

namespace tigr {

FqFn relax_fq_kernel_sswp(int layout, bool bsp, bool stats) {
    return layout == TIGR_LAYOUT_STRIDED ? pick_fq<TIGR_SSWP, TIGR_LAYOUT_STRIDED>(bsp, stats)
                                         : pick_fq<TIGR_SSWP, TIGR_LAYOUT_CONSECUTIVE>(bsp, stats);
}

}  // namespace tigr
