// frontier_sssp.cu -- the frontier relax kernels of SSSP (instantiations of frontier_kernel.cuh).
#include "frontier_kernel.cuh"

namespace tigr {

FqFn relax_fq_kernel_sssp(int layout, bool bsp, bool stats) {
    return layout == TIGR_LAYOUT_STRIDED ? pick_fq<TIGR_SSSP, TIGR_LAYOUT_STRIDED>(bsp, stats)
                                         : pick_fq<TIGR_SSSP, TIGR_LAYOUT_CONSECUTIVE>(bsp, stats);
}

}  // namespace tigr
