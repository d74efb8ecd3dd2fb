// frontier_cc.cu -- the frontier relax kernels of CC (instantiations of frontier_kernel.cuh).
#include "frontier_kernel.cuh"

namespace tigr {

FqFn relax_fq_kernel_cc(int layout, int unit, bool bsp, bool stats, bool packed) {
    return pick_fq<TIGR_CC>(layout, unit, bsp, stats, packed);
}

}  // namespace tigr
