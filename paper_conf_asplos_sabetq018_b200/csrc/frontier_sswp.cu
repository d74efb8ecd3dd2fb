// frontier_sswp.cu -- the frontier relax kernels of SSWP (instantiations of frontier_kernel.cuh).
#include "frontier_kernel.cuh"

namespace tigr {

FqFn relax_fq_kernel_sswp(int layout, int unit, bool bsp, bool stats, bool packed) {
    return pick_fq<TIGR_SSWP>(layout, unit, bsp, stats, packed);
}

}  // namespace tigr
