// frontier_sssp.cu -- the frontier relax kernels of SSSP (instantiations of frontier_kernel.cuh).
#include "frontier_kernel.cuh"

namespace tigr {

FqFn relax_fq_kernel_sssp(int layout, int unit, bool bsp, bool stats, bool packed) {
    return pick_fq<TIGR_SSSP>(layout, unit, bsp, stats, packed);
}

}  // namespace tigr
