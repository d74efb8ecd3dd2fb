// frontier_bfs.cu -- the frontier relax kernels of BFS (instantiations of frontier_kernel.cuh).
#include "frontier_kernel.cuh"

namespace tigr {

FqFn relax_fq_kernel_bfs(int layout, int unit, bool bsp, bool stats, bool packed) {
    return pick_fq<TIGR_BFS>(layout, unit, bsp, stats, packed);
}

}  // namespace tigr
