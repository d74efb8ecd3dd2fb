// standalone check of frontier.cu's warp_search + map_round on random queues (dev tool)
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cstdint>
#include <algorithm>
constexpr uint32_t kFull = 0xffffffffu, kInf = 0xffffffffu, kPad = 0xffffffffu;
#define FQ_MAP_ONLY
__device__ __forceinline__ uint32_t warp_search(const uint32_t* __restrict__ qo, uint32_t qn, uint32_t t, int lane) {
    uint32_t lo = 0, hi = qn;
    while (hi - lo > 32) {
        const uint32_t step = (hi - lo + 31) / 32;
        const uint32_t idx = lo + (uint32_t)lane * step;
        const bool p = idx < hi && __ldg(qo + idx) <= t;
        const uint32_t b = __ballot_sync(kFull, p);
        const uint32_t L = 31u - __clz(b);
        lo += L * step;
        hi = min(hi, lo + step);
    }
    const uint32_t idx = lo + (uint32_t)lane;
    const uint32_t b = __ballot_sync(kFull, idx < hi && __ldg(qo + idx) <= t);
    return lo + (31u - __clz(b));
}
__device__ __forceinline__ void map_round(const uint32_t* __restrict__ qv, const uint32_t* __restrict__ qo,
                                          uint32_t qn, uint32_t& k, uint32_t tr, int lane, uint32_t& v,
                                          uint32_t& j) {
    uint32_t idx = k + (uint32_t)lane;
    uint32_t off = idx < qn ? __ldg(qo + idx) : kInf;
    // entries starting at or before tr form a prefix of the window; its last one owns tr.
    // Rebase the window there, so that its 32 entries (>= 1 vnode each) cover tr .. tr + 31.
    const uint32_t le = __ballot_sync(kFull, off <= tr);
    const int first = 31 - __clz(le);  // le != 0: the window's first entry starts at or before tr
    if (first > 0) {                   // warp-uniform
        k += (uint32_t)first;
        idx = k + (uint32_t)lane;
        off = idx < qn ? __ldg(qo + idx) : kInf;
    }
    const uint32_t node = idx < qn ? __ldg(qv + idx) : kPad;
    uint32_t bit = 0;
    if (lane == 0) bit = 1u;
    else if (off < tr + 32u) bit = 1u << (off - tr);  // off > tr here
    const uint32_t starts = __reduce_or_sync(kFull, bit);
    const uint32_t upto = lane == 31 ? kFull : ((2u << lane) - 1u);
    const int e = __popc(starts & upto) - 1;  // window lane of this lane's entry
    v = __shfl_sync(kFull, node, e);
    const uint32_t eo = __shfl_sync(kFull, off, e);
    j = (tr + (uint32_t)lane) - eo;
    k += (uint32_t)__shfl_sync(kFull, e, 31);
}
template <int B>
__global__ void k(const uint32_t* qv, const uint32_t* qo, uint32_t qn, uint32_t qt, uint32_t* ov, uint32_t* oj) {
    const int lane = threadIdx.x & 31;
    const uint64_t warp0 = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    constexpr uint32_t kTile = 32u * B;
    const uint64_t tiles = (qt + kTile - 1) / kTile;
    for (uint64_t tile = warp0; tile < tiles; tile += nwarps) {
        const uint64_t t0 = tile * kTile;
        uint32_t k = warp_search(qo, qn, (uint32_t)t0, lane);
        if (lane == 0 && (qo[k] > t0 || (k + 32 < qn && qo[k + 32] <= t0)))
            printf("search bad: t0 %u k %u qo[k] %u qo[k+32] %u qn %u\n", (uint32_t)t0, k, qo[k], k + 32 < qn ? qo[k + 32] : 0, qn);
        uint32_t v[B], j[B];
#pragma unroll
        for (int r = 0; r < B; ++r) {
            const uint32_t tr = (uint32_t)t0 + 32u * r;
            if (tr < qt) map_round(qv, qo, qn, k, tr, lane, v[r], j[r]);
            else { v[r] = kPad; j[r] = 0; }
        }
#pragma unroll
        for (int r = 0; r < B; ++r) {
            const uint32_t t = (uint32_t)t0 + 32u * r + lane;
            if (t < qt) { ov[t] = v[r]; oj[t] = j[r]; }
        }
    }
}
int main() {
    srand(1);
    int bad = 0;
    for (int trial = 0; trial < 300 && bad < 5; ++trial) {
        uint32_t qn = 1 + rand() % 5000;
        std::vector<uint32_t> qv(qn), qo(qn);
        uint32_t t = 0;
        const int ms[] = {1, 1, 1, 2, 3, 4, 9, 33, 129, 1000};
        for (uint32_t i = 0; i < qn; ++i) { qv[i] = i * 7 + 3; qo[i] = t; t += ms[rand() % 10]; }
        uint32_t qt = t;
        uint32_t *dv, *doo, *ov, *oj;
        cudaMalloc(&dv, 4 * qn); cudaMalloc(&doo, 4 * qn); cudaMalloc(&ov, 4 * qt); cudaMalloc(&oj, 4 * qt);
        cudaMemcpy(dv, qv.data(), 4 * qn, cudaMemcpyHostToDevice);
        cudaMemcpy(doo, qo.data(), 4 * qn, cudaMemcpyHostToDevice);
        cudaMemset(ov, 0xff, 4 * qt);
        k<4><<<37, 256>>>(dv, doo, qn, qt, ov, oj);
        std::vector<uint32_t> hv(qt), hj(qt);
        cudaMemcpy(hv.data(), ov, 4 * qt, cudaMemcpyDeviceToHost);
        cudaMemcpy(hj.data(), oj, 4 * qt, cudaMemcpyDeviceToHost);
        for (uint32_t x = 0; x < qt && bad < 5; ++x) {
            uint32_t e = (uint32_t)(std::upper_bound(qo.begin(), qo.end(), x) - qo.begin()) - 1;
            if (hv[x] != qv[e] || hj[x] != x - qo[e]) {
                printf("trial %d qn %u qt %u t %u: got v %u j %u want v %u j %u\n", trial, qn, qt, x, hv[x], hj[x], qv[e], x - qo[e]);
                ++bad;
            }
        }
        cudaFree(dv); cudaFree(doo); cudaFree(ov); cudaFree(oj);
    }
    printf("err=%s bad=%d\n", cudaGetErrorString(cudaGetLastError()), bad);
}
