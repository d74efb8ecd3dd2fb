// gen.cu -- synthetic power-law (R-MAT) arc generator on the device.
//
// The paper evaluates real graphs (Table 3); this build draws R-MAT
// graphs shaped like them (BASELINE.json configs).  Counter-based:
// arc e depends only on (seed, e), so any slice of [0, m) can be drawn by any rank and the
// host generator in graphgen/ (an independent implementation of the same spec, used by the
// tests and the oracle) reproduces it bit for bit.  Spec: DESIGN.md "Generator spec".
#include "internal.cuh"

namespace tigr {
namespace {

struct U4 { uint32_t x, y, z, w; };

__device__ __forceinline__ U4 philox4x32_10(U4 c, uint32_t k0, uint32_t k1) {
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        const uint32_t lo0 = 0xD2511F53u * c.x, hi0 = __umulhi(0xD2511F53u, c.x);
        const uint32_t lo1 = 0xCD9E8D57u * c.z, hi1 = __umulhi(0xCD9E8D57u, c.z);
        c = U4{hi1 ^ c.y ^ k0, lo1, hi0 ^ c.w ^ k1, lo0};
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
    return c;
}

__global__ void k_rmat(uint64_t e0, uint64_t count, uint32_t n, uint32_t scale, uint64_t tA,
                       uint64_t tAB, uint64_t tABC, uint32_t k0, uint32_t k1, uint32_t wk0,
                       uint32_t wk1, uint32_t wmin, uint64_t wrange, uint32_t* __restrict__ src,
                       uint32_t* __restrict__ dst, uint32_t* __restrict__ w, uint32_t* err) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count;
         i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t e = e0 + i;
        const uint32_t elo = (uint32_t)e, ehi = (uint32_t)(e >> 32);
        uint32_t s = 0, d = 0;
        bool ok = false;
        for (uint32_t a = 0; a < (1u << 24) && !ok; ++a) {
            uint64_t su = 0, du = 0;
            for (uint32_t l = 0; l < scale; l += 4) {
                const U4 r4 = philox4x32_10(U4{elo, ehi, l >> 2, a}, k0, k1);
                const uint32_t words[4] = {r4.x, r4.y, r4.z, r4.w};
#pragma unroll
                for (uint32_t q = 0; q < 4; ++q) {
                    if (l + q < scale) {
                        const uint64_t r = words[q];
                        const uint64_t sb = r >= tAB;
                        const uint64_t db = (r >= tA && r < tAB) || r >= tABC;
                        su |= sb << (l + q);
                        du |= db << (l + q);
                    }
                }
            }
            if (su < n && du < n) { s = (uint32_t)su; d = (uint32_t)du; ok = true; }
        }
        if (!ok) *err = 1;
        src[i] = s;
        dst[i] = d;
        if (w) {
            const U4 r = philox4x32_10(U4{elo, ehi, 0u, 0u}, wk0, wk1);
            w[i] = wrange >= (1ull << 32) ? r.x : wmin + (uint32_t)((uint64_t)r.x % wrange);
        }
    }
}

uint64_t thresh(double x) {
    if (x <= 0.0) return 0;
    if (x >= 1.0) return 1ull << 32;
    return (uint64_t)(x * 4294967296.0);
}

}  // namespace

tigr_status rmat_range(uint32_t n, uint64_t e0, uint64_t count, double a, double b, double c,
                       uint64_t seed, uint64_t wseed, uint32_t wmin, uint32_t wmax, uint32_t* src,
                       uint32_t* dst, uint32_t* w, cudaStream_t s) {
    if (n == 0) return fail(TIGR_EINVAL, "rmat: n == 0");
    if (n > 0xFFFFFFFEu) return fail(TIGR_ERANGE, "rmat: n > 0xFFFFFFFE");
    if (wmax < wmin) return fail(TIGR_EINVAL, "rmat: wmax < wmin");
    if (count == 0) return TIGR_OK;
    uint32_t scale = 0;
    while ((1ull << scale) < n) ++scale;
    TmpBuf err;
    TIGR_TRY(err.alloc(sizeof(uint32_t), s));
    TIGR_CK(cudaMemsetAsync(err.p, 0, sizeof(uint32_t), s));
    int dev = 0, sms = 148;
    TIGR_CK(cudaGetDevice(&dev));
    TIGR_CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    const uint64_t want = (count + kBlock - 1) / kBlock;
    const unsigned grid = (unsigned)(want < (uint64_t)sms * 32 ? want : (uint64_t)sms * 32);
    k_rmat<<<grid, kBlock, 0, s>>>(e0, count, n, scale, thresh(a), thresh(a + b), thresh(a + b + c),
                                   (uint32_t)seed, (uint32_t)(seed >> 32), (uint32_t)wseed,
                                   (uint32_t)(wseed >> 32), wmin, (uint64_t)wmax - wmin + 1, src, dst, w,
                                   err.as<uint32_t>());
    TIGR_CKL("rmat");
    uint32_t herr = 0;
    TIGR_CK(cudaMemcpyAsync(&herr, err.p, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    if (herr) return fail(TIGR_EINVAL, "rmat: rejection attempt cap exceeded (degenerate a,b,c?)");
    return TIGR_OK;
}

}  // namespace tigr
