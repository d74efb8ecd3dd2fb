/*
 * graphgen/rmat.c -- seeded synthetic-input generator (host side).
 *
 * This module is the ONE place both the CPU oracle (oracle/) and the tests take
 * their input graphs from.  It holds none of the method's arithmetic (no CSR,
 * no virtual split, no relaxation): it only draws a COO edge list.  The CUDA
 * product path (paper_conf_asplos_sabetq018_b200/csrc/gen.cu) implements the
 * SAME counter-based generator independently; the GPU tests check the two are
 * bit-identical.  The paper itself loads real graphs (PAPER.md L1251-1262,
 * Table 3); R-MAT shaped like them is this build's synthetic stand-in
 * (BASELINE.json configs).
 *
 * Specification (shared by both sides):
 *   Philox4x32-10 (Salmon et al., SC'11; Random123 constants).
 *   key = (seed lo32, seed hi32); counter = (e lo32, e hi32, level/4, attempt).
 *   Word (level % 4) of the output decides recursion level `level`.
 *   r < T_A -> quadrant A (src bit 0, dst bit 0); r < T_AB -> B (0,1);
 *   r < T_ABC -> C (1,0); else D (1,1).  T_X = floor(X * 2^32) as uint64.
 *   Level l sets bit l (LSB first); s = ceil(log2 n).  An edge with
 *   src >= n or dst >= n is redrawn with attempt+1.
 *   weight(e) = wmin + philox(ctr=(e lo, e hi, 0, 0), key=(wseed lo, wseed hi)).x
 *               mod (wmax - wmin + 1)   (no mod when the range is 2^32).
 *   Duplicates and self-loops are kept, so m is exact.
 */
#include <stdint.h>
#include <stddef.h>

#define PHILOX_M0 0xD2511F53u
#define PHILOX_M1 0xCD9E8D57u
#define PHILOX_W0 0x9E3779B9u
#define PHILOX_W1 0xBB67AE85u

static inline void gg_round(uint32_t c[4], const uint32_t k[2]) {
    uint64_t p0 = (uint64_t)PHILOX_M0 * c[0];
    uint64_t p1 = (uint64_t)PHILOX_M1 * c[2];
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c[1] ^ k[0];
    uint32_t n2 = hi0 ^ c[3] ^ k[1];
    c[0] = n0; c[1] = lo1; c[2] = n2; c[3] = lo0;
}

void gg_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
    uint32_t c[4] = {ctr[0], ctr[1], ctr[2], ctr[3]};
    uint32_t k[2] = {key[0], key[1]};
    for (int r = 0; r < 10; ++r) {
        if (r) { k[0] += PHILOX_W0; k[1] += PHILOX_W1; }
        gg_round(c, k);
    }
    out[0] = c[0]; out[1] = c[1]; out[2] = c[2]; out[3] = c[3];
}

static uint32_t gg_scale(uint64_t n) {
    uint32_t s = 0;
    while (((uint64_t)1 << s) < n) ++s;
    return s;
}

static uint64_t gg_thresh(double x) {
    if (x <= 0.0) return 0;
    if (x >= 1.0) return (uint64_t)1 << 32;
    return (uint64_t)(x * 4294967296.0);
}

/* Draw edge e.  Returns 0 on success, -1 if the attempt cap is exceeded. */
static int gg_edge(uint64_t e, uint32_t s, uint64_t n, const uint32_t key[2],
                   uint64_t tA, uint64_t tAB, uint64_t tABC,
                   uint32_t* out_src, uint32_t* out_dst) {
    for (uint32_t a = 0; a < (1u << 24); ++a) {
        uint64_t su = 0, du = 0;
        uint32_t words[4] = {0, 0, 0, 0};
        for (uint32_t l = 0; l < s; ++l) {
            if ((l & 3u) == 0) {
                uint32_t ctr[4] = {(uint32_t)e, (uint32_t)(e >> 32), l >> 2, a};
                gg_philox4x32_10(ctr, key, words);
            }
            uint64_t r = words[l & 3u];
            uint64_t sb = (r >= tAB) ? 1u : 0u;
            uint64_t db = ((r >= tA && r < tAB) || r >= tABC) ? 1u : 0u;
            su |= sb << l;
            du |= db << l;
        }
        if (su < n && du < n) { *out_src = (uint32_t)su; *out_dst = (uint32_t)du; return 0; }
    }
    return -1;
}

/* Fill src/dst (and w when non-NULL) for edges [e0, e1).  Thread-safe; the
 * Python wrapper splits [0, m) across threads.  Returns 0 or -1. */
int gg_rmat_range(uint64_t n, uint64_t e0, uint64_t e1, double a, double b, double c,
                  uint64_t seed, uint64_t wseed, uint32_t wmin, uint32_t wmax,
                  uint32_t* src, uint32_t* dst, uint32_t* w) {
    if (n == 0 || n > 0xFFFFFFFEull) return -1;
    uint32_t s = gg_scale(n);
    uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
    uint32_t wkey[2] = {(uint32_t)wseed, (uint32_t)(wseed >> 32)};
    uint64_t tA = gg_thresh(a), tAB = gg_thresh(a + b), tABC = gg_thresh(a + b + c);
    uint64_t range = (uint64_t)wmax - (uint64_t)wmin + 1u;
    for (uint64_t e = e0; e < e1; ++e) {
        if (gg_edge(e, s, n, key, tA, tAB, tABC, &src[e], &dst[e]) != 0) return -1;
        if (w) {
            uint32_t ctr[4] = {(uint32_t)e, (uint32_t)(e >> 32), 0, 0}, o[4];
            gg_philox4x32_10(ctr, wkey, o);
            w[e] = (range >= ((uint64_t)1 << 32)) ? o[0] : wmin + (uint32_t)((uint64_t)o[0] % range);
        }
    }
    return 0;
}
