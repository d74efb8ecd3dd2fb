// sort.cu -- CSR construction by a stable LSD radix sort of the arcs on their source
// (Fig. 10a, "we reorder the edges during the
// construction of CSR" L1131-1132).
//
// Stable => within a source the arcs keep their input (COO) order, so the device CSR is the
// canonical one, identical element by element to a stable counting sort (and to the oracle).
// Each pass is one "onesweep" kernel: a tile of 4096 arcs is ranked in shared memory with
// warp match-any (stable), the tile's per-digit offsets come from a decoupled look-back over
// the preceding tiles, and the tile is written back grouped by digit (coalesced runs).
// No global atomics on the keys themselves, so the heavy skew of power-law sources (the
// hottest vertex owns 0.14% of all arcs at scale 24) costs nothing.  The last pass also
// counts the degrees from the runs of equal keys in its tiles; a final kernel places each arc
// into the 32-byte-aligned, padded segment of its source.
#include <algorithm>
#include <cstdlib>
#include <map>
#include <mutex>
#include <type_traits>
#include <utility>
#include <vector>

#include "internal.cuh"

namespace tigr {
namespace {

constexpr int kST = 256;                 // threads per sort tile
#ifndef TIGR_SORT_MINB
#define TIGR_SORT_MINB 3
#endif
constexpr int kSW = kST / 32;            // warps per tile
constexpr int kMaxRadix = 256;
constexpr uint64_t kFlagAgg = 1ull << 46, kFlagInc = 2ull << 46, kValMask = (1ull << 46) - 1;

template <bool W> struct ValT { typedef uint32_t T; };
template <> struct ValT<true> { typedef uint64_t T; };

// item e of the (optionally symmetrised) arc list: key = source, val = target [| weight << 32]
template <bool W>
__device__ __forceinline__ void coo_item(const uint32_t* __restrict__ src, const uint32_t* __restrict__ dst,
                                         const uint32_t* __restrict__ w, uint64_t m, uint64_t e, uint32_t& k,
                                         typename ValT<W>::T& v) {
    const bool rev = e >= m;
    const uint64_t f = rev ? e - m : e;
    const uint32_t s = src[f], d = dst[f];
    k = rev ? d : s;
    const uint32_t t = rev ? s : d;
    if constexpr (W) v = (uint64_t)t | ((uint64_t)w[f] << 32);
    else v = t;
}

// One read of the arc list before sorting: the digit histograms of every pass, the largest id
// (validation: checked on the host before any id is used as an index), and optionally the
// in-degree sketch the PageRank accumulator order uses (pr.cu): a has-in-arcs bit per node
// (a 2 MB bitmap at scale 24, tested before set, so hub targets do not serialise; measured
// 0.6 ms of the cfg4 build as a byte per node) and an in-degree count sampled
// on every 16th item.  Covers the input arcs f in [f0, f1) -- the host-input build scans each
// chunk as its copy lands (api.cu) -- and, when symmetrising (sym), their reversed items
// m + f too.  Item e: key = source, t = target.
__global__ void k_coo_scan(const uint32_t* __restrict__ src, const uint32_t* __restrict__ dst, uint64_t m,
                           uint64_t f0, uint64_t f1, int sym, int passes, int bits,
                           unsigned long long* __restrict__ hist, uint32_t* __restrict__ maxid, uint32_t n,
                           uint32_t* __restrict__ in_flag, uint32_t* __restrict__ in_sample, uint32_t klo,
                           uint32_t khi, unsigned long long* __restrict__ n_local) {
    // one arc per thread and step: measured faster (1.40 ms at cfg4) than 8 arcs per step with
    // 16-byte loads (1.59 ms; 40 registers, occupancy 97 -> 65 %): the scan is bound by the
    // shared-memory histogram atomics and the random in-flag reads, not by load latency
    __shared__ uint32_t h[4][kMaxRadix];
    for (int i = threadIdx.x; i < 4 * kMaxRadix; i += blockDim.x) (&h[0][0])[i] = 0;
    __syncthreads();
    const uint32_t mask = (1u << bits) - 1;
    uint32_t mx = 0, local = 0;
    for (uint64_t f = f0 + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; f < f1; f += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t s = src[f], d = dst[f];
        mx = max(mx, max(s, d));
        for (int dir = 0; dir <= sym; ++dir) {
            const uint64_t e = dir ? m + f : f;
            const uint32_t k = dir ? d : s, t = dir ? s : d;
            if (k < n && k >= klo && k < khi) {  // this build's source range (partitioned graphs)
                ++local;
                for (int p = 0; p < passes; ++p) atomicAdd(&h[p][(k >> (p * bits)) & mask], 1u);
            }
            if (in_flag && t < n) {
                const uint32_t bit = 1u << (t & 31);  // test first: hub targets are set once
                if (!(in_flag[t >> 5] & bit)) atomicOr(in_flag + (t >> 5), bit);
                if ((e & 15) == 0) atomicAdd(in_sample + t, 1u);
            }
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        local += __shfl_xor_sync(0xffffffffu, local, o);
    }
    if ((threadIdx.x & 31) == 0 && mx) atomicMax(maxid, mx);
    if ((threadIdx.x & 31) == 0 && local) atomicAdd(n_local, (unsigned long long)local);
    __syncthreads();
    for (int i = threadIdx.x; i < passes * kMaxRadix; i += blockDim.x) {
        const uint32_t c = (&h[0][0])[i];
        if (c) atomicAdd(&hist[i], (unsigned long long)c);
    }
}

// exclusive scan of each pass's digit counts (one block, one thread per digit)
__global__ void k_digit_base(const unsigned long long* __restrict__ hist, int passes, uint64_t* __restrict__ base) {
    __shared__ uint64_t tmp[kMaxRadix];
    for (int p = 0; p < passes; ++p) {
        tmp[threadIdx.x] = hist[p * kMaxRadix + threadIdx.x];
        __syncthreads();
        if (threadIdx.x == 0) {
            uint64_t s = 0;
            for (int d = 0; d < kMaxRadix; ++d) { const uint64_t c = tmp[d]; tmp[d] = s; s += c; }
        }
        __syncthreads();
        base[p * kMaxRadix + threadIdx.x] = tmp[threadIdx.x];
        __syncthreads();
    }
}

// look-back status words: relaxed, device-scope (the word itself carries epoch, flag and value,
// so no other data needs ordering; volatile compiled to system-scope strong loads)
__device__ __forceinline__ uint64_t status_load(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void status_store(uint64_t* p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void cp_async4(void* smem_dst, const void* gsrc) {
    const uint32_t d = (uint32_t)__cvta_generic_to_shared(smem_dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" :: "r"(d), "l"(gsrc) : "memory");
}

// Bulk (TMA-engine) tile staging: one thread arms an mbarrier with the byte count and issues a
// single cp.async.bulk per array; the other threads wait on the barrier's phase 0.
__device__ __forceinline__ void mbar_init(uint64_t* bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"((uint32_t)__cvta_generic_to_shared(bar)) : "memory");
}

__device__ __forceinline__ void bulk_load(void* smem_dst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
    const uint32_t b = (uint32_t)__cvta_generic_to_shared(bar);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(b), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"((uint32_t)__cvta_generic_to_shared(smem_dst)), "l"(gsrc), "r"(bytes), "r"(b) : "memory");
}

__device__ __forceinline__ void mbar_wait0(uint64_t* bar) {
    const uint32_t b = (uint32_t)__cvta_generic_to_shared(bar);
    uint32_t done = 0;
    while (!done)
        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
                     : "=r"(done) : "r"(b) : "memory");
}

// Lanes of the warp holding the same digit (and the same validity): one ballot per digit bit
// instead of match.any, whose result latency stalled every ranking round.
// All 8 bits are tested whatever the digit width (bits above it are 0 in every lane and leave
// the mask unchanged), so the loop has no predication; the validity ballot is only needed in
// tiles with dropped or missing items (check, warp-uniform).
__device__ __forceinline__ uint32_t match_digit(uint32_t d, bool check, bool valid) {
    uint32_t m = 0xffffffffu;
    if (check) {
        const uint32_t v = __ballot_sync(0xffffffffu, valid);
        m = valid ? v : ~v;
    }
    // per bit: the ballot, the lane's bit as a full mask s, and m &= ~(ballot ^ s) in one lop3 --
    // three instructions once ptxas has loaded the bit predicates (R2P, seven at once); the plain
    // C++ form compiled to six per bit (shift, mask, compare, mask build, vote, merge)
#pragma unroll
    for (int b = 0; b < 8; ++b)
        asm("{\n\t.reg .pred p;\n\t.reg .b32 v, s;\n\t"
            "and.b32 v, %1, %2;\n\t"
            "setp.ne.u32 p, v, 0;\n\t"
            "vote.sync.ballot.b32 v, p, 0xffffffff;\n\t"
            "selp.b32 s, -1, 0, p;\n\t"
            "lop3.b32 %0, %0, v, s, 0x90;\n\t}"
            : "+r"(m) : "r"(d), "r"(1u << b));
    return m;
}

// One pass of the stable LSD radix sort over a tile of 4096 arcs.  Values are staged into
// shared memory as soon as the tile is known (no registers held across the ranking /
// look-back); keys stay in registers; digits are recomputed from the keys.  A full tile whose
// arrays are contiguous and 16-byte aligned (bulk_ok) is staged with two bulk copies (keys via
// s_key, which is free until the reorder); other tiles with per-item 4-byte cp.async.
template <bool W, bool FIRST, int SI, bool FILT, bool DEG>
__global__ void __launch_bounds__(kST, (SI <= 16 ? TIGR_SORT_MINB : 2)) k_onesweep(const uint32_t* __restrict__ kin,
                                                  const typename ValT<W>::T* __restrict__ vin,
                                                  const uint32_t* __restrict__ src, const uint32_t* __restrict__ dst,
                                                  const uint32_t* __restrict__ w, uint64_t m, uint64_t M, int shift,
                                                  int bits, const uint64_t* __restrict__ digit_base,
                                                  uint64_t* status, uint32_t* tile_counter, uint64_t epoch,
                                                  uint32_t* __restrict__ kout, typename ValT<W>::T* __restrict__ vout,
                                                  uint32_t klo, uint32_t khi, int bulk_ok,
                                                  uint32_t* __restrict__ deg) {
    typedef typename ValT<W>::T VT;
    extern __shared__ __align__(16) unsigned char smem[];
    VT* s_vin = reinterpret_cast<VT*>(smem);                                   // tile values, input order
    VT* s_val = reinterpret_cast<VT*>(smem + sizeof(VT) * (kST * SI));         // values, digit order
    uint32_t* s_key = reinterpret_cast<uint32_t*>(smem + 2 * sizeof(VT) * (kST * SI));
    __shared__ uint32_t s_wcnt[kSW][kMaxRadix + 1];
    __shared__ uint32_t s_dstart[kMaxRadix + 1];
    __shared__ uint64_t s_gofs[kMaxRadix];
    __shared__ uint32_t s_tile;
    __shared__ uint32_t s_wsum[kSW];
    __shared__ __align__(8) uint64_t s_bar[2];  // bulk staging: keys, values

    const int t = threadIdx.x, lane = t & 31, wp = t >> 5;
    if (t == 0) {
        s_tile = atomicAdd(tile_counter, 1u);
        if (bulk_ok) {
            mbar_init(&s_bar[0]);
            mbar_init(&s_bar[1]);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
    }
    for (int i = t; i < kSW * (kMaxRadix + 1); i += kST) (&s_wcnt[0][0])[i] = 0;
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t base = (uint64_t)tile * (kST * SI);
    const int radix = 1 << bits;
    const uint32_t mask = (uint32_t)radix - 1;
    const uint32_t cnt = (M - base < (uint64_t)(kST * SI)) ? (uint32_t)(M - base) : (uint32_t)(kST * SI);

    // values -> shared memory (asynchronous, coalesced), keys -> registers; in the first pass
    // arcs whose source lies outside [klo, khi) are dropped (partitioned builds)
    uint32_t key[SI];
    uint32_t valid = 0;  // FILT: bit r = item r of this thread passed the filter
    const bool fwd_tile = base + (uint64_t)(kST * SI) <= m;  // FIRST: no reversed item in this tile
    auto keep = [&](int r) -> bool {
        if constexpr (FILT) return (valid >> r) & 1u;
        else return (uint32_t)(wp * (SI * 32) + r * 32 + lane) < cnt;
    };
    const bool bulk = bulk_ok && cnt == (uint32_t)(kST * SI) && (!FIRST || (!W && !FILT && fwd_tile));
    if (bulk) {
        if (t == 0) {
            bulk_load(s_key, FIRST ? src + base : kin + base, sizeof(uint32_t) * (kST * SI), &s_bar[0]);
            bulk_load(s_vin, FIRST ? reinterpret_cast<const VT*>(dst + base) : vin + base, sizeof(VT) * (kST * SI),
                      &s_bar[1]);
        }
        mbar_wait0(&s_bar[0]);
#pragma unroll
        for (int r = 0; r < SI; ++r) key[r] = s_key[wp * (SI * 32) + r * 32 + lane];
    } else
#pragma unroll
    for (int r = 0; r < SI; ++r) {
        const uint32_t li = wp * (SI * 32) + r * 32 + lane;
        const uint64_t idx = base + li;
        key[r] = 0;
        if (li < cnt) {
            if constexpr (FIRST) {
                // a tile wholly before the reversed half (every tile without symmetrising) reads
                // the arc list straight; only tiles that reach into it select per item
                const bool rev = !fwd_tile && idx >= m;
                const uint64_t f = rev ? idx - m : idx;
                key[r] = rev ? dst[f] : src[f];
                if (!FILT || (key[r] >= klo && key[r] < khi)) {
                    if constexpr (FILT) valid |= 1u << r;
                    uint32_t* sv = reinterpret_cast<uint32_t*>(&s_vin[li]);
                    cp_async4(sv, rev ? src + f : dst + f);
                    if constexpr (W) cp_async4(sv + 1, w + f);
                }
            } else {
                key[r] = kin[idx];
                if constexpr (W) {
                    const uint32_t* gv = reinterpret_cast<const uint32_t*>(vin + idx);
                    uint32_t* sv = reinterpret_cast<uint32_t*>(&s_vin[li]);
                    cp_async4(sv, gv);
                    cp_async4(sv + 1, gv + 1);
                } else {
                    cp_async4(&s_vin[li], vin + idx);
                }
            }
        }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
    // stable ranking within the warp's 512 items (item order = round-major, then lane): the
    // lowest lane of each digit group reserves popc(peers) slots with a shared atomic; the
    // warp issues the rounds' atomics in order, so reservations follow item order; the
    // results are broadcast after all rounds are issued (no per-round round trip).
    const uint32_t lt = (1u << lane) - 1;
    uint32_t peers[SI];
    uint32_t rank[SI / 2];  // two 16-bit ranks per register
#pragma unroll
    for (int r = 0; r < SI; ++r) {
        const bool kr = keep(r);
        const uint32_t d = kr ? (key[r] >> shift) & mask : (uint32_t)radix;
        peers[r] = match_digit(d, FILT || cnt < (uint32_t)(kST * SI), kr);
        uint32_t got = 0;
        if ((peers[r] & lt) == 0) got = atomicAdd(&s_wcnt[wp][d], (uint32_t)__popc(peers[r]));
        if (r & 1) rank[r >> 1] |= got << 16; else rank[r >> 1] = got;
    }
#pragma unroll
    for (int r = 0; r < SI; ++r) {
        const uint32_t mine = (rank[r >> 1] >> ((r & 1) * 16)) & 0xFFFFu;
        const uint32_t b = __shfl_sync(0xffffffffu, mine, __ffs(peers[r]) - 1) + __popc(peers[r] & lt);
        rank[r >> 1] = (r & 1) ? ((rank[r >> 1] & 0xFFFFu) | (b << 16)) : ((rank[r >> 1] & 0xFFFF0000u) | b);
    }
    __syncthreads();
    // per digit: exclusive prefix over warps, tile count, publish the aggregate
    uint32_t tile_cnt = 0;
    if (t < radix) {
        uint32_t s = 0;
#pragma unroll
        for (int wi = 0; wi < kSW; ++wi) {
            const uint32_t c = s_wcnt[wi][t];
            s_wcnt[wi][t] = s;
            s += c;
        }
        tile_cnt = s;
        const uint64_t word = (epoch << 48) | (tile == 0 ? kFlagInc : kFlagAgg) | (uint64_t)s;
        status_store(&status[(uint64_t)tile * kMaxRadix + t], word);
    }
    // tile-local digit starts: exclusive scan of tile_cnt over the digits (t < 256)
    {
        uint32_t v = tile_cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t u = __shfl_up_sync(0xffffffffu, v, o);
            if (lane >= o) v += u;
        }
        if (lane == 31) s_wsum[wp] = v;
        __syncthreads();
        uint32_t wofs = 0;
        for (int wi = 0; wi < wp; ++wi) wofs += s_wsum[wi];
        s_dstart[t] = wofs + v - tile_cnt;
        if (FILT && t == kST - 1) s_dstart[kMaxRadix] = wofs + v;  // the tile's kept items
    }
    if (bulk) mbar_wait0(&s_bar[1]);
    else asm volatile("cp.async.wait_all;" ::: "memory");
    __syncthreads();
    // reorder the tile by digit in shared memory (needs no global offset: done before the
    // look-back, so that the predecessors have had that much longer to publish)
#pragma unroll
    for (int r = 0; r < SI; ++r) {
        const uint32_t li = wp * (SI * 32) + r * 32 + lane;
        if (keep(r)) {
            const uint32_t d = (key[r] >> shift) & mask;
            const uint32_t lp = s_dstart[d] + s_wcnt[wp][d] + ((rank[r >> 1] >> ((r & 1) * 16)) & 0xFFFFu);
            s_key[lp] = key[r];
            s_val[lp] = s_vin[li];
        }
    }
    // decoupled look-back for this digit, kLook predecessor tiles per step: their status words
    // are loaded together (independent loads in flight) and consumed newest first until an
    // inclusive prefix is met; a predecessor that has published nothing yet is re-polled after
    // a short sleep (keeps the spinning blocks from flooding L2).  ncu showed the one-at-a-time
    // walk -- ~9 dependent L2 round trips per tile -- as a quarter of the pass.
    if (t < radix) {
        constexpr int kLook = 4;
        uint64_t excl = 0;
        if (tile > 0) {
            int64_t p = (int64_t)tile - 1;
            bool done = false;
            while (!done && p >= 0) {
                uint64_t st[kLook];
#pragma unroll
                for (int q = 0; q < kLook; ++q)
                    st[q] = (p - q >= 0) ? status_load(&status[(uint64_t)(p - q) * kMaxRadix + t]) : 0ull;
#pragma unroll
                for (int q = 0; q < kLook; ++q) {
                    if (done || p - q < 0) continue;
                    const uint64_t* sp = &status[(uint64_t)(p - q) * kMaxRadix + t];
                    while ((st[q] >> 48) != epoch || (st[q] & (3ull << 46)) == 0) {
                        __nanosleep(32);
                        st[q] = status_load(sp);
                    }
                    excl += st[q] & kValMask;
                    if (st[q] & kFlagInc) done = true;
                }
                p -= kLook;
            }
            status_store(&status[(uint64_t)tile * kMaxRadix + t], (epoch << 48) | kFlagInc | (excl + tile_cnt));
        }
        s_gofs[t] = digit_base[t] + excl - s_dstart[t];  // output position of tile item i: s_gofs[d] + i
    }
    __syncthreads();
    const uint32_t nvalid = FILT ? s_dstart[kMaxRadix] : cnt;
#pragma unroll
    for (int r = 0; r < SI; ++r) {
        const uint32_t i = r * kST + t;
        if (i < nvalid) {
            const uint32_t k = s_key[i];
            const uint32_t d = (k >> shift) & mask;
            const uint64_t pos = s_gofs[d] + i;
            kout[pos] = k;
            vout[pos] = s_val[i];
            // last pass with degree counting (DEG): the tile's input is sorted by the lower digits
            // and the stable rank adds the top one, so s_key is sorted by the whole key -- equal
            // keys are runs.  A run [i0, i1] adds i1 + 1 - i0 to its key's degree as +(i1 + 1) from
            // its last item and -i0 from its first (one atomic for a run of one); a key whose run
            // spans tiles collects one such pair per tile.
            if constexpr (DEG) {
                if (k < khi) {  // khi: the id bound in host-input run builds (ids not yet validated)
                    const bool first = i == 0 || s_key[i - 1] != k;
                    const bool last = i + 1 == nvalid || s_key[i + 1] != k;
                    if (first || last) atomicAdd(deg + k, (last ? i + 1 : 0u) - (first ? i : 0u));
                }
            }
        }
    }
}

// sorted arcs -> padded, 32-byte-aligned segments.  The thread that places a node's last arc
// (the next sorted key differs) also fills the node's pad slots up to its next span boundary
// (pads = kPad, weight 0), so no separate padding pass runs.
template <bool W>
__device__ __forceinline__ void place_pads(uint32_t v, uint64_t pos, const uint32_t* __restrict__ cptr,
                                           uint32_t* __restrict__ col, uint32_t* __restrict__ wt) {
    const uint64_t end = (uint64_t)__ldg(cptr + v + 1) * kSpan;
    for (uint64_t q = pos + 1; q < end; ++q) {
        col[q] = kPad;
        if constexpr (W) wt[q] = 0;
    }
}

template <bool W>
__global__ void k_place(const uint32_t* __restrict__ key, const typename ValT<W>::T* __restrict__ val, uint64_t M,
                        const int64_t* __restrict__ row_ptr, const uint32_t* __restrict__ cptr,
                        uint32_t* __restrict__ col, uint32_t* __restrict__ wt) {
    typedef typename ValT<W>::T VT;
    // four arcs per thread and step: 16-byte key loads, all node-record reads in flight together
    const uint64_t M4 = M / 4;
    for (uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; g < M4; g += (uint64_t)gridDim.x * blockDim.x) {
        const uint4 k4 = reinterpret_cast<const uint4*>(key)[g];
        const uint32_t v[4] = {k4.x, k4.y, k4.z, k4.w};
        const uint32_t after = 4 * g + 4 < M ? __ldg(key + 4 * g + 4) : kPad;  // key past this group
        VT x[4];
        uint64_t base[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            x[q] = val[4 * g + q];
            base[q] = (uint64_t)cptr[v[q]] * kSpan - (uint64_t)row_ptr[v[q]];
        }
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const uint64_t pos = base[q] + 4 * g + q;
            col[pos] = (uint32_t)x[q];
            if constexpr (W) wt[pos] = (uint32_t)(x[q] >> 32);
            if ((q < 3 ? v[q + 1] : after) != v[q]) place_pads<W>(v[q], pos, cptr, col, wt);
        }
    }
    for (uint64_t i = 4 * M4 + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M;
         i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t v = key[i];
        const uint64_t pos = (uint64_t)cptr[v] * kSpan + (i - (uint64_t)row_ptr[v]);
        const VT x = val[i];
        col[pos] = (uint32_t)x;
        if constexpr (W) wt[pos] = (uint32_t)(x >> 32);
        if (i + 1 == M || key[i + 1] != v) place_pads<W>(v, pos, cptr, col, wt);
    }
}

// Host-input builds in sorted runs (build_sorted_runs): after chunk c is sorted, its nodes'
// chunk-local degrees deg_c and their chunk-local run starts start_c (exclusive scan of deg_c)
// turn into delta_c[v] = (arcs of v in chunks < c) - start_c[v] (mod 2^32), so that the arc at
// chunk-local sorted index li sits at offset li + delta_c[v] of v's row: chunks are in input
// order, so the rows stay stable.  D accumulates the degrees; deg_c is cleared for the next chunk.
__global__ void k_run_delta(uint32_t n, uint32_t* __restrict__ deg_c, const uint32_t* __restrict__ start_c,
                            uint32_t* __restrict__ D, uint32_t* __restrict__ delta_c) {
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        const uint32_t pre = D[v];
        delta_c[v] = pre - start_c[v];
        D[v] = pre + deg_c[v];
        deg_c[v] = 0;
    }
}

// the sorted runs -> padded segments: the arc at chunk-local sorted index li of chunk c goes to
// offset li + delta_c[v] of v's row.  Block b owns the arcs [b, b + 1) * kRunArcs of the row space
// (row_ptr order) and places them from every chunk in turn: chunk c's arcs that land in this
// window are one contiguous range of its sorted run, found from the window's first and last
// nodes (their run starts start_c, run lengths and earlier-chunk counts pre_c = start_c + delta_c).
// So the writes of all chunks to a window happen together and its 32-byte sectors fill up in L2
// (a sweep of each chunk across all rows wrote every sector once per chunk: 2.3 ms at cfg4), and a
// hub's row is spread over many blocks.  The pad slots are written by k_pad_runs.
constexpr uint32_t kRunArcs = 16384;
constexpr int kMaxRuns = 64;

template <bool W>
__global__ void k_place_runs(const uint32_t* __restrict__ key, const typename ValT<W>::T* __restrict__ val,
                             uint64_t chunk, uint32_t nch, uint32_t n, uint64_t m, const uint32_t* __restrict__ delta,
                             const uint32_t* __restrict__ starts, const int64_t* __restrict__ row_ptr,
                             const uint32_t* __restrict__ cptr, uint32_t* __restrict__ col, uint32_t* __restrict__ wt) {
    typedef typename ValT<W>::T VT;
    __shared__ uint32_t s_lo[kMaxRuns], s_hi[kMaxRuns];
    const uint64_t nblk = (m + kRunArcs - 1) / kRunArcs;
    for (uint64_t b = blockIdx.x; b < nblk; b += gridDim.x) {
        const uint64_t g0 = b * kRunArcs, g1 = min(m, g0 + kRunArcs);
        if (threadIdx.x < nch) {
            // the nodes holding row-space arcs g0 and g1 - 1: last v with row_ptr[v] <= g
            auto owner = [&](uint64_t g) {
                uint32_t lo = 0, hi = n;  // row_ptr[lo] <= g < row_ptr[hi]
                while (hi - lo > 1) {
                    const uint32_t mid = lo + (hi - lo) / 2;
                    if ((uint64_t)__ldg(row_ptr + mid) <= g) lo = mid; else hi = mid;
                }
                return lo;
            };
            const uint32_t vf = owner(g0), vl = owner(g1 - 1);
            const int64_t r0 = (int64_t)(g0 - (uint64_t)__ldg(row_ptr + vf));
            const int64_t r1 = (int64_t)(g1 - (uint64_t)__ldg(row_ptr + vl));  // exclusive, in vl's row
            const uint32_t c = threadIdx.x;
            const uint32_t* sc = starts + (uint64_t)c * (n + 1);
            const uint32_t* dl = delta + (uint64_t)c * n;
            const uint32_t sf = __ldg(sc + vf), df = __ldg(sc + vf + 1) - sf, pf = sf + __ldg(dl + vf);
            const uint32_t sl = __ldg(sc + vl), dn = __ldg(sc + vl + 1) - sl, pl = sl + __ldg(dl + vl);
            auto clamp = [](int64_t x, int64_t hi) -> uint32_t { return (uint32_t)(x < 0 ? 0 : (x > hi ? hi : x)); };
            s_lo[c] = sf + clamp(r0 - (int64_t)pf, (int64_t)df);
            s_hi[c] = sl + clamp(r1 - (int64_t)pl, (int64_t)dn);
        }
        __syncthreads();
        for (uint32_t c = 0; c < nch; ++c) {
            const uint32_t* kc = key + c * chunk;
            const VT* vc = val + c * chunk;
            const uint32_t* dl = delta + (uint64_t)c * n;
            const uint32_t hi = s_hi[c];
            for (uint32_t i0 = s_lo[c] + threadIdx.x; i0 < hi; i0 += 4 * blockDim.x) {
                // four items per thread and step, every load issued before the first store
                uint32_t v[4];
                VT x[4];
                uint64_t pos[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const uint32_t i = i0 + q * blockDim.x;
                    v[q] = i < hi ? kc[i] : 0u;
                    x[q] = i < hi ? vc[i] : VT(0);
                }
#pragma unroll
                for (int q = 0; q < 4; ++q)
                    pos[q] = (uint64_t)__ldg(cptr + v[q]) * kSpan + (uint32_t)(i0 + q * blockDim.x + __ldg(dl + v[q]));
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    if (i0 + q * blockDim.x >= hi) break;
                    col[pos[q]] = (uint32_t)x[q];
                    if constexpr (W) wt[pos[q]] = (uint32_t)(x[q] >> 32);
                }
            }
        }
        __syncthreads();  // s_lo / s_hi reused by the next window
    }
}

// pad slots of every node: from the end of its arcs to its next 32-byte span boundary
template <bool W>
__global__ void k_pad_runs(const uint32_t* __restrict__ deg, const uint32_t* __restrict__ cptr, uint32_t n,
                           uint32_t* __restrict__ col, uint32_t* __restrict__ wt) {
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        const uint64_t end = (uint64_t)cptr[v + 1] * kSpan;
        for (uint64_t q = (uint64_t)cptr[v] * kSpan + deg[v]; q < end; ++q) {
            col[q] = kPad;
            if constexpr (W) wt[q] = 0;
        }
    }
}

unsigned sort_grid(uint64_t items) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const uint64_t want = (items + kBlock - 1) / kBlock;
    const uint64_t cap = (uint64_t)sms * 8;
    return (unsigned)(want == 0 ? 1 : (want < cap ? want : cap));
}

// Host-input builds (api.cu tigr_graph_from_coo with host pointers): the arc list reaches the
// device in chunks on a copy stream, and each chunk is scanned on the build stream as soon as
// it lands, so the PCIe transfer and the scan overlap; the sort passes need the whole list.
constexpr uint64_t kCopyChunk = 1ull << 24;  // arcs per chunk (64 MB per array)

cudaStream_t copy_stream() {
    static std::mutex mu;
    static std::map<int, cudaStream_t> streams;  // one per device, for the process lifetime
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lk(mu);
    auto it = streams.find(dev);
    if (it != streams.end()) return it->second;
    cudaStream_t cs = nullptr;
    if (cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking) != cudaSuccess) return nullptr;
    streams[dev] = cs;
    return cs;
}

template <bool W>
using OnesweepFn = void (*)(const uint32_t*, const typename ValT<W>::T*, const uint32_t*, const uint32_t*,
                            const uint32_t*, uint64_t, uint64_t, int, int, const uint64_t*, uint64_t*, uint32_t*,
                            uint64_t, uint32_t*, typename ValT<W>::T*, uint32_t, uint32_t, int, uint32_t*);

// the pass kernel: first pass (reads the arc list; optionally filtered by source range), later
// passes; the degree-counting variant for the last pass of a CSR build
template <bool W>
OnesweepFn<W> onesweep_fn(bool first, bool filt, bool deg) {
    if (first && filt) return deg ? &k_onesweep<W, true, 16, true, true> : &k_onesweep<W, true, 16, true, false>;
    if (first) return deg ? &k_onesweep<W, true, 16, false, true> : &k_onesweep<W, true, 16, false, false>;
    return deg ? &k_onesweep<W, false, 16, false, true> : &k_onesweep<W, false, 16, false, false>;
}

template <bool W>
tigr_status sort_arcs(const uint32_t* src, const uint32_t* dst, const uint32_t* w, uint64_t m, uint64_t M,
                      uint32_t n, cudaStream_t s, TmpBuf& keys_out, TmpBuf& vals_out, bool validate,
                      uint32_t* in_flag = nullptr, uint32_t* in_sample = nullptr, uint32_t klo = 0,
                      uint32_t khi = 0xFFFFFFFFu, uint64_t* M_out = nullptr, const HostArcs* host = nullptr,
                      uint32_t* deg = nullptr) {
    typedef typename ValT<W>::T VT;
    int key_bits = 0;
    while (key_bits < 32 && (1ull << key_bits) < (uint64_t)n) ++key_bits;
    const int passes = key_bits == 0 ? 1 : (key_bits + 7) / 8;
    const int bits = key_bits == 0 ? 1 : (key_bits + passes - 1) / passes;
    const bool filtered = klo != 0 || khi < n;
    constexpr int SI = 16;  // items per thread (a sweep of 12 / 16 / 20 / 24 chose 16)
    const uint64_t tile_items = (uint64_t)kST * SI;
    const uint64_t tiles = (M + tile_items - 1) / tile_items;

    TmpBuf kb[2], vb[2], hist, dbase, status, counters, maxid, nloc;
    trace(s, "sort: enter");
    for (int i = 0; i < 2; ++i) {
        TIGR_TRY(kb[i].alloc(sizeof(uint32_t) * (M ? M : 1), s));
        TIGR_TRY(vb[i].alloc(sizeof(VT) * (M ? M : 1), s));
    }
    trace(s, "sort: alloc ping-pong");
    TIGR_TRY(hist.alloc(sizeof(unsigned long long) * 4 * kMaxRadix, s));
    TIGR_TRY(dbase.alloc(sizeof(uint64_t) * 4 * kMaxRadix, s));
    TIGR_TRY(status.alloc(sizeof(uint64_t) * kMaxRadix * (tiles ? tiles : 1), s));
    TIGR_TRY(counters.alloc(sizeof(uint32_t) * 4, s));
    TIGR_CK(cudaMemsetAsync(hist.p, 0, sizeof(unsigned long long) * 4 * kMaxRadix, s));
    TIGR_CK(cudaMemsetAsync(status.p, 0, sizeof(uint64_t) * kMaxRadix * (tiles ? tiles : 1), s));
    TIGR_CK(cudaMemsetAsync(counters.p, 0, sizeof(uint32_t) * 4, s));
    TIGR_TRY(maxid.alloc(sizeof(uint32_t), s));
    TIGR_CK(cudaMemsetAsync(maxid.p, 0, sizeof(uint32_t), s));
    TIGR_TRY(nloc.alloc(sizeof(unsigned long long), s));
    TIGR_CK(cudaMemsetAsync(nloc.p, 0, sizeof(unsigned long long), s));
    trace(s, "sort: alloc+memset");
    const int sym = M > m ? 1 : 0;
    if (M && host) {  // src / dst / w are the device destinations of the host arrays
        cudaStream_t cs = copy_stream();
        if (!cs) return fail(TIGR_ECUDA, "graph_from_coo: copy stream creation failed");
        cudaEvent_t ready;
        TIGR_CK(cudaEventCreateWithFlags(&ready, cudaEventDisableTiming));
        TIGR_CK(cudaEventRecord(ready, s));  // the destinations (fresh allocations) are free on s
        TIGR_CK(cudaStreamWaitEvent(cs, ready, 0));
        cudaEventDestroy(ready);
        for (uint64_t f0 = 0; f0 < m; f0 += kCopyChunk) {
            const uint64_t f1 = std::min<uint64_t>(m, f0 + kCopyChunk);
            const size_t bytes = sizeof(uint32_t) * (f1 - f0);
            TIGR_CK(cudaMemcpyAsync(const_cast<uint32_t*>(src) + f0, host->src + f0, bytes, cudaMemcpyHostToDevice, cs));
            TIGR_CK(cudaMemcpyAsync(const_cast<uint32_t*>(dst) + f0, host->dst + f0, bytes, cudaMemcpyHostToDevice, cs));
            if (W) TIGR_CK(cudaMemcpyAsync(const_cast<uint32_t*>(w) + f0, host->w + f0, bytes, cudaMemcpyHostToDevice, cs));
            cudaEvent_t landed;
            TIGR_CK(cudaEventCreateWithFlags(&landed, cudaEventDisableTiming));
            TIGR_CK(cudaEventRecord(landed, cs));
            TIGR_CK(cudaStreamWaitEvent(s, landed, 0));
            cudaEventDestroy(landed);  // released once it has completed
            k_coo_scan<<<sort_grid(f1 - f0), kBlock, 0, s>>>(src, dst, m, f0, f1, sym, passes, bits,
                                                              hist.as<unsigned long long>(), maxid.as<uint32_t>(), n,
                                                              in_flag, in_sample, klo, khi,
                                                              nloc.as<unsigned long long>());
            TIGR_CKL("coo scan (chunk)");
        }
    } else if (M) {
        k_coo_scan<<<sort_grid(m), kBlock, 0, s>>>(src, dst, m, 0, m, sym, passes, bits, hist.as<unsigned long long>(),
                                                    maxid.as<uint32_t>(), n, in_flag, in_sample, klo, khi,
                                                    nloc.as<unsigned long long>());
        TIGR_CKL("coo scan");
    }
    uint64_t Mloc = M;  // items that survive the source-range filter
    if (M && (validate || filtered)) {
        uint32_t hmax = 0;
        unsigned long long hl = 0;
        TIGR_CK(cudaMemcpyAsync(&hmax, maxid.p, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
        TIGR_CK(cudaMemcpyAsync(&hl, nloc.p, sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
        TIGR_CK(cudaStreamSynchronize(s));
        if (validate && hmax >= n) return fail(TIGR_EINVAL, "graph_from_coo: vertex id >= n");
        Mloc = hl;
    }
    if (M_out) *M_out = Mloc;
    k_digit_base<<<1, kMaxRadix, 0, s>>>(hist.as<unsigned long long>(), passes, dbase.as<uint64_t>());
    TIGR_CKL("digit base");
    trace(s, "sort: digit histograms");
    const size_t smem = (2 * sizeof(VT) + sizeof(uint32_t)) * tile_items;
    int cur = 0;
    for (int p = 0; p < passes && M; ++p) {
        // partitioned builds: the first pass drops the arcs outside [klo, khi); the last pass
        // counts the degrees when asked to
        const auto kern = onesweep_fn<W>(p == 0, p == 0 && filtered, p == passes - 1 && deg != nullptr);
        TIGR_CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        const int out = (p == 0) ? 0 : 1 - cur;
        const uint64_t Mp = (p == 0) ? M : Mloc;  // the first pass reads (and filters) the full list
        const uint64_t tp = (Mp + tile_items - 1) / tile_items;
        if (tp == 0) break;
        // bulk tile staging needs 16-byte aligned sources (the arc arrays of the first pass may
        // be caller pointers); development builds can turn it off with TIGR_SORT_BULK=0
        const uintptr_t al = p == 0 ? ((uintptr_t)src | (uintptr_t)dst) : ((uintptr_t)kb[cur].p | (uintptr_t)vb[cur].p);
        const int bulk_ok = (al & 15) == 0 && dev_knob("TIGR_SORT_BULK", 1) != 0;
        kern<<<(unsigned)tp, kST, smem, s>>>(kb[cur].as<uint32_t>(), vb[cur].as<VT>(), src, dst, w, m, Mp, p * bits,
                                             bits, dbase.as<uint64_t>() + p * kMaxRadix, status.as<uint64_t>(),
                                             counters.as<uint32_t>() + p, (uint64_t)(p + 1), kb[out].as<uint32_t>(),
                                             vb[out].as<VT>(), klo, khi, bulk_ok, p == passes - 1 ? deg : nullptr);
        TIGR_CKL("onesweep");
        trace(s, "sort: onesweep pass");
        cur = out;
    }
    std::swap(keys_out.p, kb[cur].p);
    std::swap(keys_out.s, kb[cur].s);
    std::swap(vals_out.p, vb[cur].p);
    std::swap(vals_out.s, vb[cur].s);
    return TIGR_OK;
}

// Host-input build in sorted runs (tigr_graph_from_coo with host arrays, no symmetrising, no
// source filter): the arc list arrives in chunks on the copy stream, and each chunk is scanned
// AND fully radix-sorted on the build stream while the next chunks are still in flight.  A
// sorted chunk is a stable run; the runs are merged into the rows by k_place_runs (chunk c's
// arcs of v follow those of chunks < c: input order), so after the last chunk lands only its own
// sort, the degree scans and the placement remain -- instead of the whole three-pass sort.
// The result is element-identical to build_sorted's (same canonical stable CSR).
// Ids are validated (maxid < n) before the placement, the first step that indexes by target;
// the sort's degree counting skips ids >= n (k_onesweep's khi guard).
template <bool W>
tigr_status build_sorted_runs(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, const uint32_t* w,
                              cudaStream_t s, tigr_graph* g, const HostArcs* host, uint64_t chunk) {
    typedef typename ValT<W>::T VT;
    int key_bits = 0;
    while (key_bits < 32 && (1ull << key_bits) < (uint64_t)n) ++key_bits;
    const int passes = key_bits == 0 ? 1 : (key_bits + 7) / 8;
    const int bits = key_bits == 0 ? 1 : (key_bits + passes - 1) / passes;
    constexpr int SI = 16;
    const uint64_t tile_items = (uint64_t)kST * SI;
    const uint64_t nch = (m + chunk - 1) / chunk;
    const uint64_t ctiles = (chunk + tile_items - 1) / tile_items;
    if (nch > (uint64_t)kMaxRuns || nch * passes >= 0xFFFF) return fail(TIGR_ERANGE, "graph_from_coo: too many copy chunks");

    TmpBuf kb[2], vb[2], hist, dbase, status, counters, maxid, nloc, deg_c, delta;
    for (int i = 0; i < 2; ++i) {
        TIGR_TRY(kb[i].alloc(sizeof(uint32_t) * m, s));
        TIGR_TRY(vb[i].alloc(sizeof(VT) * m, s));
    }
    TIGR_TRY(hist.alloc(sizeof(unsigned long long) * 4 * kMaxRadix * nch, s));
    TIGR_TRY(dbase.alloc(sizeof(uint64_t) * 4 * kMaxRadix * nch, s));
    TIGR_TRY(status.alloc(sizeof(uint64_t) * kMaxRadix * ctiles, s));
    TIGR_TRY(counters.alloc(sizeof(uint32_t) * 4 * nch, s));
    TIGR_TRY(maxid.alloc(sizeof(uint32_t), s));
    TIGR_TRY(nloc.alloc(sizeof(unsigned long long), s));
    TIGR_TRY(deg_c.alloc(sizeof(uint32_t) * n, s));
    TIGR_TRY(delta.alloc(sizeof(uint32_t) * n * nch, s));
    TmpBuf starts;  // start_c of every chunk: uint32[nch][n + 1]
    TIGR_TRY(starts.alloc(sizeof(uint32_t) * ((uint64_t)n + 1) * nch, s));
    TIGR_CK(cudaMemsetAsync(hist.p, 0, sizeof(unsigned long long) * 4 * kMaxRadix * nch, s));
    TIGR_CK(cudaMemsetAsync(status.p, 0, sizeof(uint64_t) * kMaxRadix * ctiles, s));  // epoch 0 matches nothing
    TIGR_CK(cudaMemsetAsync(counters.p, 0, sizeof(uint32_t) * 4 * nch, s));
    TIGR_CK(cudaMemsetAsync(maxid.p, 0, sizeof(uint32_t), s));
    TIGR_CK(cudaMemsetAsync(nloc.p, 0, sizeof(unsigned long long), s));
    TIGR_CK(cudaMemsetAsync(deg_c.p, 0, sizeof(uint32_t) * n, s));
    uint32_t* D = g->deg.as<uint32_t>();  // zeroed by the caller

    cudaStream_t cs = copy_stream();
    if (!cs) return fail(TIGR_ECUDA, "graph_from_coo: copy stream creation failed");
    cudaEvent_t ready;
    TIGR_CK(cudaEventCreateWithFlags(&ready, cudaEventDisableTiming));
    TIGR_CK(cudaEventRecord(ready, s));  // the destinations (fresh allocations) are free on s
    TIGR_CK(cudaStreamWaitEvent(cs, ready, 0));
    cudaEventDestroy(ready);
    // every copy is queued up front, so the copy engine never waits for the build stream
    std::vector<cudaEvent_t> landed(nch);
    for (uint64_t c = 0; c < nch; ++c) {
        const uint64_t f0 = c * chunk, f1 = std::min<uint64_t>(m, f0 + chunk);
        const size_t bytes = sizeof(uint32_t) * (f1 - f0);
        TIGR_CK(cudaMemcpyAsync(const_cast<uint32_t*>(src) + f0, host->src + f0, bytes, cudaMemcpyHostToDevice, cs));
        TIGR_CK(cudaMemcpyAsync(const_cast<uint32_t*>(dst) + f0, host->dst + f0, bytes, cudaMemcpyHostToDevice, cs));
        if (W) TIGR_CK(cudaMemcpyAsync(const_cast<uint32_t*>(w) + f0, host->w + f0, bytes, cudaMemcpyHostToDevice, cs));
        TIGR_CK(cudaEventCreateWithFlags(&landed[c], cudaEventDisableTiming));
        TIGR_CK(cudaEventRecord(landed[c], cs));
    }
    const size_t smem = (2 * sizeof(VT) + sizeof(uint32_t)) * tile_items;
    for (int p = 0; p < passes; ++p)
        TIGR_CK(cudaFuncSetAttribute(onesweep_fn<W>(p == 0, false, p == passes - 1),
                                     cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int cur = 0;
    for (uint64_t c = 0; c < nch; ++c) {
        const uint64_t f0 = c * chunk, f1 = std::min<uint64_t>(m, f0 + chunk), Mc = f1 - f0;
        TIGR_CK(cudaStreamWaitEvent(s, landed[c], 0));
        cudaEventDestroy(landed[c]);  // released once it has completed
        unsigned long long* hc = hist.as<unsigned long long>() + c * 4 * kMaxRadix;
        uint64_t* bc = dbase.as<uint64_t>() + c * 4 * kMaxRadix;
        k_coo_scan<<<sort_grid(Mc), kBlock, 0, s>>>(src, dst, m, f0, f1, 0, passes, bits, hc, maxid.as<uint32_t>(), n,
                                                     g->in_flag.as<uint32_t>(), g->in_sample.as<uint32_t>(), 0,
                                                     0xFFFFFFFFu, nloc.as<unsigned long long>());
        TIGR_CKL("coo scan (run)");
        k_digit_base<<<1, kMaxRadix, 0, s>>>(hc, passes, bc);
        TIGR_CKL("digit base (run)");
        cur = 0;
        const uint64_t tp = (Mc + tile_items - 1) / tile_items;
        for (int p = 0; p < passes; ++p) {
            const int out = (p == 0) ? 0 : 1 - cur;
            const uintptr_t al = p == 0 ? ((uintptr_t)(src + f0) | (uintptr_t)(dst + f0))
                                        : ((uintptr_t)(kb[cur].as<uint32_t>() + f0) | (uintptr_t)(vb[cur].as<VT>() + f0));
            const int bulk_ok = (al & 15) == 0 && dev_knob("TIGR_SORT_BULK", 1) != 0;
            onesweep_fn<W>(p == 0, false, p == passes - 1)<<<(unsigned)tp, kST, smem, s>>>(
                kb[cur].as<uint32_t>() + f0, vb[cur].as<VT>() + f0, src + f0, dst + f0, W ? w + f0 : nullptr, Mc, Mc,
                p * bits, bits, bc + p * kMaxRadix, status.as<uint64_t>(), counters.as<uint32_t>() + c * 4 + p,
                (uint64_t)(c * passes + p + 1), kb[out].as<uint32_t>() + f0, vb[out].as<VT>() + f0, 0, n, bulk_ok,
                p == passes - 1 ? deg_c.as<uint32_t>() : nullptr);
            TIGR_CKL("onesweep (run)");
            cur = out;
        }
        uint32_t* sc = starts.as<uint32_t>() + c * ((uint64_t)n + 1);
        TIGR_TRY(exclusive_scan_u32(deg_c.as<uint32_t>(), n, SCAN_U32, 1, sc, s, nullptr));
        k_run_delta<<<grid_for(n), kBlock, 0, s>>>(n, deg_c.as<uint32_t>(), sc, D, delta.as<uint32_t>() + c * n);
        TIGR_CKL("run delta");
    }
    uint32_t hmax = 0;
    TIGR_CK(cudaMemcpyAsync(&hmax, maxid.p, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    if (hmax >= n) return fail(TIGR_EINVAL, "graph_from_coo: vertex id >= n");
    g->has_in_sketch = true;
    g->m = m;
    TIGR_TRY(g->row_ptr.alloc(sizeof(int64_t) * ((size_t)n + 1), s));
    TIGR_TRY(exclusive_scan_u64(D, n, SCAN_U32, 1, reinterpret_cast<uint64_t*>(g->row_ptr.p), s));
    TIGR_TRY(g->cptr.alloc(sizeof(uint32_t) * ((size_t)n + 1), s));
    uint64_t spans = 0;
    TIGR_TRY(exclusive_scan_u32(D, n, SCAN_CEIL_DIV, kSpan, g->cptr.as<uint32_t>(), s, &spans));
    if (spans >= (1ull << 31)) return fail(TIGR_ERANGE, "graph: padded edge spans exceed 2^31");
    g->nchunks = spans * 2;  // 16-byte chunks
    TIGR_TRY(g->col.alloc(sizeof(uint32_t) * kChunk * (g->nchunks ? g->nchunks : 1), s));
    if (W) TIGR_TRY(g->wt.alloc(sizeof(uint32_t) * kChunk * (g->nchunks ? g->nchunks : 1), s));
    const uint64_t windows = (m + kRunArcs - 1) / kRunArcs;
    k_place_runs<W><<<(unsigned)std::min<uint64_t>(windows, 1u << 20), kBlock, 0, s>>>(
        kb[cur].as<uint32_t>(), vb[cur].as<VT>(), chunk, (uint32_t)nch, n, m, delta.as<uint32_t>(),
        starts.as<uint32_t>(), g->row_ptr.as<int64_t>(), g->cptr.as<uint32_t>(), g->col.as<uint32_t>(),
        W ? g->wt.as<uint32_t>() : nullptr);
    TIGR_CKL("place (runs)");
    k_pad_runs<W><<<grid_for(n), kBlock, 0, s>>>(D, g->cptr.as<uint32_t>(), n, g->col.as<uint32_t>(),
                                                  W ? g->wt.as<uint32_t>() : nullptr);
    TIGR_CKL("pads (runs)");
    return TIGR_OK;
}

template <bool W>
tigr_status build_sorted(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, const uint32_t* w,
                         int symmetrize, cudaStream_t s, tigr_graph* g, uint32_t klo, uint32_t khi,
                         const HostArcs* host) {
    typedef typename ValT<W>::T VT;
    const uint64_t Mall = symmetrize ? 2 * m : m;
    uint64_t M = Mall;
    TmpBuf keys, vals;
    keys.s = vals.s = s;
    const size_t fw = ((size_t)n + 31) / 32 + 1;  // in_flag bitmap words
    TIGR_TRY(g->in_flag.alloc(sizeof(uint32_t) * fw, s));
    TIGR_TRY(g->in_sample.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    TIGR_CK(cudaMemsetAsync(g->in_flag.p, 0, sizeof(uint32_t) * fw, s));
    TIGR_CK(cudaMemsetAsync(g->in_sample.p, 0, sizeof(uint32_t) * n, s));
    // degrees: counted by the last radix pass from the runs of equal keys in its tiles
    TIGR_TRY(g->deg.alloc(sizeof(uint32_t) * (n ? n : 1), s));
    TIGR_CK(cudaMemsetAsync(g->deg.p, 0, sizeof(uint32_t) * n, s));
    // host arrays, whole graph, more than one copy chunk: sort the chunks as they land
    const uint64_t run_chunk = std::max<uint64_t>(kCopyChunk, ((m / 64 + (1u << 20) - 1) >> 20) << 20);
    if (host && !symmetrize && klo == 0 && khi >= n && m > run_chunk && dev_knob("TIGR_HOST_RUNS", 1))
        return build_sorted_runs<W>(n, m, src, dst, w, s, g, host, run_chunk);
    TIGR_TRY(sort_arcs<W>(src, dst, w, m, Mall, n, s, keys, vals, true, g->in_flag.as<uint32_t>(),
                          g->in_sample.as<uint32_t>(), klo, khi, &M, host, g->deg.as<uint32_t>()));
    g->has_in_sketch = true;
    g->m = M;  // arcs of this build's source range (all arcs unless partitioned)
    // node array, padded chunk offsets, edge buffers
    TIGR_TRY(g->row_ptr.alloc(sizeof(int64_t) * ((size_t)n + 1), s));
    TIGR_TRY(exclusive_scan_u64(g->deg.as<uint32_t>(), n, SCAN_U32, 1, reinterpret_cast<uint64_t*>(g->row_ptr.p), s));
    TIGR_TRY(g->cptr.alloc(sizeof(uint32_t) * ((size_t)n + 1), s));
    uint64_t nch = 0;
    TIGR_TRY(exclusive_scan_u32(g->deg.as<uint32_t>(), n, SCAN_CEIL_DIV, kSpan, g->cptr.as<uint32_t>(), s, &nch));
    if (nch >= (1ull << 31)) return fail(TIGR_ERANGE, "graph: padded edge spans exceed 2^31");
    nch *= 2;  // 16-byte chunks
    g->nchunks = nch;
    trace(s, "csr: deg+scans");
    TIGR_TRY(g->col.alloc(sizeof(uint32_t) * kChunk * (nch ? nch : 1), s));
    if (W) TIGR_TRY(g->wt.alloc(sizeof(uint32_t) * kChunk * (nch ? nch : 1), s));
    if (M) {
        k_place<W><<<sort_grid(M), kBlock, 0, s>>>(keys.as<uint32_t>(), vals.as<VT>(), M, g->row_ptr.as<int64_t>(),
                                                    g->cptr.as<uint32_t>(), g->col.as<uint32_t>(),
                                                    W ? g->wt.as<uint32_t>() : nullptr);
        TIGR_CKL("place");
    }
    trace(s, "csr: place");
    return TIGR_OK;
}

constexpr int kCutBuckets = 16384;

// histogram of the arc sources over kCutBuckets contiguous vertex ranges (per-block shared copy)
__global__ void k_src_hist(const uint32_t* __restrict__ src, const uint32_t* __restrict__ dst, uint64_t m, uint64_t M,
                           int shift, unsigned long long* __restrict__ hist) {
    extern __shared__ uint32_t sh[];
    for (int i = threadIdx.x; i < kCutBuckets; i += blockDim.x) sh[i] = 0;
    __syncthreads();
    for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < M; e += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t k = e < m ? src[e] : dst[e - m];
        atomicAdd(&sh[min((uint32_t)(k >> shift), (uint32_t)kCutBuckets - 1)], 1u);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < kCutBuckets; i += blockDim.x)
        if (sh[i]) atomicAdd(&hist[i], (unsigned long long)sh[i]);
}

}  // namespace

// Source-vertex cuts for nranks partitions with ~equal arc counts, at a granularity of
// n / 16384 vertices (deterministic: every rank computes the same cuts from the same arcs).
tigr_status coo_source_cuts(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, int symmetrize,
                            int nranks, cudaStream_t s, uint32_t* cuts) {
    const uint64_t M = symmetrize ? 2 * m : m;
    int key_bits = 0;
    while (key_bits < 32 && (1ull << key_bits) < (uint64_t)n) ++key_bits;
    const int shift = key_bits > 14 ? key_bits - 14 : 0;
    TmpBuf hist;
    TIGR_TRY(hist.alloc(sizeof(unsigned long long) * kCutBuckets, s));
    TIGR_CK(cudaMemsetAsync(hist.p, 0, sizeof(unsigned long long) * kCutBuckets, s));
    if (M) {
        TIGR_CK(cudaFuncSetAttribute(k_src_hist, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)(sizeof(uint32_t) * kCutBuckets)));
        k_src_hist<<<sort_grid(M), kBlock, sizeof(uint32_t) * kCutBuckets, s>>>(src, dst, m, M, shift,
                                                                               hist.as<unsigned long long>());
        TIGR_CKL("source histogram");
    }
    std::vector<unsigned long long> h(kCutBuckets);
    TIGR_CK(cudaMemcpyAsync(h.data(), hist.p, sizeof(unsigned long long) * kCutBuckets, cudaMemcpyDeviceToHost, s));
    TIGR_CK(cudaStreamSynchronize(s));
    cuts[0] = 0;
    cuts[nranks] = n;
    unsigned long long acc = 0;
    int b = 0;
    for (int r = 1; r < nranks; ++r) {
        const unsigned long long target = (unsigned long long)((unsigned __int128)M * (unsigned)r / (unsigned)nranks);
        while (b < kCutBuckets && acc + h[b] <= target) acc += h[b++];
        // bucket b straddles the target: cut at the nearer of its two boundaries
        uint64_t v = (uint64_t)b << shift;
        if (b < kCutBuckets && target - acc > acc + h[b] - target) v = (uint64_t)(b + 1) << shift;
        cuts[r] = (uint32_t)std::min<uint64_t>(std::max<uint64_t>(v, cuts[r - 1]), n);
    }
    return TIGR_OK;
}

// Stable sort of (key, value) u32 pairs by key (keys < key_limit); results owned by the TmpBufs.
tigr_status sort_pairs_u32(const uint32_t* keys, const uint32_t* vals, uint64_t count, uint32_t key_limit,
                           cudaStream_t s, TmpBuf& keys_out, TmpBuf& vals_out) {
    keys_out.s = vals_out.s = s;
    return sort_arcs<false>(keys, vals, nullptr, count, count, key_limit, s, keys_out, vals_out, false);
}

// Stable device CSR build from an arc list (device pointers).  Caller validated ids < n.
tigr_status csr_build_sorted(uint32_t n, uint64_t m, const uint32_t* src, const uint32_t* dst, const uint32_t* w,
                             int symmetrize, cudaStream_t s, tigr_graph* g, uint32_t klo, uint32_t khi,
                             const HostArcs* host) {
    if (w) return build_sorted<true>(n, m, src, dst, w, symmetrize, s, g, klo, khi, host);
    return build_sorted<false>(n, m, src, dst, w, symmetrize, s, g, klo, khi, host);
}

}  // namespace tigr
