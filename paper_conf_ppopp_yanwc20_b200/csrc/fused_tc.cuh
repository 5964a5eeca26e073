// fused_tc.cuh -- fused Winograd F(2x2,3x3) with the Winograd-domain GEMM on
// tcgen05 tensor cores (TF32 or 3xTF32), accumulators in TMEM.
//
// Paper: same method and steps as the FP32 kernel (Eq. 5-8;
// Alg. 1); the paper has no tensor-core path and notes that "the data
// layout needs a redesign" for one (Sec. 8.3).  This is that redesign.
//
// Tile: 128 filters (UMMA M) x 32 tiles*images nu (UMMA N) x all 16 xi.
// TMEM: 16 accumulators D(xi) of 128 lanes x 32 columns = all 512 columns.
// Persistent (one CTA per SM, tiles blockIdx.x, +gridDim.x, ...), warp-specialised:
//   * warp 12 (U producer): 64 KB bulk copies of the pre-arranged transformed
//     filter per channel block into a 2-slot ring;
//   * warp 14 (x producer): TMA box of raw x (n:32, w:4, h:4, c:8) per channel
//     block (zero fill = implicit padding, Sec. 3.5), L2 prefetch ahead;
//   * warps 8-11 (ITF): V = B^T d B (Eq. 6) for the 8 x 32 (c, nu) tiles of a
//     block, rounded to TF32 (3xTF32: big + small planes), stored as the
//     K-major UMMA B operand.  A lane owns one nu and 4 channels: its raw-x reads
//     are 32 consecutive floats per warp (conflict-free) and its V stores are one
//     16 B core-matrix row per xi (a quarter-warp writes 128 contiguous bytes);
//     MM = 128: two warp pairs take alternate channel blocks; MM = 64: one warp
//     pair per nu-half;
//   * warp 13 (MMA, one thread): per xi, D(xi) += U(xi) * V(xi) (3xTF32:
//     big*big + big*small + small*big); tcgen05.commit frees smem slots;
//   * warps 0-7 (epilogue): warps w and w + 4 share TMEM lane quadrant w % 4 and
//     split its columns (nu 0-15 / 16-31 of every accumulator): tcgen05.ld, OTF
//     (Eq. 8) into registers, release TMEM to the next tile's MMAs, then
//     coalesced stores -- overlapping the next tile's main loop.  Eight warps
//     drain TMEM about twice as fast as four (tile-boundary stall).
// Every hand-off between thread groups is an mbarrier on which each producing lane
// arrives itself (racecheck-clean; scripts/microbench/racecheck_mbar_repro.cu).
// All hand-offs are mbarriers; the producers run ahead across tile boundaries.
#pragma once
#include <cuda.h>

#include <cstdint>

#include "wino_ptx.cuh"
#include "wino_transforms.cuh"

namespace wino {
namespace tc {

#ifdef WINO_TC_TRACE
// Debug-only event trace (CTA 0): [event][cb] = clock64 at the event.
constexpr int TRACE_EVENTS = 8, TRACE_CB = 128;
__device__ unsigned long long g_trace[TRACE_EVENTS * TRACE_CB];
#define TC_TRACE(ev, cb)                                                                         \
    do {                                                                                         \
        if (blockIdx.x == 0 && (cb) < TRACE_CB) g_trace[(ev) * TRACE_CB + (cb)] = clock64();    \
    } while (0)
#else
#define TC_TRACE(ev, cb) \
    do {                 \
    } while (0)
#endif

constexpr int BN = 32;         // nu per UMMA (N); a tile has 128 / MM such halves
// MM (template) = filters per tile = UMMA M: 128, or 64 with TWO accumulators per
// xi interleaved in TMEM lanes (rows 0-15 of each 32-lane quadrant hold nu-half 0,
// lanes 16-31 hold nu-half 1; scripts/microbench/umma_m64.cu) -> tile 64 x 64.
constexpr int BC = 8;          // channels per block (UMMA K for tf32)
constexpr int EPI_WARPS = 8;   // warps 0..7: epilogue (TMEM lane quadrant warp % 4, column half warp / 4)
constexpr int ITF_WARP0 = 8;   // warps 8..11: ITF
constexpr int ITF_WARPS = 4;
constexpr int PROD_WARP = 12;  // bulk-copy producer of the transformed filter U
constexpr int MMA_WARP = 13;   // tcgen05.mma issuer
constexpr int XPROD_WARP = 14; // TMA / cp.async producer of raw x
constexpr int NT = 512;        // 16 warps (warp 15 idle; warpgroup-granular register split)
constexpr int REG_EPI = 168, REG_ITF = 120, REG_PROD = 56;  // 256*168 + 128*120 + 128*56 = 65536
template <int MM>
constexpr int a_tile() { return MM * BC * 4; }  // one (xi, plane) A operand: 4 / 2 KB
constexpr int B_TILE = BN * BC * 4;  // one (xi, plane, nu-half) B operand: 1 KB
constexpr int XS_BYTES = BC * 16 * BN * 4;  // raw x box: 16 KB
constexpr int X_PREFETCH = 6;               // channel blocks of x prefetched into L2 ahead
// U ring unit: 64 KB = all 16 xi (TF32) or 8 xi x 2 planes (3xTF32) of one channel
// block.  A bulk copy occupies the SM's copy engine for ~360 cycles whatever its
// size up to 32 KB (scripts/microbench/bulk_bw.cu: 11 / 23 / 45 / 90 B/clk/SM for
// 4 / 8 / 16 / 32 KB copies, ~110 B/clk for 64 KB), so the ring uses the largest
// copies that still leave two slots in flight.
template <int P>
constexpr int xi_per_unit() { return P == 1 ? 16 : 8; }

// u_tc layout (written by tc_filter_kernel, read with bulk copies):
//   [cb = C/8][kb = K/MM][xi 16][plane P][m/8][c/4 2][m%8 8][c%4 4]  fp32
// i.e. per (cb, kb, xi, plane) one K-major SWIZZLE_NONE UMMA A tile of MM rows
// (LBO = 128 B between the two 16 B K-chunks, SBO = 256 B between 8-row groups).
__host__ __device__ inline size_t u_tc_floats(int C, int K, int planes, int MM) {
    return size_t((C + BC - 1) / BC) * ((K + MM - 1) / MM) * 16 * planes * (MM * BC);
}
// Tile height used for a shape: the filter transform and the conv must agree.
#ifdef WINO_TC_MM64_ALL
__host__ __device__ inline int tc_mm(int, int planes) { return planes == 1 ? 64 : 128; }  // A/B builds
#else
__host__ __device__ inline int tc_mm(int K, int planes) { return (planes == 1 && K <= 64) ? 64 : 128; }
#endif

// FTF (Eq. 5) straight into the tensor-core operand layout, rounded to TF32 (reading R8;
// 3xTF32 also stores small = rna(u - big)).  Block = 8 channels x 32 filters, one (c, k) per
// thread (9 coalesced loads along k); results staged in shared memory so that every store is
// a 16 B core-matrix row (4 channels of one filter).  Grid (Kp/32, ceil(C/8)).  Pads K and C
// with zeros.
template <int P, int MM>
__global__ void __launch_bounds__(256) tc_filter_kernel(const float* __restrict__ w, float* __restrict__ u_tc,
                                                        int C, int K) {
    __shared__ __align__(16) float st[16][P][32][BC];  // [xi][plane][k][c]
    const int kl = threadIdx.x & 31, cl = threadIdx.x >> 5;
    const int k = blockIdx.x * 32 + kl, cb = blockIdx.y, c = cb * BC + cl;
    float t[16];
    if (c < C && k < K) {
        float g[9];
        const float* wc = w + (size_t)c * 9 * K + k;
#pragma unroll
        for (int e = 0; e < 9; ++e) g[e] = __ldg(wc + (size_t)e * K);
        ftf_4x4(g, t);
    } else {
#pragma unroll
        for (int e = 0; e < 16; ++e) t[e] = 0.f;
    }
#pragma unroll
    for (int xi = 0; xi < 16; ++xi) {
        const float big = to_tf32(t[xi]);
        st[xi][0][kl][cl] = big;
        if (P == 2) st[xi][P - 1][kl][cl] = to_tf32(t[xi] - big);
    }
    __syncthreads();
    const int Kp = ((K + MM - 1) / MM) * MM, nkb = Kp / MM;
#pragma unroll
    for (int r = 0; r < 4 * P; ++r) {  // 16 xi x P planes x 32 filters x 2 chunks of 4 channels
        const int row = r * 256 + threadIdx.x;
        const int ch = row & 1, rk = (row >> 1) & 31, pl = (row >> 6) % P, xi = (row >> 6) / P;
        const int kk = blockIdx.x * 32 + rk;
        if (kk >= Kp) continue;
        const int kb = kk / MM, m = kk % MM;
        const size_t base = ((((size_t)cb * nkb + kb) * 16 + xi) * P + pl) * (MM * BC);
        *reinterpret_cast<float4*>(u_tc + base + (m >> 3) * 64 + ch * 32 + (m & 7) * 4) =
            *reinterpret_cast<const float4*>(&st[xi][pl][rk][ch * 4]);
    }
}

struct __align__(64) Params {
    CUtensorMap tmx;  // x (C,H,W,N) as (N, W, H, C), box (32, 4, 4, 8)   [TMA x path]
    const float* __restrict__ x;
    const float* __restrict__ u_tc;
    float* __restrict__ y;
    int N, C, H, W, K;
    int TW, NV;
    int num_kb;     // ceil(K/MM)
    int num_cb;     // ceil(C/8)
    int num_tiles;  // ceil(NV/(32*NH)) * num_kb
    // stream-K (SK = true, same scheme as fused_tc16.cuh): units = tile * num_cb + cb, CTA b takes
    // [b*q + min(b, r), ...); pieces of cut tiles leave partial outputs in sk_ws (2 x 64 KiB per CTA)
    float* __restrict__ sk_ws;
    int sk_q, sk_r;
};

__host__ __device__ __forceinline__ int sk_start(const Params& p, int b) { return b * p.sk_q + min(b, p.sk_r); }

// The (tile, channel-block range) pieces of a CTA, identical in every warp role.
template <bool SK>
struct Segs {
    int a, b, n = 0;
    __device__ __forceinline__ explicit Segs(const Params& p) {
        if constexpr (SK) {
            a = sk_start(p, blockIdx.x);
            b = sk_start(p, blockIdx.x + 1);
        } else {
            a = blockIdx.x;
            b = gridDim.x;
        }
    }
    __device__ __forceinline__ bool next(const Params& p, int& tile, int& lo, int& hi) {
        if constexpr (SK) {
            if (a >= b) return false;
            tile = a / p.num_cb;
            lo = a - tile * p.num_cb;
            hi = min(p.num_cb, lo + (b - a));
            a += hi - lo;
        } else {
            if (a >= p.num_tiles) return false;
            tile = a;
            lo = 0;
            hi = p.num_cb;
            a += b;
        }
        ++n;
        return true;
    }
};

template <int P, int MM, int XM>
struct Cfg {
    static constexpr int NH = 128 / MM;                         // nu-halves per tile (32 nu each)
    static constexpr int XPU = xi_per_unit<P>();
    static constexpr int UNITS_PER_CB = 16 / XPU;
    static constexpr int A_TILE = a_tile<MM>();
    static constexpr int UNIT = XPU * P * A_TILE;               // 64 KB (MM=128) / 32 KB (MM=64)
    static constexpr int U_SLOTS = (MM == 64 && XM >= 2) ? 3 : 2;
    static constexpr int X_SLOTS = 2;                           // raw x boxes in flight (L2-prefetched)
    static constexpr int X_SLOT = NH * XS_BYTES;
    static constexpr int V_SLOT = 16 * NH * P * B_TILE;        // 16 / 32 KB
    static constexpr int TAB = (XM >= 2) ? 0 : 16 * BN * NH * 4;  // cp.async gather table
    static constexpr int OFF_U = 0;
    static constexpr int OFF_X = OFF_U + U_SLOTS * UNIT;
    static constexpr int OFF_V = OFF_X + X_SLOTS * X_SLOT;
    static constexpr int OFF_TAB = OFF_V + 2 * V_SLOT;
    static constexpr int OFF_BAR = OFF_TAB + TAB;
    // u_full/u_empty[U_SLOTS], x_full/x_empty[X_SLOTS], v_full[2], v_empty[2], acc_full, acc_empty
    static constexpr int NBAR = 2 * U_SLOTS + 2 * X_SLOTS + 6;
    static constexpr int OFF_TMEM = OFF_BAR + NBAR * 8;
    static constexpr int BYTES = OFF_TMEM + 16;
    static_assert(BYTES <= 232448, "shared memory budget");
};

// XM: 2 = TMA x box (N % 32 == 0), 3 = 32/N TMA boxes per nu-half (N in {4, 8, 16}: the
// per-rank batches of batch sharding), 1 = cp.async 16 B gather, 0 = cp.async 4 B gather
template <int P, int XM, int MM, bool SK = false>
__global__ void __launch_bounds__(NT, 1) fused_tc_kernel(const __grid_constant__ Params p) {
    using G = Cfg<P, MM, XM>;
    constexpr int NH = G::NH;
    constexpr int TN = BN * NH;  // nu per tile
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t* const su = smem + G::OFF_U;
    float* const sx = reinterpret_cast<float*>(smem + G::OFF_X);
    uint8_t* const sv = smem + G::OFF_V;
    int* const xtab = reinterpret_cast<int*>(smem + G::OFF_TAB);
    uint64_t* const bars = reinterpret_cast<uint64_t*>(smem + G::OFF_BAR);
    uint64_t* const u_full = bars;
    uint64_t* const u_empty = bars + G::U_SLOTS;
    uint64_t* const x_full = bars + 2 * G::U_SLOTS;
    uint64_t* const x_empty = x_full + G::X_SLOTS;
    uint64_t* const v_full = x_empty + G::X_SLOTS;
    uint64_t* const v_empty = v_full + 2;
    uint64_t* const acc_full = v_full + 4;
    uint64_t* const acc_empty = acc_full + 1;
    uint32_t* const tmem_slot = reinterpret_cast<uint32_t*>(smem + G::OFF_TMEM);

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

    if (tid == 0) {
        for (int s = 0; s < G::U_SLOTS; ++s) {
            mbar_init(&u_full[s], 1);
            mbar_init(&u_empty[s], 1);
        }
        // ITF lanes per channel block: MM = 128 one warp pair (the pairs alternate blocks),
        // MM = 64 both pairs (one per nu-half); the gather path's x producer arrives per lane
        constexpr int ITF_LANES = (NH == 1 ? 2 : 4) * 32;
        for (int s = 0; s < G::X_SLOTS; ++s) {
            mbar_init(&x_full[s], XM >= 2 ? 1 : 32);
            mbar_init(&x_empty[s], ITF_LANES);
        }
        for (int s = 0; s < 2; ++s) {
            mbar_init(&v_full[s], ITF_LANES);
            mbar_init(&v_empty[s], 1);
        }
        mbar_init(acc_full, 1);
        mbar_init(acc_empty, EPI_WARPS * 32);
        fence_mbar_init();
        if constexpr (XM >= 2) tma_prefetch_desc(&p.tmx);
    }
    if (warp == 0) tmem_alloc(tmem_slot, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    const size_t HWN = (size_t)p.H * p.W * p.N;

    if (warp >= PROD_WARP) {
        setmaxnreg_dec<REG_PROD>();
        if (warp == XPROD_WARP) {
            // --------------------------- raw-x producer ---------------------------
            int gcb = 0;  // channel blocks issued so far (all tiles)
            Segs<SK> segs(p);
            int tile, lo, hi;
            while (segs.next(p, tile, lo, hi)) {
                const int nu0 = (tile / p.num_kb) * TN;
                int tma_n0[NH], tma_w0[NH], tma_h0[NH];
                if constexpr (XM == 3) {
                    // first image tile of each half; the half's 32/N boxes are tiles t0 .. t0 + 32/N - 1
#pragma unroll
                    for (int h = 0; h < NH; ++h) tma_n0[h] = (nu0 + h * BN) / p.N;
                } else if constexpr (XM == 2) {
#pragma unroll
                    for (int h = 0; h < NH; ++h) {  // N % 32 == 0: each half = 32 consecutive n of one image tile
                        const int nuh = nu0 + h * BN;
                        const int t = nuh < p.NV ? nuh / p.N : 0;
                        tma_n0[h] = nuh < p.NV ? nuh - t * p.N : 0;
                        const int th = t / p.TW, tw = t - th * p.TW;
                        tma_w0[h] = nuh < p.NV ? 2 * tw - 1 : -8;  // -1: TMA zero fill = padding (Sec. 3.5);
                        tma_h0[h] = nuh < p.NV ? 2 * th - 1 : -8;  // -8: half past NV -> all zeros
                    }
                    // x streams from HBM (first touch): warm L2 a few blocks ahead
                    if (lane == 0)
                        for (int cb = lo; cb < lo + X_PREFETCH && cb < hi; ++cb)
#pragma unroll
                            for (int h = 0; h < NH; ++h)
                                tma_prefetch_l2_4d(&p.tmx, tma_n0[h], tma_w0[h], tma_h0[h], cb * BC);
                } else {
                    // gather offsets (h*W+w)*N+n of the 4x4 window element pos of local nu (-1: padding)
                    __syncwarp();
                    for (int e = lane; e < 16 * TN; e += 32) {
                        const int hh = e / (16 * BN), r = e % (16 * BN);
                        const int pos = r / BN, nl = r % BN, nu = nu0 + hh * BN + nl;
                        int off = -1;
                        if (nu < p.NV) {
                            const int t = nu / p.N, n = nu - t * p.N;
                            const int th = t / p.TW, tw = t - th * p.TW;
                            const int h = 2 * th - 1 + (pos >> 2), w = 2 * tw - 1 + (pos & 3);
                            if (h >= 0 && h < p.H && w >= 0 && w < p.W) off = (h * p.W + w) * p.N + n;
                        }
                        xtab[e] = off;
                    }
                    __syncwarp();
                }
                for (int cb = lo; cb < hi; ++cb, ++gcb) {
                    const int xs = gcb % G::X_SLOTS;
                    if (gcb >= G::X_SLOTS) mbar_wait(&x_empty[xs], ((gcb / G::X_SLOTS) - 1) & 1);
                    float* xdst = sx + xs * (G::X_SLOT / 4);
                    if constexpr (XM == 3) {
                        if (lane == 0) {
                            mbar_arrive_expect_tx(&x_full[xs], G::X_SLOT);
                            const int nbox = BN / p.N;
#pragma unroll
                            for (int h = 0; h < NH; ++h)
                                for (int b = 0; b < nbox; ++b) {
                                    const int t = tma_n0[h] + b;
                                    const bool live = t * p.N < p.NV;
                                    const int th = t / p.TW, tw = t - th * p.TW;
                                    // -1: zero fill = padding (Sec. 3.5); -8: tile past the end -> zeros
                                    tma_load_4d(xdst + h * (XS_BYTES / 4) + b * (BC * 16 * p.N), &p.tmx, &x_full[xs], 0,
                                                live ? 2 * tw - 1 : -8, live ? 2 * th - 1 : -8, cb * BC);
                                }
                        }
                    } else if constexpr (XM == 2) {
                        if (lane == 0) {
                            mbar_arrive_expect_tx(&x_full[xs], G::X_SLOT);
#pragma unroll
                            for (int h = 0; h < NH; ++h) {
                                if (cb + X_PREFETCH < hi)
                                    tma_prefetch_l2_4d(&p.tmx, tma_n0[h], tma_w0[h], tma_h0[h], (cb + X_PREFETCH) * BC);
                                tma_load_4d(xdst + h * (XS_BYTES / 4), &p.tmx, &x_full[xs], tma_n0[h], tma_w0[h],
                                            tma_h0[h], cb * BC);
                            }
                        }
                    } else {
                        constexpr int VX = XM == 1 ? 4 : 1;
                        constexpr int PER_C = 16 * BN / VX;  // vectors per (half, channel)
                        for (int e = lane; e < NH * BC * PER_C; e += 32) {
                            const int hh = e / (BC * PER_C), r0 = e % (BC * PER_C);
                            const int cl = r0 / PER_C, r = (r0 % PER_C) * VX;
                            const int c = cb * BC + cl;
                            const int off = xtab[hh * 16 * BN + r];
                            const bool ok = (c < p.C) && (off >= 0);
                            const float* src = ok ? p.x + (size_t)c * HWN + off : p.x;
                            const uint32_t dst = smem_u32(xdst + hh * (XS_BYTES / 4) + cl * 16 * BN + r);
                            if constexpr (VX == 4) cp_async16(dst, src, ok);
                            else cp_async4(dst, src, ok);
                        }
                        cp_async_wait_all();
                        mbar_arrive(&x_full[xs]);  // every lane: its own copies have landed
                    }
                }
            }
        } else if (warp == PROD_WARP) {
            // ------------------------ transformed-filter producer -----------------
            int unit = 0;
            Segs<SK> segs(p);
            int tile, lo, hi;
            while (segs.next(p, tile, lo, hi)) {
                const int kb = tile % p.num_kb;
                for (int cb = lo; cb < hi; ++cb) {
                    for (int h = 0; h < G::UNITS_PER_CB; ++h, ++unit) {
                        const int us = unit % G::U_SLOTS;
                        if (unit >= G::U_SLOTS) mbar_wait(&u_empty[us], ((unit / G::U_SLOTS) - 1) & 1);
                        if (lane == 0) {
                            const float* src =
                                p.u_tc + ((((size_t)cb * p.num_kb + kb) * 16 + h * G::XPU) * P) * (MM * BC);
                            mbar_arrive_expect_tx(&u_full[us], G::UNIT);
                            bulk_load(su + us * G::UNIT, src, G::UNIT, &u_full[us]);
                        }
                    }
                }
            }
        } else if (warp == MMA_WARP) {
            // ------------------------------ MMA issuer ----------------------------
            constexpr uint32_t IDESC = umma_idesc_tf32(MM, BN);
            int unit = 0, gcb = 0, it = 0;
            Segs<SK> segs(p);
            int tile, lo, hi;
            for (; segs.next(p, tile, lo, hi); ++it) {
                if (it > 0) mbar_wait(acc_empty, (it - 1) & 1);  // epilogue drained TMEM
                tc_fence_after();
                for (int cb = lo; cb < hi; ++cb, ++gcb) {
                    const int vs = gcb & 1;
                    mbar_wait(&v_full[vs], (gcb >> 1) & 1);
                    for (int half = 0; half < G::UNITS_PER_CB; ++half, ++unit) {
                        const int us = unit % G::U_SLOTS;
                        mbar_wait(&u_full[us], (unit / G::U_SLOTS) & 1);
                        tc_fence_after();
                        if (lane == 0) {
                            const uint32_t ubase = smem_u32(su + us * G::UNIT);
                            const uint32_t vbase = smem_u32(sv + vs * G::V_SLOT);
#pragma unroll
                            for (int q = 0; q < G::XPU; ++q) {
                                const int xi = half * G::XPU + q;
                                const uint32_t a0 = ubase + (q * P) * G::A_TILE;
                                const uint64_t ab = umma_desc(a0, 128, 256);
#pragma unroll
                                for (int h = 0; h < NH; ++h) {
                                    // nu-half h accumulates in TMEM lanes 16h.. of each quadrant (MM = 64)
                                    const uint32_t d = tmem + xi * BN + ((uint32_t)(16 * h) << 16);
                                    const uint32_t b0 = vbase + ((xi * NH + h) * P) * B_TILE;
                                    const uint64_t bb = umma_desc(b0, 128, 256);
                                    umma_tf32(d, ab, bb, IDESC, cb > lo ? 1u : 0u);
                                    if constexpr (P == 2) {
                                        const uint64_t as = umma_desc(a0 + G::A_TILE, 128, 256);
                                        const uint64_t bs = umma_desc(b0 + B_TILE, 128, 256);
                                        umma_tf32(d, ab, bs, IDESC, 1u);
                                        umma_tf32(d, as, bb, IDESC, 1u);
                                    }
                                }
                            }
                            umma_commit(&u_empty[us]);
                            if (half == G::UNITS_PER_CB - 1) umma_commit(&v_empty[vs]);
                        }
                        __syncwarp();
                    }
                }
                if (lane == 0) umma_commit(acc_full);
                __syncwarp();
            }
        }
    } else if (warp >= ITF_WARP0) {
        setmaxnreg_dec<REG_ITF>();
        // ------------------------------ ITF warps -----------------------------
        // lane = nu of the half; warp iw: channels 4 (iw & 1) .. +3; MM = 128: warp pair iw >> 1
        // takes the channel blocks of its parity; MM = 64: warp pair iw >> 1 = nu-half
        const int iw = warp - ITF_WARP0;
        const int grp = NH == 1 ? (iw >> 1) : 0;
        const int hh = NH == 1 ? 0 : (iw >> 1);
        const int cq = iw & 1;
        const int nl = lane;
        // K-major core-matrix row of (nu, channels 4cq..4cq+3): [nu/8][c/4][nu%8][c%4]
        const uint32_t voff = (nl >> 3) * 256 + cq * 128 + (nl & 7) * 16;
        // raw x of (4cq, nl): [c][pos][n32] (XM != 3) or [box][c][pos][n:N] (XM == 3)
        const int xnb = XM == 3 ? p.N : BN;
        const int xoff = (nl / xnb) * (BC * 16 * xnb) + 4 * cq * 16 * xnb + nl % xnb;
        int gcb = 0;
        Segs<SK> segs(p);
        int tile, lo, hi;
        while (segs.next(p, tile, lo, hi)) {
            for (int cb = lo; cb < hi; ++cb, ++gcb) {
                if (NH == 1 && (gcb & 1) != grp) continue;
                const int xs = gcb % G::X_SLOTS, vs = gcb & 1;
                mbar_wait(&x_full[xs], (gcb / G::X_SLOTS) & 1);
                const float* xsrc = sx + xs * (G::X_SLOT / 4) + hh * (XS_BYTES / 4) + xoff;
                float t[4][16];
#pragma unroll
                for (int c = 0; c < 4; ++c) {
                    float d[16];
#pragma unroll
                    for (int e = 0; e < 16; ++e) d[e] = xsrc[(c * 16 + e) * xnb];
                    itf_4x4(d, t[c]);
                }
                // generic-proxy reads of a TMA-filled slot -> fence.proxy.async before releasing it: the
                // next TMA write (async proxy) is otherwise not ordered after them
                fence_proxy_async_smem();
                mbar_arrive(&x_empty[xs]);  // this lane's reads of the x slot are done
                if (gcb >= 2) mbar_wait(&v_empty[vs], ((gcb >> 1) - 1) & 1);
                uint8_t* vdst = sv + vs * G::V_SLOT + voff;
#pragma unroll
                for (int xi = 0; xi < 16; ++xi) {
                    const float b0 = to_tf32(t[0][xi]), b1 = to_tf32(t[1][xi]);
                    const float b2 = to_tf32(t[2][xi]), b3 = to_tf32(t[3][xi]);
                    uint8_t* dst = vdst + ((xi * NH + hh) * P) * B_TILE;
                    *reinterpret_cast<float4*>(dst) = make_float4(b0, b1, b2, b3);
                    if constexpr (P == 2)
                        *reinterpret_cast<float4*>(dst + B_TILE) =
                            make_float4(to_tf32(t[0][xi] - b0), to_tf32(t[1][xi] - b1), to_tf32(t[2][xi] - b2),
                                        to_tf32(t[3][xi] - b3));
                }
                fence_proxy_async_smem();  // generic smem writes -> visible to the tensor core (async proxy)
                mbar_arrive(&v_full[vs]);
            }
        }
    } else {
        setmaxnreg_inc<REG_EPI>();
        // ------------------------------ epilogue ------------------------------
        // thread = TMEM lane = filter k of the tile; nu 16 eh .. 16 eh + 15 of each accumulator
        // MM = 128: lane = filter; MM = 64: lanes 0-15 -> filters of nu-half 0, 16-31 -> nu-half 1
        constexpr int EN = BN / 2;  // nu per thread
        const int qd = warp & 3, eh = warp >> 2;
        const int kl = (MM == 128) ? qd * 32 + lane : qd * 16 + (lane & 15);
        const int hsel = (MM == 128) ? 0 : (lane >> 4);
        const uint32_t trow = tmem + ((uint32_t)(qd * 32) << 16) + eh * EN;
        const size_t dW = (size_t)p.W * p.N;
        int it = 0;
        Segs<SK> segs(p);
        int tile, lo, hi;
        for (; segs.next(p, tile, lo, hi); ++it) {
            const int k = (tile % p.num_kb) * MM + kl;
            const int nu0 = (tile / p.num_kb) * TN + hsel * BN + eh * EN;
            mbar_wait(acc_full, it & 1);
            tc_fence_after();
            float o[EN][4];  // OTF results of this filter for its 16 nu
#pragma unroll
            for (int ch = 0; ch < EN / 4; ++ch) {
                float m[16][4];
#pragma unroll
                for (int xi = 0; xi < 16; ++xi) tmem_ld4(trow + xi * BN + ch * 4, m[xi]);
                tmem_ld_wait();
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    float mm[16];
#pragma unroll
                    for (int xi = 0; xi < 16; ++xi) mm[xi] = m[xi][j];
                    otf_2x2(mm, o[ch * 4 + j]);
                }
            }
            tc_fence_before();
            mbar_arrive(acc_empty);  // TMEM free for the next tile's MMAs (after this lane's loads)
            if (SK && hi - lo != p.num_cb) {
                // piece of a cut tile: partial outputs -> slot 2b (the CTA's first piece) or 2b + 1
                // (its last), [kl][output][nu of the tile]; tc_fixup_kernel adds them
                float* wk = p.sk_ws + ((size_t)(2 * blockIdx.x + (segs.n > 1 ? 1 : 0)) * MM + kl) * (4 * TN) +
                            hsel * BN + eh * EN;
#pragma unroll
                for (int q = 0; q < 4; ++q)
#pragma unroll
                    for (int j = 0; j < EN; j += 4)
                        *reinterpret_cast<float4*>(wk + q * TN + j) =
                            make_float4(o[j][q], o[j + 1][q], o[j + 2][q], o[j + 3][q]);
                continue;
            }
            if (k >= p.K || nu0 >= p.NV) continue;
            if constexpr (XM == 2) {
                // N % 32 == 0: the 32 nu of a half are 32 consecutive n of one image tile -> 64 B per thread
                const int t = nu0 / p.N, n = nu0 - t * p.N;
                const int th = t / p.TW, tw = t - th * p.TW;
                const int i0 = 2 * th, j0 = 2 * tw;
                float* yk = p.y + (size_t)k * HWN + ((size_t)i0 * p.W + j0) * p.N + n;
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int a = q >> 1, b = q & 1;
                    if (i0 + a >= p.H || j0 + b >= p.W) continue;  // odd H/W (L1155)
                    float* dst = yk + a * dW + b * p.N;
#pragma unroll
                    for (int j = 0; j < EN; j += 4)
                        *reinterpret_cast<float4*>(dst + j) = make_float4(o[j][q], o[j + 1][q], o[j + 2][q], o[j + 3][q]);
                }
            } else if constexpr (XM == 3) {
                // N | 32, N % 4 == 0: every group of 4 nu is 4 consecutive n of one image tile
#pragma unroll
                for (int j = 0; j < EN; j += 4) {
                    const int nu = nu0 + j;
                    if (nu >= p.NV) break;
                    const int t = nu / p.N, n = nu - t * p.N;
                    const int th = t / p.TW, tw = t - th * p.TW;
                    const int i0 = 2 * th, j0 = 2 * tw;
                    float* yk = p.y + (size_t)k * HWN + ((size_t)i0 * p.W + j0) * p.N + n;
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const int a = q >> 1, b = q & 1;
                        if (i0 + a >= p.H || j0 + b >= p.W) continue;  // odd H/W (L1155)
                        *reinterpret_cast<float4*>(yk + a * dW + b * p.N) =
                            make_float4(o[j][q], o[j + 1][q], o[j + 2][q], o[j + 3][q]);
                    }
                }
            } else {
#pragma unroll
                for (int j = 0; j < EN; ++j) {
                    const int nu = nu0 + j;
                    if (nu >= p.NV) break;
                    const int t = nu / p.N, n = nu - t * p.N;
                    const int th = t / p.TW, tw = t - th * p.TW;
                    const int i0 = 2 * th, j0 = 2 * tw;
                    float* yk = p.y + (size_t)k * HWN + ((size_t)i0 * p.W + j0) * p.N + n;
                    yk[0] = o[j][0];
                    if (j0 + 1 < p.W) yk[p.N] = o[j][1];
                    if (i0 + 1 < p.H) yk[dW] = o[j][2];
                    if (i0 + 1 < p.H && j0 + 1 < p.W) yk[dW + p.N] = o[j][3];
                }
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tmem_dealloc(tmem, 512);
}

// Stream-K fixup (as tc16_fixup_kernel): blocks 16i .. 16i+15 handle the tile cut by the range
// boundary of CTA i + 1 when it is the first boundary inside that tile; y = sum of the pieces'
// partials in CTA order.
constexpr int FIX_PARTS = 16;
template <int MM>
__global__ void __launch_bounds__(256) tc_fixup_kernel(const __grid_constant__ Params p, int G) {
    constexpr int TN = BN * (128 / MM);
    constexpr int PER = MM * TN / FIX_PARTS / 256;
    __shared__ int slots[256];
    __shared__ int nseg;
    const int b = blockIdx.x / FIX_PARTS + 1, part = blockIdx.x % FIX_PARTS;
    const int ub = sk_start(p, b);
    const int tile = ub / p.num_cb;
    const int t0 = tile * p.num_cb, t1 = t0 + p.num_cb;
    if (ub == t0 || sk_start(p, b - 1) > t0) return;
    if (threadIdx.x == 0) {
        int b0 = b - 1;
        while (b0 > 0 && sk_start(p, b0) > t0) --b0;
        int ns = 0, c0 = sk_start(p, b0);
        for (int c = b0; c < G && c0 < t1 && ns < 256; ++c) {
            const int c1 = sk_start(p, c + 1);
            if (c1 > c0) slots[ns++] = 2 * c + (c0 < t0 ? 1 : 0);
            c0 = c1;
        }
        nseg = ns;
    }
    __syncthreads();
    const int ns = nseg;
    const int kb = tile % p.num_kb, nb = tile / p.num_kb;
    const size_t HWN = (size_t)p.H * p.W * p.N, dW = (size_t)p.W * p.N;
    constexpr size_t SLOT = (size_t)MM * 4 * TN;
    float o[PER][4];
#pragma unroll
    for (int i = 0; i < PER; ++i)
#pragma unroll
        for (int q = 0; q < 4; ++q) o[i][q] = 0.f;
    for (int sidx = 0; sidx < ns; ++sidx) {
        const float* wk = p.sk_ws + slots[sidx] * SLOT;
        float v[PER][4];
#pragma unroll
        for (int i = 0; i < PER; ++i) {
            const int e = (part * PER + i) * 256 + threadIdx.x, kl = e / TN, j = e - kl * TN;
#pragma unroll
            for (int q = 0; q < 4; ++q) v[i][q] = wk[((size_t)kl * 4 + q) * TN + j];
        }
#pragma unroll
        for (int i = 0; i < PER; ++i)
#pragma unroll
            for (int q = 0; q < 4; ++q) o[i][q] += v[i][q];
    }
#pragma unroll
    for (int i = 0; i < PER; ++i) {
        const int e = (part * PER + i) * 256 + threadIdx.x, kl = e / TN, j = e - kl * TN;
        const int k = kb * MM + kl, nu = nb * TN + j;
        if (k >= p.K || nu >= p.NV) continue;
        const int t = nu / p.N, n = nu - t * p.N;
        const int th = t / p.TW, tw = t - th * p.TW;
        const int i0 = 2 * th, j0 = 2 * tw;
        float* yk = p.y + (size_t)k * HWN + ((size_t)i0 * p.W + j0) * p.N + n;
        yk[0] = o[i][0];
        if (j0 + 1 < p.W) yk[p.N] = o[i][1];
        if (i0 + 1 < p.H) yk[dW] = o[i][2];
        if (i0 + 1 < p.H && j0 + 1 < p.W) yk[dW + p.N] = o[i][3];
    }
}

}  // namespace tc
}  // namespace wino
