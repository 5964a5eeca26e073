// fused_tc16.cuh -- NEXT row N4: fused Winograd F(2x2,3x3) with FP16 or BF16
// operands on tcgen05 tensor cores (kind::f16, FP32 accumulators in TMEM).
//
// Paper: "The implementation can be ported to the fp16 version by increasing bn
// to 64.  To further increase the throughput with newly introduced tensor core,
// the data layout needs a redesign" (Sec. 8.3).  Same method (Eq. 5-8,
// L191-207); x, w, y are stored in the 16-bit type, the transforms and the
// accumulation run in FP32, the Winograd-domain operands U, V and the output y
// are rounded to the 16-bit type (round-to-nearest-even; reading R18).
//
// Tile: 128 filters (UMMA M) x 32 nu (UMMA N) x all 16 xi, channel blocks of 16
// (one UMMA K step per xi).  The 16-bit operands carry twice the channels of the
// TF32 kernel (fused_tc.cuh) in the same shared-memory bytes, so the per-block
// operand traffic that bounds that kernel (Sec. 7.3 of DESIGN.md) buys twice the
// Winograd-domain work here.
// Warp roles (persistent, one CTA per SM, 512 threads):
//   * warps 0-3   epilogue: tcgen05.ld of the 16 accumulators, OTF (Eq. 8) in
//                 FP32 registers, TMEM released, 16-bit stores of y;
//   * warps 4-7 / 8-11  two ITF groups taking alternate channel blocks: each
//                 thread transforms 2 channels x 2 nu (V = B^T d B, Eq. 6, FP32)
//                 and stores c-pairs of V as 32-bit words of the K-major B operand;
//   * warp 12     bulk copy of the pre-arranged 16-bit U (64 KB per block);
//   * warp 13     one thread issues tcgen05.mma.kind::f16 per xi;
//   * warp 14     TMA of raw x (n:32, w:4, h:4, c:16), zero fill = padding (Sec. 3.5).
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include <cstdint>

#include "wino_ptx.cuh"
#include "wino_transforms.cuh"

namespace wino {
namespace tc16 {

#ifdef WINO_TC16_TRACE
// Debug-only event trace (CTA 0): [event][gcb] = clock64 at the event.
constexpr int TRACE_EVENTS = 8, TRACE_CB = 256;
__device__ unsigned long long g_trace16[TRACE_EVENTS * TRACE_CB];
#define TC16_TRACE(ev, cb)                                                                          \
    do {                                                                                           \
        if (blockIdx.x == 0 && (cb) < TRACE_CB) g_trace16[(ev) * TRACE_CB + (cb)] = clock64();     \
    } while (0)
#else
#define TC16_TRACE(ev, cb) \
    do {                   \
    } while (0)
#endif

constexpr int BN = 32;    // nu per UMMA (N); a tile has NH = 128 / MM such halves
constexpr int BC = 16;    // channels per block (UMMA K of kind::f16)
constexpr int EPI_WARPS = 4, ITF_WARP0 = 4, ITF_WARPS = 8, ITF_GROUP = 4;
constexpr int PROD_WARP = 12, MMA_WARP = 13, XPROD_WARP = 14;
constexpr int NT = 512;
constexpr int REG_EPI = 216, REG_ITF = 112, REG_PROD = 56;  // 128*216 + 256*112 + 128*56 = 63488
constexpr int V_SBO = 256;                // 8-row group stride of the V operand
constexpr int B_TILE = (BN / 8) * V_SBO;  // one (xi, nu-half) of V: 1 KB, [nu/8][c/8 (LBO 128)][nu%8][c%8]
constexpr int XS_BYTES = BC * 16 * BN * 2;  // raw x of one block and nu-half: 16 KB, [c][pos][nu]

// Per tile height MM (filters = UMMA M):
//  * MM = 128: tile 128 k x 32 nu; the two ITF groups take alternate channel blocks; x slot =
//    gcb % 4 (each group owns two slots and consumes them in order, so an mbarrier phase
//    parity never aliases a fill that has not landed while the groups drift apart).
//  * MM = 64: tile 64 k x 64 nu (two nu-halves; their M = 64 accumulators interleave in TMEM
//    lanes 0-15 / 16-31 of each quadrant, scripts/microbench/umma_m64.cu); ITF group g
//    transforms nu-half g of every channel block.  Half the filter bytes per (k, nu) pair.
template <int MM>
struct Cfg {
    static constexpr int NH = 128 / MM;
    static constexpr int TN = BN * NH;
    static constexpr int A_TILE = MM * BC * 2;  // one xi of U, [m/8][c/8][m%8][c%8]
    static constexpr int UNIT = 16 * A_TILE;    // one channel block of U: 64 / 32 KB
    static constexpr int U_SLOTS = NH == 1 ? 2 : 3;
    static constexpr int X_SLOTS = NH == 1 ? 4 : 2;
    static constexpr int V_SLOTS = 2;
    static constexpr int X_SLOT = NH * XS_BYTES;
    static constexpr int V_SLOT = 16 * NH * B_TILE;
    static constexpr int ITF_PER_X = NH == 1 ? ITF_GROUP : ITF_WARPS;  // warps consuming one x / V slot
    static constexpr int OFF_U = 0;
    static constexpr int OFF_X = OFF_U + U_SLOTS * UNIT;
    static constexpr int OFF_V = OFF_X + X_SLOTS * X_SLOT;
    static constexpr int OFF_BAR = OFF_V + V_SLOTS * V_SLOT;
    static constexpr int NBAR = 2 * U_SLOTS + 2 * X_SLOTS + 2 * V_SLOTS + 2;
    static constexpr int OFF_TMEM = OFF_BAR + NBAR * 8;
    static constexpr int BYTES = OFF_TMEM + 16;
    static_assert(BYTES <= 232448, "shared memory budget");
};

// Tile height of a shape (the filter transform and the conv must agree).
__host__ __device__ inline int tc16_mm(int K) {
#if defined(WINO_TC16_MM)
    return WINO_TC16_MM;  // A/B builds
#else
    return K <= 64 ? 64 : 128;
#endif
}
// u_h layout (written by tc16_filter_kernel, read with bulk copies):
//   [cb = ceil(C/16)][kb = ceil(K/MM)][xi 16][m/8][c/8 2][m%8 8][c%8 8]  16-bit
// i.e. per (cb, kb, xi) one K-major SWIZZLE_NONE UMMA A tile (LBO 128 B, SBO 256 B).
__host__ __device__ inline size_t u_h_elems(int C, int K) {
    const int mm = tc16_mm(K);
    return size_t((C + BC - 1) / BC) * ((K + mm - 1) / mm) * 16 * (mm * BC);
}

// 16-bit type helpers: DT 0 = IEEE fp16, 1 = bf16.
template <int DT>
__device__ __forceinline__ float2 unpack2(uint32_t w) {
    if constexpr (DT == 0) {
        __half2 h = *reinterpret_cast<__half2*>(&w);
        return __half22float2(h);
    } else {
        return make_float2(__uint_as_float(w << 16), __uint_as_float(w & 0xffff0000u));
    }
}
template <int DT>
__device__ __forceinline__ uint32_t pack2(float lo, float hi) {  // round-to-nearest-even
    if constexpr (DT == 0) {
        __half2 h = __floats2half2_rn(lo, hi);
        return *reinterpret_cast<uint32_t*>(&h);
    } else {
        __nv_bfloat162 h = __floats2bfloat162_rn(lo, hi);
        return *reinterpret_cast<uint32_t*>(&h);
    }
}
template <int DT>
__device__ __forceinline__ float to_f(uint16_t v) {
    if constexpr (DT == 0) return __half2float(__ushort_as_half(v));
    else return __uint_as_float(uint32_t(v) << 16);
}
template <int DT>
__device__ __forceinline__ uint16_t from_f(float v) {
    if constexpr (DT == 0) return __half_as_ushort(__float2half_rn(v));
    else return __bfloat16_as_ushort(__float2bfloat16_rn(v));
}

// D f32, A/B fp16 (0) or bf16 (1), both K-major.
__host__ __device__ constexpr uint32_t umma_idesc_f16(int dt, int M, int N) {
    return (1u << 4) | (uint32_t(dt) << 7) | (uint32_t(dt) << 10) | (uint32_t(N >> 3) << 17) |
           (uint32_t(M >> 4) << 24);
}
__device__ __forceinline__ void umma_f16(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(d_tmem),
        "l"(a), "l"(b), "r"(idesc), "r"(acc)
        : "memory");
}

// FTF (Eq. 5) from 16-bit w (C,3,3,K) in FP32, rounded to the 16-bit type, straight into the
// operand layout above.  Block = 8 channels x 32 filters, one (c, k) per thread (9 coalesced
// loads along k); the 16 results go through shared memory so that every store is a 16 B
// core-matrix row (8 channels of one filter), consecutive filters consecutive rows.
// Grid (ceil(Kp/32), ceil(C/16)*2).  Pads C and K with zeros.
template <int DT, int MM>
__global__ void __launch_bounds__(256) tc16_filter_kernel(const uint16_t* __restrict__ w, uint16_t* __restrict__ u,
                                                          int C, int K) {
    __shared__ __align__(16) uint16_t st[16][32][8];  // [xi][k][c]
    const int kl = threadIdx.x & 31, cl = threadIdx.x >> 5;
    const int k = blockIdx.x * 32 + kl, c8 = blockIdx.y, c = c8 * 8 + cl;
    float t[16];
    if (c < C && k < K) {
        float g[9];
        const uint16_t* wc = w + (size_t)c * 9 * K + k;
#pragma unroll
        for (int e = 0; e < 9; ++e) g[e] = to_f<DT>(wc[(size_t)e * K]);
        ftf_4x4(g, t);
    } else {
#pragma unroll
        for (int e = 0; e < 16; ++e) t[e] = 0.f;
    }
#pragma unroll
    for (int xi = 0; xi < 16; ++xi) st[xi][kl][cl] = from_f<DT>(t[xi]);
    __syncthreads();
    const int Kp = ((K + MM - 1) / MM) * MM, nkb = Kp / MM;
    const int cb = c8 / (BC / 8), ch = c8 % (BC / 8);
#pragma unroll
    for (int r = 0; r < 2; ++r) {  // 16 xi x 32 rows = 512 rows of 16 B, 2 per thread
        const int row = r * 256 + threadIdx.x, xi = row >> 5, rk = row & 31;
        const int kk = blockIdx.x * 32 + rk;
        if (kk >= Kp) continue;
        const int kb = kk / MM, m = kk % MM;
        const size_t base = (((size_t)cb * nkb + kb) * 16 + xi) * (MM * BC);
        *reinterpret_cast<uint4*>(u + base + (m >> 3) * 128 + ch * 64 + (m & 7) * 8) =
            *reinterpret_cast<const uint4*>(&st[xi][rk][0]);
    }
}

struct __align__(64) Params {
    CUtensorMap tmx;  // x (C,H,W,N) 16-bit as (N, W, H, C), box (32 or N, 4, 4, 16)   [TMA paths]
    const uint16_t* __restrict__ x;
    const uint16_t* __restrict__ u;
    uint16_t* __restrict__ y;
    int N, C, H, W, K;
    int TW, NV;
    int num_kb, num_cb, num_tiles;
    // stream-K (SK = true): units = tile * num_cb + cb; CTA b takes [b*q + min(b, r), ...); pieces
    // of cut tiles leave FP32 partial outputs in sk_ws (2 slots of MM x 4 x TN floats per CTA)
    float* __restrict__ sk_ws;
    int sk_q, sk_r;
};

__host__ __device__ __forceinline__ int sk_start(const Params& p, int b) { return b * p.sk_q + min(b, p.sk_r); }

// The (tile, channel-block range) pieces a CTA processes, identical in every warp role:
// persistent tiles blockIdx.x, +gridDim.x, ... (whole tiles), or the CTA's stream-K range.
template <bool SK>
struct Segs {
    int a, b, n = 0;  // cursor, end (SK) / stride; pieces handed out so far
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

// XM: 2 = one TMA box per nu-half (N % 32 == 0), 3 = 32/N boxes per half (N in {8, 16}),
// 0 = generic gather by the x-producer warp (a 16-bit box needs >= 8 images: 16 B rows)
template <int DT, int XM, int MM, bool SK = false>
__global__ void __launch_bounds__(NT, 1) fused_tc16_kernel(const __grid_constant__ Params p) {
    using G = Cfg<MM>;
    constexpr int NH = G::NH, TN = G::TN;
    constexpr int U_SLOTS = G::U_SLOTS, X_SLOTS = G::X_SLOTS, V_SLOTS = G::V_SLOTS;
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t* const su = smem + G::OFF_U;
    uint8_t* const sx = smem + G::OFF_X;
    uint8_t* const sv = smem + G::OFF_V;
    uint64_t* const bars = reinterpret_cast<uint64_t*>(smem + G::OFF_BAR);
    uint64_t* const u_full = bars;
    uint64_t* const u_empty = bars + U_SLOTS;
    uint64_t* const x_full = bars + 2 * U_SLOTS;
    uint64_t* const x_empty = x_full + X_SLOTS;
    uint64_t* const v_full = x_empty + X_SLOTS;
    uint64_t* const v_empty = v_full + V_SLOTS;
    uint64_t* const acc_full = v_empty + V_SLOTS;
    uint64_t* const acc_empty = acc_full + 1;
    uint32_t* const tmem_slot = reinterpret_cast<uint32_t*>(smem + G::OFF_TMEM);

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

    if (tid == 0) {
        for (int s = 0; s < U_SLOTS; ++s) {
            mbar_init(&u_full[s], 1);
            mbar_init(&u_empty[s], 1);
        }
        for (int s = 0; s < X_SLOTS; ++s) {
            mbar_init(&x_full[s], XM == 0 ? 32 : 1);  // gather: every lane releases its own stores
            mbar_init(&x_empty[s], G::ITF_PER_X);
        }
        for (int s = 0; s < V_SLOTS; ++s) {
            mbar_init(&v_full[s], G::ITF_PER_X);
            mbar_init(&v_empty[s], 1);
        }
        mbar_init(acc_full, 1);
        mbar_init(acc_empty, EPI_WARPS);
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
            int gcb = 0;
            Segs<SK> segs(p);
            int tile, lo, hi;
            while (segs.next(p, tile, lo, hi)) {
                const int nu0 = (tile / p.num_kb) * TN;
                int tn0[NH], tw0[NH], th0[NH];
                if constexpr (XM == 2) {
                    // N % 32 == 0: each nu-half = 32 consecutive n of one image tile
#pragma unroll
                    for (int h = 0; h < NH; ++h) {
                        const int nuh = nu0 + h * BN;
                        tn0[h] = 0;
                        tw0[h] = -8;  // half past NV -> all zeros
                        th0[h] = -8;
                        if (nuh < p.NV) {
                            const int t = nuh / p.N;
                            tn0[h] = nuh - t * p.N;
                            const int th = t / p.TW, tw = t - th * p.TW;
                            tw0[h] = 2 * tw - 1;  // -1: TMA zero fill = padding (Sec. 3.5)
                            th0[h] = 2 * th - 1;
                        }
                    }
                    if (lane == 0)
                        for (int cb = lo; cb < lo + 4 && cb < hi; ++cb)
#pragma unroll
                            for (int h = 0; h < NH; ++h) tma_prefetch_l2_4d(&p.tmx, tn0[h], tw0[h], th0[h], cb * BC);
                }
                for (int cb = lo; cb < hi; ++cb, ++gcb) {
                    const int xs = gcb % X_SLOTS;
                    if (gcb >= X_SLOTS) mbar_wait(&x_empty[xs], ((gcb / X_SLOTS) - 1) & 1);
                    uint8_t* xdst = sx + xs * G::X_SLOT;
                    if (lane == 0) TC16_TRACE(0, gcb);
                    if constexpr (XM == 2) {
                        if (lane == 0) {
                            mbar_arrive_expect_tx(&x_full[xs], G::X_SLOT);
#pragma unroll
                            for (int h = 0; h < NH; ++h) {
                                if (cb + 4 < hi) tma_prefetch_l2_4d(&p.tmx, tn0[h], tw0[h], th0[h], (cb + 4) * BC);
                                tma_load_4d(xdst + h * XS_BYTES, &p.tmx, &x_full[xs], tn0[h], tw0[h], th0[h], cb * BC);
                            }
                        }
                    } else if constexpr (XM == 3) {
                        if (lane == 0) {
                            mbar_arrive_expect_tx(&x_full[xs], G::X_SLOT);
                            const int nbox = TN / p.N, t0 = nu0 / p.N;
                            for (int b = 0; b < nbox; ++b) {
                                const int t = t0 + b;
                                const bool live = t * p.N < p.NV;
                                const int th = t / p.TW, tw = t - th * p.TW;
                                // [box][c][pos][n:N]; -8: tile past the end -> zeros
                                tma_load_4d(xdst + b * (BC * 16 * p.N * 2), &p.tmx, &x_full[xs], 0,
                                            live ? 2 * tw - 1 : -8, live ? 2 * th - 1 : -8, cb * BC);
                            }
                        }
                    } else {
                        // generic gather: lane = local nu of each half, layout [h][c][pos][nu]; the 16
                        // window offsets are computed once per half, then 16 independent loads per channel
#pragma unroll 1
                        for (int h = 0; h < NH; ++h) {
                            const int gnu = nu0 + h * BN + lane;
                            const bool glive = gnu < p.NV;
                            const int gt = glive ? gnu / p.N : 0, gn = glive ? gnu - gt * p.N : 0;
                            const int gh0 = 2 * (gt / p.TW) - 1, gw0 = 2 * (gt % p.TW) - 1;
                            int off[16];
#pragma unroll
                            for (int pos = 0; pos < 16; ++pos) {
                                const int hh = gh0 + (pos >> 2), ww = gw0 + (pos & 3);
                                off[pos] = (glive && hh >= 0 && hh < p.H && ww >= 0 && ww < p.W)
                                               ? (hh * p.W + ww) * p.N + gn
                                               : -1;
                            }
                            uint16_t* xd = reinterpret_cast<uint16_t*>(xdst + h * XS_BYTES) + lane;
#pragma unroll 1
                            for (int cl = 0; cl < BC; ++cl) {
                                const int c = cb * BC + cl;
                                const uint16_t* xc = p.x + (size_t)(c < p.C ? c : 0) * HWN;
                                uint16_t v[16];
#pragma unroll
                                for (int pos = 0; pos < 16; ++pos) v[pos] = (c < p.C && off[pos] >= 0) ? xc[off[pos]] : 0;
#pragma unroll
                                for (int pos = 0; pos < 16; ++pos) xd[(cl * 16 + pos) * BN] = v[pos];
                            }
                        }
                        mbar_arrive(&x_full[xs]);
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
                for (int cb = lo; cb < hi; ++cb, ++unit) {
                    const int us = unit % U_SLOTS;
                    if (unit >= U_SLOTS) mbar_wait(&u_empty[us], ((unit / U_SLOTS) - 1) & 1);
                    if (lane == 0) {
                        TC16_TRACE(1, unit);
                        const uint16_t* src = p.u + (((size_t)cb * p.num_kb + kb) * 16) * (MM * BC);
                        mbar_arrive_expect_tx(&u_full[us], G::UNIT);
                        bulk_load(su + us * G::UNIT, src, G::UNIT, &u_full[us]);
                    }
                }
            }
        } else if (warp == MMA_WARP) {
            // ------------------------------ MMA issuer ----------------------------
            constexpr uint32_t IDESC = umma_idesc_f16(DT, MM, BN);
            int unit = 0, gcb = 0, it = 0;
            Segs<SK> segs(p);
            int tile, lo, hi;
            for (; segs.next(p, tile, lo, hi); ++it) {
                if (it > 0) mbar_wait(acc_empty, (it - 1) & 1);  // epilogue drained TMEM
                tc_fence_after();
                for (int cb = lo; cb < hi; ++cb, ++gcb, ++unit) {
                    const int vs = gcb & 1, us = unit % U_SLOTS;
                    mbar_wait(&v_full[vs], (gcb >> 1) & 1);
                    if (lane == 0) TC16_TRACE(4, gcb);
                    mbar_wait(&u_full[us], (unit / U_SLOTS) & 1);
                    tc_fence_after();
                    if (lane == 0) {
                        TC16_TRACE(5, gcb);
                        const uint32_t ubase = smem_u32(su + us * G::UNIT);
                        const uint32_t vbase = smem_u32(sv + vs * G::V_SLOT);
#pragma unroll
                        for (int xi = 0; xi < 16; ++xi) {
                            const uint64_t ad = umma_desc(ubase + xi * G::A_TILE, 128, 256);
#pragma unroll
                            for (int h = 0; h < NH; ++h) {
                                // nu-half h accumulates in TMEM lanes 16h.. of each quadrant (MM = 64)
                                const uint64_t bd = umma_desc(vbase + (xi * NH + h) * B_TILE, 128, V_SBO);
                                umma_f16(tmem + xi * BN + ((uint32_t)(16 * h) << 16), ad, bd, IDESC,
                                         cb > lo ? 1u : 0u);
                            }
                        }
                        umma_commit(&u_empty[us]);
                        umma_commit(&v_empty[vs]);
                    }
                    __syncwarp();
                }
                if (lane == 0) umma_commit(acc_full);
                __syncwarp();
            }
        }
    } else if (warp >= ITF_WARP0) {
        setmaxnreg_dec<REG_ITF>();
        // ------------------------------ ITF warps -----------------------------
        // group g (warps 4-7 / 8-11): MM = 128 -> channel blocks gcb % 2 == g; MM = 64 -> nu-half g.
        // Thread -> channels (2cp, 2cp+1) x nu (2np, 2np+1) of its half.
        const int g = (warp - ITF_WARP0) / ITF_GROUP, gw = (warp - ITF_WARP0) % ITF_GROUP;
        const int hh = NH == 2 ? g : 0;
        const int cp = 2 * gw + (lane >> 4), np = lane & 15;
        // raw x word (nu pair) of channel c, window element pos:
        //   XM 0/2: [h][c][pos][nu32] -> word h*4096 + c*256 + pos*16 + np; lanes 16-31 read pos^1
        //           first (pos*16 words apart -> the two half-warps hit disjoint banks)
        //   XM 3:   [box][c][pos][n:N] -> word box*(BC*8N) + c*8N + pos*N/2 + (n/2)
        const int par = (XM == 3) ? 0 : (lane >> 4);
        int wbase, wc, wp;
        if constexpr (XM == 3) {
            const int nu = hh * BN + 2 * np, b = nu / p.N, n = nu - b * p.N;
            wbase = b * (BC * 8 * p.N) + (n >> 1);
            wc = 8 * p.N;
            wp = p.N >> 1;
        } else {
            wbase = hh * (XS_BYTES / 4) + np;
            wc = 256;
            wp = 16;
        }
        // V word (row nu, K pair cp) at byte (nu/8)*V_SBO + (cp/4)*128 + (nu%8)*16 + (cp%4)*4; lanes with
        // (np/4) odd store their nu+1 row first (2-way instead of 4-way bank conflicts)
        const int sw = (np >> 2) & 1;
        const uint32_t voff0 = hh * B_TILE + ((2 * np) >> 3) * V_SBO + (cp >> 2) * 128 + ((2 * np) & 7) * 16 + (cp & 3) * 4;
        int gcb = 0;
        Segs<SK> segs(p);
        int tile, lo, hi;
        while (segs.next(p, tile, lo, hi)) {
            for (int cb = lo; cb < hi; ++cb, ++gcb) {
                if (NH == 1 && (gcb & 1) != g) continue;
                const int xs = gcb % X_SLOTS, vs = gcb & 1;
                mbar_wait(&x_full[xs], (gcb / X_SLOTS) & 1);
                const uint32_t* xw = reinterpret_cast<const uint32_t*>(sx + xs * G::X_SLOT) + wbase;
                uint32_t r[2][16];
#pragma unroll
                for (int j = 0; j < 2; ++j) {
                    const uint32_t* xc = xw + (2 * cp + j) * wc;
#pragma unroll
                    for (int e = 0; e < 16; ++e) r[j][e] = xc[(e ^ par) * wp];
                }
                // V = B^T d B (Eq. 6) in FP32 for the 4 tiles, packed as c-pairs, BEFORE waiting
                // for the V slot (the transform overlaps the tensor cores' use of the slot)
                uint32_t vw[2][16];
#pragma unroll
                for (int i = 0; i < 2; ++i) {  // nu = 2np + i
                    float d0[16], d1[16], v0[16], v1[16];
#pragma unroll
                    for (int e = 0; e < 16; ++e) {
                        // the upper half-warp loaded pos e^1 into slot e
                        const uint32_t a0 = r[0][e], a1 = r[0][e ^ 1], b0 = r[1][e], b1 = r[1][e ^ 1];
                        const float2 a = unpack2<DT>(par ? a1 : a0), b = unpack2<DT>(par ? b1 : b0);
                        d0[e] = i ? a.y : a.x;
                        d1[e] = i ? b.y : b.x;
                    }
                    itf_4x4(d0, v0);
                    itf_4x4(d1, v1);
#pragma unroll
                    for (int xi = 0; xi < 16; ++xi) vw[i][xi] = pack2<DT>(v0[xi], v1[xi]);
                }
                // generic-proxy reads of a TMA-filled slot -> fence.proxy.async before releasing it: the
                // next TMA write (async proxy) is otherwise not ordered after them
                fence_proxy_async_smem();
                __syncwarp();
                if (lane == 0) mbar_arrive(&x_empty[xs]);  // the x slot can be refilled
                if (gcb >= 2) mbar_wait(&v_empty[vs], ((gcb >> 1) - 1) & 1);
                uint8_t* vdst = sv + vs * G::V_SLOT + voff0;
#pragma unroll
                for (int s = 0; s < 2; ++s)
#pragma unroll
                    for (int xi = 0; xi < 16; ++xi) {
                        const uint32_t val = sw ? vw[s ^ 1][xi] : vw[s][xi];
                        *reinterpret_cast<uint32_t*>(vdst + xi * NH * B_TILE + (s ^ sw) * 16) = val;
                    }
                fence_proxy_async_smem();  // generic smem writes -> visible to the tensor core (async proxy)
                __syncwarp();
                if (lane == 0) mbar_arrive(&v_full[vs]);
#ifdef WINO_TC16_TRACE
                if (lane == 0) TC16_TRACE(gw == 0 ? 2 : gw == 1 ? 3 : gw == 2 ? 6 : 7, gcb);  // v_full arrival per warp
#endif
            }
        }
    } else {
        setmaxnreg_inc<REG_EPI>();
        // ------------------------------ epilogue ------------------------------
        // MM = 128: TMEM lane = filter; MM = 64: lanes 0-15 -> filters of nu-half 0, 16-31 -> nu-half 1
        const int kl = (MM == 128) ? warp * 32 + lane : warp * 16 + (lane & 15);
        const int hsel = (MM == 128) ? 0 : (lane >> 4);
        const uint32_t trow = tmem + ((uint32_t)(warp * 32) << 16);
        const size_t dW = (size_t)p.W * p.N;
        int it = 0;
        Segs<SK> segs(p);
        int tile, lo, hi;
        for (; segs.next(p, tile, lo, hi); ++it) {
            const int k = (tile % p.num_kb) * MM + kl;
            const int nu0 = (tile / p.num_kb) * TN + hsel * BN;
            mbar_wait(acc_full, it & 1);
            tc_fence_after();
            float o[BN][4];
#pragma unroll
            for (int ch = 0; ch < BN / 4; ++ch) {
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
            __syncwarp();
            if (lane == 0) mbar_arrive(acc_empty);  // TMEM free for the next tile's MMAs
            if (SK && hi - lo != p.num_cb) {
                // piece of a cut tile: FP32 partial outputs -> slot 2b (the CTA's first piece) or
                // 2b + 1 (its last), [kl][output][nu of the tile]; tc16_fixup_kernel adds and rounds
                float* wk = p.sk_ws + ((size_t)(2 * blockIdx.x + (segs.n > 1 ? 1 : 0)) * MM + kl) * (4 * TN) + hsel * BN;
#pragma unroll
                for (int q = 0; q < 4; ++q)
#pragma unroll
                    for (int j = 0; j < BN; j += 4)
                        *reinterpret_cast<float4*>(wk + q * TN + j) =
                            make_float4(o[j][q], o[j + 1][q], o[j + 2][q], o[j + 3][q]);
                continue;
            }
            if (k >= p.K || nu0 >= p.NV) continue;
            if constexpr (XM == 2 || XM == 3) {
                // groups of 8 nu = 8 consecutive n of one image tile (N % 8 == 0) -> 16 B stores
#pragma unroll
                for (int j = 0; j < BN; j += 8) {
                    const int nu = nu0 + j;
                    if (nu >= p.NV) break;
                    const int t = nu / p.N, n = nu - t * p.N;
                    const int th = t / p.TW, tw = t - th * p.TW;
                    const int i0 = 2 * th, j0 = 2 * tw;
                    uint16_t* yk = p.y + (size_t)k * HWN + ((size_t)i0 * p.W + j0) * p.N + n;
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const int a = q >> 1, b = q & 1;
                        if (i0 + a >= p.H || j0 + b >= p.W) continue;  // odd H/W (L1155)
                        uint4 v;
                        v.x = pack2<DT>(o[j][q], o[j + 1][q]);
                        v.y = pack2<DT>(o[j + 2][q], o[j + 3][q]);
                        v.z = pack2<DT>(o[j + 4][q], o[j + 5][q]);
                        v.w = pack2<DT>(o[j + 6][q], o[j + 7][q]);
                        *reinterpret_cast<uint4*>(yk + a * dW + b * p.N) = v;
                    }
                }
            } else {
#pragma unroll
                for (int j = 0; j < BN; ++j) {
                    const int nu = nu0 + j;
                    if (nu >= p.NV) break;
                    const int t = nu / p.N, n = nu - t * p.N;
                    const int th = t / p.TW, tw = t - th * p.TW;
                    const int i0 = 2 * th, j0 = 2 * tw;
                    uint16_t* yk = p.y + (size_t)k * HWN + ((size_t)i0 * p.W + j0) * p.N + n;
                    yk[0] = from_f<DT>(o[j][0]);
                    if (j0 + 1 < p.W) yk[p.N] = from_f<DT>(o[j][1]);
                    if (i0 + 1 < p.H) yk[dW] = from_f<DT>(o[j][2]);
                    if (i0 + 1 < p.H && j0 + 1 < p.W) yk[dW + p.N] = from_f<DT>(o[j][3]);
                }
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tmem_dealloc(tmem, 512);
}

// Stream-K fixup: blocks 16i .. 16i+15 handle the tile cut by the range boundary of CTA b = i + 1
// (when it is the first boundary inside that tile), 1/16 of its MM x TN outputs each:
// y = RNE(sum of the pieces' FP32 partials in CTA order).  Each thread owns 4 (filter, nu)
// outputs and issues all their loads before adding (latency-bound otherwise).
constexpr int FIX_PARTS = 16;
template <int DT, int MM>
__global__ void __launch_bounds__(256) tc16_fixup_kernel(const __grid_constant__ Params p, int G) {
    constexpr int TN = Cfg<MM>::TN;
    constexpr int PER = MM * TN / FIX_PARTS / 256;  // outputs per thread (4)
    __shared__ int slots[256];
    __shared__ int nseg;
    const int b = blockIdx.x / FIX_PARTS + 1, part = blockIdx.x % FIX_PARTS;
    const int ub = sk_start(p, b);
    const int tile = ub / p.num_cb;
    const int t0 = tile * p.num_cb, t1 = t0 + p.num_cb;
    if (ub == t0 || sk_start(p, b - 1) > t0) return;  // no cut, or an earlier boundary owns it
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
    for (int sidx = 0; sidx < ns; ++sidx) {  // CTA order
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
        uint16_t* yk = p.y + (size_t)k * HWN + ((size_t)i0 * p.W + j0) * p.N + n;
        yk[0] = from_f<DT>(o[i][0]);
        if (j0 + 1 < p.W) yk[p.N] = from_f<DT>(o[i][1]);
        if (i0 + 1 < p.H) yk[dW] = from_f<DT>(o[i][2]);
        if (i0 + 1 < p.H && j0 + 1 < p.W) yk[dW + p.N] = from_f<DT>(o[i][3]);
    }
}

}  // namespace tc16
}  // namespace wino
