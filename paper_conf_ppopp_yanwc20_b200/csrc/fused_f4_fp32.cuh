// fused_f4_fp32.cuh -- NEXT row N1: fused Winograd F(4x4,3x3) forward convolution, FP32 FFMA.
//
// The paper limits itself to F(2x2,3x3) (L117) and expects "greater speedup in
// the future if the fused F(4x4,3x3) is well optimized" (Sec. 8.1);
// SURVEY 8(f) ranks it first among the next rows.  Same structure as the
// persistent warp-specialised F(2x2) kernel (fused_fp32_ws.cuh) with alpha = 6:
// 6x6 input windows at stride 4, 36 Winograd elements xi, 4x4 outputs per tile,
// 36 EWMM multiplications per 16 outputs (2.25 per output vs 4 for F(2x2) and 9
// for direct convolution).  Matrices: Lavin-Gray F(4x4,3x3) (points 0, +-1, +-2,
// inf), as pinned in oracle/exact.py.
//
//   * tile: 64 filters x 16 nu (16 consecutive n of one image tile, N % 16 == 0)
//     x 36 xi; stage = 4 channels (u box (k:64, xi:36, c:4), x box (n:16, w:6,
//     h:6, c:4), both TMA with out-of-bounds zero fill = implicit padding);
//   * 3 compute warpgroups (12 warps, 152 registers): warp w owns xi = 3w..3w+2,
//     each lane an 8 (k) x 4 (nu) block of each -> 96 accumulators;
//   * producer warpgroup (56 registers): warp 12 issues TMA, warps 13-14 run
//     the 6x6 input transform (two passes to stay within 56 registers);
//   * OTF through a 4-round epilogue buffer (16 filters per round).
// TMA path when N % 16 == 0 and K % 4 == 0.  Any other shape (the paper claims generality
// for every N, K, C, with peak speed only at the multiples, L1281) takes the generic path
// (GEN = true): the producer warp gathers the same [c][pos][nu] x stage with 4-byte
// cp.async from a per-tile table of window offsets (-1 = padding: zero fill, Sec. 3.5) and
// the [c][xi][k] u stage with 16-byte (K % 4 == 0) or 4-byte cp.async, every lane arriving on
// the stage barrier once its copies have landed (cp.async groups, one stage behind).
#pragma once
#include <cuda.h>

#include <cstdint>

#include "wino_ptx.cuh"

namespace wino {
namespace f4 {

constexpr int NXI = 36;
constexpr int BK = 64, BN = 16, BC = 4;
constexpr int NT = 512;
constexpr int COMPUTE_WARPS = 12, COMPUTE_THREADS = 384;
constexpr int S = 3, SV = 2;
constexpr int REG_COMPUTE = 152, REG_PRODUCER = 56;  // 384*152 + 128*56 = 65536
constexpr int ITF_WARPS = 2;                         // warps 13, 14 (warp 15 idle)
constexpr int US_FLOATS = BC * NXI * BK;             // [c][xi][k]    36 KB
constexpr int XS_FLOATS = BC * NXI * BN;             // [c][pos][nu]   9 KB
constexpr int STAGE_FLOATS = US_FLOATS + XS_FLOATS;
constexpr int VS_FLOATS = NXI * BC * BN;             // [xi][c][nu]    9 KB
constexpr int ER_KROWS = 16, ER_LD = BN + 4;
constexpr int ER_FLOATS = NXI * ER_KROWS * ER_LD;    // [xi][16 k][20]
constexpr int XTAB = NXI * BN;  // generic path: window offsets of a tile's 16 nu x 36 positions
struct Smem {
    static constexpr int ep_offset = (S * STAGE_FLOATS + SV * VS_FLOATS) * 4;
    static constexpr int tab_offset = ep_offset + ER_FLOATS * 4;
    static constexpr int bar_offset = tab_offset + XTAB * 4;
    static constexpr int bytes = bar_offset + (2 * S + 2 * SV) * 8;
    static_assert(bytes <= 232448, "shared memory budget");
};

// ---- F(4x4,3x3) transforms (compile-time matrices; zero terms fold away) ----
__device__ constexpr float kG4[6][3] = {{0.25f, 0, 0},
                                        {-1.0f / 6, -1.0f / 6, -1.0f / 6},
                                        {-1.0f / 6, 1.0f / 6, -1.0f / 6},
                                        {1.0f / 24, 1.0f / 12, 1.0f / 6},
                                        {1.0f / 24, -1.0f / 12, 1.0f / 6},
                                        {0, 0, 1}};

// u4 = G4 g G4^T, g row-major 3x3 -> u row-major 6x6 (xi = 6 r' + s')
__device__ __forceinline__ void ftf4(const float g[9], float u[36]) {
    float t[6][3];
#pragma unroll
    for (int a = 0; a < 6; ++a)
#pragma unroll
        for (int b = 0; b < 3; ++b) {
            float s = 0.f;
#pragma unroll
            for (int m = 0; m < 3; ++m)
                if (kG4[a][m] != 0.f) s = fmaf(kG4[a][m], g[m * 3 + b], s);
            t[a][b] = s;
        }
#pragma unroll
    for (int a = 0; a < 6; ++a)
#pragma unroll
        for (int b = 0; b < 6; ++b) {
            float s = 0.f;
#pragma unroll
            for (int m = 0; m < 3; ++m)
                if (kG4[b][m] != 0.f) s = fmaf(t[a][m], kG4[b][m], s);
            u[a * 6 + b] = s;
        }
}

// 6-vector transforms, factorised (12 and 10 flops instead of 22 and 18):
//   B4^T rows: (4,0,-5,0,1,0) (0,-4,-4,1,1,0) (0,4,-4,-1,1,0) (0,-2,-1,2,1,0) (0,2,-1,-2,1,0) (0,4,0,-5,0,1)
//   r1,r2 = (d4-4d2) +- (d3-4d1);  r3,r4 = (d4-d2) +- 2(d3-d1)
__device__ __forceinline__ void bt4_vec(const float d[6], float r[6]) {
    const float p = fmaf(-4.f, d[2], d[4]), q = fmaf(-4.f, d[1], d[3]);
    const float e = d[4] - d[2], f = d[3] - d[1];
    r[0] = fmaf(4.f, d[0], fmaf(-5.f, d[2], d[4]));
    r[1] = p + q;
    r[2] = p - q;
    r[3] = fmaf(2.f, f, e);
    r[4] = fmaf(-2.f, f, e);
    r[5] = fmaf(4.f, d[1], fmaf(-5.f, d[3], d[5]));
}
//   A4^T rows: (1,1,1,1,1,0) (0,1,-1,2,-2,0) (0,1,1,4,4,0) (0,1,-1,8,-8,1)
__device__ __forceinline__ void at4_vec(const float m[6], float r[4]) {
    const float s12 = m[1] + m[2], d12 = m[1] - m[2], s34 = m[3] + m[4], d34 = m[3] - m[4];
    r[0] = m[0] + s12 + s34;
    r[1] = fmaf(2.f, d34, d12);
    r[2] = fmaf(4.f, s34, s12);
    r[3] = fmaf(8.f, d34, d12) + m[5];
}

struct __align__(64) Params {
    CUtensorMap tmx;  // x (C,H,W,N) as 4-d (N, W, H, C), box (16, 6, 6, 4)
    CUtensorMap tmu;  // u4 (C,36,K) as 3-d (K, 36, C), box (64, 36, 4)
    float* __restrict__ y;
    const float* __restrict__ x;   // generic path: gathered with cp.async
    const float* __restrict__ u4;  // generic path
    int u_vec;                     // generic path: K % 4 == 0 -> 16-byte u copies
    int N, C, H, W, K;
    int TW;      // ceil(W/4)
    int NV;      // N * ceil(H/4) * ceil(W/4)
    int num_kb;  // ceil(K/64)
    int num_it;  // ceil(C/4)
    int num_tiles;
    // stream-K (SK = true; the scheme of fused_fp32_ws.cuh): units = tile * num_it + g, CTA b takes
    // [b*q + min(b, r), ...); pieces of cut tiles leave their 16 partial outputs per (k, nu) in
    // sk_ws: 2 slots of [64 k][16 outputs][16 nu] floats (64 KiB) per CTA
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
            tile = a / p.num_it;
            lo = a - tile * p.num_it;
            hi = min(p.num_it, lo + (b - a));
            a += hi - lo;
        } else {
            if (a >= p.num_tiles) return false;
            tile = a;
            lo = 0;
            hi = p.num_it;
            a += b;
        }
        ++n;
        return true;
    }
};

// FTF for F(4x4): u4 (C,6,6,K)
__global__ void __launch_bounds__(256) ftf4_kernel(const float* __restrict__ w, float* __restrict__ u, int C, int K) {
    const long idx = (long)blockIdx.x * 256 + threadIdx.x;
    if (idx >= (long)C * K) return;
    const int c = (int)(idx / K), k = (int)(idx - (long)c * K);
    float g[9], t[36];
#pragma unroll
    for (int e = 0; e < 9; ++e) g[e] = __ldg(w + ((size_t)c * 9 + e) * K + k);
    ftf4(g, t);
#pragma unroll
    for (int e = 0; e < 36; ++e) u[((size_t)c * 36 + e) * K + k] = t[e];
}

template <bool SK = false, bool GEN = false>
__global__ void __launch_bounds__(NT, 1) fused_f4_kernel(const __grid_constant__ Params p) {
    extern __shared__ __align__(1024) float smem[];
    float* const vs = smem + S * STAGE_FLOATS;
    float* const ep = reinterpret_cast<float*>(reinterpret_cast<char*>(smem) + Smem::ep_offset);
    int* const xtab = reinterpret_cast<int*>(reinterpret_cast<char*>(smem) + Smem::tab_offset);
    uint64_t* const full = reinterpret_cast<uint64_t*>(reinterpret_cast<char*>(smem) + Smem::bar_offset);
    uint64_t* const empty = full + S;
    uint64_t* const vfull = empty + S;
    uint64_t* const vempty = vfull + SV;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

    if (tid == 0) {
        if constexpr (!GEN) {
            tma_prefetch_desc(&p.tmx);
            tma_prefetch_desc(&p.tmu);
        }
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], GEN ? 32 : 1);
            mbar_init(&empty[s], COMPUTE_WARPS + ITF_WARPS);
        }
        for (int s = 0; s < SV; ++s) {
            mbar_init(&vfull[s], ITF_WARPS);
            mbar_init(&vempty[s], COMPUTE_WARPS);
        }
        fence_mbar_init();
    }
    __syncthreads();

    if (warp >= COMPUTE_WARPS) {
        setmaxnreg_dec<REG_PRODUCER>();
        if (warp == COMPUTE_WARPS && GEN) {
            // ------------------ generic gather (any N, K): all 32 lanes ------------------
            const size_t HWN = (size_t)p.H * p.W * p.N;
            int G = 0;
            Segs<SK> segs(p);
            int tile, lo, hi;
            while (segs.next(p, tile, lo, hi)) {
                const int k0 = (tile % p.num_kb) * BK, nu0 = (tile / p.num_kb) * BN;
                // window offset (h*W + w)*N + n of position pos of local nu (-1: padding / past NV);
                // only this warp reads the table, and it has issued every copy of the previous tile
                __syncwarp();
                for (int e = lane; e < XTAB; e += 32) {
                    const int pos = e / BN, nl = e % BN, nu = nu0 + nl;
                    int off = -1;
                    if (nu < p.NV) {
                        const int t = nu / p.N, n = nu - t * p.N;
                        const int th = t / p.TW, tw = t - th * p.TW;
                        const int h = 4 * th - 1 + pos / 6, w = 4 * tw - 1 + pos % 6;
                        if (h >= 0 && h < p.H && w >= 0 && w < p.W) off = (h * p.W + w) * p.N + n;
                    }
                    xtab[e] = off;
                }
                __syncwarp();
                for (int g = lo; g < hi; ++g, ++G) {
                    const int slot = G % S;
                    if (G >= S) mbar_wait(&empty[slot], ((G / S) - 1) & 1);
                    float* us = smem + slot * STAGE_FLOATS;
                    float* xs = us + US_FLOATS;
                    for (int e = lane; e < XS_FLOATS; e += 32) {  // [c][pos][nu]
                        const int c = g * BC + e / XTAB, off = xtab[e % XTAB];
                        const bool ok = c < p.C && off >= 0;
                        cp_async4(smem_u32(xs + e), ok ? p.x + (size_t)c * HWN + off : p.x, ok);
                    }
                    if (p.u_vec) {
                        for (int e = lane; e < US_FLOATS / 4; e += 32) {  // [c][xi][k], 4 k per copy
                            const int c = g * BC + e / (NXI * BK / 4), r = e % (NXI * BK / 4);
                            const int xi = r / (BK / 4), k = k0 + 4 * (r % (BK / 4));
                            const bool ok = c < p.C && k < p.K;
                            cp_async16(smem_u32(us + 4 * e), ok ? p.u4 + ((size_t)c * NXI + xi) * p.K + k : p.u4, ok);
                        }
                    } else {
                        for (int e = lane; e < US_FLOATS; e += 32) {
                            const int c = g * BC + e / (NXI * BK), r = e % (NXI * BK);
                            const int xi = r / BK, k = k0 + r % BK;
                            const bool ok = c < p.C && k < p.K;
                            cp_async4(smem_u32(us + e), ok ? p.u4 + ((size_t)c * NXI + xi) * p.K + k : p.u4, ok);
                        }
                    }
                    cp_async_commit();
                    if (G > 0) {  // the previous stage's copies (one group behind) have landed
                        cp_async_wait<1>();
                        mbar_arrive(&full[(G - 1) % S]);
                    }
                }
            }
            if (G > 0) {
                cp_async_wait<0>();
                mbar_arrive(&full[(G - 1) % S]);
            }
            return;
        }
        if (warp == COMPUTE_WARPS) {
            // ---------------------------- TMA issue ----------------------------
            if (lane == 0) {
                constexpr uint32_t kBytes = (US_FLOATS + XS_FLOATS) * 4;
                int G = 0;
                Segs<SK> segs(p);
                int tile, lo, hi;
                while (segs.next(p, tile, lo, hi)) {
                    const int k0 = (tile % p.num_kb) * BK, nu0 = (tile / p.num_kb) * BN;
                    const int t = nu0 / p.N, n0 = nu0 - t * p.N;
                    const int th = t / p.TW, tw = t - th * p.TW;
                    for (int g = lo; g < hi; ++g, ++G) {
                        const int slot = G % S;
                        if (G >= S) mbar_wait(&empty[slot], ((G / S) - 1) & 1);
                        float* us = smem + slot * STAGE_FLOATS;
                        mbar_arrive_expect_tx(&full[slot], kBytes);
                        tma_load_3d(us, &p.tmu, &full[slot], k0, 0, g * BC);
                        // window origin (4th-1, 4tw-1); -1 and past-the-end: TMA zero fill
                        tma_load_4d(us + US_FLOATS, &p.tmx, &full[slot], n0, 4 * tw - 1, 4 * th - 1, g * BC);
                    }
                }
            }
            return;
        }
        if (warp > COMPUTE_WARPS + ITF_WARPS) return;
        // ------------------- ITF: 6x6 input transform, 64 tiles / stage -------------------
        const int it_thr = tid - (COMPUTE_WARPS + 1) * 32;  // 0..63
        const int c = it_thr >> 4, nl = it_thr & 15;
        int G = 0;
        Segs<SK> segs(p);
        int tile, lo, hi;
        while (segs.next(p, tile, lo, hi)) {
            for (int g = lo; g < hi; ++g, ++G) {
                const int slot = G % S, vb = G % SV;
                mbar_wait(&full[slot], (G / S) & 1);
                if (G >= SV) mbar_wait(&vempty[vb], ((G / SV) - 1) & 1);
                const float* xs = smem + slot * STAGE_FLOATS + US_FLOATS + c * NXI * BN + nl;
                float* v = vs + vb * VS_FLOATS + c * BN + nl;
                float t[6][6];  // t = B^T d, column by column
#pragma unroll
                for (int b = 0; b < 6; ++b) {
                    float col[6], r[6];
#pragma unroll
                    for (int a = 0; a < 6; ++a) col[a] = xs[(a * 6 + b) * BN];
                    bt4_vec(col, r);
#pragma unroll
                    for (int a = 0; a < 6; ++a) t[a][b] = r[a];
                }
#pragma unroll
                for (int a = 0; a < 6; ++a) {  // V = t B, row by row
                    float r[6];
                    bt4_vec(t[a], r);
#pragma unroll
                    for (int b = 0; b < 6; ++b) v[((a * 6 + b) * BC) * BN] = r[b];
                }
                fence_proxy_async_smem();  // generic reads of the TMA slot before its async-proxy refill
                __syncwarp();
                if (lane == 0) {
                    mbar_arrive(&empty[slot]);
                    mbar_arrive(&vfull[vb]);
                }
            }
        }
        return;
    }

    // ================================ compute ================================
    setmaxnreg_inc<REG_COMPUTE>();
    // lane -> (k-group, nu-group) chosen so both operand loads are 2-wavefront LDS.128:
    // lanes sharing an address are adjacent pairs / at most 2 distinct per quarter-warp
    // (scripts/microbench/lds_wave.cu; lane>>2 / lane&3 costs 4 wavefronts for the nu load)
    const int fo = 4 * ((lane & 15) >> 1);              // k: fo..fo+3, fo+32..fo+35 (8 k-groups)
    const int io = 4 * ((lane & 1) + 2 * (lane >> 4));  // nu: io..io+3                 (4 nu-groups)
    const int xi0 = 3 * warp;
    const size_t HWN = (size_t)p.H * p.W * p.N;
    const size_t dW = (size_t)p.W * p.N;
    int G = 0;
    Segs<SK> segs(p);
    int tile, lo, hi;
    while (segs.next(p, tile, lo, hi)) {
        const int k0 = (tile % p.num_kb) * BK, nu0 = (tile / p.num_kb) * BN;
        // stream-K piece of a cut tile -> workspace slot 2b (the CTA's first piece) or 2b + 1
        const int sk_slot = (SK && hi - lo != p.num_it) ? 2 * static_cast<int>(blockIdx.x) + (segs.n > 1 ? 1 : 0) : -1;
        float acc[3][8][4];
#pragma unroll
        for (int q = 0; q < 3; ++q)
#pragma unroll
            for (int i = 0; i < 8; ++i)
#pragma unroll
                for (int j = 0; j < 4; ++j) acc[q][i][j] = 0.f;
        for (int g = lo; g < hi; ++g, ++G) {
            const int slot = G % S, vb = G % SV;
            mbar_wait(&full[slot], (G / S) & 1);
            mbar_wait(&vfull[vb], (G / SV) & 1);
            const float* us = smem + slot * STAGE_FLOATS + xi0 * BK + fo;
            const float* v = vs + vb * VS_FLOATS + xi0 * BC * BN + io;
#pragma unroll
            for (int c = 0; c < BC; ++c) {
#pragma unroll
                for (int q = 0; q < 3; ++q) {
                    const float4 a = *reinterpret_cast<const float4*>(us + (c * NXI + q) * BK);
                    const float4 b = *reinterpret_cast<const float4*>(us + (c * NXI + q) * BK + 32);
                    const float4 gv = *reinterpret_cast<const float4*>(v + (q * BC + c) * BN);
                    const float f[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
                    const float gg[4] = {gv.x, gv.y, gv.z, gv.w};
                    // bank-aware order (see fused_fp32.cuh): acc packed with parity opposite to gg
#pragma unroll
                    for (int i = 0; i < 8; ++i)
#pragma unroll
                        for (int jj = 0; jj < 4; ++jj) {
                            const int j = (i & 1) ? 3 - jj : jj;
                            acc[q][i][j] = fmaf(f[i], gg[j], acc[q][i][j]);
                        }
                }
            }
            fence_proxy_async_smem();  // generic reads of the TMA slot before its async-proxy refill
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(&empty[slot]);
                mbar_arrive(&vempty[vb]);
            }
        }

        // ---- OTF: 4 rounds of 16 filters through the epilogue buffer ----
#pragma unroll
        for (int rd = 0; rd < 4; ++rd) {
            named_bar_sync(1, COMPUTE_THREADS);
#pragma unroll
            for (int q = 0; q < 3; ++q)
#pragma unroll
                for (int ii = 0; ii < 2; ++ii) {
                    const int i = (rd >> 1) * 4 + (rd & 1) * 2 + ii;
                    const int r = (fo >> 2) * 2 + ii;
                    *reinterpret_cast<float4*>(ep + ((xi0 + q) * ER_KROWS + r) * ER_LD + io) =
                        make_float4(acc[q][i][1], acc[q][i][0], acc[q][i][3], acc[q][i][2]);
                }
            named_bar_sync(1, COMPUTE_THREADS);
            if (tid < ER_KROWS * BN) {  // one (k, nu) per thread
                const int r = tid >> 4, nl = tid & 15;
                const int kl = (r >> 1) * 4 + (rd & 1) * 2 + (r & 1) + (rd >> 1) * 32;
                const int k = k0 + kl, nu = nu0 + nl;
                if (k < p.K && nu < p.NV) {
                    const int t = nu / p.N, n = nu - t * p.N;
                    const int th = t / p.TW, tw = t - th * p.TW;
                    const int i0 = 4 * th, j0 = 4 * tw;
                    float tt[4][6];  // A^T M, column by column
#pragma unroll
                    for (int b = 0; b < 6; ++b) {
                        float col[6], o[4];
#pragma unroll
                        for (int a = 0; a < 6; ++a) col[a] = ep[((a * 6 + b) * ER_KROWS + r) * ER_LD + (nl ^ 1)];
                        at4_vec(col, o);
#pragma unroll
                        for (int a = 0; a < 4; ++a) tt[a][b] = o[a];
                    }
                    float* yk = p.y + (size_t)k * HWN + ((size_t)i0 * p.W + j0) * p.N + n;
                    float* wk = SK ? p.sk_ws + ((size_t)sk_slot * BK + kl) * (16 * BN) + nl : nullptr;
#pragma unroll
                    for (int a = 0; a < 4; ++a) {
                        float o[4];
                        at4_vec(tt[a], o);
#pragma unroll
                        for (int b = 0; b < 4; ++b) {
                            if (SK && sk_slot >= 0) wk[(a * 4 + b) * BN] = o[b];  // partial: [kl][a*4+b][nu]
                            else if (i0 + a < p.H && j0 + b < p.W) yk[a * dW + b * p.N] = o[b];
                        }
                    }
                }
            }
        }
    }
}

// Stream-K fixup: blocks 16i .. 16i+15 handle the tile cut by the range boundary of CTA i + 1
// when it is the first boundary inside that tile, 1/16 of its 64 k x 16 nu x 16 outputs each:
// y = sum of the pieces' partials in CTA order (deterministic).
constexpr int FIX_PARTS = 16;
__global__ void __launch_bounds__(256) f4_fixup_kernel(const __grid_constant__ Params p, int G) {
    constexpr int PER = BK * BN * 16 / FIX_PARTS / 256;  // 4 outputs per thread
    __shared__ int slots[256];
    __shared__ int nseg;
    const int b = blockIdx.x / FIX_PARTS + 1, part = blockIdx.x % FIX_PARTS;
    const int ub = sk_start(p, b);
    const int tile = ub / p.num_it;
    const int t0 = tile * p.num_it, t1 = t0 + p.num_it;
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
    constexpr size_t SLOT = (size_t)BK * 16 * BN;
    float o[PER];
#pragma unroll
    for (int i = 0; i < PER; ++i) o[i] = 0.f;
    for (int sidx = 0; sidx < ns; ++sidx) {
        const float* wk = p.sk_ws + slots[sidx] * SLOT;
        float v[PER];
#pragma unroll
        for (int i = 0; i < PER; ++i) v[i] = wk[(part * PER + i) * 256 + threadIdx.x];  // [kl][a*4+b][nu]
#pragma unroll
        for (int i = 0; i < PER; ++i) o[i] += v[i];
    }
#pragma unroll
    for (int i = 0; i < PER; ++i) {
        const int e = (part * PER + i) * 256 + threadIdx.x;
        const int nl = e % BN, ab = (e / BN) % 16, kl = e / (16 * BN);
        const int k = kb * BK + kl, nu = nb * BN + nl;
        if (k >= p.K || nu >= p.NV) continue;
        const int t = nu / p.N, n = nu - t * p.N;
        const int th = t / p.TW, tw = t - th * p.TW;
        const int a = ab >> 2, bb = ab & 3, i0 = 4 * th + a, j0 = 4 * tw + bb;
        if (i0 < p.H && j0 < p.W) p.y[(size_t)k * HWN + (size_t)i0 * dW + (size_t)j0 * p.N + n] = o[i];
    }
}

}  // namespace f4
}  // namespace wino
