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
// Used when N % 16 == 0 and K % 4 == 0 (other shapes: WINO_ERR_UNSUPPORTED).
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
struct Smem {
    static constexpr int ep_offset = (S * STAGE_FLOATS + SV * VS_FLOATS) * 4;
    static constexpr int bar_offset = ep_offset + ER_FLOATS * 4;
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
    int N, C, H, W, K;
    int TW;      // ceil(W/4)
    int NV;      // N * ceil(H/4) * ceil(W/4)
    int num_kb;  // ceil(K/64)
    int num_it;  // ceil(C/4)
    int num_tiles;
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

__global__ void __launch_bounds__(NT, 1) fused_f4_kernel(const __grid_constant__ Params p) {
    extern __shared__ __align__(1024) float smem[];
    float* const vs = smem + S * STAGE_FLOATS;
    float* const ep = reinterpret_cast<float*>(reinterpret_cast<char*>(smem) + Smem::ep_offset);
    uint64_t* const full = reinterpret_cast<uint64_t*>(reinterpret_cast<char*>(smem) + Smem::bar_offset);
    uint64_t* const empty = full + S;
    uint64_t* const vfull = empty + S;
    uint64_t* const vempty = vfull + SV;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int NIT = p.num_it;

    if (tid == 0) {
        tma_prefetch_desc(&p.tmx);
        tma_prefetch_desc(&p.tmu);
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
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
        if (warp == COMPUTE_WARPS) {
            // ---------------------------- TMA issue ----------------------------
            if (lane == 0) {
                constexpr uint32_t kBytes = (US_FLOATS + XS_FLOATS) * 4;
                int G = 0;
                for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
                    const int k0 = (tile % p.num_kb) * BK, nu0 = (tile / p.num_kb) * BN;
                    const int t = nu0 / p.N, n0 = nu0 - t * p.N;
                    const int th = t / p.TW, tw = t - th * p.TW;
                    for (int g = 0; g < NIT; ++g, ++G) {
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
        for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
            for (int g = 0; g < NIT; ++g, ++G) {
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
    for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
        const int k0 = (tile % p.num_kb) * BK, nu0 = (tile / p.num_kb) * BN;
        float acc[3][8][4];
#pragma unroll
        for (int q = 0; q < 3; ++q)
#pragma unroll
            for (int i = 0; i < 8; ++i)
#pragma unroll
                for (int j = 0; j < 4; ++j) acc[q][i][j] = 0.f;
        for (int g = 0; g < NIT; ++g, ++G) {
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
#pragma unroll
                    for (int a = 0; a < 4; ++a) {
                        float o[4];
                        at4_vec(tt[a], o);
#pragma unroll
                        for (int b = 0; b < 4; ++b)
                            if (i0 + a < p.H && j0 + b < p.W) yk[a * dW + b * p.N] = o[b];
                    }
                }
            }
        }
    }
}

}  // namespace f4
}  // namespace wino
