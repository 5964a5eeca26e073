// nonfused_tc.cuh -- NEXT row N3 with the library's own tensor-core GEMM: the NON-fused
// Winograd F(2x2,3x3) forward convolution as four launches,
//   1. nf_arrange_u_kernel  u (C,4,4,K)   -> Ug [16*P][K][Cp4]   (TF32-rounded; P = 2: + residual plane)
//   2. nf_itf_kernel        x (C,H,W,N)   -> V  [16*P][NV][Cp4]  (Eq. 6, TF32-rounded, c contiguous)
//   3. nf_gemm_kernel       M[xi][k][nu] = sum_c V[xi][nu][c] * Ug[xi][k][c]   (Eq. 7, tcgen05 kind::tf32)
//   4. otf_nf_kernel        M [16][K][NV] -> y (K,H,W,N)          (Eq. 8, nonfused.cuh)
// The paper: "store intermediate results in global memory (non-fused version) ... can utilize
// optimized batched matrix multiplication routines.  However, it needs significant amount of
// global memory as workspace and data loading can be the new bottleneck" (Sec. 9; the
// Sec. 8.1 cost model L1245-1269).  Here the 16 batched GEMMs are this file's kernel, not a
// library's.
//
// GEMM (one CTA per (128 nu) x (BNK k) tile of one xi): the Winograd-domain operands are both
// stored K-major (channel c contiguous) so tcgen05 reads them straight from TMA-filled shared
// memory with the 128-byte swizzle: A = V[xi] rows nu (UMMA M = 128), B = Ug[xi] rows k (UMMA N =
// BNK <= 256), K = 8 channels per instruction, 32 channels (one 128 B swizzle atom) per pipeline
// stage.  D[nu][k] lives in TMEM (128 lanes x BNK columns); the epilogue reads it with
// tcgen05.ld (lane = nu, so each column store is a coalesced 128 B row of M[xi][k][.]).
// Operands past C, NV or K are zero-filled by TMA (out-of-bounds boxes), so the workspaces need
// no padding beyond the 16-byte row pitch Cp4 = 4 ceil(C/4).
// 3xTF32 (P = 2, the FP32-accuracy non-fused variant): big = rna(v), small = rna(v - big) for both
// operands; D += Vb Ub + Vb Us + Vs Ub (reading R8).
#pragma once
#include <cuda.h>

#include <cstdint>

#include "wino_ptx.cuh"
#include "wino_transforms.cuh"

namespace wino {
namespace nftc {

constexpr int BM = 128;        // nu per tile (UMMA M, TMEM lanes)
constexpr int BKC = 32;        // channels per stage: one 128 B swizzle atom row
constexpr int GEMM_THREADS = 128;
constexpr int A_TILE = BM * BKC * 4;  // 16 KB per plane

__host__ __device__ inline int cp4(int C) { return (C + 3) & ~3; }
// N of the UMMA (filters per tile): K rounded up to 16 up to 256, else 256
__host__ __device__ inline int gemm_bnk(int K) { return K <= 256 ? ((K + 15) / 16) * 16 : 256; }
__host__ __device__ inline int tmem_cols(int bnk) { return bnk <= 32 ? 32 : bnk <= 64 ? 64 : bnk <= 128 ? 128 : 256; }
template <int P>
__host__ __device__ inline int gemm_stages(int bnk) {
    const int stage = P * (A_TILE + bnk * BKC * 4);
    const int s = (200 * 1024) / stage;
    return s > 6 ? 6 : s;
}
// stages actually used: no more than the K loop has chunks (short K loops -> smaller CTAs, more
// of them per SM to overlap one tile's epilogue with another's loads)
template <int P>
__host__ __device__ inline int gemm_stages_for(int bnk, int nchunks) {
    if (nchunks <= 4) {  // short K loop (C <= 128): <= 75 KB per CTA so that >= 3 CTAs share an SM
        const int per = (75 * 1024) / (P * (A_TILE + bnk * BKC * 4));
        const int s = nchunks < per ? nchunks : per;
        return s < 2 ? 2 : s;
    }
    return gemm_stages<P>(bnk);
}
template <int P>
__host__ __device__ inline int gemm_smem_bytes(int bnk, int stages) {
    return 1024 /* alignment slack */ + stages * P * (A_TILE + bnk * BKC * 4) + 256;
}

// SWIZZLE_128B K-major shared-memory matrix descriptor (sm_100): start >> 4, LBO unused (1),
// SBO = 1024 B between 8-row groups, version 1 (bit 46), layout type 2 = SWIZZLE_128B (bits 61-63).
__device__ __forceinline__ uint64_t desc_sw128(uint32_t saddr) {
    return uint64_t((saddr >> 4) & 0x3FFF) | (uint64_t(1) << 16) | (uint64_t(1024 >> 4) << 32) |
           (uint64_t(1) << 46) | (uint64_t(2) << 61);
}

// 32 lanes x 32 bit, 16 consecutive columns per thread
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t r[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];\n"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
}

struct __align__(64) GemmParams {
    CUtensorMap tmv;  // V  (Cp4 pitch): dims (C, NV, 16P), box (32, 128, 1), SWIZZLE_128B
    CUtensorMap tmu;  // Ug (Cp4 pitch): dims (C, K, 16P),  box (32, BNK, 1), SWIZZLE_128B
    float* __restrict__ m;  // M [16][K][NV]
    int K, NV, C, bnk, stages, nchunks;
};

// grid (ceil(NV/128), ceil(K/BNK), 16).  Warp 0 lane 0: TMA producer; warp 1 lane 0: MMA issuer;
// all 4 warps: epilogue (warp w reads TMEM lanes 32w..32w+31).
template <int P>
__global__ void __launch_bounds__(GEMM_THREADS) nf_gemm_kernel(const __grid_constant__ GemmParams p) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    const int S = p.stages, BNK = p.bnk;
    const int b_tile = BNK * BKC * 4;
    const int stage_bytes = P * (A_TILE + b_tile);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + S * stage_bytes);
    uint64_t* empty = full + S;
    uint64_t* acc = empty + S;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(acc + 1);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int nu0 = blockIdx.x * BM, k0 = blockIdx.y * BNK, xi = blockIdx.z;
    const int ncols = tmem_cols(BNK);

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], 1);
        }
        mbar_init(acc, 1);
        fence_mbar_init();
        tma_prefetch_desc(&p.tmv);
        tma_prefetch_desc(&p.tmu);
    }
    if (warp == 0) tmem_alloc(tmem_slot, ncols);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;

    if (warp == 0 && lane == 0) {
        // ------------------------------ TMA producer ------------------------------
        for (int it = 0; it < p.nchunks; ++it) {
            const int s = it % S;
            if (it >= S) mbar_wait(&empty[s], ((it / S) - 1) & 1);
            uint8_t* st = smem + s * stage_bytes;
            mbar_arrive_expect_tx(&full[s], stage_bytes);
#pragma unroll
            for (int pl = 0; pl < P; ++pl) {
                tma_load_3d(st + pl * A_TILE, &p.tmv, &full[s], it * BKC, nu0, xi * P + pl);
                tma_load_3d(st + P * A_TILE + pl * b_tile, &p.tmu, &full[s], it * BKC, k0, xi * P + pl);
            }
        }
    } else if (warp == 1 && lane == 0) {
        // ------------------------------- MMA issuer -------------------------------
        const uint32_t idesc = umma_idesc_tf32(BM, BNK);
        for (int it = 0; it < p.nchunks; ++it) {
            const int s = it % S;
            mbar_wait(&full[s], (it / S) & 1);
            tc_fence_after();
            const uint32_t a0 = smem_u32(smem + s * stage_bytes);
            const uint32_t b0 = a0 + P * A_TILE;
#pragma unroll
            for (int ks = 0; ks < BKC / 8; ++ks) {  // 4 K-steps of 8 channels (32 B) in the swizzle atom
                const uint64_t ab = desc_sw128(a0 + ks * 32), bb = desc_sw128(b0 + ks * 32);
                umma_tf32(tmem, ab, bb, idesc, (it | ks) ? 1u : 0u);
                if constexpr (P == 2) {
                    const uint64_t as = desc_sw128(a0 + A_TILE + ks * 32), bs = desc_sw128(b0 + b_tile + ks * 32);
                    umma_tf32(tmem, ab, bs, idesc, 1u);
                    umma_tf32(tmem, as, bb, idesc, 1u);
                }
            }
            umma_commit(&empty[s]);  // the stage is free once these MMAs have read it
        }
        umma_commit(acc);
    }
    __syncwarp();
    // --------------------------------- epilogue ---------------------------------
    mbar_wait(acc, 0);
    tc_fence_after();
    const int nu = nu0 + warp * 32 + lane;
    const uint32_t trow = tmem + ((uint32_t)(warp * 32) << 16);
    float* mrow = p.m + (size_t)xi * p.K * p.NV + nu;
    for (int c0 = 0; c0 < BNK; c0 += 16) {
        uint32_t r[16];
        tmem_ld16(trow + c0, r);
        tmem_ld_wait();
        if (nu < p.NV) {
#pragma unroll
            for (int j = 0; j < 16; ++j) {
                const int k = k0 + c0 + j;
                if (k < p.K) mrow[(size_t)k * p.NV] = __uint_as_float(r[j]);  // 128 B rows across the warp
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tmem_dealloc(tmem, ncols);
}

// u (C,4,4,K) -> Ug[xi*P + plane][k][c] (pitch Cp4), TF32-rounded (+ residual plane).  Block = 32 k
// x 32 c of one xi through a padded shared tile: reads along k, writes along c (both coalesced).
template <int P>
__global__ void __launch_bounds__(256) nf_arrange_u_kernel(const float* __restrict__ u, float* __restrict__ ug,
                                                           int C, int K) {
    __shared__ float t[32][33];
    const int xi = blockIdx.z, k0 = blockIdx.x * 32, c0 = blockIdx.y * 32;
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    const int C4 = cp4(C);
#pragma unroll
    for (int j = 0; j < 32; j += 8) {
        const int c = c0 + ty + j, k = k0 + tx;
        t[ty + j][tx] = (c < C && k < K) ? u[((size_t)c * 16 + xi) * K + k] : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < 32; j += 8) {
        const int k = k0 + ty + j, c = c0 + tx;
        if (k < K && c < C4) {
            const float v = t[tx][ty + j];
            const float big = to_tf32(v);
            ug[((size_t)(xi * P) * K + k) * C4 + c] = big;
            if (P == 2) ug[((size_t)(xi * P + 1) * K + k) * C4 + c] = to_tf32(v - big);
        }
    }
}

// x (C,H,W,N) -> V[xi*P + plane][nu][c] (pitch Cp4), Eq. 6 + TF32 rounding (+ residual plane).
// Block = 32 nu x 32 c: a warp transforms 32 consecutive nu of one channel (coalesced window loads
// along n; zero outside the image = implicit padding, Sec. 3.5), the 16 results go through a
// padded shared tile per xi and leave as 128 B rows along c.
constexpr int ITF_SMEM = 16 * 32 * 33 * 4;
template <int P>
__global__ void __launch_bounds__(256) nf_itf_kernel(const float* __restrict__ x, float* __restrict__ v, int N, int C,
                                                     int H, int W, int TW, int NV) {
    extern __shared__ float sv[];  // [xi][c 32][nu 33]
    const int nu0 = blockIdx.x * 32, c0 = blockIdx.y * 32;
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5;
    const int nu = nu0 + lane;
    const int C4 = cp4(C);
    int th = 0, tw = 0, n = 0;
    if (nu < NV) {
        const int t = nu / N;
        n = nu - t * N;
        th = t / TW;
        tw = t - th * TW;
    }
#pragma unroll 1
    for (int j = 0; j < 4; ++j) {
        const int cl = wp + 8 * j, c = c0 + cl;
        float d[16], o[16];
        const float* xc = x + (size_t)c * H * W * N + n;
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            const int h = 2 * th - 1 + a;
#pragma unroll
            for (int b = 0; b < 4; ++b) {
                const int w = 2 * tw - 1 + b;
                d[4 * a + b] = (nu < NV && c < C && h >= 0 && h < H && w >= 0 && w < W)
                                   ? __ldg(xc + ((size_t)h * W + w) * N) : 0.f;
            }
        }
        itf_4x4(d, o);
#pragma unroll
        for (int e = 0; e < 16; ++e) sv[(e * 32 + cl) * 33 + lane] = o[e];
    }
    __syncthreads();
    // write-out: for each xi, 32 nu rows of 32 c (a warp writes one row per step)
    for (int r = wp; r < 16 * 32; r += 8) {
        const int e = r >> 5, nl = r & 31, nuo = nu0 + nl, c = c0 + lane;
        if (nuo >= NV || c >= C4) continue;
        const float val = sv[(e * 32 + lane) * 33 + nl];
        const float big = to_tf32(val);
        v[((size_t)(e * P) * NV + nuo) * C4 + c] = big;
        if (P == 2) v[((size_t)(e * P + 1) * NV + nuo) * C4 + c] = to_tf32(val - big);
    }
}

}  // namespace nftc
}  // namespace wino
