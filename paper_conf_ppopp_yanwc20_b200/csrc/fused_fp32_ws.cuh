// fused_fp32_ws.cuh -- persistent, warp-specialised variant of the fused FP32 kernel (sm_100a).
//
// Same method, tiling and FFMA micro-kernel as fused_fp32.cuh (Yan, Wang & Chu,
// Sec. 3-4, Alg. 1), re-organised for Blackwell:
//   * warpgroups 0-1 (8 warps, 208 registers each via setmaxnreg) only run the
//     16-batched GEMM (LDS.128 fragments + FFMA, Fig. 3 arrangement, bank-aware
//     order) and the output transform;
//   * warpgroup 2 (88 registers): one warp issues the TMA boxes, two perform
//     the ITF (Eq. 6) of the coming stages (LDS.128 / STS.128 along nu) into a
//     ring of V buffers;
//   * stages are handed over with mbarriers (full / empty / V-full / V-empty),
//     so the compute warps never wait at a CTA-wide barrier and never stall on
//     the ITF's load-to-use latency (the paper interleaves ITF and FFMA in one
//     instruction stream by hand, Sec. 6; here another warpgroup does it);
//   * persistent: one CTA per SM walks tiles blockIdx.x, +gridDim.x, ...; the
//     producer runs ahead across tile boundaries, so the next tile's loads and
//     ITF overlap this tile's epilogue.  The epilogue therefore has its own
//     shared buffer and runs in 4 rounds (16 filters each) -- the paper's
//     4-round OTF (L479-499), here to leave room for the pipeline ring.
// Used when both operands can be TMA boxes (N % 32 == 0, K % 4 == 0).
#pragma once
#include <cuda.h>

#include <cstdint>

#include "fused_fp32.cuh"
#include "wino_ptx.cuh"
#include "wino_transforms.cuh"

namespace wino {
namespace fp32ws {

using fp32::BC;
using fp32::BK;
using fp32::BN;
using fp32::Params;
using fp32::STAGE_FLOATS;
using fp32::US_FLOATS;
using fp32::VS_FLOATS;
using fp32::XS_FLOATS;

constexpr int NT = 384;             // 2 compute warpgroups + 1 producer/ITF warpgroup
constexpr int COMPUTE_THREADS = 256;
constexpr int S = 3;                // TMA stage ring (u 32 KB + raw x 16 KB per stage)
constexpr int SV = 2;               // V ring (16 KB each)
constexpr int REG_COMPUTE = 208, REG_PRODUCER = 88;  // 256*208 + 128*88 = 64512 <= 65536
constexpr int ITF_WARPS = 2;        // warps 9..10 (float4 along nu); warp 8 only issues TMA; 11 idle
constexpr int ER_LD = BN + 4;       // padded row of the epilogue buffer
constexpr int ER_KROWS = 16;        // filters per epilogue round
constexpr int ER_FLOATS = 16 * ER_KROWS * ER_LD;  // [xi][16 k][36]

struct Smem {
    static constexpr int ep_offset = (S * STAGE_FLOATS + SV * VS_FLOATS) * 4;
    static constexpr int bar_offset = ep_offset + ER_FLOATS * 4;
    // full[S], empty[S], vfull[SV], vempty[SV]
    static constexpr int bytes = bar_offset + (2 * S + 2 * SV) * 8;
};

__global__ void __launch_bounds__(NT, 1) fused_fp32_ws_kernel(const __grid_constant__ Params p, int num_tiles) {
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
            mbar_init(&empty[s], 8 + ITF_WARPS);  // 8 compute warps (u) + ITF warps (raw x)
        }
        for (int s = 0; s < SV; ++s) {
            mbar_init(&vfull[s], ITF_WARPS);
            mbar_init(&vempty[s], 8);
        }
        fence_mbar_init();
    }
    __syncthreads();

    if (warp >= 8) {
        // ============================ producer / ITF ============================
        setmaxnreg_dec<REG_PRODUCER>();
        if (warp == 8) {
            // ---------------- TMA issue (one elected lane) ----------------
            if (lane == 0) {
                constexpr uint32_t kBytes = (US_FLOATS + XS_FLOATS) * 4;
                int G = 0;  // global stage counter across tiles
                for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x) {
                    const int kb = tile % p.num_kb, nb = tile / p.num_kb;
                    const int k0 = kb * BK, nu0 = nb * BN;
                    // N % 32 == 0 -> the tile's 32 nu are 32 consecutive n of one image tile
                    const int t = nu0 / p.N;
                    const int n0 = nu0 - t * p.N;
                    const int th = t / p.TW, tw = t - th * p.TW;
                    const int w0 = 2 * tw - 1, h0 = 2 * th - 1;  // -1: TMA zero fill = padding (Sec. 3.5)
                    for (int g = 0; g < NIT; ++g, ++G) {
                        const int slot = G % S;
                        if (G >= S) mbar_wait(&empty[slot], ((G / S) - 1) & 1);
                        float* us = smem + slot * STAGE_FLOATS;
                        mbar_arrive_expect_tx(&full[slot], kBytes);
                        tma_load_3d(us, &p.tmu, &full[slot], k0, 0, g * BC);
                        tma_load_4d(us + US_FLOATS, &p.tmx, &full[slot], n0, w0, h0, g * BC);
                    }
                }
            }
            return;
        }
        // ---------------- ITF (Sec. 4.2) on warps 9..10 ----------------
        // 256 (c, nu) tiles per stage; a thread transforms 4 consecutive nu of one
        // channel with LDS.128 / STS.128 (a quarter-warp covers one 128 B row:
        // conflict-free): lane -> (c = 4 (w - 9) + lane / 8, nu4 = lane % 8).
        if (warp > 8 + ITF_WARPS) return;
        const int c = 4 * (warp - 9) + (lane >> 3), n4 = 4 * (lane & 7);
        int G = 0;
        for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x) {
            for (int g = 0; g < NIT; ++g, ++G) {
                const int slot = G % S, vb = G % SV;
                mbar_wait(&full[slot], (G / S) & 1);
                if (G >= SV) mbar_wait(&vempty[vb], ((G / SV) - 1) & 1);
                const float* xs = smem + slot * STAGE_FLOATS + US_FLOATS + c * 16 * BN + n4;
                float* v = vs + vb * VS_FLOATS + c * BN + n4;
                float d[4][16];
#pragma unroll
                for (int e = 0; e < 16; ++e) {
                    const float4 q = *reinterpret_cast<const float4*>(xs + e * BN);
                    d[0][e] = q.x; d[1][e] = q.y; d[2][e] = q.z; d[3][e] = q.w;
                }
                float t[4][16];
#pragma unroll
                for (int j = 0; j < 4; ++j) itf_4x4(d[j], t[j]);
#pragma unroll
                for (int e = 0; e < 16; ++e)
                    *reinterpret_cast<float4*>(v + e * BC * BN) = make_float4(t[0][e], t[1][e], t[2][e], t[3][e]);
                __syncwarp();
                if (lane == 0) {
                    mbar_arrive(&empty[slot]);  // raw x of this slot consumed
                    mbar_arrive(&vfull[vb]);
                }
            }
        }
        return;
    }

    // ================================ compute ================================
    setmaxnreg_inc<REG_COMPUTE>();
    const int fo = 4 * ((lane & 15) >> 1);             // k offset: fo..fo+3, fo+32..fo+35 (Fig. 3)
    const int io = 4 * ((lane & 1) + 2 * (lane >> 4));  // nu offset: io..io+3, io+16..io+19
    const int xi0 = 2 * warp;
    const size_t HWN = (size_t)p.H * p.W * p.N;
    const size_t dW = (size_t)p.W * p.N;

    auto load_frag = [&](const float* us, const float* v, int c, float f[2][8], float g[2][8]) {
#pragma unroll
        for (int q = 0; q < 2; ++q) {
            const float4 a = *reinterpret_cast<const float4*>(us + (c * 16 + q) * BK);
            const float4 b = *reinterpret_cast<const float4*>(us + (c * 16 + q) * BK + 32);
            const float4 va = *reinterpret_cast<const float4*>(v + (q * BC + c) * BN);
            const float4 vb = *reinterpret_cast<const float4*>(v + (q * BC + c) * BN + 16);
            f[q][0] = a.x; f[q][1] = a.y; f[q][2] = a.z; f[q][3] = a.w;
            f[q][4] = b.x; f[q][5] = b.y; f[q][6] = b.z; f[q][7] = b.w;
            g[q][0] = va.x; g[q][1] = va.y; g[q][2] = va.z; g[q][3] = va.w;
            g[q][4] = vb.x; g[q][5] = vb.y; g[q][6] = vb.z; g[q][7] = vb.w;
        }
    };

    int G = 0;
    for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x) {
        const int kb = tile % p.num_kb, nb = tile / p.num_kb;
        const int k0 = kb * BK, nu0 = nb * BN;
        float acc[2][8][8];
#pragma unroll
        for (int q = 0; q < 2; ++q)
#pragma unroll
            for (int i = 0; i < 8; ++i)
#pragma unroll
                for (int j = 0; j < 8; ++j) acc[q][i][j] = 0.f;
        // register-bank-aware order: see fused_fp32.cuh (paper Fig. 4 rule re-derived for sm_100)
        auto ffma_block = [&](const float f[2][8], const float g[2][8]) {
#pragma unroll
            for (int q = 0; q < 2; ++q)
#pragma unroll
                for (int i = 0; i < 8; ++i)
#pragma unroll
                    for (int jj = 0; jj < 8; ++jj) {
                        const int j = (i & 1) ? 7 - jj : jj;
                        acc[q][i][j] = fmaf(f[q][i], g[q][j], acc[q][i][j]);
                    }
        };
        for (int g = 0; g < NIT; ++g, ++G) {
            const int slot = G % S, vb = G % SV;
            mbar_wait(&full[slot], (G / S) & 1);
            mbar_wait(&vfull[vb], (G / SV) & 1);
            const float* us = smem + slot * STAGE_FLOATS + xi0 * BK + fo;
            const float* v = vs + vb * VS_FLOATS + xi0 * BC * BN + io;
            float fa[2][8], ga[2][8], fb[2][8], gb[2][8];
            load_frag(us, v, 0, fa, ga);
#pragma unroll
            for (int c = 0; c < BC; c += 2) {
                load_frag(us, v, c + 1, fb, gb);
                ffma_block(fa, ga);
                if (c + 2 < BC) load_frag(us, v, c + 2, fa, ga);
                ffma_block(fb, gb);
            }
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(&empty[slot]);  // u of this slot consumed
                mbar_arrive(&vempty[vb]);
            }
        }

        // ---- OTF (Sec. 4.4) in 4 rounds of 16 filters through the epilogue buffer ----
        const int nu = nu0 + lane;
        int t = 0, n = 0, i0 = 0, j0 = 0;
        if (nu < p.NV) {
            t = nu / p.N;
            n = nu - t * p.N;
            const int th = t / p.TW, tw = t - th * p.TW;
            i0 = 2 * th;
            j0 = 2 * tw;
        }
        const bool okr = i0 + 1 < p.H, okc = j0 + 1 < p.W;  // odd H/W: drop extra outputs (L1155)
        const size_t base = ((size_t)i0 * p.W + j0) * p.N + n;
#pragma unroll
        for (int rd = 0; rd < 4; ++rd) {
            // round rd stores accumulator rows i in {2(rd&1), 2(rd&1)+1} of half rd>>1:
            // filters kl = fo + (i&3) + 32*(i>>2); in the buffer row = (fo>>2)*2 + (i&1)
            named_bar_sync(1, COMPUTE_THREADS);  // previous round's readers are done
#pragma unroll
            for (int q = 0; q < 2; ++q)
#pragma unroll
                for (int ii = 0; ii < 2; ++ii) {
                    const int i = (rd >> 1) * 4 + (rd & 1) * 2 + ii;
                    const int r = (fo >> 2) * 2 + ii;
                    float* row = ep + ((xi0 + q) * ER_KROWS + r) * ER_LD + io;
                    *reinterpret_cast<float4*>(row) =
                        make_float4(acc[q][i][1], acc[q][i][0], acc[q][i][3], acc[q][i][2]);
                    *reinterpret_cast<float4*>(row + 16) =
                        make_float4(acc[q][i][5], acc[q][i][4], acc[q][i][7], acc[q][i][6]);
                }
            named_bar_sync(1, COMPUTE_THREADS);
            if (nu < p.NV) {
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int r = warp + 8 * h;  // buffer row 0..15
                    const int kl = (r >> 1) * 4 + (rd & 1) * 2 + (r & 1) + (rd >> 1) * 32;
                    const int k = k0 + kl;
                    if (k < p.K) {
                        float m[16], o[4];
#pragma unroll
                        for (int e = 0; e < 16; ++e) m[e] = ep[(e * ER_KROWS + r) * ER_LD + (lane ^ 1)];
                        otf_2x2(m, o);
                        float* yk = p.y + (size_t)k * HWN + base;
                        yk[0] = o[0];
                        if (okc) yk[p.N] = o[1];
                        if (okr) yk[dW] = o[2];
                        if (okr && okc) yk[dW + p.N] = o[3];
                    }
                }
            }
        }
    }
}

}  // namespace fp32ws
}  // namespace wino
