// fused_fp32.cuh -- fused ITF + 16-batched GEMM (FFMA) + OTF kernel for sm_100a.
//
// Yan, Wang & Chu (PPoPP'20): workflow Sec. 3.1 (L209), cache blocking
// Sec. 3.2-3.3 (L211-217, bk=64, bn=32, bc=8), software pipelining Sec. 3.4
// (L323-333), implicit zero padding Sec. 3.5 (L335), thread-block workload and
// Algorithm 1 (L339-355), ITF Sec. 4.2 (L357-359), batched GEMM, lane
// arrangement and register-bank-aware FFMA order Sec. 4.3 / Fig. 3-4
// (L361-477), OTF through shared memory Sec. 4.4 (L479-503).
//
// B200 redesign:
//  * global->shared staging is an S-deep ring filled by TMA tiled loads
//    (cp.async.bulk.tensor, completion on an mbarrier): one elected thread moves
//    a (k:64, xi:16, c:8) box of u and a (n:32, w:4, h:4, c:8) box of raw x per
//    stage; TMA's out-of-bounds zero fill IS the implicit padding of Sec. 3.5
//    (negative / past-the-end h, w coordinates) and also pads the C and K tails.
//    This removes the paper's 48 prefetch registers and predicate masks
//    (Table 5).  Shapes TMA cannot express (N % 32 != 0 for x,
//    K % 4 != 0 for u) fall back to cp.async with src-size-0 zero fill and a
//    per-CTA gather table -- still on the GPU, never on the host;
//  * nu = (tile, n) is flattened with n fastest, so any N works and small
//    per-rank batches still fill CTAs (the paper assumes 32 consecutive n);
//  * B200's 227 KB of shared memory holds all 128 KB of accumulators at once,
//    so the OTF transpose runs in ONE round instead of the paper's 4 (L499).
#pragma once
#include <cuda.h>

#include <cstdint>

#include "wino_ptx.cuh"
#include "wino_transforms.cuh"

namespace wino {
namespace fp32 {

constexpr int BK = 64;   // filters per CTA   (Sec. 3.3)
constexpr int BN = 32;   // tiles*images per CTA
constexpr int BC = 8;    // channels per pipeline step
constexpr int US_FLOATS = BC * 16 * BK;  // transformed-filter stage [c][xi][k]
constexpr int XS_FLOATS = BC * 16 * BN;  // raw-input stage        [c][pos][nu]
constexpr int STAGE_FLOATS = US_FLOATS + XS_FLOATS;
constexpr int VS_FLOATS = 16 * BC * BN;  // transformed input      [xi][c][nu] (Table 4 (16,bc,bn))
constexpr int EP_LD = BN + 4;            // padded row of the OTF transpose buffer
constexpr int EP_FLOATS = 16 * BK * EP_LD;
constexpr int TAB_INTS = 16 * BN;        // per-CTA gather/padding table (cp.async x path)

// how a stage's operand reaches shared memory
enum LoadMode : int { LD_CP4B = 0, LD_CP16B = 1, LD_TMA = 2 };

template <int S>
struct Smem {
    static constexpr int main_floats = S * STAGE_FLOATS + 2 * VS_FLOATS;
    static_assert(EP_FLOATS <= main_floats, "OTF buffer must fit in the pipeline buffers");
    static constexpr int bar_offset = (main_floats + TAB_INTS) * 4;
    static constexpr int bytes = bar_offset + S * 8;
};

struct __align__(64) Params {
    CUtensorMap tmx;  // x (C,H,W,N) as 4-d (N, W, H, C), box (32, 4, 4, BC)   [LD_TMA only]
    CUtensorMap tmu;  // u (C,16,ldu) as 3-d (K, 16, C),  box (BK, 16, BC)      [LD_TMA only]
    const float* __restrict__ x;  // (C,H,W,N)
    const float* __restrict__ u;  // (C,4,4,K)
    float* __restrict__ y;        // (K,H,W,N)
    int N, C, H, W, K;
    int ldu;     // row stride of u in elements (>= K; > K when u is a K-slice)
    int TW;      // ceil(W/2)
    int NV;      // N * ceil(H/2) * ceil(W/2)
    int num_kb;  // ceil(K/BK)
    int num_it;  // ceil(C/BC)
    int xnb;     // n-extent of one x TMA box: 32, or N when N | 32 (WS kernel: 32/xnb boxes per stage)
    int split;   // split-C factor S = cluster size (WS kernel; 1 = no split)
    int itf_map[64];  // WS kernel, N | 32: ITF task of thread (warp-9)*32+lane: c | n4 << 3 | xoff << 8
    // Generic kernel: element strides of x (c, n, h, w) and y (k, n, h, w), so any dense
    // layout works (CHWN / KHWN: the paper's, Table 4; NCHW / NKHW: Sec. 8.4), and
    // the order of nu = (tile, n): tfast = 0 -> n fastest (CHWN), 1 -> tile fastest (NCHW:
    // neighbouring lanes read / write neighbouring pixels of one image).
    long long xs_c, xs_n, xs_h, xs_w, ys_k, ys_n, ys_h, ys_w;
    int tfast;
    int T;  // ceil(H/2) * ceil(W/2)
    // WS kernel, stream-K mode: the (tile, channel block) iteration space of sk_total units is
    // cut into gridDim.x equal contiguous ranges; partial tiles go to sk_ws (2 slots of
    // 64 k x 4 outputs x 32 nu per CTA) and are summed by sk_fixup_kernel.
    float* __restrict__ sk_ws;
    unsigned* __restrict__ sk_flags;  // arrival counter per CTA holding a cut tile's block 0 (zero between launches)
    long long sk_total;  // tiles * num_it  (< 2^31)
    int sk_q, sk_r;      // sk_total = gridDim * sk_q + sk_r: CTA b's range starts at b*q + min(b, r)
};

// XPW = Winograd elements xi per warp: 2 -> 8 warps / 256 threads (the paper's
// Sec. 4 / Alg. 1 shape, 2 x 64 accumulators per thread); 1 -> 16 warps / 512
// threads with 64 accumulators each (same CTA tile, twice the warps per
// scheduler to hide LDS / barrier latency).
template <int XPW>
__host__ __device__ constexpr int threads_for() { return 512 / XPW; }

template <int XM, int UM, int S, int XPW>
__global__ void __launch_bounds__(threads_for<XPW>(), 1) fused_fp32_kernel(const __grid_constant__ Params p) {
    constexpr int NT = threads_for<XPW>();
    constexpr int NWARP = NT / 32;
    constexpr bool kTma = (XM == LD_TMA) || (UM == LD_TMA);
    constexpr uint32_t kTmaBytes = (XM == LD_TMA ? XS_FLOATS * 4 : 0) + (UM == LD_TMA ? US_FLOATS * 4 : 0);
    extern __shared__ __align__(1024) float smem[];
    float* const vs = smem + S * STAGE_FLOATS;
    int* const xtab = reinterpret_cast<int*>(vs + 2 * VS_FLOATS);
    uint64_t* const bar = reinterpret_cast<uint64_t*>(reinterpret_cast<char*>(smem) + Smem<S>::bar_offset);

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // k-block fastest: the CTAs resident at once share input tiles through L2
    const int kb = blockIdx.x % p.num_kb;
    const int nb = blockIdx.x / p.num_kb;
    const int k0 = kb * BK, nu0 = nb * BN;

    if constexpr (kTma) {
        if (tid == 0) {
            if constexpr (XM == LD_TMA) tma_prefetch_desc(&p.tmx);
            if constexpr (UM == LD_TMA) tma_prefetch_desc(&p.tmu);
#pragma unroll
            for (int s = 0; s < S; ++s) mbar_init(&bar[s], 1);
            fence_mbar_init();
        }
    }
    // TMA x box origin: N % 32 == 0, so the CTA's 32 nu are 32 consecutive n of one tile
    int tma_n0 = 0, tma_w0 = 0, tma_h0 = 0;
    if constexpr (XM == LD_TMA) {
        const int t = nu0 / p.N;
        tma_n0 = nu0 - t * p.N;
        const int th = t / p.TW, tw = t - th * p.TW;
        tma_w0 = 2 * tw - 1;  // may be -1: TMA zero-fills (implicit padding, Sec. 3.5)
        tma_h0 = 2 * th - 1;
    } else {
        // Spatial gather offsets (h*W+w)*N+n of the 4x4 window element `pos` of
        // local tile nu, or -1 where the window leaves the image (zero padding).
        for (int e = tid; e < TAB_INTS; e += NT) {
            const int pos = e / BN, nl = e % BN, nu = nu0 + nl;
            int off = -1;
            if (nu < p.NV) {
                int t, n;
                if (p.tfast) n = nu / p.T, t = nu - n * p.T;
                else t = nu / p.N, n = nu - t * p.N;
                const int th = t / p.TW, tw = t - th * p.TW;
                const int h = 2 * th - 1 + (pos >> 2), w = 2 * tw - 1 + (pos & 3);
                if (h >= 0 && h < p.H && w >= 0 && w < p.W) off = (int)(n * p.xs_n + h * p.xs_h + w * p.xs_w);
            }
            xtab[e] = off;
        }
    }
    __syncthreads();

    // ---- producer: one pipeline stage = BC channels of u and raw x ----------
    auto issue_stage = [&](int it, int slot) {
        const int c0 = it * BC;
        float* us = smem + slot * STAGE_FLOATS;
        float* xs = us + US_FLOATS;
        if constexpr (kTma) {
            if (tid == 0) {
                fence_proxy_async_smem();  // prior generic reads of this slot before async writes
                mbar_arrive_expect_tx(&bar[slot], kTmaBytes);
                if constexpr (UM == LD_TMA) tma_load_3d(us, &p.tmu, &bar[slot], k0, 0, c0);
                if constexpr (XM == LD_TMA) tma_load_4d(xs, &p.tmx, &bar[slot], tma_n0, tma_w0, tma_h0, c0);
            }
        }
        if constexpr (UM != LD_TMA) {
            constexpr int VU = UM == LD_CP16B ? 4 : 1;
            constexpr int UV_ROW = BK / VU;
            constexpr int U_PER_THREAD = BC * 16 * UV_ROW / NT;
#pragma unroll
            for (int j = 0; j < U_PER_THREAD; ++j) {
                const int idx = tid + j * NT;
                const int row = idx / UV_ROW, col = (idx % UV_ROW) * VU;
                const int c = c0 + row / 16, k = k0 + col;
                const bool ok = (c < p.C) && (k < p.K);
                const float* src = ok ? p.u + ((size_t)c * 16 + (row & 15)) * p.ldu + k : p.u;
                const uint32_t dst = smem_u32(us + row * BK + col);
                if constexpr (VU == 4) cp_async16(dst, src, ok);
                else cp_async4(dst, src, ok);
            }
        }
        if constexpr (XM != LD_TMA) {
            constexpr int VX = XM == LD_CP16B ? 4 : 1;
            constexpr int XV_C = 16 * BN / VX;
            constexpr int X_PER_THREAD = BC * XV_C / NT;
#pragma unroll
            for (int j = 0; j < X_PER_THREAD; ++j) {
                const int idx = tid + j * NT;
                const int cl = idx / XV_C, e = (idx % XV_C) * VX;
                const int c = c0 + cl;
                const int off = xtab[e];
                const bool ok = (c < p.C) && (off >= 0);
                const float* src = ok ? p.x + c * p.xs_c + off : p.x;
                const uint32_t dst = smem_u32(xs + cl * 16 * BN + e);
                if constexpr (VX == 4) cp_async16(dst, src, ok);
                else cp_async4(dst, src, ok);
            }
        }
    };
    auto wait_tma = [&](int it) {
        if constexpr (kTma) mbar_wait(&bar[it % S], (it / S) & 1);
    };

    // ---- ITF (Sec. 4.2): one (c, nu) tile per thread, raw [c][pos][nu] ->
    //      V [xi][c][nu]; lanes run along nu so both sides are conflict-free.
    //      Split into load / transform+store halves so the main loop can
    //      interleave them with the FFMA stream of the previous stage.
    const int itf_c = tid >> 5, itf_n = tid & 31;
    auto itf_load = [&](int slot, float d[16]) {
        const float* xs = smem + slot * STAGE_FLOATS + US_FLOATS + itf_c * 16 * BN + itf_n;
#pragma unroll
        for (int e = 0; e < 16; ++e) d[e] = xs[e * BN];
    };
    auto itf_store = [&](int vbuf, const float d[16]) {
        float t[16];
        itf_4x4(d, t);
        float* v = vs + vbuf * VS_FLOATS + itf_c * BN + itf_n;
#pragma unroll
        for (int e = 0; e < 16; ++e) v[e * BC * BN] = t[e];
    };

    // ---- EWMM as 16-batched GEMM (Sec. 4.3): warp w owns xi = XPW*w .. +XPW-1;
    //      the lane owns an 8(k) x 8(nu) block of each, Fig. 3 lane arrangement.
    const int fo = 4 * ((lane & 15) >> 1);             // k offset: fo..fo+3, fo+32..fo+35
    const int io = 4 * ((lane & 1) + 2 * (lane >> 4));  // nu offset: io..io+3, io+16..io+19
    const int xi0 = XPW * warp;
    float acc[XPW][8][8];
#pragma unroll
    for (int q = 0; q < XPW; ++q)
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
            for (int j = 0; j < 8; ++j) acc[q][i][j] = 0.f;

    // fragments of one channel c: f = u[c][xi][k-block], g = V[xi][c][nu-block]
    auto load_frag = [&](const float* us, const float* v, int c, float f[XPW][8], float g[XPW][8]) {
#pragma unroll
        for (int q = 0; q < XPW; ++q) {
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
    // Register-bank-aware FFMA order (the paper's Fig. 4 rule, L469-477,
    // re-derived for sm_100: an FFMA costs max(#even, #odd) register reads
    // among operands not served by the reuse cache).  f[i] is reused along a
    // row; acc[i][j] is packed with parity opposite to g[j] (see the swapped
    // float4 packing in the OTF store) and rows snake so the row change reuses
    // g[j_end] instead of f[i].
    auto ffma_block = [&](const float f[XPW][8], const float g[XPW][8]) {
#pragma unroll
        for (int q = 0; q < XPW; ++q)
#pragma unroll
            for (int i = 0; i < 8; ++i)
#pragma unroll
                for (int jj = 0; jj < 8; ++jj) {
                    const int j = (i & 1) ? 7 - jj : jj;
                    acc[q][i][j] = fmaf(f[q][i], g[q][j], acc[q][i][j]);
                }
    };
    // One pipeline step: GEMM over the BC channels of stage `slot` / V buffer
    // `vbuf`, with fragments double-buffered in registers (Sec. 3.4:
    // "hide the latency of LDS with software pipelining") and, when do_itf,
    // the ITF of the next stage woven into the FFMA stream.
    auto gemm_stage = [&](int slot, int vbuf, bool do_itf, int itf_slot, int itf_vbuf) {
        const float* us = smem + slot * STAGE_FLOATS + xi0 * BK + fo;
        const float* v = vs + vbuf * VS_FLOATS + xi0 * BC * BN + io;
        float fa[XPW][8], ga[XPW][8], fb[XPW][8], gb[XPW][8], d[16];
        do_itf = do_itf && (tid < BC * BN);  // warp-uniform: one (c, nu) tile per thread
        load_frag(us, v, 0, fa, ga);
        if (do_itf) itf_load(itf_slot, d);
#pragma unroll
        for (int c = 0; c < BC; c += 2) {
            load_frag(us, v, c + 1, fb, gb);
            ffma_block(fa, ga);
            if (c == 0 && do_itf) itf_store(itf_vbuf, d);
            if (c + 2 < BC) load_frag(us, v, c + 2, fa, ga);
            ffma_block(fb, gb);
        }
    };

    // ---- main loop (Algorithm 1 lines 6-16) with an S-stage ring -----------
    const int NIT = p.num_it;
#pragma unroll
    for (int s = 0; s < S - 1; ++s) {
        if (s < NIT) issue_stage(s, s);
        cp_async_commit();
    }
    cp_async_wait<S - 2>();
    wait_tma(0);
    __syncthreads();
    if (tid < BC * BN) {
        float d[16];
        itf_load(0, d);
        itf_store(0, d);
    }

    for (int it = 0; it < NIT; ++it) {
        cp_async_wait<S - 3>();
        if (it + 1 < NIT) wait_tma(it + 1);  // stage it+1 landed
        // the slot refilled below was read through the generic proxy; a TMA refill is an
        // async-proxy write, ordered after those reads only through fence.proxy.async
        if (XM == LD_TMA || UM == LD_TMA) fence_proxy_async_smem();
        __syncthreads();                      // V[it&1] complete; slot (it-1)%S free
        const int nxt = it + S - 1;
        if (nxt < NIT) issue_stage(nxt, nxt % S);
        cp_async_commit();
        gemm_stage(it % S, it & 1, it + 1 < NIT, (it + 1) % S, (it + 1) & 1);
    }
    cp_async_wait<0>();
    __syncthreads();

    // ---- OTF (Sec. 4.4): accumulators -> smem [xi][k][nu] in one round ------
    // Columns are stored pair-swapped (nu^1), matching the register packing
    // chosen for bank-conflict-free FFMAs; the reader undoes it.
    float* ep = smem;
#pragma unroll
    for (int q = 0; q < XPW; ++q)
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int kl = fo + (i & 3) + (i >> 2) * 32;
            float* row = ep + ((xi0 + q) * BK + kl) * EP_LD + io;
            *reinterpret_cast<float4*>(row) =
                make_float4(acc[q][i][1], acc[q][i][0], acc[q][i][3], acc[q][i][2]);
            *reinterpret_cast<float4*>(row + 16) =
                make_float4(acc[q][i][5], acc[q][i][4], acc[q][i][7], acc[q][i][6]);
        }
    __syncthreads();

    const int nu = nu0 + lane;
    if (nu < p.NV) {
        int t, n;
        if (p.tfast) n = nu / p.T, t = nu - n * p.T;
        else t = nu / p.N, n = nu - t * p.N;
        const int th = t / p.TW, tw = t - th * p.TW;
        const int i0 = 2 * th, j0 = 2 * tw;
        const bool okr = i0 + 1 < p.H, okc = j0 + 1 < p.W;  // odd H/W: drop extra outputs (L1155)
        const long long base = n * p.ys_n + i0 * p.ys_h + j0 * p.ys_w;
        const long long dW = p.ys_h, dN = p.ys_w;
#pragma unroll 2
        for (int r = 0; r < BK / NWARP; ++r) {
            const int kl = warp + NWARP * r, k = k0 + kl;
            if (k >= p.K) break;
            float m[16], o[4];
#pragma unroll
            for (int e = 0; e < 16; ++e) m[e] = ep[(e * BK + kl) * EP_LD + (lane ^ 1)];
            otf_2x2(m, o);
            float* yk = p.y + k * p.ys_k + base;
            yk[0] = o[0];
            if (okc) yk[dN] = o[1];
            if (okr) yk[dW] = o[2];
            if (okr && okc) yk[dW + dN] = o[3];
        }
    }
}

}  // namespace fp32
}  // namespace wino
