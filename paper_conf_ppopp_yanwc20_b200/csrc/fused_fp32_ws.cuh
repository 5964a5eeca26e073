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
// Used when both operands can be TMA boxes (N % 32 == 0 or N in {4, 8, 16}; K % 4 == 0).
//
// Small per-rank batches (batch sharding): with N | 32 a 32-nu tile
// spans 32/N consecutive image tiles, loaded as 32/N boxes (n:N, w:4, h:4, c:8).
// Split-C (SPLIT = true): when there are too few (k, nu) tiles to fill 148 SMs,
// a thread-block cluster of S CTAs shares each tile, CTA r accumulating channel
// blocks [r*NIT/S, (r+1)*NIT/S).  The output transform is linear (Eq. 8), so each
// CTA applies it to its partial M and the S partial 2x2 outputs are summed (the 4
// outputs per (k, nu) are reduced instead of the 16 M).  CTA r owns filters
// [r*64/S, (r+1)*64/S) of the tile: every CTA pushes its partial outputs of those
// filters into slot [its rank] of CTA r's receive buffer with st.async (remote,
// fire-and-forget, byte-counted on CTA r's mbarrier), and CTA r's compute warps sum
// the S slots from LOCAL shared memory in rank order 0..S-1 and store y --
// deterministic, no atomics, no global workspace.  Pull-based reads of
// the peers' buffers were measured ~4x slower (DSMEM reads queue behind the remote
// SM's LDS traffic; scripts/ws_trace.py), and so was a dedicated reducer warp in the
// producer warpgroup (its shared-memory loads queue behind the compute warps').
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
#ifndef WS_X_PREFETCH
#define WS_X_PREFETCH 0  // channel blocks of x prefetched into L2 ahead of the TMA loads (A/B knob)
#endif
#ifndef WS_XBAR
#define WS_XBAR 0  // 1: raw x gets its own stage barrier (issued before u), so the ITF need not wait for u
#endif
#ifndef WS_EPI_ROUNDS
#define WS_EPI_ROUNDS 4  // OTF rounds of the non-split epilogue: 4 (16 filters, 3-stage ring) or 2 (A/B)
#endif
constexpr int S = WS_EPI_ROUNDS == 2 ? 2 : 3;  // TMA stage ring (u 32 KB + raw x 16 KB per stage)
constexpr int SV = 2;               // V ring (16 KB each)
constexpr int REG_COMPUTE = 208, REG_PRODUCER = 88;  // 256*208 + 128*88 = 64512 <= 65536
constexpr int ITF_WARPS = 2;        // warps 9..10 (float4 along nu); warp 8 only issues TMA; 11 idle
constexpr int ER_LD = BN + 4;       // padded row of the epilogue buffer
constexpr int MAX_SPLIT = 8;        // portable cluster size
constexpr uint32_t kSplitTileBytes = BK * BN * 4 * 4;  // S slots x 64/S filters x 32 nu x 16 B

#ifdef WINO_WS_TRACE
// debug builds only: clock64 events of CTA 0 per tile (scripts/ws_trace.py)
__device__ unsigned long long g_ws_trace[8][64];
#define WS_TR(e, T) \
    do { if (blockIdx.x == 0 && (T) < 64) g_ws_trace[e][T] = clock64(); } while (0)
#else
#define WS_TR(e, T) do { } while (0)
#endif
#ifdef WINO_WS_CTATRACE
// debug builds only: %globaltimer (ns) per CTA: entry, first stage landed, last main loop done, exit
__device__ unsigned long long g_cta_trace[256][4];
__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
#define WS_CT(e) do { if (blockIdx.x < 256) g_cta_trace[blockIdx.x][e] = gtimer(); } while (0)
#else
#define WS_CT(e) do { } while (0)
#endif

// Epilogue geometry: RR accumulator rows per thread per round -> 8*RR filters per
// round, 8/RR rounds.  Without split RR = 2 (4 rounds of 16 filters, L499).  With
// split RR = 1 (8 rounds of 8) so that the whole tile's partial outputs fit: the
// rounds fill yp[64 k][4 outputs][32 nu] (32 KB), then ONE cluster exchange per
// tile (a per-round exchange is latency-bound: ~8 DSMEM round trips per tile).
template <bool SPLIT>
struct Smem {
    static constexpr int RR = SPLIT ? 1 : 8 / WS_EPI_ROUNDS;
    static constexpr int ER_KROWS = 8 * RR;
    static constexpr int ER_FLOATS = 16 * ER_KROWS * ER_LD;  // [xi][8RR k][36]
    // split receive buffer [S slots][64/S owned filters][32 nu][4 outputs] = 32 KB for any S
    static constexpr int YP_FLOATS = SPLIT ? BK * 4 * BN : 0;
    static constexpr int ep_offset = (S * STAGE_FLOATS + SV * VS_FLOATS) * 4;
    static constexpr int yp_offset = ep_offset + ER_FLOATS * 4;
    static constexpr int bar_offset = yp_offset + YP_FLOATS * 4;
    // full[S], empty[S], vfull[SV], vempty[SV], yready, yfree; then 2 ints (stream-K reduction)
    static constexpr int sk_offset = bar_offset + (2 * S + 2 * SV + 2 + (WS_XBAR ? S : 0)) * 8;
    static constexpr int bytes = sk_offset + 16;
};

// ITF loop of warps 9..10 (Sec. 4.2): raw x of every stage -> V = B^T d B in the V ring.
__device__ __forceinline__ void itf_loop(float* smem, float* vs, uint64_t* full, uint64_t* empty, uint64_t* vfull,
                                         uint64_t* vempty, int xoff, int xpos, int voff, int NIT, int first,
                                         int num_tiles, int stride, int lane) {
        int G = 0;
        for (int tile = first; tile < num_tiles; tile += stride) {
            for (int g = 0; g < NIT; ++g, ++G) {
                const int slot = G % S, vb = G % SV;
                mbar_wait(&full[slot], (G / S) & 1);
                if (G >= SV) mbar_wait(&vempty[vb], ((G / SV) - 1) & 1);
                const float* xs = smem + slot * STAGE_FLOATS + US_FLOATS + xoff;
                float* v = vs + vb * VS_FLOATS + voff;
                float d[4][16];
#pragma unroll
                for (int e = 0; e < 16; ++e) {
                    const float4 q = *reinterpret_cast<const float4*>(xs + e * xpos);
                    d[0][e] = q.x; d[1][e] = q.y; d[2][e] = q.z; d[3][e] = q.w;
                }
                float t[4][16];
#pragma unroll
                for (int j = 0; j < 4; ++j) itf_4x4(d[j], t[j]);
#pragma unroll
                for (int e = 0; e < 16; ++e)
                    *reinterpret_cast<float4*>(v + e * BC * BN) = make_float4(t[0][e], t[1][e], t[2][e], t[3][e]);
                fence_proxy_async_smem();  // generic reads of the TMA slot before its async-proxy refill
                __syncwarp();
                if (lane == 0) {
                    mbar_arrive(&empty[slot]);  // raw x of this slot consumed
                    mbar_arrive(&vfull[vb]);
                }
            }
        }
}
// Stream-K (SK = true): CTA b of G takes units [b*total/G, (b+1)*total/G) of the flattened
// (tile, channel block) space, unit = tile * NIT + g.  A tile is cut into segments at CTA
// boundaries; a segment covering the whole tile stores y.  A segment of a cut tile stores its
// partial OTF outputs (Eq. 8 is linear) in sk_ws: slot 2b if it starts inside the tile (it is
// then CTA b's first segment), slot 2b + 1 if it holds the tile's channel block 0 (CTA b's last
// segment, or its only one).  Each segment then counts itself on the tile's arrival counter
// (indexed by the CTA holding block 0); the LAST segment to arrive sums all the tile's partials in
// CTA order (deterministic) with every compute thread and stores y, and resets the counter --
// no fixup launch, no CTA ever waits for another.
// (the first total % G CTAs get one unit more; no division on the device)
__host__ __device__ __forceinline__ int sk_start(const Params& p, int b) { return b * p.sk_q + min(b, p.sk_r); }
// The pi-th segment of CTA b's range in PROCESSING order: its first segment, then its last, then the
// whole tiles in between.  Both ends of a range are (possibly) cut tiles, so every CTA handles its
// cut segments first: all pieces of a cut tile arrive early, and the reduction by the last one to
// arrive overlaps the other CTAs' whole tiles instead of adding a tail to the launch.
__device__ __forceinline__ bool sk_piece(const Params& p, int b, int pi, int& tile, int& g_lo, int& nst) {
    const int s = sk_start(p, b), e = sk_start(p, b + 1);
    if (s >= e) return false;
    const int tf = s / p.num_it, tl = (e - 1) / p.num_it;
    int t;
    if (pi == 0) {
        t = tf;
    } else if (pi == 1) {
        if (tl == tf) return false;
        t = tl;
    } else {
        t = tf + pi - 1;
        if (t >= tl) return false;
    }
    const int u0 = max(s, t * p.num_it), u1 = min(e, (t + 1) * p.num_it);
    tile = t;
    g_lo = u0 - t * p.num_it;
    nst = u1 - u0;
    return true;
}
// Stream-K cut tile: this segment's partials are in the workspace; count the segment on the tile's
// arrival counter; the last of the tile's segments sums them in CTA order and stores y.  Called by
// the 256 compute threads (named barrier 1).  sh: 2 ints of shared memory.
__device__ __noinline__ void sk_arrive(const Params& p, int tile, int k0, int nu0, int* sh, int tid) {
    // The 256 threads' partial outputs are ordered before thread 0's acq_rel atomic by the barrier
    // (release is cumulative over what thread 0 has observed); on the reducing side thread 0's
    // acquire is carried to the other threads by the second barrier.
    named_bar_sync(1, COMPUTE_THREADS);
    if (tid == 0) {
        const int t0 = tile * p.num_it, t1 = t0 + p.num_it;
        int b0 = static_cast<int>(blockIdx.x);
        while (sk_start(p, b0) > t0) --b0;  // the CTA holding channel block 0 (slot 2 b0 + 1)
        int nc = 0;                         // CTAs starting inside the tile (slots 2c)
        while (b0 + nc + 1 < static_cast<int>(gridDim.x) && sk_start(p, b0 + nc + 1) < t1) ++nc;
        const unsigned seen = atom_add_acq_rel_gpu(p.sk_flags + b0, 1u);
        const bool last = seen == static_cast<unsigned>(nc);
        if (last) p.sk_flags[b0] = 0u;  // every segment has arrived: reset for the next launch
        sh[0] = last ? b0 : -1;
        sh[1] = nc;
    }
    named_bar_sync(1, COMPUTE_THREADS);
    const int b0 = sh[0], nc = sh[1];
    if (b0 < 0) return;
    // 64 k x 32 nu (k, nu) pairs, 8 per thread, nu = lane: coalesced [slot][kl][output][nu] rows
    constexpr int PER = BK * BN / COMPUTE_THREADS;
    const int nl = tid & 31, kr = tid >> 5;
    float o[PER][4];
#pragma unroll
    for (int j = 0; j < PER; ++j) {
        const float* w = p.sk_ws + ((size_t)(2 * b0 + 1) * BK + kr + 8 * j) * (4 * BN) + nl;
#pragma unroll
        for (int q = 0; q < 4; ++q) o[j][q] = __ldcg(w + q * BN);
    }
    int c = 1;
    for (; c + 1 <= nc; c += 2) {  // two pieces' loads in flight per step; adds in CTA order (deterministic)
        float v0[PER][4], v1[PER][4];
#pragma unroll
        for (int j = 0; j < PER; ++j) {
            const float* w0 = p.sk_ws + ((size_t)(2 * (b0 + c)) * BK + kr + 8 * j) * (4 * BN) + nl;
            const float* w1 = w0 + (size_t)2 * BK * 4 * BN;
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                v0[j][q] = __ldcg(w0 + q * BN);
                v1[j][q] = __ldcg(w1 + q * BN);
            }
        }
#pragma unroll
        for (int j = 0; j < PER; ++j)
#pragma unroll
            for (int q = 0; q < 4; ++q) o[j][q] = (o[j][q] + v0[j][q]) + v1[j][q];
    }
    if (c == nc) {
#pragma unroll
        for (int j = 0; j < PER; ++j) {
            const float* w = p.sk_ws + ((size_t)(2 * (b0 + c)) * BK + kr + 8 * j) * (4 * BN) + nl;
#pragma unroll
            for (int q = 0; q < 4; ++q) o[j][q] += __ldcg(w + q * BN);
        }
    }
    const int nu = nu0 + nl;
    if (nu >= p.NV) return;
    const int t = nu / p.N, n = nu - t * p.N;
    const int th = t / p.TW, tw = t - th * p.TW;
    const int i0 = 2 * th, j0 = 2 * tw;
    const bool okr = i0 + 1 < p.H, okc = j0 + 1 < p.W;  // odd H/W (L1155)
    const size_t HWN = (size_t)p.H * p.W * p.N, dW = (size_t)p.W * p.N;
#pragma unroll
    for (int j = 0; j < PER; ++j) {
        const int k = k0 + kr + 8 * j;
        if (k >= p.K) continue;
        float* yk = p.y + (size_t)k * HWN + ((size_t)i0 * p.W + j0) * p.N + n;
        yk[0] = o[j][0];
        if (okc) yk[p.N] = o[j][1];
        if (okr) yk[dW] = o[j][2];
        if (okr && okc) yk[dW + p.N] = o[j][3];
    }
}

// BOX32: N % 32 == 0 (one x box per stage, compile-time ITF strides); else N | 32
// (32/N boxes, runtime strides -- costs the 88-register ITF warps one spill).
template <bool SPLIT, bool BOX32, bool SK = false>
__global__ void __launch_bounds__(NT, 1) fused_fp32_ws_kernel(const __grid_constant__ Params p, int num_tiles) {
    using SM = Smem<SPLIT>;
    constexpr int RR = SM::RR, ER_KROWS = SM::ER_KROWS;
    extern __shared__ __align__(1024) float smem[];
    float* const vs = smem + S * STAGE_FLOATS;
    float* const ep = reinterpret_cast<float*>(reinterpret_cast<char*>(smem) + SM::ep_offset);
    float* const yp = reinterpret_cast<float*>(reinterpret_cast<char*>(smem) + SM::yp_offset);
    uint64_t* const full = reinterpret_cast<uint64_t*>(reinterpret_cast<char*>(smem) + SM::bar_offset);
    uint64_t* const empty = full + S;
    uint64_t* const vfull = empty + S;
    uint64_t* const vempty = vfull + SV;
    uint64_t* const yready = vempty + SV;  // split: all S slots of this CTA's receive buffer landed (tx bytes)
    uint64_t* const yfree = yready + 1;    // split: every owner has consumed this CTA's slots of the last tile
    uint64_t* const xfull = WS_XBAR ? yfree + 1 : full;  // raw x landed (WS_XBAR), else shares full
    int* const sk_sh = reinterpret_cast<int*>(reinterpret_cast<char*>(smem) + SM::sk_offset);

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) WS_CT(0);
    // split-C: cluster = S consecutive CTAs sharing each tile; rank r takes channel
    // blocks [it_lo, it_hi).  Without split every CTA is its own "cluster".
    const int nsplit = SPLIT ? p.split : 1;
    const int crank = SPLIT ? static_cast<int>(cluster_ctarank()) : 0;
    // first tile / tile stride of this cluster.  Re-derived from blockIdx / gridDim at each
    // use rather than held in registers: two more live registers across the compute
    // warps' main loop change ptxas' accumulator assignment and cost ~20% more FFMA
    // register-bank conflicts (scripts/sass_bank.py: 1.14 -> 1.35 reads per FFMA).
#define WS_CID (SPLIT ? static_cast<int>(blockIdx.x) / p.split : static_cast<int>(blockIdx.x))
#define WS_NCL (SPLIT ? static_cast<int>(gridDim.x) / p.split : static_cast<int>(gridDim.x))
    const int it_lo = crank * p.num_it / nsplit, it_hi = (crank + 1) * p.num_it / nsplit;
    const int NIT = it_hi - it_lo;

    if (tid == 0) {
        tma_prefetch_desc(&p.tmx);
        tma_prefetch_desc(&p.tmu);
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            if (WS_XBAR) mbar_init(&xfull[s], 1);
            mbar_init(&empty[s], 8 + ITF_WARPS);  // 8 compute warps (u) + ITF warps (raw x)
        }
        for (int s = 0; s < SV; ++s) {
            mbar_init(&vfull[s], ITF_WARPS);
            mbar_init(&vempty[s], 8);
        }
        if (SPLIT) {
            mbar_init(yready, 1);       // one arrive.expect_tx per tile (+ S x 64/S x 512 B of st.async)
            mbar_init(yfree, nsplit);   // one arrival per owner CTA
        }
        fence_mbar_init();
    }
    if constexpr (SPLIT) {
        if (tid == 0) mbar_arrive_expect_tx(yready, kSplitTileBytes);  // tile 0's partials
        cluster_sync_all();  // peers' barriers initialised before any remote arrive / st.async
    }
    else __syncthreads();

    if (warp >= 8) {
        // ============================ producer / ITF ============================
        setmaxnreg_dec<REG_PRODUCER>();
        if (warp == 8) {
            // ---------------- TMA issue (one elected lane) ----------------
            if (lane == 0) {
                constexpr uint32_t kBytes = (US_FLOATS + XS_FLOATS) * 4;
                int G = 0;  // global stage counter across tiles
                int pi = 0;  // stream-K: segment index in processing order (sk_piece)
                for (int tile = SK ? 0 : WS_CID;;) {
                    int g_lo = it_lo, g_hi = it_hi;
                    if constexpr (SK) {
                        int nst;
                        if (!sk_piece(p, blockIdx.x, pi++, tile, g_lo, nst)) break;
                        g_hi = g_lo + nst;
                    } else if (tile >= num_tiles) {
                        break;
                    }
                    const int kb = tile % p.num_kb, nb = tile / p.num_kb;
                    const int k0 = kb * BK, nu0 = nb * BN;
                    // N % 32 == 0: the tile's 32 nu are 32 consecutive n of one image tile (one box);
                    // N | 32: 32/N consecutive image tiles, one (n:N) box each -> [box][c][pos][n]
                    const int t0 = nu0 / p.N;
                    const int n0 = nu0 - t0 * p.N;
                    const int nbox = BOX32 ? 1 : BN / p.xnb;
#if WS_X_PREFETCH > 0
                    if (BOX32) {  // x streams from HBM on first touch: warm L2 a few stages ahead
                        const int th = t0 / p.TW, tw = t0 - th * p.TW;
                        for (int g = g_lo; g < g_lo + WS_X_PREFETCH && g < g_hi; ++g)
                            tma_prefetch_l2_4d(&p.tmx, n0, 2 * tw - 1, 2 * th - 1, g * BC);
                    }
#endif
                    for (int g = g_lo; g < g_hi; ++g, ++G) {
                        const int slot = G % S;
                        if (G >= S) mbar_wait(&empty[slot], ((G / S) - 1) & 1);
                        float* us = smem + slot * STAGE_FLOATS;
                        if (WS_XBAR) {
                            mbar_arrive_expect_tx(&xfull[slot], XS_FLOATS * 4);
                            mbar_arrive_expect_tx(&full[slot], US_FLOATS * 4);
                        } else {
                            mbar_arrive_expect_tx(&full[slot], kBytes);
                            tma_load_3d(us, &p.tmu, &full[slot], k0, 0, g * BC);
                        }
#if WS_X_PREFETCH > 0
                        if (BOX32 && g + WS_X_PREFETCH < g_hi) {
                            const int th = t0 / p.TW, tw = t0 - th * p.TW;
                            tma_prefetch_l2_4d(&p.tmx, n0, 2 * tw - 1, 2 * th - 1, (g + WS_X_PREFETCH) * BC);
                        }
#endif
                        for (int b = 0; b < nbox; ++b) {
                            const int t = t0 + b;
                            const int th = t / p.TW, tw = t - th * p.TW;
                            // -1 / past the end: TMA zero fill = implicit padding (Sec. 3.5).
                            // BOX32: map (n, w, h, c) -> [c][pos][n]; small N: map (n, c, w, h)
                            // -> [pos][c][n] per box (see the ITF lane map below)
                            if (BOX32)
                                tma_load_4d(us + US_FLOATS, &p.tmx, &xfull[slot], n0, 2 * tw - 1, 2 * th - 1, g * BC);
                            else
                                tma_load_4d(us + US_FLOATS + b * (BC * 16 * p.xnb), &p.tmx, &xfull[slot], 0, g * BC,
                                            2 * tw - 1, 2 * th - 1);
                        }
                        if (WS_XBAR) tma_load_3d(us, &p.tmu, &full[slot], k0, 0, g * BC);  // u after x
                    }
                    if constexpr (!SK) tile += WS_NCL;
                }
            }
            return;
        }
        // ---------------- ITF (Sec. 4.2) on warps 9..10 ----------------
        // 256 (c, nu) tiles per stage; a thread transforms 4 consecutive nu of one
        // channel with LDS.128 / STS.128 (a quarter-warp covers one 128 B row:
        // conflict-free): lane -> (c = 4 (w - 9) + lane / 8, nu4 = lane % 8).
        if (warp == 11) return;  // idle
        // Small N (N | 32, boxes [b][pos][c][n]): the 8 lanes of a quarter-warp (one LDS.128 /
        // STS.128 wavefront) take task i = b*Q + h (Q = N/4 quads per row, h = quad) with
        // channel c = (b + j) % 8 in quarter j: raw reads hit bank group (c*Q + h) % 8 and V
        // writes (b*Q + h) % 8 -- both distinct across the 8 lanes, so conflict-free.  The map
        // comes precomputed in Params: computing it here (or calling the ITF out of line)
        // perturbs ptxas' register assignment of the compute warps' FFMA stream.
        int c, n4, xoff, xpos;
        if (BOX32) {
            c = 4 * (warp - 9) + (lane >> 3);
            n4 = 4 * (lane & 7);
            xoff = c * 16 * BN + n4;  // [c][pos][n]
            xpos = BN;
        } else {
            const int m = p.itf_map[(warp - 9) * 32 + lane];  // host-computed (wino_api.cu)
            c = m & 7;
            n4 = (m >> 3) & 31;
            xoff = m >> 8;
            xpos = BC * p.xnb;
        }
        if (SK)  // one run of this CTA's stages (the ITF does not depend on the tile)
            itf_loop(smem, vs, xfull, empty, vfull, vempty, xoff, xpos, c * BN + n4,
                     sk_start(p, blockIdx.x + 1) - sk_start(p, blockIdx.x),
                     0, 1, 1, lane);
        else if (BOX32)
            itf_loop(smem, vs, xfull, empty, vfull, vempty, xoff, xpos, c * BN + n4, NIT, WS_CID, num_tiles, WS_NCL,
                     lane);
        else
            itf_loop(smem, vs, xfull, empty, vfull, vempty, xoff, xpos, c * BN + n4, NIT, WS_CID, num_tiles, WS_NCL,
                     lane);
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
    int pi = 0;  // stream-K: segment index in processing order (sk_piece), live across the main loop
    for (int tile = SK ? 0 : WS_CID;; tile += SK ? 0 : WS_NCL) {
        int nst = NIT;     // channel blocks of this tile handled here
        int sk_slot = -1;  // stream-K: -1 whole tile -> y; else the workspace slot of this cut segment:
                           // 2b (starts inside the tile) or 2b + 1 (holds the tile's channel block 0)
        if constexpr (SK) {
            int g_lo;
            if (!sk_piece(p, blockIdx.x, pi++, tile, g_lo, nst)) break;
            if (nst != p.num_it) sk_slot = 2 * static_cast<int>(blockIdx.x) + (g_lo > 0 ? 0 : 1);
        } else if (tile >= num_tiles) {
            break;
        }
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
#ifdef WINO_WS_TRACE
        const int Ttr = (tile - WS_CID) / WS_NCL;
        if (tid == 0) WS_TR(0, Ttr);
#endif
        for (int g = 0; g < nst; ++g, ++G) {
            const int slot = G % S, vb = G % SV;
            mbar_wait(&full[slot], (G / S) & 1);
            mbar_wait(&vfull[vb], (G / SV) & 1);
#ifdef WINO_WS_CTATRACE
            if (tid == 0 && G == 0) WS_CT(1);
#endif
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
            fence_proxy_async_smem();  // generic reads of the TMA slot before its async-proxy refill (7.6)
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(&empty[slot]);  // u of this slot consumed
                mbar_arrive(&vempty[vb]);
            }
        }

        if (tid == 0) WS_CT(2);
        // ---- OTF (Sec. 4.4) through the epilogue buffer ----
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
#ifdef WINO_WS_TRACE
        if (!SPLIT && tid == 0) WS_TR(1, (tile - WS_CID) / WS_NCL);
#endif
        if constexpr (!SPLIT) {
            // 4 rounds of 16 filters (the paper's 4-round OTF, L499).  NOTE: ptxas' register
            // assignment of the accumulators (and so the FFMA bank conflicts of the main
            // loop) is sensitive to this code's shape: keep it as is.
#pragma unroll
            for (int rd = 0; rd < 8 / RR; ++rd) {
                // round rd stores accumulator rows i = 4*rd_hi + RR*rd_lo + ii (ii < RR) of half rd_hi:
                // filters kl = fo + (i&3) + 32*(i>>2); in the buffer row = (fo>>2)*RR + ii
                // (RR = 2: 4 rounds of 16 filters, the paper's 4-round OTF, L499)
                const int rd_hi = RR == 2 ? (rd >> 1) : rd, rd_lo = RR == 2 ? (rd & 1) : 0;
                named_bar_sync(1, COMPUTE_THREADS);  // previous round's readers are done
#pragma unroll
                for (int q = 0; q < 2; ++q)
#pragma unroll
                    for (int ii = 0; ii < RR; ++ii) {
                        const int i = rd_hi * 4 + rd_lo * RR + ii;
                        const int r = (fo >> 2) * RR + ii;
                        float* row = ep + ((xi0 + q) * ER_KROWS + r) * ER_LD + io;
                        *reinterpret_cast<float4*>(row) =
                            make_float4(acc[q][i][1], acc[q][i][0], acc[q][i][3], acc[q][i][2]);
                        *reinterpret_cast<float4*>(row + 16) =
                            make_float4(acc[q][i][5], acc[q][i][4], acc[q][i][7], acc[q][i][6]);
                    }
                named_bar_sync(1, COMPUTE_THREADS);
                // branch-free reads (all 2 RR x 16 LDS issue back to back), predicated stores; one
                // store pattern for y and for a cut segment's workspace slot [slot][kl][output][nu]
                float m[RR][16], o[RR][4];
#pragma unroll
                for (int h = 0; h < RR; ++h)
#pragma unroll
                    for (int e = 0; e < 16; ++e) m[h][e] = ep[(e * ER_KROWS + warp + 8 * h) * ER_LD + (lane ^ 1)];
#pragma unroll
                for (int h = 0; h < RR; ++h) otf_2x2(m[h], o[h]);
                const bool cut = SK && sk_slot >= 0;
#pragma unroll
                for (int h = 0; h < RR; ++h) {
                    const int r = warp + 8 * h;  // buffer row 0..8RR-1
                    const int kl = (r / RR) * 4 + rd_lo * RR + (r % RR) + rd_hi * 32;
                    if (nu < p.NV && k0 + kl < p.K) {
                        float* d = cut ? p.sk_ws + ((size_t)sk_slot * BK + kl) * (4 * BN) + lane
                                       : p.y + (size_t)(k0 + kl) * HWN + base;
                        d[0] = o[h][0];
                        if (cut || okc) d[cut ? BN : p.N] = o[h][1];
                        if (cut || okr) d[cut ? 2 * BN : dW] = o[h][2];
                        if (cut || (okr && okc)) d[cut ? 3 * BN : dW + p.N] = o[h][3];
                    }
                }
            }
            if (SK && sk_slot >= 0) sk_arrive(p, tile, k0, nu0, sk_sh, tid);
#ifdef WINO_WS_TRACE
            if (tid == 0) WS_TR(3, (tile - WS_CID) / WS_NCL);
#endif
        } else {
            // 8 rounds of 8 filters: round rd stores accumulator row i = rd (filters
            // kl = fo + (rd&3) + 32*(rd>>2)) into buffer row fo>>2; the OTF of buffer row
            // `warp` (filter 4*warp + (rd&3) + 32*(rd>>2)) goes to yp[kl][o][nu]
            // peers done reading this CTA's yp of its previous tile (T = this CTA's tile count
            // so far, re-derived rather than kept live across the main loop)
            const int T = (tile - WS_CID) / WS_NCL;
            if (tid == 0) WS_TR(1, T);
            if (T > 0) mbar_wait_cluster(yfree, (T - 1) & 1);  // owners consumed our previous partials
            if (tid == 0) WS_TR(2, T);
            const int rows = BK / nsplit;
            const uint32_t yb = smem_u32(yp), ybar = smem_u32(yready);
#pragma unroll
            for (int rd = 0; rd < 8; ++rd) {
                named_bar_sync(1, COMPUTE_THREADS);
#pragma unroll
                for (int q = 0; q < 2; ++q) {
                    float* row = ep + ((xi0 + q) * ER_KROWS + (fo >> 2)) * ER_LD + io;
                    *reinterpret_cast<float4*>(row) =
                        make_float4(acc[q][rd][1], acc[q][rd][0], acc[q][rd][3], acc[q][rd][2]);
                    *reinterpret_cast<float4*>(row + 16) =
                        make_float4(acc[q][rd][5], acc[q][rd][4], acc[q][rd][7], acc[q][rd][6]);
                }
                named_bar_sync(1, COMPUTE_THREADS);
                const int kl = 4 * warp + (rd & 3) + 32 * (rd >> 2);
                float m[16], o[4];
#pragma unroll
                for (int e = 0; e < 16; ++e) m[e] = ep[(e * ER_KROWS + warp) * ER_LD + (lane ^ 1)];
                otf_2x2(m, o);
                // -> slot [crank] of the owner of filter kl: [slot][kl % rows][nu][4]
                const int owner = kl / rows;
                const uint32_t dst = yb + (uint32_t)((((crank * rows + kl - owner * rows) * BN) + lane) * 16);
                st_async4(mapa_shared(dst, owner), o[0], o[1], o[2], o[3], mapa_shared(ybar, owner));
            }
        }
        if constexpr (SPLIT) {
            // all S partials of this CTA's filters landed -> sum the S slots and store.  Warp w
            // takes owned filters w + 8i: always 8 (filter, slot) pairs per thread (64/S filters
            // x S slots / 8 warps), all 8 loads issued before the first add; the slots are
            // added by a fixed pairwise tree ((s0+s1)+(s2+s3))+... (deterministic).
            const int T = (tile - WS_CID) / WS_NCL;
            mbar_wait_cluster(yready, T & 1);
            if (tid == 0) WS_TR(5, T);
            {
                const int rows = BK / nsplit, lg = nsplit == 2 ? 1 : (nsplit == 4 ? 2 : 3);
                const float4* yb4 = reinterpret_cast<const float4*>(yp) + lane;
                float4 v[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) {  // j = i * S + q: filter warp + 8i, slot q
                    const int q = j & (nsplit - 1), r = warp + 8 * (j >> lg);
                    v[j] = yb4[(q * rows + r) * BN];
                }
                auto add4 = [](float4& a, const float4& b) { a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w; };
#pragma unroll
                for (int j = 0; j < 8; j += 2) add4(v[j], v[j + 1]);
                if (nsplit >= 4) {
#pragma unroll
                    for (int j = 0; j < 8; j += 4) add4(v[j], v[j + 2]);
                }
                if (nsplit >= 8) add4(v[0], v[4]);
                if (nu < p.NV) {
#pragma unroll
                    for (int j = 0; j < 8; ++j) {
                        if (j & (nsplit - 1)) continue;
                        const int k = k0 + crank * rows + warp + 8 * (j >> lg);
                        if (k >= p.K) continue;
                        float* yk = p.y + (size_t)k * HWN + base;
                        yk[0] = v[j].x;
                        if (okc) yk[p.N] = v[j].y;
                        if (okr) yk[dW] = v[j].z;
                        if (okr && okc) yk[dW + p.N] = v[j].w;
                    }
                }
            }
            fence_proxy_async_smem();  // generic reads of the slots before the peers' next st.async into them
            named_bar_sync(1, COMPUTE_THREADS);  // every slot consumed
            if (warp == 0) {
                if (lane == 0) mbar_arrive_expect_tx(yready, kSplitTileBytes);  // next tile's partials
                if (lane < nsplit) mbar_arrive_cluster(mapa_shared(smem_u32(yfree), lane));
            }
            if (tid == 0) WS_TR(6, T);
#ifdef WINO_WS_TRACE
            if (tid == 0) WS_TR(3, (tile - WS_CID) / WS_NCL);
#endif
        }
    }
    if (tid == 0) WS_CT(3);
    if constexpr (SPLIT) {
        // peers may still be reading this CTA's yp: exit only after they all signalled
        const int T = num_tiles > WS_CID ? (num_tiles - WS_CID + WS_NCL - 1) / WS_NCL : 0;  // tiles done
        if (T > 0) mbar_wait_cluster(yfree, (T - 1) & 1);
    }
}

#undef WS_CID
#undef WS_NCL

}  // namespace fp32ws
}  // namespace wino
