// fused_fp32_ml.cuh -- several independent layers in ONE persistent stream-K launch of the
// warp-specialised FP32 kernel (same method, tile, pipeline, FFMA micro-kernel and OTF as
// fused_fp32_ws.cuh; Yan, Wang & Chu Sec. 3-4, Alg. 1).
//
// The (tile, channel block) units of every layer are concatenated and cut into one contiguous
// range per CTA (stream-K over the whole step).  The host cuts on a WORK model, not on units
// (ml_cut in wino_api.cu): a unit costs more when N | 32 (32/N TMA boxes of N-float rows per
// stage) and every tile adds one OTF epilogue, so a layer with few channels per tile (conv2: 8
// blocks) or a small batch shard is not under-charged.  Consequences for a step of L layers:
//   * one pipeline fill and one tail per step instead of one per layer (a batch-sharded rank
//     runs each layer for only 10-40 us);
//   * a CTA has at most two cut tiles in the whole step (one at each end of its range) instead
//     of up to two per layer;
//   * layers may differ in every dimension, in N % 32 == 0 vs N | 32 (x box mode, per layer at
//     run time) and in C, K (per-layer TMA maps).
// Cut tiles are reduced inside the kernel exactly as in fused_fp32_ws.cuh (the last piece to
// arrive sums the pieces' partial outputs in CTA order; no fixup launch).  Every CTA's range is
// non-empty, so the pieces of a cut tile belong to consecutive CTAs.
#pragma once
#include <cuda.h>

#include <cstdint>

#include "fused_fp32_ws.cuh"
#include "wino_ptx.cuh"
#include "wino_transforms.cuh"

namespace wino {
namespace fp32ml {

using fp32::BC;
using fp32::BK;
using fp32::BN;
using fp32::STAGE_FLOATS;
using fp32::US_FLOATS;
using fp32::VS_FLOATS;
using fp32::XS_FLOATS;
using fp32ws::COMPUTE_THREADS;
using fp32ws::ER_LD;
using fp32ws::ITF_WARPS;
using fp32ws::NT;
using fp32ws::REG_COMPUTE;
using fp32ws::REG_PRODUCER;
using fp32ws::S;
using fp32ws::SV;
using SM = fp32ws::Smem<false>;

// Piece records: the TMA producer computes each segment (ml_piece) and publishes {u0, u1, l} in a
// ring of PR records before arming the segment's first stage; the ITF and compute warps read it
// after their wait on that stage's full barrier (the producer's arrive releases the store), so
// neither runs the piece arithmetic (dependent parameter loads and divisions: ~1.5 us per tile
// when every warp re-derived it).  The producer is at most S stages -- so S segments -- ahead of
// the slowest consumer, so a record is rewritten only after its segment is finished.
constexpr int PR = 4;
static_assert(PR > fp32ws::S, "piece ring must outlive the TMA ring");
// The record also carries what the epilogue needs of the layer, so the compute warps never index
// the parameter block with a run-time layer number (dependent constant-cache loads, ~12 % of a
// shared tile's epilogue samples).
struct __align__(16) PieceRec {
    int u0, u1, l, sk_slot;  // global units [u0, u1) of layer l; cut-segment workspace slot or -1
    int k0, nu0, K, NV;      // tile origin, layer K and NV
    int N, TW, H, W;
    float* y;
    int pad[2];
};
constexpr int REC_OFFSET = (SM::bytes + 15) / 16 * 16;
constexpr int SMEM_BYTES = REC_OFFSET + PR * static_cast<int>(sizeof(PieceRec));

constexpr int MAX_LAYERS = 4;
constexpr int MAX_GRID = 160;  // CTAs of one launch (B200: 148 SMs, one CTA each)

struct __align__(64) Layer {
    CUtensorMap tmx;  // x: (N, W, H, C) box (32, 4, 4, 8) when N % 32 == 0, else (n, c, w, h) box (N, 8, 4, 4)
    CUtensorMap tmu;  // u: (K, 16, C) box (64, 16, 8)
    CUtensorMap tmv;  // vmode: V = B^T d B of every tile, (NV, C, 16) box (32, 8, 16) -> the V ring as is
    float* __restrict__ y;
    int N, C, H, W, K;
    int TW, NV, num_kb, num_it, xnb;
    int vg, vr, vlc;   // nu-tile order (ml_nu_tile): ~vg CTAs share the layer, vr nu-tiles each
    int ng_s;          // nu-tiles in that order; the dynamic tail's nu-tiles [ng_s, ng) keep their own index
    int unit0;         // global index of the layer's first unit (tile * num_it + g)
    int vmode;         // 1: V comes transformed from ml_itf_kernel (small N), the ITF warps idle
    int itf_map[64];   // N | 32: ITF task map of the 64 ITF lanes (as fp32::Params::itf_map)
};

struct __align__(64) Params {
    Layer L[MAX_LAYERS];
    int nl;
    // CTA b's units are [start[b], start[b+1]): cut on the host by a work model (unit cost per x
    // box mode + one epilogue per tile), strictly increasing (no empty range)
    int start[MAX_GRID + 1];
    float* __restrict__ sk_ws;          // 2 partial-tile slots per CTA
    unsigned* __restrict__ sk_flags;    // one arrival counter per CTA (zero between launches)
    // Dynamic tail: units [start[grid], start[grid] + dyn_n * dyn_nu) are dyn_n whole tiles of the last
    // layer that the producers grab one at a time from dyn_ctr[0] after their static range (per-CTA
    // speed differences -- DRAM latency, cut tiles -- no longer set the launch's tail); dyn_ctr[1]
    // counts the producers done, the last one resets both words (zero between launches).
    int dyn_n, dyn_nu;
    unsigned* __restrict__ dyn_ctr;
};

__device__ __forceinline__ int layer_of(const Params& p, int u) {
    int l = 0;
    while (l + 1 < p.nl && p.L[l + 1].unit0 <= u) ++l;
    return l;
}

// Order of a layer's nu-tiles along its unit sequence.  Each CTA of the persistent launch walks its
// own contiguous range, so in natural order the ~vg CTAs sharing a layer would stream vg distant
// regions of x at once, and the Winograd tiles' overlap (Sec. 3.5: neighbouring 4x4 input patches
// share 2 rows / columns) would be re-read from DRAM after eviction (whole ResNet step in one launch:
// 1.21 GB of DRAM reads for 310 MB of x and u).  Instead sequence position s (column s / vr ~ one
// CTA's share, row s % vr ~ its step) maps to nu-tile row * vg + column, so that at each step the
// CTAs work on ~vg neighbouring nu-tiles, as a one-tile-per-CTA grid would (step reads 0.57 GB;
// DESIGN.md 7.11).  A bijection on [0, ng_s) with ng_s = (vg - 1) * vr + vlc, 1 <= vlc <= vr.
__device__ __forceinline__ int ml_nu_tile(const Layer& L, int s) {
    if (s >= L.ng_s) return s;  // dynamic tail: consecutive grabs take neighbouring nu-tiles
    const int c = s / L.vr, r = s - c * L.vr;
    return r < L.vlc ? r * L.vg + c : L.vlc * L.vg + (r - L.vlc) * (L.vg - 1) + c;
}

// The pi-th segment of CTA b's range in processing order: its first segment, its last, then the
// whole tiles in between (across layers) -- as fp32ws::sk_piece, re-derived from (b, pi) at every
// use so that nothing but pi stays live across the compute warps' main loop.
// Out: layer l, global units [u0, u1) (one tile's channel blocks).  false: no such segment.
__device__ __forceinline__ bool ml_piece(const Params& p, int b, int pi, int& l, int& u0, int& u1) {
    const int s = p.start[b], e = p.start[b + 1];
    const int lf = layer_of(p, s);
    const int nf = p.L[lf].num_it, bf = p.L[lf].unit0;
    const int fe = min(bf + ((s - bf) / nf + 1) * nf, e);  // end of the first segment
    if (pi == 0) {
        l = lf;
        u0 = s;
        u1 = fe;
        return true;
    }
    if (fe >= e) return false;
    const int ll = layer_of(p, e - 1);
    const int nl_ = p.L[ll].num_it, bl = p.L[ll].unit0;
    const int ls = bl + ((e - 1 - bl) / nl_) * nl_;  // start of the last segment (>= fe: a tile start)
    if (pi == 1) {
        l = ll;
        u0 = ls;
        u1 = e;
        return true;
    }
    int m = pi - 2;
    for (int k = layer_of(p, fe); k <= ll; ++k) {  // whole tiles in [fe, ls), layer by layer
        const int n_k = p.L[k].num_it;
        const int a = max(fe, p.L[k].unit0);
        const int z = k + 1 < p.nl ? min(ls, p.L[k + 1].unit0) : ls;
        const int nt = z > a ? (z - a) / n_k : 0;
        if (m < nt) {
            l = k;
            u0 = a + m * n_k;
            u1 = u0 + n_k;
            return true;
        }
        m -= nt;
    }
    return false;
}

// cut tile of layer l starting at global unit t0: count this piece; the last one to arrive sums
// all pieces in CTA order and stores y (as fp32ws::sk_arrive; called by the 256 compute threads)
__device__ __noinline__ void ml_arrive(const Params& p, int l, int t0, int k0, int nu0, int* sh, int tid) {
    const Layer& L = p.L[l];
    named_bar_sync(1, COMPUTE_THREADS);
    if (tid == 0) {
        const int t1 = t0 + L.num_it;
        int b0 = static_cast<int>(blockIdx.x);
        while (p.start[b0] > t0) --b0;  // the CTA holding channel block 0 (slot 2 b0 + 1)
        int nc = 0;                     // CTAs starting inside the tile (slots 2c)
        while (b0 + nc + 1 < static_cast<int>(gridDim.x) && p.start[b0 + nc + 1] < t1) ++nc;
        const unsigned seen = atom_add_acq_rel_gpu(p.sk_flags + b0, 1u);
        const bool last = seen == static_cast<unsigned>(nc);
        if (last) p.sk_flags[b0] = 0u;
        sh[0] = last ? b0 : -1;
        sh[1] = nc;
    }
    named_bar_sync(1, COMPUTE_THREADS);
    const int b0 = sh[0], nc = sh[1];
    if (b0 < 0) return;
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
    for (; c + 1 <= nc; c += 2) {
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
    if (nu >= L.NV) return;
    const int t = nu / L.N, n = nu - t * L.N;
    const int th = t / L.TW, tw = t - th * L.TW;
    const int i0 = 2 * th, j0 = 2 * tw;
    const bool okr = i0 + 1 < L.H, okc = j0 + 1 < L.W;  // odd H/W (L1155)
    const size_t HWN = (size_t)L.H * L.W * L.N, dW = (size_t)L.W * L.N;
#pragma unroll
    for (int j = 0; j < PER; ++j) {
        const int k = k0 + kr + 8 * j;
        if (k >= L.K) continue;
        float* yk = L.y + (size_t)k * HWN + ((size_t)i0 * L.W + j0) * L.N + n;
        yk[0] = o[j][0];
        if (okc) yk[L.N] = o[j][1];
        if (okr) yk[dW] = o[j][2];
        if (okr && okc) yk[dW + L.N] = o[j][3];
    }
}

// Input transform of the vmode layers ahead of the fused launch (Sec. 4.2's ITF, Eq. 6, with the
// expression tree of itf_4x4 so V is bit-identical to the ITF warps'): thread (row r of V, c, 4
// consecutive nu) reads the two rows of its 4x4 patch that row r of B^T combines, as float4 along n
// (N % 4 == 0; zero outside the image = the implicit padding of Sec. 3.5), and writes
// V[4r..4r+3][c][nu..nu+3] as float4 -- a warp stores 512 contiguous bytes per xi.
struct ItfJob {
    const float* __restrict__ x;
    float* __restrict__ v;
    int N, C, H, W, TW, NV;
    int first;  // first thread index of this job (C * NV / 4 threads per V row, blockIdx.y = row)
};
struct ItfJobs {
    ItfJob j[MAX_LAYERS];
    int n;
    int total;
};

__global__ void __launch_bounds__(256) ml_itf_kernel(const __grid_constant__ ItfJobs p) {
    const int row = blockIdx.y;  // row of V = B^T row: (d[i0] - d[i1]) for rows 0, 2, 3, (d[i0] + d[i1]) for row 1
    const int i0 = row == 0 ? 0 : (row == 2 ? 2 : 1), i1 = row == 0 ? 2 : (row == 2 ? 1 : (row == 1 ? 2 : 3));
    for (int i = blockIdx.x * 256 + threadIdx.x; i < p.total; i += gridDim.x * 256) {
        int a = 0;
        while (a + 1 < p.n && p.j[a + 1].first <= i) ++a;
        const ItfJob& J = p.j[a];
        const int nq = J.NV >> 2, r = i - J.first;
        const int c = r / nq, nu = 4 * (r - c * nq);
        const int t = nu / J.N, n = nu - t * J.N;
        const int th = t / J.TW, tw = t - th * J.TW;
        const int ha = 2 * th - 1 + i0, hb = 2 * th - 1 + i1, w0 = 2 * tw - 1;
        const float* xa = J.x + ((c * J.H + ha) * J.W + w0) * J.N + n;  // < 2^31 floats (kMaxElems)
        const float* xb = xa + (i1 - i0) * J.W * J.N;
        const bool oka = ha >= 0 && ha < J.H, okb = hb >= 0 && hb < J.H;
        float4 tr[4];  // row `row` of B^T d
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const bool okw = w0 + j >= 0 && w0 + j < J.W;
            float4 d0 = make_float4(0.f, 0.f, 0.f, 0.f), d1 = d0;
            if (okw && oka) d0 = __ldg(reinterpret_cast<const float4*>(xa + j * J.N));
            if (okw && okb) d1 = __ldg(reinterpret_cast<const float4*>(xb + j * J.N));
            tr[j] = row == 1 ? make_float4(d0.x + d1.x, d0.y + d1.y, d0.z + d1.z, d0.w + d1.w)
                             : make_float4(d0.x - d1.x, d0.y - d1.y, d0.z - d1.z, d0.w - d1.w);
        }
        auto sub = [](float4 u, float4 w) { return make_float4(u.x - w.x, u.y - w.y, u.z - w.z, u.w - w.w); };
        auto add = [](float4 u, float4 w) { return make_float4(u.x + w.x, u.y + w.y, u.z + w.z, u.w + w.w); };
        const size_t plane = static_cast<size_t>(J.C) * J.NV;
        float* vo = J.v + 4 * row * plane + static_cast<size_t>(c) * J.NV + nu;
        __stcg(reinterpret_cast<float4*>(vo), sub(tr[0], tr[2]));
        __stcg(reinterpret_cast<float4*>(vo + plane), add(tr[1], tr[2]));
        __stcg(reinterpret_cast<float4*>(vo + 2 * plane), sub(tr[2], tr[1]));
        __stcg(reinterpret_cast<float4*>(vo + 3 * plane), sub(tr[1], tr[3]));
    }
}

#ifdef WINO_WS_CTATRACE
__device__ unsigned long long g_ml_piece_trace[4][96][4];  // CTAs 0, 40, 80, 120: per piece t0, loop end, epi end, nst
#define ML_PT(pi, e, v) do { const int cs_ = blockIdx.x % 40 == 0 ? blockIdx.x / 40 : -1; \
    if (cs_ >= 0 && cs_ < 4 && (pi) < 96) g_ml_piece_trace[cs_][pi][e] = (v); } while (0)
#define ML_CT(e, v) do { if (blockIdx.x < 256) fp32ws::g_cta_trace[blockIdx.x][e] = (v); } while (0)
#else
#define ML_PT(pi, e, v) do { } while (0)
#define ML_CT(e, v) do { } while (0)
#endif

__global__ void __launch_bounds__(NT, 1) fused_fp32_ml_kernel(const __grid_constant__ Params p) {
    constexpr int RR = SM::RR, ER_KROWS = SM::ER_KROWS;
    extern __shared__ __align__(1024) float smem[];
    float* const vs = smem + S * STAGE_FLOATS;
    float* const ep = reinterpret_cast<float*>(reinterpret_cast<char*>(smem) + SM::ep_offset);
    uint64_t* const full = reinterpret_cast<uint64_t*>(reinterpret_cast<char*>(smem) + SM::bar_offset);
    uint64_t* const empty = full + S;
    uint64_t* const vfull = empty + S;
    uint64_t* const vempty = vfull + SV;
    int* const sk_sh = reinterpret_cast<int*>(reinterpret_cast<char*>(smem) + SM::sk_offset);
    PieceRec* const rec = reinterpret_cast<PieceRec*>(reinterpret_cast<char*>(smem) + REC_OFFSET);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
#ifdef WINO_WS_CTATRACE
    if (tid == 0) ML_CT(0, fp32ws::gtimer());
#endif

    if (tid == 0) {
        for (int l = 0; l < p.nl; ++l) {
            tma_prefetch_desc(p.L[l].vmode ? &p.L[l].tmv : &p.L[l].tmx);
            tma_prefetch_desc(&p.L[l].tmu);
        }
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
                // L2 priority: u is re-read by every tile of its layer (y is stored with .cs)
                const uint64_t pol_keep = l2_policy_evict_last();
                int G = 0;
                int l, u0, u1;
                bool dyn = false;  // past the static range: grabbing whole tiles of the dynamic tail
                for (int pi = 0;; ++pi) {
                    if (!dyn && !ml_piece(p, blockIdx.x, pi, l, u0, u1)) dyn = true;
                    if (dyn) {
                        const unsigned t = p.dyn_n > 0 ? atomicAdd(p.dyn_ctr, 1u) : 0u;
                        if (static_cast<int>(t) >= p.dyn_n) {
                            if (p.dyn_n > 0 && atomicAdd(p.dyn_ctr + 1, 1u) == gridDim.x - 1) {
                                p.dyn_ctr[0] = 0u;  // every producer made its last grab: reset for the next call
                                p.dyn_ctr[1] = 0u;
                            }
                            // terminal record, published through one empty stage: the consumers stop
                            const int slot = G % S;
                            if (G >= S) mbar_wait(&empty[slot], ((G / S) - 1) & 1);
                            rec[pi % PR].l = -1;
                            mbar_arrive(&full[slot]);
                            break;
                        }
                        l = p.nl - 1;
                        u0 = p.start[gridDim.x] + static_cast<int>(t) * p.dyn_nu;
                        u1 = u0 + p.dyn_nu;
                    }
                    const Layer& L = p.L[l];
                    const int lu = u0 - L.unit0;
                    const int tile = lu / L.num_it, g_lo = lu - tile * L.num_it, g_hi = g_lo + (u1 - u0);
                    const int kb = tile % L.num_kb, nb = tile / L.num_kb;
                    const int k0 = kb * BK, nu0 = ml_nu_tile(L, nb) * BN;
                    if (G >= S) mbar_wait(&empty[G % S], ((G / S) - 1) & 1);  // (re-checked below: free)
                    PieceRec& R = rec[pi % PR];
                    R.u0 = u0;
                    R.u1 = u1;
                    R.l = l;
                    R.sk_slot = u1 - u0 == L.num_it ? -1 : 2 * static_cast<int>(blockIdx.x) + (g_lo > 0 ? 0 : 1);
                    R.k0 = k0;
                    R.nu0 = nu0;
                    R.K = L.K;
                    R.NV = L.NV;
                    R.N = L.N;
                    R.TW = L.TW;
                    R.H = L.H;
                    R.W = L.W;
                    R.y = L.y;
                    const int t0 = nu0 / L.N, n0 = nu0 - t0 * L.N;
                    const bool box32 = L.xnb == BN;
                    const int nbox = box32 ? 1 : BN / L.xnb;
                    if (L.vmode) {  // u into the stage, V (16 KB, 128 B rows) straight into the V ring
                        for (int g = g_lo; g < g_hi; ++g, ++G) {
                            const int slot = G % S, vb = G % SV;
                            if (G >= S) mbar_wait(&empty[slot], ((G / S) - 1) & 1);
                            float* us = smem + slot * STAGE_FLOATS;
                            mbar_arrive_expect_tx(&full[slot], US_FLOATS * 4);
                            tma_load_3d_hint(us, &L.tmu, &full[slot], k0, 0, g * BC, pol_keep);
                            if (G >= SV) mbar_wait(&vempty[vb], ((G / SV) - 1) & 1);
                            mbar_arrive_expect_tx(&vfull[vb], VS_FLOATS * 4);
                            tma_load_3d(vs + vb * VS_FLOATS, &L.tmv, &vfull[vb], nu0, g * BC, 0);
                            mbar_arrive(&vfull[vb]);  // vfull counts ITF_WARPS = 2 arrivals
                        }
                        continue;
                    }
                    for (int g = g_lo; g < g_hi; ++g, ++G) {
                        const int slot = G % S;
                        if (G >= S) mbar_wait(&empty[slot], ((G / S) - 1) & 1);
                        float* us = smem + slot * STAGE_FLOATS;
                        mbar_arrive_expect_tx(&full[slot], kBytes);
                        tma_load_3d_hint(us, &L.tmu, &full[slot], k0, 0, g * BC, pol_keep);
                        for (int b = 0; b < nbox; ++b) {
                            const int t = t0 + b;
                            const int th = t / L.TW, tw = t - th * L.TW;
                            // -1 / past the end: TMA zero fill = implicit padding (Sec. 3.5)
                            float* dst = us + US_FLOATS + (box32 ? 0 : b * (BC * 16 * L.xnb));
                            const int c0 = box32 ? n0 : 0, c1 = box32 ? 2 * tw - 1 : g * BC;
                            const int c2 = box32 ? 2 * th - 1 : 2 * tw - 1, c3 = box32 ? g * BC : 2 * th - 1;
                            tma_load_4d(dst, &L.tmx, &full[slot], c0, c1, c2, c3);
                        }
                    }
                }
            }
            return;
        }
        if (warp == 11) return;  // idle
        // ---------------- ITF (Sec. 4.2) on warps 9..10 ----------------
        // lane map per layer: N % 32 == 0 -> (c = 4 (w - 9) + lane / 8, nu4 = lane % 8) on [c][pos][n];
        // N | 32 -> the host-computed conflict-free map of fp32::Params::itf_map on [box][pos][c][n]
        int G = 0;
        for (int pi = 0;; ++pi) {
            mbar_wait(&full[G % S], (G / S) & 1);  // the segment's first stage: its record is published
            if (rec[pi % PR].l < 0) break;         // terminal record (no stage behind it)
            const int u0 = rec[pi % PR].u0, u1 = rec[pi % PR].u1;
            const Layer& L = p.L[rec[pi % PR].l];
            if (L.vmode) {  // no raw x: only keep the stage hand-off (the producer waits on our arrival)
                for (int g = u0; g < u1; ++g, ++G) {
                    mbar_wait(&full[G % S], (G / S) & 1);
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&empty[G % S]);
                }
                continue;
            }
            int c, n4, xoff, xpos;
            if (L.xnb == BN) {
                c = 4 * (warp - 9) + (lane >> 3);
                n4 = 4 * (lane & 7);
                xoff = c * 16 * BN + n4;
                xpos = BN;
            } else {
                const int m = L.itf_map[(warp - 9) * 32 + lane];
                c = m & 7;
                n4 = (m >> 3) & 31;
                xoff = m >> 8;
                xpos = BC * L.xnb;
            }
            const int voff = c * BN + n4;
            for (int g = u0; g < u1; ++g, ++G) {
                const int slot = G % S, vb = G % SV;
                mbar_wait(&full[slot], (G / S) & 1);
                if (G >= SV) mbar_wait(&vempty[vb], ((G / SV) - 1) & 1);
                const float* xs = smem + slot * STAGE_FLOATS + US_FLOATS + xoff;
                float* v = vs + vb * VS_FLOATS + voff;
                float d[4][16];
#pragma unroll
                for (int e = 0; e < 16; ++e) {
                    const float4 q = *reinterpret_cast<const float4*>(xs + e * xpos);
                    d[0][e] = q.x;
                    d[1][e] = q.y;
                    d[2][e] = q.z;
                    d[3][e] = q.w;
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
                    mbar_arrive(&empty[slot]);
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
    for (int pi = 0;; ++pi) {
        mbar_wait(&full[G % S], (G / S) & 1);  // the segment's first stage: its record is published
        if (rec[pi % PR].l < 0) break;         // terminal record (no stage behind it)
        const int nst = rec[pi % PR].u1 - rec[pi % PR].u0;
#ifdef WINO_WS_CTATRACE
        if (tid == 0) { ML_PT(pi, 0, fp32ws::gtimer()); ML_PT(pi, 3, nst); }
#endif
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
        for (int g = 0; g < nst; ++g, ++G) {
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
            fence_proxy_async_smem();  // generic reads of the TMA slot before its async-proxy refill (7.6)
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(&empty[slot]);
                mbar_arrive(&vempty[vb]);
            }
        }

#ifdef WINO_WS_CTATRACE
        if (tid == 0) ML_PT(pi, 1, fp32ws::gtimer());
#endif
        // ---- OTF (Sec. 4.4): 4 rounds of 16 filters through the epilogue buffer (L499) ----
        const PieceRec& R = rec[pi % PR];
        // -1: whole tile -> y; else this cut segment's workspace slot: 2b (starts inside the
        // tile) or 2b + 1 (holds the tile's channel block 0)
        const int sk_slot = R.sk_slot;
        const int k0 = R.k0, nu0 = R.nu0, LK = R.K, LN = R.N, LNV = R.NV, LH = R.H, LW = R.W;
        float* const Ly = R.y;
        const int nu = nu0 + lane;
        const bool nu_ok = nu < LNV;
        int n = 0, i0 = 0, j0 = 0;
        if (nu_ok) {
            const int t = nu / LN;
            n = nu - t * LN;
            const int th = t / R.TW, tw = t - th * R.TW;
            i0 = 2 * th;
            j0 = 2 * tw;
        }
        const bool okr = i0 + 1 < LH, okc = j0 + 1 < LW;  // odd H/W: drop extra outputs (L1155)
        const size_t base = ((size_t)i0 * LW + j0) * LN + n;
        const size_t HWN = (size_t)LH * LW * LN, dW = (size_t)LW * LN;
        // one store pattern for both destinations (y, or this cut segment's workspace slot
        // [slot][kl][output][nu]); the round's reads are branch-free so the 2 RR x 16 LDS issue back to
        // back and only the stores are predicated
        const bool cut = sk_slot >= 0;
        const size_t o1 = cut ? BN : LN, o2 = cut ? 2 * BN : dW, o3 = cut ? 3 * BN : dW + LN;
        const bool p1 = cut || okc, p2 = cut || okr, p3 = cut || (okr && okc);
        float* const dst0 = cut ? p.sk_ws + (size_t)sk_slot * BK * (4 * BN) + lane : Ly + (size_t)k0 * HWN + base;
        const size_t dk = cut ? 4 * BN : HWN;  // per filter
#pragma unroll
        for (int rd = 0; rd < 8 / RR; ++rd) {
            const int rd_hi = RR == 2 ? (rd >> 1) : rd, rd_lo = RR == 2 ? (rd & 1) : 0;
            named_bar_sync(1, COMPUTE_THREADS);  // previous round's readers are done
#pragma unroll
            for (int q = 0; q < 2; ++q)
#pragma unroll
                for (int ii = 0; ii < RR; ++ii) {
                    const int i = rd_hi * 4 + rd_lo * RR + ii;
                    const int r = (fo >> 2) * RR + ii;
                    float* row = ep + ((xi0 + q) * ER_KROWS + r) * ER_LD + io;
                    *reinterpret_cast<float4*>(row) = make_float4(acc[q][i][1], acc[q][i][0], acc[q][i][3], acc[q][i][2]);
                    *reinterpret_cast<float4*>(row + 16) =
                        make_float4(acc[q][i][5], acc[q][i][4], acc[q][i][7], acc[q][i][6]);
                }
            named_bar_sync(1, COMPUTE_THREADS);
            float m[RR][16], o[RR][4];
#pragma unroll
            for (int h = 0; h < RR; ++h)
#pragma unroll
                for (int e = 0; e < 16; ++e) m[h][e] = ep[(e * ER_KROWS + warp + 8 * h) * ER_LD + (lane ^ 1)];
#pragma unroll
            for (int h = 0; h < RR; ++h) otf_2x2(m[h], o[h]);
#pragma unroll
            for (int h = 0; h < RR; ++h) {
                const int r = warp + 8 * h;
                const int kl = (r / RR) * 4 + rd_lo * RR + (r % RR) + rd_hi * 32;
                if (nu_ok && k0 + kl < LK) {  // y is never re-read here: stream it past L2 (st.global.cs)
                    float* d = dst0 + (size_t)kl * dk;
                    __stcs(d, o[h][0]);
                    if (p1) __stcs(d + o1, o[h][1]);
                    if (p2) __stcs(d + o2, o[h][2]);
                    if (p3) __stcs(d + o3, o[h][3]);
                }
            }
        }
        if (sk_slot >= 0) {
            const Layer& L = p.L[R.l];
            ml_arrive(p, R.l, L.unit0 + ((R.u0 - L.unit0) / L.num_it) * L.num_it, k0, nu0, sk_sh, tid);
        }
#ifdef WINO_WS_CTATRACE
        if (tid == 0) ML_PT(pi, 2, fp32ws::gtimer());
#endif
    }
#ifdef WINO_WS_CTATRACE
    if (tid == 0) {
        ML_CT(3, fp32ws::gtimer());
        ML_CT(1, static_cast<unsigned long long>(p.start[blockIdx.x]));
        ML_CT(2, static_cast<unsigned long long>(p.start[blockIdx.x + 1]));
    }
#endif
}

}  // namespace fp32ml
}  // namespace wino
