// wino_api.cu -- the C ABI of libwino.so (declared in include/wino.h).
//
// Argument validation, shape -> kernel-variant dispatch, launches.  Every step
// of the computation runs in the CUDA kernels included below; there is no host
// or CPU fallback anywhere in this library.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <atomic>
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <vector>

#include "../../include/wino.h"
#include "ftf.cuh"
#include "fused_fp32.cuh"
#include "fused_fp32_ws.cuh"
#include "fused_fp32_ml.cuh"
#include "fused_tc.cuh"
#include "fused_tc16.cuh"
#include "fused_f4_fp32.cuh"
#include "nonfused.cuh"
#include "nonfused_tc.cuh"
#include "layout.cuh"


namespace {

thread_local int g_last_cuda_error = 0;

constexpr int kMaxDevices = 64;
constexpr int kStages = 3;  // smem ring depth of the FP32 kernel
#ifndef WINO_XPW
#define WINO_XPW 2
#endif
constexpr int kXpw = WINO_XPW;  // Winograd elements per warp (2: 256 threads, 1: 512 threads)

wino_status_t cuda_fail(cudaError_t e) {
    g_last_cuda_error = static_cast<int>(e);
    return WINO_ERR_CUDA;
}

// Per-device capability cache: 0 unknown, 1 sm_100, 2 other.
std::atomic<int> g_dev_cap[kMaxDevices];

wino_status_t check_device(int* dev_out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_fail(e);
    if (dev < 0 || dev >= kMaxDevices) return WINO_ERR_UNSUPPORTED;
    int cap = g_dev_cap[dev].load(std::memory_order_acquire);
    if (cap == 0) {
        int major = 0, minor = 0;
        if ((e = cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev)) != cudaSuccess)
            return cuda_fail(e);
        if ((e = cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev)) != cudaSuccess)
            return cuda_fail(e);
        cap = (major == 10 && minor == 0) ? 1 : 2;
        g_dev_cap[dev].store(cap, std::memory_order_release);
    }
    *dev_out = dev;
    return cap == 1 ? WINO_OK : WINO_ERR_UNSUPPORTED;
}

// SM count per device (cached).
std::atomic<int> g_sm_count[kMaxDevices];
int sm_count(int dev) {
    int n = g_sm_count[dev].load(std::memory_order_relaxed);
    if (n == 0) {
        if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0) n = 148;
        g_sm_count[dev].store(n, std::memory_order_relaxed);
    }
    return n;
}

// Opt-in to >48 KB dynamic shared memory once per (device, kernel instance).
std::mutex g_attr_mu;
template <typename Kern>
wino_status_t ensure_smem_attr(Kern kern, int dev, int bytes, std::atomic<uint64_t>& done_mask) {
    const uint64_t bit = 1ull << dev;
    if (done_mask.load(std::memory_order_acquire) & bit) return WINO_OK;
    std::lock_guard<std::mutex> lk(g_attr_mu);
    if (done_mask.load(std::memory_order_relaxed) & bit) return WINO_OK;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e != cudaSuccess) return cuda_fail(e);
    done_mask.fetch_or(bit, std::memory_order_release);
    return WINO_OK;
}

bool overlaps(const void* a, size_t na, const void* b, size_t nb) {
    const uintptr_t pa = reinterpret_cast<uintptr_t>(a), pb = reinterpret_cast<uintptr_t>(b);
    return pa < pb + nb && pb < pa + na;
}

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

size_t round_up256(size_t b) { return (b + 255) & ~size_t(255); }

// stream-K workspace of the tensor-core kernels: 2 slots of MM x 4 x TN FP32 partials (64 KiB each) per CTA
size_t tc16_sk_bytes(int ctas) { return size_t(ctas) * 2 * 128 * 4 * 32 * sizeof(float); }
// stream-K pays for the 16-bit kernel only when whole tiles would leave most SMs idle: its pieces
// run ~1.5x slower per channel block than the persistent schedule (measured: conv5 at P = 1
// 38.9 -> 52 us, conv2 175 -> 204 us; at P = 8 conv5 with 8 tiles 325 -> 42 us)
// stream-K workspace of the F(4x4) kernel: 2 slots of 64 k x 16 outputs x 16 nu floats per CTA
size_t f4_sk_bytes(int ctas) { return size_t(ctas) * 2 * 64 * 16 * 16 * sizeof(float); }
bool tc16_sk_pays(int64_t tiles, int ncb, int sms) {
    const double units = double(tiles) * ncb, reg = std::ceil(double(tiles) / sms) * ncb;
    return 2 * tiles <= sms && 1.5 * std::ceil(units / sms) + 3.0 < 0.9 * reg;
}

constexpr int64_t kMaxElems = (int64_t(1) << 31) - 1;

// Shape checks common to every conv entry point.
wino_status_t check_shape(int N, int C, int H, int W, int K, int pad, int stride) {
    if (N <= 0 || C <= 0 || H <= 0 || W <= 0 || K <= 0) return WINO_ERR_INVALID_ARG;
    if (pad != 1 || stride != 1) return WINO_ERR_UNSUPPORTED;
    const int64_t hw = int64_t(H) * W;
    const int64_t xe = int64_t(C) * hw * N, ye = int64_t(K) * hw * N, ue = int64_t(16) * C * K;
    const int64_t nv = int64_t(N) * ((H + 1) / 2) * ((W + 1) / 2);
    if (xe > kMaxElems || ye > kMaxElems || ue > kMaxElems || nv > kMaxElems) return WINO_ERR_TOO_LARGE;
    return WINO_OK;
}

// Co-resident clusters of `split` CTAs of the warp-specialised kernel (1 CTA per SM).
// Measured with cudaOccupancyMaxActiveClusters on the device when one is current
// (cached); without a device (host-only planning) the B200 values.
std::atomic<int> g_clusters[kMaxDevices][4];
int cluster_slots(int split, int dev);

struct Fp32Plan {
    int load_x, load_u;  // wino::fp32::LoadMode (generic kernel)
    bool ws;             // warp-specialised persistent kernel
    int xnb;             // x TMA box n-extent (ws)
    int split;           // split-C factor = cluster size (ws)
    int64_t tiles;       // (k, nu) tiles
    int64_t grid;        // CTAs launched
    int threads, smem;
    bool sk = false;     // stream-K WS kernel (+ fixup kernel); needs the workspace
};

// Stream-K workspace: 2 partial-tile slots (64 k x 4 outputs x 32 nu fp32) per CTA, then one
// arrival counter per CTA (zero between launches; see fused_fp32_ws.cuh).
size_t sk_slot_bytes() { return size_t(wino::fp32::BK) * 4 * wino::fp32::BN * sizeof(float); }
// slots, one arrival counter per CTA, and 2 words for the multi-layer launch's dynamic tail (dyn_ctr)
size_t sk_workspace_bytes(int ctas) { return size_t(ctas) * 2 * sk_slot_bytes() + round_up256(size_t(ctas) * 4 + 8); }
// The arrival counters sit after the slots of a FULL grid (one CTA per SM) whatever the grid of a
// launch: a smaller grid's counters would otherwise land on slots that an earlier launch on the
// same workspace left non-zero.
unsigned* sk_flags_of(void* ws, int dev) {
    return reinterpret_cast<unsigned*>(static_cast<char*>(ws) + 2 * sk_slot_bytes() * size_t(sm_count(dev)));
}

int log2_small(int s) { return s == 1 ? 0 : s == 2 ? 1 : s == 4 ? 2 : 3; }
// planner cost of the stream-K plan beyond its units, in channel-block times: up to two partial
// epilogues per CTA plus the last-arrival reductions (fitted to scripts/sk_ab.py)
constexpr double kSkFixupBlocks = 4.0;

// Shape -> kernel / tiling / split-C.  force_split: 0 = choose, else 1, 2, 4 or 8.
// The split model: a cluster of S CTAs shares a tile, each CTA runs ceil(NIT/S)
// channel blocks plus an epilogue worth ~E channel blocks (E measured: the
// DSMEM-reduced epilogue of the split kernel costs about one block more than the
// plain one); time ~ waves(S) * (ceil(NIT/S) + E(S)), waves = ceil(tiles/clusters).
// sk_mode: 0 = no stream-K (no workspace), 1 = planner's choice, 2 = force stream-K.
Fp32Plan plan_fp32(int N, int C, int H, int W, int K, bool u_tma_ok, int dev, int force_split, int sk_mode = 0) {
    using namespace wino::fp32;
    Fp32Plan p;
    p.load_x = (N % 32 == 0) ? LD_TMA : (N % 4 == 0 ? LD_CP16B : LD_CP4B);
    p.load_u = (K % 4 == 0 && u_tma_ok) ? LD_TMA : LD_CP4B;
    const int64_t nv = int64_t(N) * ((H + 1) / 2) * ((W + 1) / 2);
    const int64_t nb = (nv + BN - 1) / BN;
    const int64_t kb = (K + BK - 1) / BK;
    p.tiles = nb * kb;
    p.xnb = (N % 32 == 0) ? 32 : N;
    p.ws = p.load_u == LD_TMA && (N % 32 == 0 || N == 4 || N == 8 || N == 16);
#ifdef WINO_NO_WS
    p.ws = false;
#endif
    p.split = 1;
    if (!p.ws) {
        p.grid = p.tiles;
        p.threads = threads_for<kXpw>();
        p.smem = Smem<kStages>::bytes;
        return p;
    }
    const int nit = (C + BC - 1) / BC;
    const int sms = cluster_slots(1, dev);
    if (double(p.tiles) * nit >= 2147483647.0) sk_mode = 0;  // stream-K unit indices are 32-bit
    if (sk_mode == 2 && force_split <= 1) {
        p.sk = true;
    } else if (force_split > 0) {
        p.split = force_split;
    } else {
        double best = 0;
        for (int s = 1; s <= wino::fp32ws::MAX_SPLIT; s *= 2) {
            if (s > 1 && nit < 2 * s) break;  // keep >= 2 channel blocks per CTA
            const int cl = cluster_slots(s, dev);
            if (cl <= 0) continue;
            const double waves = double((p.tiles + cl - 1) / cl);
            // epilogue in channel-block times: plain 0.5; the cluster reduction 1.5 for S = 2, 4 and
            // 5 for S = 8 (8 partials per output; fitted to scripts/sk_ab.py)
            const double est = waves * (double((nit + s - 1) / s) + (s == 1 ? 0.5 : (s == 8 ? 5.0 : 1.5)));
            if (s == 1 || est < best * 0.97) {
                best = est;
                p.split = s;
            }
        }
        if (sk_mode == 1) {
            // stream-K: equal shares of the tiles x channel blocks units on every SM, a tile
            // epilogue per tile plus up to two partial ones per CTA, and the fixup launch
            const double units = double(p.tiles) * nit;
            const double est = std::ceil(units / sms) + (double(p.tiles) / sms + 1.0) * 0.5 + kSkFixupBlocks;
            if (est < best * 0.97 && units >= 2.0 * sms) {
                p.sk = true;
                p.split = 1;
            }
        }
    }
    if (p.sk) {
        p.split = 1;
        p.grid = sms;  // one CTA per SM (the workspace holds 2 slots + a counter per SM)
        p.threads = wino::fp32ws::NT;
        p.smem = wino::fp32ws::Smem<false>::bytes;
        return p;
    }
    const int64_t cl = cluster_slots(p.split, dev);
    p.grid = (p.tiles < cl ? p.tiles : cl) * p.split;
    p.threads = wino::fp32ws::NT;
    p.smem = p.split > 1 ? wino::fp32ws::Smem<true>::bytes : wino::fp32ws::Smem<false>::bytes;
    return p;
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no -lcuda).
PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
    static std::atomic<void*> fn{nullptr};
    void* f = fn.load(std::memory_order_acquire);
    if (!f) {
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            return nullptr;
        fn.store(f, std::memory_order_release);
    }
    return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(f);
}

// fp32 tensor map, dims innermost first; strides (bytes, dims 1..rank-1) default to dense.
bool encode_map(CUtensorMap* m, const void* base, int rank, const cuuint64_t* dims, const cuuint32_t* box,
                const cuuint64_t* strides_in = nullptr,
                CUtensorMapDataType dtype = CU_TENSOR_MAP_DATA_TYPE_FLOAT32, int esize = 4,
                CUtensorMapSwizzle swizzle = CU_TENSOR_MAP_SWIZZLE_NONE) {
    auto enc = tensor_map_encoder();
    if (!enc) return false;
    cuuint64_t strides[4];
    cuuint64_t acc = esize;
    for (int i = 0; i < rank - 1; ++i) {
        acc *= dims[i];
        strides[i] = strides_in ? strides_in[i] : acc;
    }
    cuuint32_t estr[5] = {1, 1, 1, 1, 1};
    CUresult r = enc(m, dtype, rank, const_cast<void*>(base), dims, strides, box, estr,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, swizzle, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);  // OOB elements read as zero
    return r == CUDA_SUCCESS;
}

std::atomic<uint64_t> g_attr_fp32[3][3];
std::atomic<uint64_t> g_attr_f4[2];

template <int XM, int UM>
wino_status_t launch_fp32(const wino::fp32::Params& prm, int64_t ctas, int smem, int dev, cudaStream_t st) {
    auto kern = wino::fp32::fused_fp32_kernel<XM, UM, kStages, kXpw>;
    wino_status_t s = ensure_smem_attr(kern, dev, smem, g_attr_fp32[XM][UM]);
    if (s != WINO_OK) return s;
    kern<<<dim3(static_cast<unsigned>(ctas)), wino::fp32::threads_for<kXpw>(), smem, st>>>(prm);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}

}  // namespace

namespace {
std::atomic<uint64_t> g_attr_tc[2][4][2][2];  // [P-1][XM][MM == 64][SK]
template <int P, int XM, int MM, bool SK = false>
wino_status_t launch_tc(const wino::tc::Params& prm, int64_t ctas, int dev, cudaStream_t st) {
    auto kern = wino::tc::fused_tc_kernel<P, XM, MM, SK>;
    const int smem = wino::tc::Cfg<P, MM, XM>::BYTES;
    wino_status_t s = ensure_smem_attr(kern, dev, smem, g_attr_tc[P - 1][XM][MM == 64][SK]);
    if (s != WINO_OK) return s;
    kern<<<dim3(static_cast<unsigned>(ctas)), wino::tc::NT, smem, st>>>(prm);
    cudaError_t e = cudaGetLastError();
    if (e == cudaSuccess && SK && ctas > 1) {
        wino::tc::tc_fixup_kernel<MM><<<dim3(static_cast<unsigned>(wino::tc::FIX_PARTS * (ctas - 1))), 256, 0, st>>>(
            prm, static_cast<int>(ctas));
        e = cudaGetLastError();
    }
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}
}  // namespace

namespace {
int cluster_slots(int split, int dev) {
    // host-only default: B200 (148 SMs); clusters of 8 measured 18
    static const int kDefault[4] = {148, 74, 37, 18};
    const int li = log2_small(split);
    if (dev < 0 || dev >= kMaxDevices) return kDefault[li];
    int n = g_clusters[dev][li].load(std::memory_order_relaxed);
    if (n != 0) return n;
    n = kDefault[li];
    if (split == 1) {
        n = sm_count(dev);
    } else {
        auto kern = wino::fp32ws::fused_fp32_ws_kernel<true, true>;
        const int smem = wino::fp32ws::Smem<true>::bytes;
        if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) == cudaSuccess) {
            cudaLaunchConfig_t cfg = {};
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = split;
            at[0].val.clusterDim.y = 1;
            at[0].val.clusterDim.z = 1;
            cfg.gridDim = dim3(split * 64);
            cfg.blockDim = dim3(wino::fp32ws::NT);
            cfg.dynamicSmemBytes = smem;
            cfg.attrs = at;
            cfg.numAttrs = 1;
            int q = 0;
            if (cudaOccupancyMaxActiveClusters(&q, kern, &cfg) == cudaSuccess && q > 0) n = q;
        }
        cudaGetLastError();  // a failed query must not leak into the caller's error state
    }
    g_clusters[dev][li].store(n, std::memory_order_relaxed);
    return n;
}

std::atomic<uint64_t> g_attr_ws_k[2][2];
std::atomic<uint64_t> g_attr_ws_sk[2];
}  // namespace

// FP32 fused conv on validated arguments; u may be a K-slice of a wider (C,4,4,ldu) array.
// force_split: 0 = planner's choice, else the split-C factor (1, 2, 4, 8).
// nchw: x (N,C,H,W) / y (N,K,H,W) instead of the paper's CHWN / KHWN (generic kernel).
// sk_mode / ws: stream-K (0 = off, 1 = planner's choice, 2 = forced) when ws holds
// sk_workspace_bytes(SM count) bytes.
wino_status_t launch_fwd_fp32(const float* x_dev, const float* u_dev, int ldu, float* y_dev, int N, int C, int H,
                              int W, int K, int dev, cudaStream_t st, int force_split = 0, bool nchw = false,
                              int sk_mode = 0, void* ws = nullptr, size_t ws_bytes = 0) {
    using namespace wino::fp32;
    const bool u_tma_ok = ldu % 4 == 0 && aligned16(u_dev);
    const bool ws_ok = ws != nullptr && aligned16(ws) && ws_bytes >= sk_workspace_bytes(sm_count(dev));
    Fp32Plan pl = plan_fp32(N, C, H, W, K, u_tma_ok, dev, force_split, ws_ok && !nchw ? sk_mode : 0);
    if (nchw) {  // strided gathers (Sec. 8.4: "offsets ... need to be recomputed")
        pl.ws = false;
        pl.split = 1;
        pl.load_x = LD_CP4B;
        pl.grid = pl.tiles;
        pl.threads = threads_for<kXpw>();
        pl.smem = Smem<kStages>::bytes;
    }
    Params prm;
    std::memset(&prm, 0, sizeof(prm));
    prm.x = x_dev;
    prm.u = u_dev;
    prm.y = y_dev;
    prm.N = N;
    prm.C = C;
    prm.H = H;
    prm.W = W;
    prm.K = K;
    prm.ldu = ldu;
    prm.TW = (W + 1) / 2;
    prm.NV = N * ((H + 1) / 2) * prm.TW;
    prm.num_kb = (K + BK - 1) / BK;
    prm.num_it = (C + BC - 1) / BC;
    prm.xnb = pl.ws ? pl.xnb : BN;
    prm.split = pl.split;
    prm.T = ((H + 1) / 2) * prm.TW;
    const long long hw = (long long)H * W;
    if (nchw) {
        prm.xs_c = hw, prm.xs_n = (long long)C * hw, prm.xs_h = W, prm.xs_w = 1;
        prm.ys_k = hw, prm.ys_n = (long long)K * hw, prm.ys_h = W, prm.ys_w = 1;
        prm.tfast = 1;
    } else {
        prm.xs_c = hw * N, prm.xs_n = 1, prm.xs_h = (long long)W * N, prm.xs_w = N;
        prm.ys_k = hw * N, prm.ys_n = 1, prm.ys_h = (long long)W * N, prm.ys_w = N;
        prm.tfast = 0;
    }
    if (pl.ws && prm.xnb < BN) {
        // ITF lane map of the small-N WS kernel (conflict-free LDS.128 / STS.128, see fused_fp32_ws.cuh)
        const int Q = prm.xnb / 4;
        for (int t = 0; t < 64; ++t) {
            const int j = t / 8, i = t % 8, b = i / Q, h = i % Q;
            const int c = (b + j) % 8, n4 = b * prm.xnb + 4 * h;
            const int xoff = b * (BC * 16 * prm.xnb) + c * prm.xnb + 4 * h;  // [b][pos][c][n]
            prm.itf_map[t] = c | (n4 << 3) | (xoff << 8);
        }
        // small N: x viewed as (n, c, w, h) so that a box lands as [pos][c][n] (conflict-free ITF)
        const cuuint64_t dims[4] = {cuuint64_t(N), cuuint64_t(C), cuuint64_t(W), cuuint64_t(H)};
        const cuuint64_t strides[3] = {cuuint64_t(H) * W * N * 4, cuuint64_t(N) * 4, cuuint64_t(W) * N * 4};
        const cuuint32_t box[4] = {cuuint32_t(prm.xnb), BC, 4, 4};
        if (!encode_map(&prm.tmx, x_dev, 4, dims, box, strides)) return cuda_fail(cudaErrorInvalidValue);
    } else if (pl.ws || pl.load_x == LD_TMA) {
        const cuuint64_t dims[4] = {cuuint64_t(N), cuuint64_t(W), cuuint64_t(H), cuuint64_t(C)};
        const cuuint32_t box[4] = {BN, 4, 4, BC};
        if (!encode_map(&prm.tmx, x_dev, 4, dims, box)) return cuda_fail(cudaErrorInvalidValue);
    }
    if (pl.load_u == LD_TMA) {
        const cuuint64_t dims[3] = {cuuint64_t(K), 16, cuuint64_t(C)};
        const cuuint64_t strides[2] = {cuuint64_t(ldu) * 4, cuuint64_t(16) * ldu * 4};
        const cuuint32_t box[3] = {BK, 16, BC};
        if (!encode_map(&prm.tmu, u_dev, 3, dims, box, strides)) return cuda_fail(cudaErrorInvalidValue);
    }
    const int64_t g = pl.tiles;
    const int sm = pl.smem;
    const bool box32 = prm.xnb == BN;
    if (pl.ws && pl.sk) {  // stream-K: equal unit ranges on every SM + fixup of the cut tiles
        prm.sk_ws = static_cast<float*>(ws);
        // 2 partial-tile slots per CTA, then one arrival counter per CTA (zero between launches)
        prm.sk_flags = sk_flags_of(ws, dev);
        prm.sk_total = pl.tiles * prm.num_it;  // < 2^31 (planner)
        prm.sk_q = static_cast<int>(prm.sk_total / pl.grid);
        prm.sk_r = static_cast<int>(prm.sk_total % pl.grid);
        auto kern = box32 ? wino::fp32ws::fused_fp32_ws_kernel<false, true, true>
                          : wino::fp32ws::fused_fp32_ws_kernel<false, false, true>;
        wino_status_t s = ensure_smem_attr(kern, dev, sm, g_attr_ws_sk[box32]);
        if (s != WINO_OK) return s;
        kern<<<dim3(static_cast<unsigned>(pl.grid)), wino::fp32ws::NT, sm, st>>>(prm, static_cast<int>(g));
        cudaError_t e = cudaGetLastError();  // the cut tiles are summed inside the kernel (no fixup launch)
        return e == cudaSuccess ? WINO_OK : cuda_fail(e);
    }
    if (pl.ws && pl.split == 1) {  // warp-specialised persistent kernel, one CTA per SM
        auto kern = box32 ? wino::fp32ws::fused_fp32_ws_kernel<false, true>
                          : wino::fp32ws::fused_fp32_ws_kernel<false, false>;
        wino_status_t s = ensure_smem_attr(kern, dev, sm, g_attr_ws_k[0][box32]);
        if (s != WINO_OK) return s;
        kern<<<dim3(static_cast<unsigned>(pl.grid)), wino::fp32ws::NT, sm, st>>>(prm, static_cast<int>(g));
        cudaError_t e = cudaGetLastError();
        return e == cudaSuccess ? WINO_OK : cuda_fail(e);
    }
    if (pl.ws) {  // split-C: clusters of pl.split CTAs, partial outputs reduced through DSMEM
        auto kern = box32 ? wino::fp32ws::fused_fp32_ws_kernel<true, true>
                          : wino::fp32ws::fused_fp32_ws_kernel<true, false>;
        wino_status_t s = ensure_smem_attr(kern, dev, sm, g_attr_ws_k[1][box32]);
        if (s != WINO_OK) return s;
        cudaLaunchConfig_t cfg = {};
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = pl.split;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.gridDim = dim3(static_cast<unsigned>(pl.grid));
        cfg.blockDim = dim3(wino::fp32ws::NT);
        cfg.dynamicSmemBytes = sm;
        cfg.stream = st;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        cudaError_t e = cudaLaunchKernelEx(&cfg, kern, prm, static_cast<int>(g));
        return e == cudaSuccess ? WINO_OK : cuda_fail(e);
    }
    switch (pl.load_x * 3 + pl.load_u) {
        case LD_TMA * 3 + LD_TMA: return launch_fp32<LD_TMA, LD_TMA>(prm, g, sm, dev, st);
        case LD_TMA * 3 + LD_CP4B: return launch_fp32<LD_TMA, LD_CP4B>(prm, g, sm, dev, st);
        case LD_CP16B * 3 + LD_TMA: return launch_fp32<LD_CP16B, LD_TMA>(prm, g, sm, dev, st);
        case LD_CP16B * 3 + LD_CP4B: return launch_fp32<LD_CP16B, LD_CP4B>(prm, g, sm, dev, st);
        case LD_CP4B * 3 + LD_TMA: return launch_fp32<LD_CP4B, LD_TMA>(prm, g, sm, dev, st);
        default: return launch_fp32<LD_CP4B, LD_CP4B>(prm, g, sm, dev, st);
    }
}

// Copy-in / copy-out helper streams of the multi-layer host path, one pair per
// device, created on first use (non-blocking, so they never sync with stream 0).
std::mutex g_stream_mu;
cudaStream_t g_s_in[kMaxDevices], g_s_out[kMaxDevices];
wino_status_t helper_streams(int dev, cudaStream_t* in, cudaStream_t* out) {
    std::lock_guard<std::mutex> lk(g_stream_mu);
    if (!g_s_in[dev]) {
        cudaError_t e = cudaStreamCreateWithFlags(&g_s_in[dev], cudaStreamNonBlocking);
        if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&g_s_out[dev], cudaStreamNonBlocking);
        if (e != cudaSuccess) return cuda_fail(e);
    }
    *in = g_s_in[dev];
    *out = g_s_out[dev];
    return WINO_OK;
}

// Events used for cross-stream ordering within one call, all created before anything is
// queued (the count is known from the layer list) and destroyed at the end of the call
// (CUDA releases an event once the work recorded on it completes).
struct EventPool {
    cudaEvent_t* ev = nullptr;
    int n = 0, cap = 0;
    cudaError_t reserve(int count) {
        ev = new (std::nothrow) cudaEvent_t[count];
        if (!ev) return cudaErrorMemoryAllocation;
        for (; cap < count; ++cap) {
            cudaError_t e = cudaEventCreateWithFlags(&ev[cap], cudaEventDisableTiming);
            if (e != cudaSuccess) return e;
        }
        return cudaSuccess;
    }
    cudaEvent_t get() { return n < cap ? ev[n++] : nullptr; }
    ~EventPool() {
        for (int i = 0; i < cap; ++i) cudaEventDestroy(ev[i]);
        delete[] ev;
    }
};


extern "C" {

int wino_version(void) { return 100; }  // 0.1.0

const char* wino_status_string(wino_status_t s) {
    switch (s) {
        case WINO_OK: return "WINO_OK";
        case WINO_ERR_INVALID_ARG: return "WINO_ERR_INVALID_ARG";
        case WINO_ERR_UNSUPPORTED: return "WINO_ERR_UNSUPPORTED";
        case WINO_ERR_MISALIGNED: return "WINO_ERR_MISALIGNED";
        case WINO_ERR_TOO_LARGE: return "WINO_ERR_TOO_LARGE";
        case WINO_ERR_CUDA: return "WINO_ERR_CUDA";
    }
    return "WINO_ERR_UNKNOWN";
}

int wino_last_cuda_error(void) { return g_last_cuda_error; }

#ifdef WINO_WS_TRACE
int wino_debug_cluster_slots(int split) {
    int dev = 0;
    cudaGetDevice(&dev);
    return cluster_slots(split, dev);
}
int wino_debug_ws_trace(unsigned long long* host, int n) {
    return (int)cudaMemcpyFromSymbol(host, wino::fp32ws::g_ws_trace, sizeof(unsigned long long) * n);
}
#endif
#ifdef WINO_WS_CTATRACE
int wino_debug_cta_trace(unsigned long long* host, int n) {
    return (int)cudaMemcpyFromSymbol(host, wino::fp32ws::g_cta_trace, sizeof(unsigned long long) * n);
}
int wino_debug_ml_piece_trace(unsigned long long* host, int n) {
    return (int)cudaMemcpyFromSymbol(host, wino::fp32ml::g_ml_piece_trace, sizeof(unsigned long long) * n);
}
#endif
#ifdef WINO_TC16_TRACE
int wino_debug_tc16_trace(unsigned long long* host, int n) {
    return (int)cudaMemcpyFromSymbol(host, wino::tc16::g_trace16, sizeof(unsigned long long) * n);
}
#endif
#ifdef WINO_TC_TRACE
// debug builds only: copy the tcgen05 kernel's CTA-0 event trace to the host
int wino_debug_tc_trace(unsigned long long* host, int n) {
    return (int)cudaMemcpyFromSymbol(host, wino::tc::g_trace, sizeof(unsigned long long) * n);
}
#endif

size_t wino_filter_workspace_bytes(int C, int K) {
    if (C <= 0 || K <= 0) return 0;
    return size_t(16) * size_t(C) * size_t(K) * sizeof(float);
}

wino_status_t wino_filter_transform(const float* w_dev, float* u_dev, int C, int K, wino_stream_t stream) {
    if (!w_dev || !u_dev || C <= 0 || K <= 0) return WINO_ERR_INVALID_ARG;
    if (int64_t(16) * C * K > kMaxElems) return WINO_ERR_TOO_LARGE;
    if (!aligned16(w_dev) || !aligned16(u_dev)) return WINO_ERR_MISALIGNED;
    if (overlaps(w_dev, size_t(9) * C * K * 4, u_dev, size_t(16) * C * K * 4)) return WINO_ERR_INVALID_ARG;
    int dev;
    wino_status_t s = check_device(&dev);
    if (s != WINO_OK) return s;
    const wino_ftf_job_t job = {w_dev, u_dev, C, K};  // one job of the (vectorised) multi-layer FTF kernel
    return wino_filter_transform_multi(&job, 1, stream);
}

wino_status_t wino_filter_transform_multi(const wino_ftf_job_t* jobs, int n, wino_stream_t stream) {
    if (!jobs || n <= 0 || n > wino::FTF_MAX_JOBS) return WINO_ERR_INVALID_ARG;
    wino::FtfJobs J;
    std::memset(&J, 0, sizeof(J));
    J.n = n;
    unsigned blocks = 0;
    for (int j = 0; j < n; ++j) {
        const wino_ftf_job_t& b = jobs[j];
        if (!b.w || !b.u || b.C <= 0 || b.K <= 0) return WINO_ERR_INVALID_ARG;
        if (int64_t(16) * b.C * b.K > kMaxElems) return WINO_ERR_TOO_LARGE;
        if (!aligned16(b.w) || !aligned16(b.u)) return WINO_ERR_MISALIGNED;
        if (overlaps(b.w, size_t(9) * b.C * b.K * 4, b.u, size_t(16) * b.C * b.K * 4)) return WINO_ERR_INVALID_ARG;
        for (int i = 0; i < n; ++i) {  // an output must not overlap another output or any input
            if (i == j || !jobs[i].w || !jobs[i].u) continue;
            if (overlaps(b.u, size_t(16) * b.C * b.K * 4, jobs[i].u, size_t(16) * jobs[i].C * jobs[i].K * 4) ||
                overlaps(b.u, size_t(16) * b.C * b.K * 4, jobs[i].w, size_t(9) * jobs[i].C * jobs[i].K * 4))
                return WINO_ERR_INVALID_ARG;
        }
        J.w[j] = b.w;
        J.u[j] = b.u;
        J.C[j] = b.C;
        J.K[j] = b.K;
        J.vec[j] = b.K % 4 == 0 ? 1 : 0;  // 4 consecutive k per thread (the pointers are 16-byte aligned)
        J.first[j] = blocks;
        const int64_t nb = (int64_t(b.C) * (J.vec[j] ? b.K / 4 : b.K) + wino::FTF_THREADS - 1) / wino::FTF_THREADS;
        if (int64_t(blocks) + nb > 0x7fffffff) return WINO_ERR_TOO_LARGE;
        blocks += static_cast<unsigned>(nb);
    }
    J.first[n] = blocks;
    int dev;
    wino_status_t s = check_device(&dev);
    if (s != WINO_OK) return s;
    wino::ftf_multi_kernel<<<blocks, wino::FTF_THREADS, 0, reinterpret_cast<cudaStream_t>(stream)>>>(J);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}

wino_status_t wino_plan(int N, int C, int H, int W, int K, int variant, wino_plan_t* plan) {
    if (!plan) return WINO_ERR_INVALID_ARG;
    wino_status_t s = check_shape(N, C, H, W, K, 1, 1);
    if (s != WINO_OK) return s;
    std::memset(plan, 0, sizeof(*plan));
    if (variant == 1 || variant == 2 || variant == 6 || variant == 7) {  // tcgen05 TF32 / 3xTF32 (+ workspace)
        using namespace wino::tc;
        const bool with_ws = variant >= 6;
        variant = with_ws ? variant - 5 : variant;
        const int64_t nv = int64_t(N) * ((H + 1) / 2) * ((W + 1) / 2);
        const int mm = tc_mm(K, variant == 2 ? 2 : 1);
        plan->variant = variant;
        plan->bk = mm;
        plan->bn = BN * (128 / mm);
        plan->bc = BC;
        plan->load_x = (N % 32 == 0 || N == 4 || N == 8 || N == 16) ? 2 : (N % 4 == 0 ? 1 : 0);
        plan->load_u = 3;  // bulk copy of the pre-arranged operand tiles
        plan->split_c = 1;
        plan->ctas = ((nv + plan->bn - 1) / plan->bn) * ((K + mm - 1) / mm);  // tiles (persistent grid <= #SMs)
        plan->threads = NT;
        plan->smem_bytes = variant == 1 ? (mm == 64 ? Cfg<1, 64, 2>::BYTES : Cfg<1, 128, 2>::BYTES) : Cfg<2, 128, 2>::BYTES;
        plan->launches = 1;
        if (with_ws && plan->load_x == 2) {
            int dev = -1, sms = 148;  // host-only planning unless an sm_100 device is current
            if (check_device(&dev) == WINO_OK) sms = sm_count(dev);
            else cudaGetLastError();
            sms = sms < 256 ? sms : 256;
            if (tc16_sk_pays(plan->ctas, (C + BC - 1) / BC, sms)) {
                plan->stream_k = 1;
                plan->launches = 2;
                plan->ctas = sms;
            }
            plan->variant = variant + 5;
        }
        return WINO_OK;
    }
    if (variant == 3 || variant == 5) {  // tcgen05 kind::f16 (FP16 / BF16, NEXT row N4); 5: with workspace
        using namespace wino::tc16;
        const int64_t nv = int64_t(N) * ((H + 1) / 2) * ((W + 1) / 2);
        const int mm = tc16_mm(K), tn = BN * (128 / mm);
        plan->variant = 3;
        plan->bk = mm;
        plan->bn = tn;
        plan->bc = BC;
        plan->load_x = (N % 32 == 0 || N == 8 || N == 16) ? 2 : 0;
        plan->load_u = 3;
        plan->split_c = 1;
        plan->ctas = ((nv + tn - 1) / tn) * ((K + mm - 1) / mm);
        plan->threads = NT;
        plan->smem_bytes = mm == 64 ? Cfg<64>::BYTES : Cfg<128>::BYTES;
        plan->launches = 1;
        int dev = -1, sms = 148;  // host-only planning unless an sm_100 device is current
        if (check_device(&dev) == WINO_OK) sms = sm_count(dev);
        else cudaGetLastError();
        sms = sms < 256 ? sms : 256;
        if (variant == 5 && tc16_sk_pays(plan->ctas, (C + BC - 1) / BC, sms)) {
            plan->stream_k = 1;
            plan->launches = 2;
            plan->ctas = sms;
        }
        plan->variant = variant;
        return WINO_OK;
    }
    if (variant != 0 && variant != 4) return WINO_ERR_UNSUPPORTED;
    int dev = -1;  // host-only planning unless an sm_100 device is current
    {
        int d;
        if (check_device(&d) == WINO_OK) dev = d;
        else cudaGetLastError();
    }
    Fp32Plan p = plan_fp32(N, C, H, W, K, true, dev, 0, variant == 4 ? 1 : 0);
    plan->variant = variant;
    plan->bk = wino::fp32::BK;
    plan->bn = wino::fp32::BN;
    plan->bc = wino::fp32::BC;
    plan->load_x = p.ws ? 2 : p.load_x;
    plan->load_u = p.load_u;
    plan->split_c = p.split;
    plan->ctas = p.sk ? p.grid : p.tiles * p.split;
    plan->threads = p.threads;
    plan->smem_bytes = p.smem;
    plan->launches = 1;  // the FP32 stream-K plan reduces its cut tiles in the kernel
    plan->stream_k = p.sk ? 1 : 0;
    return WINO_OK;
}

wino_status_t wino_conv2d_f2x3_fwd(const float* x_dev, const float* u_dev, float* y_dev, int N, int C, int H,
                                   int W, int K, int pad, int stride, wino_stream_t stream) {
    if (!x_dev || !u_dev || !y_dev) return WINO_ERR_INVALID_ARG;
    wino_status_t s = check_shape(N, C, H, W, K, pad, stride);
    if (s != WINO_OK) return s;
    if (!aligned16(x_dev) || !aligned16(u_dev) || !aligned16(y_dev)) return WINO_ERR_MISALIGNED;
    const size_t hwn = size_t(H) * W * N;
    const size_t yb = size_t(K) * hwn * 4;
    if (overlaps(y_dev, yb, x_dev, size_t(C) * hwn * 4) || overlaps(y_dev, yb, u_dev, size_t(16) * C * K * 4))
        return WINO_ERR_INVALID_ARG;
    int dev;
    if ((s = check_device(&dev)) != WINO_OK) return s;
    return launch_fwd_fp32(x_dev, u_dev, K, y_dev, N, C, H, W, K, dev, reinterpret_cast<cudaStream_t>(stream));
}

wino_status_t wino_conv2d_f2x3_fwd_split(const float* x_dev, const float* u_dev, float* y_dev, int N, int C, int H,
                                         int W, int K, int pad, int stride, int split_c, wino_stream_t stream) {
    if (split_c != 0 && split_c != 1 && split_c != 2 && split_c != 4 && split_c != 8) return WINO_ERR_INVALID_ARG;
    if (!x_dev || !u_dev || !y_dev) return WINO_ERR_INVALID_ARG;
    wino_status_t s = check_shape(N, C, H, W, K, pad, stride);
    if (s != WINO_OK) return s;
    if (!aligned16(x_dev) || !aligned16(u_dev) || !aligned16(y_dev)) return WINO_ERR_MISALIGNED;
    const size_t hwn = size_t(H) * W * N;
    const size_t yb = size_t(K) * hwn * 4;
    if (overlaps(y_dev, yb, x_dev, size_t(C) * hwn * 4) || overlaps(y_dev, yb, u_dev, size_t(16) * C * K * 4))
        return WINO_ERR_INVALID_ARG;
    int dev;
    if ((s = check_device(&dev)) != WINO_OK) return s;
    return launch_fwd_fp32(x_dev, u_dev, K, y_dev, N, C, H, W, K, dev, reinterpret_cast<cudaStream_t>(stream),
                           split_c);
}

size_t wino_conv_workspace_bytes(int N, int C, int H, int W, int K) {
    if (check_shape(N, C, H, W, K, 1, 1) != WINO_OK) return 0;
    int dev = -1, sms = 148;  // host-only query: B200
    if (check_device(&dev) == WINO_OK) sms = sm_count(dev);
    else cudaGetLastError();
    return sk_workspace_bytes(sms);
}

wino_status_t wino_conv2d_f2x3_fwd_ws(const float* x_dev, const float* u_dev, float* y_dev, int N, int C, int H,
                                      int W, int K, int pad, int stride, int sk, void* ws_dev, size_t ws_bytes,
                                      wino_stream_t stream) {
    if (sk < 0 || sk > 2) return WINO_ERR_INVALID_ARG;
    if (!x_dev || !u_dev || !y_dev || (ws_bytes > 0 && !ws_dev)) return WINO_ERR_INVALID_ARG;
    wino_status_t s = check_shape(N, C, H, W, K, pad, stride);
    if (s != WINO_OK) return s;
    if (!aligned16(x_dev) || !aligned16(u_dev) || !aligned16(y_dev) || (ws_dev && !aligned16(ws_dev)))
        return WINO_ERR_MISALIGNED;
    const size_t hwn = size_t(H) * W * N;
    const size_t yb = size_t(K) * hwn * 4, xb = size_t(C) * hwn * 4, ub = size_t(16) * C * K * 4;
    if (overlaps(y_dev, yb, x_dev, xb) || overlaps(y_dev, yb, u_dev, ub)) return WINO_ERR_INVALID_ARG;
    if (ws_dev && (overlaps(ws_dev, ws_bytes, x_dev, xb) || overlaps(ws_dev, ws_bytes, u_dev, ub) ||
                   overlaps(ws_dev, ws_bytes, y_dev, yb)))
        return WINO_ERR_INVALID_ARG;
    int dev;
    if ((s = check_device(&dev)) != WINO_OK) return s;
    if (sk == 2 && ws_bytes < sk_workspace_bytes(sm_count(dev))) return WINO_ERR_INVALID_ARG;
    const int mode = sk == 0 ? 1 : (sk == 1 ? 0 : 2);  // API 0 auto / 1 off / 2 force -> planner 1 / 0 / 2
    return launch_fwd_fp32(x_dev, u_dev, K, y_dev, N, C, H, W, K, dev, reinterpret_cast<cudaStream_t>(stream), 0,
                           false, mode, ws_dev, ws_bytes);
}

}  // extern "C"

namespace {
std::atomic<uint64_t> g_attr_ml;
// Work model of the multi-layer cut, in units of one N % 32 == 0 channel block (~1.5 us of one
// SM), fitted to per-CTA / per-piece timelines of the ResNet step and its batch shards
// (scripts/ml_trace.py): small-N box modes move x in 32/N boxes of N-float rows
// (N = 16 / 8 / 4: 1.07 / 1.31 / 1.65 blocks), vmode layers skip the raw-x staging and the ITF
// (0.93), and each tile's 4-round OTF epilogue costs ~1.65 blocks (~2.5 us).
// Costs in channel-block times: [0] epilogue per tile, [1] vmode unit, [2..4] N = 16 / 8 / 4 x-box units.
// WINO_ML_COSTS="e,v,n16,n8,n4" overrides them (A/B of the work model only, scripts/gpu.sh; read once).
struct MlCosts {
    double c[5] = {1.65, 0.93, 1.07, 1.31, 1.65};
    MlCosts() {
        if (const char* e = std::getenv("WINO_ML_COSTS"))
            std::sscanf(e, "%lf,%lf,%lf,%lf,%lf", &c[0], &c[1], &c[2], &c[3], &c[4]);
    }
};
const MlCosts& ml_costs() {
    static const MlCosts m;
    return m;
}
double ml_epi_cost() { return ml_costs().c[0]; }
double ml_unit_cost(int xnb, bool vmode) {
    const double* c = ml_costs().c;
    return vmode ? c[1] : (xnb >= 32 ? 1.0 : (xnb == 16 ? c[2] : (xnb == 8 ? c[3] : c[4])));
}
// A job joins the shared persistent launch when the warp-specialised kernel takes it (N % 32 == 0
// or N in {4, 8, 16}; K % 4 == 0) and it has fewer than 64 tiles per SM; a layer that big fills
// the GPU on its own and gains nothing from sharing (ResNet conv2 at N = 256, 42 tiles per SM:
// shared 1129.5 vs alone 1131.5 us for the step, scripts/ml_ab.py).
#ifndef WINO_ML_ALONE_TILES_PER_SM  // A/B builds only (scripts/ml_ab.py)
#define WINO_ML_ALONE_TILES_PER_SM 64
#endif
bool ml_shares_launch(const wino_conv_job_t& J, int sms) {
    using namespace wino::fp32ml;
    if (J.K % 4 != 0 || !(J.N % 32 == 0 || J.N == 4 || J.N == 8 || J.N == 16)) return false;
    const long long nv = static_cast<long long>(J.N) * ((J.H + 1) / 2) * ((J.W + 1) / 2);
    const long long tiles = ((nv + BN - 1) / BN) * ((J.K + BK - 1) / BK);
    return tiles < static_cast<long long>(WINO_ML_ALONE_TILES_PER_SM) * sms;
}
// vmode (N = 4, 8): the small-N x boxes (rows of 16 / 32 B, 8 / 4 TMA boxes per stage) cost a
// shared layer 1.65 / 1.31 channel-block times; instead ml_itf_kernel transforms the (small) x into
// V once per call and the fused kernel loads V tiles with one 16 KB box of 128 B rows per stage.
#ifndef WINO_ML_VMODE_MAX_N  // A/B builds only (scripts/ml_ab.py)
#define WINO_ML_VMODE_MAX_N 8
#endif
constexpr int kMlVModeMaxN = WINO_ML_VMODE_MAX_N;
bool ml_vmode(const wino_conv_job_t& J) { return J.N % 32 != 0 && J.N <= kMlVModeMaxN; }
size_t ml_v_bytes(const wino_conv_job_t& J) {
    const size_t nv = size_t(J.N) * ((J.H + 1) / 2) * ((J.W + 1) / 2);
    return round_up256(size_t(16) * J.C * nv * 4);
}
size_t ml_multi_ws_bytes(const wino_conv_job_t* jobs, int n, int sms) {
    size_t b = sk_workspace_bytes(sms);
    for (int i = 0; i < n; ++i)
        if (ml_shares_launch(jobs[i], sms) && ml_vmode(jobs[i])) b += ml_v_bytes(jobs[i]);
    return b;
}
}  // namespace

extern "C" {

size_t wino_conv_multi_workspace_bytes(const wino_conv_job_t* jobs, int n) {
    if (!jobs || n <= 0) return 0;
    for (int i = 0; i < n; ++i)
        if (check_shape(jobs[i].N, jobs[i].C, jobs[i].H, jobs[i].W, jobs[i].K, 1, 1) != WINO_OK) return 0;
    int dev = -1, sms = 148;
    if (check_device(&dev) == WINO_OK) sms = sm_count(dev);
    else cudaGetLastError();
    return ml_multi_ws_bytes(jobs, n, sms);
}

}  // extern "C"

namespace {
// One multi-layer stream-K launch (and its vmode input transform), prepared on the host.
struct MlLaunch {
    wino::fp32ml::Params prm;
    wino::fp32ml::ItfJobs itf;
    int grid;
};
// Layers [0, n) of jobs (n <= 4, all warp-specialised eligible) as one multi-layer launch; vbuf[i]:
// the V buffer of a vmode layer (else unused).  Nothing is queued.
wino_status_t prepare_multi_fp32(const wino_conv_job_t* jobs, float* const* vbuf, int n, void* ws, int dev,
                                 MlLaunch& out) {
    using namespace wino::fp32ml;
    Params& prm = out.prm;
    std::memset(&prm, 0, sizeof(prm));
    prm.nl = n;
    ItfJobs& itf = out.itf;
    std::memset(&itf, 0, sizeof(itf));
    long long units = 0;
    double cu[MAX_LAYERS], per_tile[MAX_LAYERS], work0[MAX_LAYERS + 1];
    work0[0] = 0.0;
    for (int i = 0; i < n; ++i) {
        const wino_conv_job_t& J = jobs[i];
        Layer& L = prm.L[i];
        L.y = J.y;
        L.N = J.N;
        L.C = J.C;
        L.H = J.H;
        L.W = J.W;
        L.K = J.K;
        L.TW = (J.W + 1) / 2;
        L.NV = J.N * ((J.H + 1) / 2) * L.TW;
        L.num_kb = (J.K + BK - 1) / BK;
        L.num_it = (J.C + BC - 1) / BC;
        const long long tiles = static_cast<long long>((L.NV + BN - 1) / BN) * L.num_kb;
        L.xnb = J.N % 32 == 0 ? BN : J.N;
        L.unit0 = static_cast<int>(units < 2147483647LL ? units : 0);
        units += tiles * L.num_it;
        L.vmode = ml_vmode(J) ? 1 : 0;
        cu[i] = ml_unit_cost(L.xnb, L.vmode);
        per_tile[i] = L.num_it * cu[i] + ml_epi_cost();
        work0[i + 1] = work0[i] + tiles * per_tile[i];
        if (L.vmode) {  // V[xi][c][nu] from ml_itf_kernel: (NV, C, 16) box (32, 8, 16) = the V ring slot
            ItfJob& T = itf.j[itf.n++];
            T.x = J.x;
            T.v = vbuf[i];
            T.N = J.N;
            T.C = J.C;
            T.H = J.H;
            T.W = J.W;
            T.TW = L.TW;
            T.NV = L.NV;
            T.first = itf.total;
            itf.total += J.C * (L.NV / 4);  // < 2^31: C * NV <= C * H * W * N <= kMaxElems
            const cuuint64_t dims[3] = {cuuint64_t(L.NV), cuuint64_t(J.C), 16};
            const cuuint64_t strides[2] = {cuuint64_t(L.NV) * 4, cuuint64_t(J.C) * L.NV * 4};
            const cuuint32_t box[3] = {BN, BC, 16};
            if (!encode_map(&L.tmv, vbuf[i], 3, dims, box, strides)) return cuda_fail(cudaErrorInvalidValue);
        } else if (L.xnb < BN) {  // small N: (n, c, w, h) boxes + the conflict-free ITF map (as launch_fwd_fp32)
            const int Q = L.xnb / 4;
            for (int t = 0; t < 64; ++t) {
                const int j = t / 8, ii = t % 8, b = ii / Q, h = ii % Q;
                const int c = (b + j) % 8, n4 = b * L.xnb + 4 * h;
                const int xoff = b * (BC * 16 * L.xnb) + c * L.xnb + 4 * h;
                L.itf_map[t] = c | (n4 << 3) | (xoff << 8);
            }
            const cuuint64_t dims[4] = {cuuint64_t(J.N), cuuint64_t(J.C), cuuint64_t(J.W), cuuint64_t(J.H)};
            const cuuint64_t strides[3] = {cuuint64_t(J.H) * J.W * J.N * 4, cuuint64_t(J.N) * 4,
                                           cuuint64_t(J.W) * J.N * 4};
            const cuuint32_t box[4] = {cuuint32_t(L.xnb), BC, 4, 4};
            if (!encode_map(&L.tmx, J.x, 4, dims, box, strides)) return cuda_fail(cudaErrorInvalidValue);
        } else {
            const cuuint64_t dims[4] = {cuuint64_t(J.N), cuuint64_t(J.W), cuuint64_t(J.H), cuuint64_t(J.C)};
            const cuuint32_t box[4] = {BN, 4, 4, BC};
            if (!encode_map(&L.tmx, J.x, 4, dims, box)) return cuda_fail(cudaErrorInvalidValue);
        }
        const cuuint64_t udims[3] = {cuuint64_t(J.K), 16, cuuint64_t(J.C)};
        const cuuint64_t ustrides[2] = {cuuint64_t(J.K) * 4, cuuint64_t(16) * J.K * 4};
        const cuuint32_t ubox[3] = {BK, 16, BC};
        if (!encode_map(&L.tmu, J.u, 3, udims, ubox, ustrides)) return cuda_fail(cudaErrorInvalidValue);
    }
    if (units >= 2147483647LL) return WINO_ERR_TOO_LARGE;
    // one CTA per SM; CTA b starts at the first unit whose work position reaches b / grid of the
    // static total, then pushed up so that every range is non-empty.  The last ~6 % of the work --
    // whole tiles of the last layer -- is the dynamic tail the CTAs grab after their static ranges.
    const int sms = sm_count(dev) < MAX_GRID ? sm_count(dev) : MAX_GRID;
    const int grid = units < sms ? static_cast<int>(units) : sms;
    long long dyn = 0;
    {
        static const double frac = [] {
            const char* e = std::getenv("WINO_ML_DYN");  // A/B of the tail fraction (0: off)
            return e ? std::atof(e) : 0.08;
        }();
        const Layer& Lz = prm.L[n - 1];
        const long long tiles_z = static_cast<long long>((Lz.NV + BN - 1) / BN) * Lz.num_kb;
        dyn = static_cast<long long>(frac * work0[n] / per_tile[n - 1]);
        if (dyn > tiles_z - 1) dyn = tiles_z - 1;
        if (units - dyn * Lz.num_it < 2LL * grid) dyn = 0;  // keep every static range at >= 2 units
        // a tail pays only when each CTA can grab a few tiles of it (P = 8 shard, 0.6 tile per CTA at
        // 6 %: 176 vs 171 us; the P = 1 step with ~6 tiles per CTA: 1128 vs 1139 us, scripts: DESIGN 7.11)
        if (dyn < 3LL * grid) dyn = 0;
        dyn = dyn / Lz.num_kb * Lz.num_kb;  // whole nu-tiles (all their filter blocks)
    }
    const long long units_static = units - dyn * prm.L[n - 1].num_it;
    const double total = work0[n] - dyn * per_tile[n - 1];
    for (int i = 0; i < n; ++i) {  // nu-tile order (ml_nu_tile): the CTAs' shares of each layer
        Layer& L = prm.L[i];
        // the last layer's dynamic tail (whole nu-tiles at the end) keeps the identity order
        const int ng = (L.NV + BN - 1) / BN - (i == n - 1 ? static_cast<int>(dyn / L.num_kb) : 0);
        L.ng_s = ng;
        const double wl = work0[i + 1] - work0[i] - (i == n - 1 ? dyn * per_tile[i] : 0.0);
        long long g = std::llround(wl * grid / total);
        g = g < 1 ? 1 : (g > ng ? ng : g);
        L.vr = static_cast<int>((ng + g - 1) / g);
        L.vg = (ng + L.vr - 1) / L.vr;
        L.vlc = ng - (L.vg - 1) * L.vr;
    }
    for (int b = 0; b <= grid; ++b) {
        long long u = units_static;
        if (b < grid) {
            const double w = total * b / grid;
            int i = 0;
            while (i + 1 < n && work0[i + 1] <= w) ++i;
            const Layer& L = prm.L[i];
            const double local = w - work0[i];
            const long long tile = static_cast<long long>(local / per_tile[i]);
            long long g = static_cast<long long>(std::ceil((local - tile * per_tile[i]) / cu[i] - 1e-9));
            if (g > L.num_it) g = L.num_it;
            if (g < 0) g = 0;
            u = L.unit0 + tile * L.num_it + g;
        }
        if (b > 0 && u <= prm.start[b - 1]) u = prm.start[b - 1] + 1;  // non-empty ranges
        if (u > units_static - (grid - b)) u = units_static - (grid - b);
        prm.start[b] = static_cast<int>(u);
    }
    prm.sk_ws = static_cast<float*>(ws);
    prm.sk_flags = sk_flags_of(ws, dev);
    prm.dyn_n = static_cast<int>(dyn);
    prm.dyn_nu = prm.L[n - 1].num_it;
    prm.dyn_ctr = sk_flags_of(ws, dev) + sm_count(dev);
    out.grid = grid;
    return WINO_OK;
}
// the vmode input transform of a prepared launch (reads x only)
wino_status_t launch_ml_itf(const MlLaunch& L, int dev, cudaStream_t st) {
    if (L.itf.n == 0) return WINO_OK;
    int blocks = (L.itf.total + 255) / 256;
    if (blocks > 2 * sm_count(dev)) blocks = 2 * sm_count(dev);
    wino::fp32ml::ml_itf_kernel<<<dim3(static_cast<unsigned>(blocks), 4), 256, 0, st>>>(L.itf);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}
wino_status_t launch_ml(const MlLaunch& L, int dev, cudaStream_t st) {
    const int smem = wino::fp32ml::SMEM_BYTES;
    wino_status_t s = ensure_smem_attr(wino::fp32ml::fused_fp32_ml_kernel, dev, smem, g_attr_ml);
    if (s != WINO_OK) return s;
    wino::fp32ml::fused_fp32_ml_kernel<<<dim3(static_cast<unsigned>(L.grid)), wino::fp32ws::NT, smem, st>>>(L.prm);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}
}  // namespace

extern "C" {

wino_status_t wino_conv2d_f2x3_fwd_multi(const wino_conv_job_t* jobs, int n, void* ws_dev, size_t ws_bytes,
                                         void* u_ready, wino_stream_t stream) {
    if (!jobs || n <= 0 || !ws_dev) return WINO_ERR_INVALID_ARG;
    if (!aligned16(ws_dev)) return WINO_ERR_MISALIGNED;
    for (int i = 0; i < n; ++i) {
        const wino_conv_job_t& J = jobs[i];
        if (!J.x || !J.u || !J.y) return WINO_ERR_INVALID_ARG;
        wino_status_t s = check_shape(J.N, J.C, J.H, J.W, J.K, 1, 1);
        if (s != WINO_OK) return s;
        if (!aligned16(J.x) || !aligned16(J.u) || !aligned16(J.y)) return WINO_ERR_MISALIGNED;
    }
    for (int i = 0; i < n; ++i) {  // outputs overlap nothing else; the workspace overlaps nothing
        const wino_conv_job_t& A = jobs[i];
        const size_t hwn = size_t(A.H) * A.W * A.N;
        const size_t yb = size_t(A.K) * hwn * 4, xb = size_t(A.C) * hwn * 4, ub = size_t(16) * A.C * A.K * 4;
        if (overlaps(ws_dev, ws_bytes, A.x, xb) || overlaps(ws_dev, ws_bytes, A.u, ub) ||
            overlaps(ws_dev, ws_bytes, A.y, yb))
            return WINO_ERR_INVALID_ARG;
        for (int j = 0; j < n; ++j) {
            const wino_conv_job_t& B = jobs[j];
            const size_t hwn_b = size_t(B.H) * B.W * B.N;
            if (overlaps(A.y, yb, B.x, size_t(B.C) * hwn_b * 4) || overlaps(A.y, yb, B.u, size_t(16) * B.C * B.K * 4))
                return WINO_ERR_INVALID_ARG;
            if (j != i && overlaps(A.y, yb, B.y, size_t(B.K) * hwn_b * 4)) return WINO_ERR_INVALID_ARG;
        }
    }
    int dev;
    wino_status_t s = check_device(&dev);
    if (s != WINO_OK) return s;
    const int sms = sm_count(dev);
    if (ws_bytes < ml_multi_ws_bytes(jobs, n, sms)) return WINO_ERR_INVALID_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    // 1. plan every shared launch (groups of <= 4 in job order); the other jobs run alone
    wino_conv_job_t group[wino::fp32ml::MAX_LAYERS];
    float* vbuf[wino::fp32ml::MAX_LAYERS];
    char* vnext = static_cast<char*>(ws_dev) + sk_workspace_bytes(sms);  // V buffers of vmode layers
    std::vector<MlLaunch> ml;
    std::vector<int> alone;
    int m = 0;
    for (int i = 0; i <= n; ++i) {
        if ((i == n || m == wino::fp32ml::MAX_LAYERS) && m > 0) {
            ml.emplace_back();
            if ((s = prepare_multi_fp32(group, vbuf, m, ws_dev, dev, ml.back())) != WINO_OK) return s;
            m = 0;
        }
        if (i == n) break;
        const wino_conv_job_t& J = jobs[i];
        if (ml_shares_launch(J, sms)) {
            vbuf[m] = nullptr;
            if (ml_vmode(J)) {
                vbuf[m] = reinterpret_cast<float*>(vnext);
                vnext += ml_v_bytes(J);
            }
            group[m++] = J;
        } else {
            alone.push_back(i);
        }
    }
    // 2. work that reads x only (the vmode input transforms), then wait for u, then the convolutions
    for (const MlLaunch& L : ml)
        if ((s = launch_ml_itf(L, dev, st)) != WINO_OK) return s;
    if (u_ready) {
        cudaError_t e = cudaStreamWaitEvent(st, static_cast<cudaEvent_t>(u_ready), 0);
        if (e != cudaSuccess) return cuda_fail(e);
    }
    for (const MlLaunch& L : ml)
        if ((s = launch_ml(L, dev, st)) != WINO_OK) return s;
    for (int i : alone) {
        const wino_conv_job_t& J = jobs[i];
        if ((s = launch_fwd_fp32(J.x, J.u, J.K, J.y, J.N, J.C, J.H, J.W, J.K, dev, st, 0, false, 1, ws_dev,
                                 ws_bytes)) != WINO_OK)
            return s;
    }
    return WINO_OK;
}

int wino_conv_multi_launches(const wino_conv_job_t* jobs, int n) {
    if (!jobs || n <= 0) return -1;
    int dev = -1, sms = 148;
    if (check_device(&dev) == WINO_OK) sms = sm_count(dev);
    else cudaGetLastError();
    int launches = 0, m = 0;
    bool group_v = false;  // the current group has a vmode layer (+ one ml_itf_kernel launch)
    for (int i = 0; i < n; ++i) {
        const wino_conv_job_t& J = jobs[i];
        if (ml_shares_launch(J, sms)) {
            if (m == 0) {
                launches += 1;
                group_v = false;
            }
            if (ml_vmode(J) && !group_v) {
                launches += 1;
                group_v = true;
            }
            m = (m + 1) % wino::fp32ml::MAX_LAYERS;
        } else {
            wino_plan_t pl;
            if (wino_plan(J.N, J.C, J.H, J.W, J.K, 4, &pl) != WINO_OK) return -1;
            launches += pl.launches;
        }
    }
    return launches;
}

wino_status_t wino_filter_transform_kcrs(const float* w_kcrs_dev, float* u_dev, int C, int K, wino_stream_t stream) {
    if (!w_kcrs_dev || !u_dev || C <= 0 || K <= 0) return WINO_ERR_INVALID_ARG;
    if (int64_t(16) * C * K > kMaxElems) return WINO_ERR_TOO_LARGE;
    if (!aligned16(w_kcrs_dev) || !aligned16(u_dev)) return WINO_ERR_MISALIGNED;
    if (overlaps(w_kcrs_dev, size_t(9) * C * K * 4, u_dev, size_t(16) * C * K * 4)) return WINO_ERR_INVALID_ARG;
    int dev;
    wino_status_t s = check_device(&dev);
    if (s != WINO_OK) return s;
    const int64_t n = int64_t(C) * K;
    const unsigned blocks = static_cast<unsigned>((n + wino::FTF_THREADS - 1) / wino::FTF_THREADS);
    wino::ftf_kcrs_kernel<<<blocks, wino::FTF_THREADS, 0, reinterpret_cast<cudaStream_t>(stream)>>>(w_kcrs_dev,
                                                                                                   u_dev, C, K);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}

wino_status_t wino_conv2d_f2x3_fwd_nchw(const float* x_nchw_dev, const float* u_dev, float* y_nkhw_dev, int N, int C,
                                        int H, int W, int K, int pad, int stride, wino_stream_t stream) {
    if (!x_nchw_dev || !u_dev || !y_nkhw_dev) return WINO_ERR_INVALID_ARG;
    wino_status_t s = check_shape(N, C, H, W, K, pad, stride);
    if (s != WINO_OK) return s;
    if (!aligned16(x_nchw_dev) || !aligned16(u_dev) || !aligned16(y_nkhw_dev)) return WINO_ERR_MISALIGNED;
    const size_t hwn = size_t(H) * W * N;
    const size_t yb = size_t(K) * hwn * 4;
    if (overlaps(y_nkhw_dev, yb, x_nchw_dev, size_t(C) * hwn * 4) ||
        overlaps(y_nkhw_dev, yb, u_dev, size_t(16) * C * K * 4))
        return WINO_ERR_INVALID_ARG;
    int dev;
    if ((s = check_device(&dev)) != WINO_OK) return s;
    return launch_fwd_fp32(x_nchw_dev, u_dev, K, y_nkhw_dev, N, C, H, W, K, dev,
                           reinterpret_cast<cudaStream_t>(stream), 1, true);
}

extern "C++" {
namespace {
size_t round256(size_t b) { return (b + 255) & ~size_t(255); }
cudaError_t transpose2d(const float* in, float* out, int R, long long S, cudaStream_t st) {
    // 1-D grid over (row tile, column tile) pairs: R * S < 2^31 elements, so < 2^21 tiles
    const long long tiles = ((S + wino::TR_TILE - 1) / wino::TR_TILE) * ((R + wino::TR_TILE - 1) / wino::TR_TILE);
    wino::transpose2d_kernel<<<dim3(static_cast<unsigned>(tiles)), dim3(wino::TR_TILE, wino::TR_ROWS), 0, st>>>(
        in, out, R, S);
    return cudaGetLastError();
}
}  // namespace
}  // extern "C++"

size_t wino_nchw_workspace_bytes(int N, int C, int H, int W, int K) {
    if (check_shape(N, C, H, W, K, 1, 1) != WINO_OK) return 0;
    const size_t hwn = size_t(H) * W * N;
    return round256(size_t(C) * hwn * 4) + round256(size_t(K) * hwn * 4) + wino_conv_workspace_bytes(N, C, H, W, K);
}

wino_status_t wino_conv2d_f2x3_fwd_nchw_ws(const float* x_nchw_dev, const float* u_dev, float* y_nkhw_dev, int N,
                                           int C, int H, int W, int K, int pad, int stride, void* ws_dev,
                                           size_t ws_bytes, wino_stream_t stream) {
    if (!x_nchw_dev || !u_dev || !y_nkhw_dev || !ws_dev) return WINO_ERR_INVALID_ARG;
    wino_status_t s = check_shape(N, C, H, W, K, pad, stride);
    if (s != WINO_OK) return s;
    if (!aligned16(x_nchw_dev) || !aligned16(u_dev) || !aligned16(y_nkhw_dev) || !aligned16(ws_dev))
        return WINO_ERR_MISALIGNED;
    const size_t hwn = size_t(H) * W * N;
    const size_t xb = size_t(C) * hwn * 4, yb = size_t(K) * hwn * 4, ub = size_t(16) * C * K * 4;
    if (overlaps(y_nkhw_dev, yb, x_nchw_dev, xb) || overlaps(y_nkhw_dev, yb, u_dev, ub)) return WINO_ERR_INVALID_ARG;
    const size_t need = wino_nchw_workspace_bytes(N, C, H, W, K);
    if (ws_bytes < need) return WINO_ERR_INVALID_ARG;
    if (overlaps(ws_dev, ws_bytes, x_nchw_dev, xb) || overlaps(ws_dev, ws_bytes, u_dev, ub) ||
        overlaps(ws_dev, ws_bytes, y_nkhw_dev, yb))
        return WINO_ERR_INVALID_ARG;
    int dev;
    if ((s = check_device(&dev)) != WINO_OK) return s;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    float* xc = static_cast<float*>(ws_dev);                                          // (C,H,W,N)
    float* yc = reinterpret_cast<float*>(static_cast<char*>(ws_dev) + round256(xb));  // (K,H,W,N)
    void* wsk = static_cast<char*>(ws_dev) + round256(xb) + round256(yb);
    const size_t wsk_bytes = ws_bytes - round256(xb) - round256(yb);
    cudaError_t e = transpose2d(x_nchw_dev, xc, N, (long long)C * H * W, st);  // (N, CHW) -> (CHW, N)
    if (e != cudaSuccess) return cuda_fail(e);
    s = launch_fwd_fp32(xc, u_dev, K, yc, N, C, H, W, K, dev, st, 0, false, 1, wsk, wsk_bytes);
    if (s != WINO_OK) return s;
    e = transpose2d(yc, y_nkhw_dev, K * H * W, N, st);  // (KHW, N) -> (N, KHW)
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}

size_t wino_filter_workspace_bytes_tc(int C, int K, wino_tc_mode_t mode) {
    if (C <= 0 || K <= 0 || (mode != WINO_TC_TF32 && mode != WINO_TC_3XTF32)) return 0;
    const int planes = mode == WINO_TC_3XTF32 ? 2 : 1;
    return wino::tc::u_tc_floats(C, K, planes, wino::tc::tc_mm(K, planes)) * sizeof(float);
}

wino_status_t wino_filter_transform_tc(const float* w_dev, float* u_tc_dev, int C, int K, wino_tc_mode_t mode,
                                       wino_stream_t stream) {
    if (!w_dev || !u_tc_dev || C <= 0 || K <= 0) return WINO_ERR_INVALID_ARG;
    if (mode != WINO_TC_TF32 && mode != WINO_TC_3XTF32) return WINO_ERR_INVALID_ARG;
    const size_t ub = wino_filter_workspace_bytes_tc(C, K, mode);
    if (ub / 4 > size_t(kMaxElems)) return WINO_ERR_TOO_LARGE;
    if (!aligned16(w_dev) || !aligned16(u_tc_dev)) return WINO_ERR_MISALIGNED;
    if (overlaps(w_dev, size_t(9) * C * K * 4, u_tc_dev, ub)) return WINO_ERR_INVALID_ARG;
    int dev;
    wino_status_t s = check_device(&dev);
    if (s != WINO_OK) return s;
    const int planes = mode == WINO_TC_3XTF32 ? 2 : 1;
    const int mm = wino::tc::tc_mm(K, planes);
    const int64_t Kp = ((K + mm - 1) / mm) * mm;
    const dim3 blocks(static_cast<unsigned>(Kp / 32), static_cast<unsigned>((C + wino::tc::BC - 1) / wino::tc::BC));
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    if (planes == 1 && mm == 64) wino::tc::tc_filter_kernel<1, 64><<<blocks, 256, 0, st>>>(w_dev, u_tc_dev, C, K);
    else if (planes == 1) wino::tc::tc_filter_kernel<1, 128><<<blocks, 256, 0, st>>>(w_dev, u_tc_dev, C, K);
    else wino::tc::tc_filter_kernel<2, 128><<<blocks, 256, 0, st>>>(w_dev, u_tc_dev, C, K);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}


extern "C++" {
namespace {
// sk: 0 = never, 1 = planner's choice, 2 = always (TMA x paths; needs ws >= tc16_sk_bytes(SMs))
wino_status_t conv_tc(const float* x_dev, const float* u_tc_dev, float* y_dev, int N, int C, int H, int W, int K,
                      int pad, int stride, wino_tc_mode_t mode, int sk, void* ws_dev, size_t ws_bytes,
                      wino_stream_t stream) {
    if (!x_dev || !u_tc_dev || !y_dev) return WINO_ERR_INVALID_ARG;
    if (mode != WINO_TC_TF32 && mode != WINO_TC_3XTF32) return WINO_ERR_INVALID_ARG;
    wino_status_t s = check_shape(N, C, H, W, K, pad, stride);
    if (s != WINO_OK) return s;
    if (!aligned16(x_dev) || !aligned16(u_tc_dev) || !aligned16(y_dev) || (ws_dev && !aligned16(ws_dev)))
        return WINO_ERR_MISALIGNED;
    const size_t hwn = size_t(H) * W * N;
    const size_t yb = size_t(K) * hwn * 4;
    if (overlaps(y_dev, yb, x_dev, size_t(C) * hwn * 4) ||
        overlaps(y_dev, yb, u_tc_dev, wino_filter_workspace_bytes_tc(C, K, mode)))
        return WINO_ERR_INVALID_ARG;
    int dev;
    if ((s = check_device(&dev)) != WINO_OK) return s;
    using namespace wino::tc;
    Params prm;
    std::memset(&prm, 0, sizeof(prm));
    prm.x = x_dev;
    prm.u_tc = u_tc_dev;
    prm.y = y_dev;
    prm.N = N;
    prm.C = C;
    prm.H = H;
    prm.W = W;
    prm.K = K;
    prm.TW = (W + 1) / 2;
    prm.NV = N * ((H + 1) / 2) * prm.TW;
    const int planes = mode == WINO_TC_3XTF32 ? 2 : 1;
    const int mm = tc_mm(K, planes);
    const int tn = BN * (128 / mm);
    prm.num_kb = (K + mm - 1) / mm;
    prm.num_cb = (C + BC - 1) / BC;
    prm.num_tiles = ((prm.NV + tn - 1) / tn) * prm.num_kb;
    const int xm = (N % 32 == 0) ? 2 : ((N == 4 || N == 8 || N == 16) ? 3 : (N % 4 == 0 ? 1 : 0));
    if (xm >= 2) {
        const cuuint64_t dims[4] = {cuuint64_t(N), cuuint64_t(W), cuuint64_t(H), cuuint64_t(C)};
        const cuuint32_t box[4] = {cuuint32_t(xm == 2 ? BN : N), 4, 4, BC};
        if (!encode_map(&prm.tmx, x_dev, 4, dims, box)) return cuda_fail(cudaErrorInvalidValue);
    }
    const int sms = sm_count(dev) < 256 ? sm_count(dev) : 256;
    int64_t ctas = prm.num_tiles < sms ? prm.num_tiles : sms;  // persistent
    if (ws_dev && (overlaps(ws_dev, ws_bytes, x_dev, size_t(C) * hwn * 4) || overlaps(ws_dev, ws_bytes, y_dev, yb) ||
                   overlaps(ws_dev, ws_bytes, u_tc_dev, wino_filter_workspace_bytes_tc(C, K, mode))))
        return WINO_ERR_INVALID_ARG;
    const double units = double(prm.num_tiles) * prm.num_cb;
    // (the 64-filter tiles' stream-K plan was fenced off in round 1 after intermittent wrong partials;
    // the cause was a missing fence.proxy.async between the ITF's generic reads of a raw-x slot and
    // its TMA refill, DESIGN.md 7.6 -- fixed in every kernel, so both tile heights take stream-K)
    const bool sk_ok = xm >= 2 && ws_dev && ws_bytes >= tc16_sk_bytes(sms) && units < 2147483647.0;
    if (sk == 2 && !sk_ok) return WINO_ERR_INVALID_ARG;
    const bool use_sk = sk == 2 || (sk == 1 && sk_ok && tc16_sk_pays(prm.num_tiles, prm.num_cb, sms));
    if (use_sk) {  // stream-K: equal (tile, channel block) ranges on every SM + fixup
        ctas = sms;
        prm.sk_ws = static_cast<float*>(ws_dev);
        prm.sk_q = static_cast<int>(int64_t(units) / sms);
        prm.sk_r = static_cast<int>(int64_t(units) % sms);
    }
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    if (use_sk) {
        if (mode == WINO_TC_TF32 && mm == 64)
            return xm == 3 ? launch_tc<1, 3, 64, true>(prm, ctas, dev, st) : launch_tc<1, 2, 64, true>(prm, ctas, dev, st);
        if (mode == WINO_TC_TF32)
            return xm == 3 ? launch_tc<1, 3, 128, true>(prm, ctas, dev, st)
                           : launch_tc<1, 2, 128, true>(prm, ctas, dev, st);
        return xm == 3 ? launch_tc<2, 3, 128, true>(prm, ctas, dev, st) : launch_tc<2, 2, 128, true>(prm, ctas, dev, st);
    }
    if (mode == WINO_TC_TF32 && mm == 64) {
        if (xm == 3) return launch_tc<1, 3, 64>(prm, ctas, dev, st);
        if (xm == 2) return launch_tc<1, 2, 64>(prm, ctas, dev, st);
        if (xm == 1) return launch_tc<1, 1, 64>(prm, ctas, dev, st);
        return launch_tc<1, 0, 64>(prm, ctas, dev, st);
    }
    if (mode == WINO_TC_TF32) {
        if (xm == 3) return launch_tc<1, 3, 128>(prm, ctas, dev, st);
        if (xm == 2) return launch_tc<1, 2, 128>(prm, ctas, dev, st);
        if (xm == 1) return launch_tc<1, 1, 128>(prm, ctas, dev, st);
        return launch_tc<1, 0, 128>(prm, ctas, dev, st);
    }
    if (xm == 3) return launch_tc<2, 3, 128>(prm, ctas, dev, st);
    if (xm == 2) return launch_tc<2, 2, 128>(prm, ctas, dev, st);
    if (xm == 1) return launch_tc<2, 1, 128>(prm, ctas, dev, st);
    return launch_tc<2, 0, 128>(prm, ctas, dev, st);
}
}  // namespace
}  // extern "C++"

wino_status_t wino_conv2d_f2x3_fwd_tc(const float* x_dev, const float* u_tc_dev, float* y_dev, int N, int C, int H,
                                      int W, int K, int pad, int stride, wino_tc_mode_t mode,
                                      wino_stream_t stream) {
    return conv_tc(x_dev, u_tc_dev, y_dev, N, C, H, W, K, pad, stride, mode, 0, nullptr, 0, stream);
}

size_t wino_tc_workspace_bytes(int N, int C, int H, int W, int K) { return wino_half_workspace_bytes(N, C, H, W, K); }

wino_status_t wino_conv2d_f2x3_fwd_tc_ws(const float* x_dev, const float* u_tc_dev, float* y_dev, int N, int C,
                                         int H, int W, int K, int pad, int stride, wino_tc_mode_t mode, int sk,
                                         void* ws_dev, size_t ws_bytes, wino_stream_t stream) {
    if (sk < 0 || sk > 2 || (ws_bytes > 0 && !ws_dev)) return WINO_ERR_INVALID_ARG;
    const int m = sk == 0 ? 1 : (sk == 1 ? 0 : 2);  // API 0 auto / 1 off / 2 force
    return conv_tc(x_dev, u_tc_dev, y_dev, N, C, H, W, K, pad, stride, mode, m, ws_dev, ws_bytes, stream);
}


extern "C++" {
namespace {
std::atomic<uint64_t> g_attr_tc16[2][4][2][2];  // [DT][XM 0..3][MM == 64][SK]
template <int DT, int XM, int MM, bool SK>
wino_status_t launch_tc16(const wino::tc16::Params& prm, int64_t ctas, int dev, cudaStream_t st) {
    auto kern = wino::tc16::fused_tc16_kernel<DT, XM, MM, SK>;
    constexpr int smem = wino::tc16::Cfg<MM>::BYTES;
    wino_status_t s = ensure_smem_attr(kern, dev, smem, g_attr_tc16[DT][XM][MM == 64][SK]);
    if (s != WINO_OK) return s;
    kern<<<dim3(static_cast<unsigned>(ctas)), wino::tc16::NT, smem, st>>>(prm);
    cudaError_t e = cudaGetLastError();
    if (e == cudaSuccess && SK && ctas > 1) {
        wino::tc16::tc16_fixup_kernel<DT, MM><<<dim3(static_cast<unsigned>(wino::tc16::FIX_PARTS * (ctas - 1))), 256, 0,
                                                st>>>(
            prm, static_cast<int>(ctas));
        e = cudaGetLastError();
    }
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}
bool half_type_ok(wino_half_t t) { return t == WINO_HALF_FP16 || t == WINO_HALF_BF16; }
template <int DT, int MM>
wino_status_t launch_tc16_xm(const wino::tc16::Params& prm, int xm, bool sk, int64_t ctas, int dev,
                             cudaStream_t st) {
    if (sk) {
        if (xm == 2) return launch_tc16<DT, 2, MM, true>(prm, ctas, dev, st);
        if (xm == 3) return launch_tc16<DT, 3, MM, true>(prm, ctas, dev, st);
        return launch_tc16<DT, 0, MM, true>(prm, ctas, dev, st);
    }
    if (xm == 2) return launch_tc16<DT, 2, MM, false>(prm, ctas, dev, st);
    if (xm == 3) return launch_tc16<DT, 3, MM, false>(prm, ctas, dev, st);
    return launch_tc16<DT, 0, MM, false>(prm, ctas, dev, st);
}

}  // namespace
}  // extern "C++"

size_t wino_filter_workspace_bytes_half(int C, int K) {
    if (C <= 0 || K <= 0) return 0;
    return wino::tc16::u_h_elems(C, K) * 2;
}

wino_status_t wino_filter_transform_half(const void* w_dev, void* u_h_dev, int C, int K, wino_half_t type,
                                         wino_stream_t stream) {
    if (!w_dev || !u_h_dev || C <= 0 || K <= 0 || !half_type_ok(type)) return WINO_ERR_INVALID_ARG;
    const size_t ub = wino_filter_workspace_bytes_half(C, K);
    if (ub / 2 > size_t(kMaxElems) || int64_t(9) * C * K > kMaxElems) return WINO_ERR_TOO_LARGE;
    if (!aligned16(w_dev) || !aligned16(u_h_dev)) return WINO_ERR_MISALIGNED;
    if (overlaps(w_dev, size_t(9) * C * K * 2, u_h_dev, ub)) return WINO_ERR_INVALID_ARG;
    int dev;
    wino_status_t s = check_device(&dev);
    if (s != WINO_OK) return s;
    using namespace wino::tc16;
    const int mm = tc16_mm(K);
    const int64_t Kp = ((K + mm - 1) / mm) * mm, C8 = ((C + BC - 1) / BC) * (BC / 8);
    const dim3 blocks(static_cast<unsigned>(Kp / 32), static_cast<unsigned>(C8));
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    const uint16_t* w = static_cast<const uint16_t*>(w_dev);
    uint16_t* u = static_cast<uint16_t*>(u_h_dev);
    if (type == WINO_HALF_FP16) {
        if (mm == 64) tc16_filter_kernel<0, 64><<<blocks, 256, 0, st>>>(w, u, C, K);
        else tc16_filter_kernel<0, 128><<<blocks, 256, 0, st>>>(w, u, C, K);
    } else {
        if (mm == 64) tc16_filter_kernel<1, 64><<<blocks, 256, 0, st>>>(w, u, C, K);
        else tc16_filter_kernel<1, 128><<<blocks, 256, 0, st>>>(w, u, C, K);
    }
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}

extern "C++" {
namespace {
// sk: 0 = never, 1 = planner's choice, 2 = always (stream-K needs ws >= tc16_sk_bytes(SMs))
wino_status_t conv_half(const void* x_dev, const void* u_h_dev, void* y_dev, int N, int C, int H, int W, int K,
                        int pad, int stride, wino_half_t type, int sk, void* ws_dev, size_t ws_bytes,
                        wino_stream_t stream) {
    if (!x_dev || !u_h_dev || !y_dev || !half_type_ok(type)) return WINO_ERR_INVALID_ARG;
    wino_status_t s = check_shape(N, C, H, W, K, pad, stride);
    if (s != WINO_OK) return s;
    if (wino_filter_workspace_bytes_half(C, K) / 2 > size_t(kMaxElems)) return WINO_ERR_TOO_LARGE;
    if (!aligned16(x_dev) || !aligned16(u_h_dev) || !aligned16(y_dev) || (ws_dev && !aligned16(ws_dev)))
        return WINO_ERR_MISALIGNED;
    const size_t hwn = size_t(H) * W * N;
    const size_t yb = size_t(K) * hwn * 2, xb = size_t(C) * hwn * 2, ub = wino_filter_workspace_bytes_half(C, K);
    if (overlaps(y_dev, yb, x_dev, xb) || overlaps(y_dev, yb, u_h_dev, ub)) return WINO_ERR_INVALID_ARG;
    if (ws_dev && (overlaps(ws_dev, ws_bytes, x_dev, xb) || overlaps(ws_dev, ws_bytes, u_h_dev, ub) ||
                   overlaps(ws_dev, ws_bytes, y_dev, yb)))
        return WINO_ERR_INVALID_ARG;
    int dev;
    if ((s = check_device(&dev)) != WINO_OK) return s;
    using namespace wino::tc16;
    Params prm;
    std::memset(&prm, 0, sizeof(prm));
    prm.x = static_cast<const uint16_t*>(x_dev);
    prm.u = static_cast<const uint16_t*>(u_h_dev);
    prm.y = static_cast<uint16_t*>(y_dev);
    prm.N = N;
    prm.C = C;
    prm.H = H;
    prm.W = W;
    prm.K = K;
    prm.TW = (W + 1) / 2;
    prm.NV = N * ((H + 1) / 2) * prm.TW;
    const int mm = tc16_mm(K), tn = BN * (128 / mm);
    prm.num_kb = (K + mm - 1) / mm;
    prm.num_cb = (C + BC - 1) / BC;
    prm.num_tiles = ((prm.NV + tn - 1) / tn) * prm.num_kb;
    const int xm = (N % 32 == 0) ? 2 : ((N == 8 || N == 16) ? 3 : 0);
    const CUtensorMapDataType dt =
        type == WINO_HALF_FP16 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16;
    if (xm >= 2) {
        const cuuint64_t dims[4] = {cuuint64_t(N), cuuint64_t(W), cuuint64_t(H), cuuint64_t(C)};
        const cuuint32_t box[4] = {cuuint32_t(xm == 2 ? BN : N), 4, 4, BC};
        if (!encode_map(&prm.tmx, x_dev, 4, dims, box, nullptr, dt, 2)) return cuda_fail(cudaErrorInvalidValue);
    }
    const int sms = sm_count(dev) < 256 ? sm_count(dev) : 256;
    int64_t ctas = prm.num_tiles < sms ? prm.num_tiles : sms;  // persistent
    // stream-K: equal (tile, channel block) ranges on every SM when the tiles leave SMs idle or
    // end in a partial wave (estimate in channel-block times: waves x blocks vs units / SMs + 3)
    const double units = double(prm.num_tiles) * prm.num_cb;
    const bool sk_ok = ws_dev && ws_bytes >= tc16_sk_bytes(sms) && units < 2147483647.0;
    if (sk == 2 && !sk_ok) return WINO_ERR_INVALID_ARG;
    const bool use_sk = sk == 2 || (sk == 1 && sk_ok && tc16_sk_pays(prm.num_tiles, prm.num_cb, sms));
    if (use_sk) {
        ctas = sms;
        prm.sk_ws = static_cast<float*>(ws_dev);
        prm.sk_q = static_cast<int>(int64_t(units) / sms);
        prm.sk_r = static_cast<int>(int64_t(units) % sms);
    }
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    if (type == WINO_HALF_FP16)
        return mm == 64 ? launch_tc16_xm<0, 64>(prm, xm, use_sk, ctas, dev, st)
                        : launch_tc16_xm<0, 128>(prm, xm, use_sk, ctas, dev, st);
    return mm == 64 ? launch_tc16_xm<1, 64>(prm, xm, use_sk, ctas, dev, st)
                    : launch_tc16_xm<1, 128>(prm, xm, use_sk, ctas, dev, st);
}
}  // namespace
}  // extern "C++"

wino_status_t wino_conv2d_f2x3_fwd_half(const void* x_dev, const void* u_h_dev, void* y_dev, int N, int C, int H,
                                        int W, int K, int pad, int stride, wino_half_t type, wino_stream_t stream) {
    return conv_half(x_dev, u_h_dev, y_dev, N, C, H, W, K, pad, stride, type, 0, nullptr, 0, stream);
}

size_t wino_half_workspace_bytes(int N, int C, int H, int W, int K) {
    if (check_shape(N, C, H, W, K, 1, 1) != WINO_OK) return 0;
    int dev = -1, sms = 148;
    if (check_device(&dev) == WINO_OK) sms = sm_count(dev);
    else cudaGetLastError();
    return tc16_sk_bytes(sms < 256 ? sms : 256);
}

wino_status_t wino_conv2d_f2x3_fwd_half_ws(const void* x_dev, const void* u_h_dev, void* y_dev, int N, int C, int H,
                                           int W, int K, int pad, int stride, wino_half_t type, int sk,
                                           void* ws_dev, size_t ws_bytes, wino_stream_t stream) {
    if (sk < 0 || sk > 2 || (ws_bytes > 0 && !ws_dev)) return WINO_ERR_INVALID_ARG;
    const int mode = sk == 0 ? 1 : (sk == 1 ? 0 : 2);  // API 0 auto / 1 off / 2 force
    return conv_half(x_dev, u_h_dev, y_dev, N, C, H, W, K, pad, stride, type, mode, ws_dev, ws_bytes, stream);
}

size_t wino_host_workspace_bytes(int N, int C, int H, int W, int K) {
    if (check_shape(N, C, H, W, K, 1, 1) != WINO_OK) return 0;
    const size_t hwn = size_t(H) * W * N;
    return round_up256(size_t(C) * hwn * 4) + round_up256(size_t(9) * C * K * 4) +
           round_up256(size_t(16) * C * K * 4) + round_up256(size_t(K) * hwn * 4);
}

wino_status_t wino_conv2d_f2x3_fwd_host(const float* x_host, const float* w_host, float* y_host, int N, int C,
                                        int H, int W, int K, int pad, int stride, void* ws_dev, size_t ws_bytes,
                                        wino_stream_t stream) {
    if (!x_host || !w_host || !y_host || !ws_dev) return WINO_ERR_INVALID_ARG;
    wino_status_t s = check_shape(N, C, H, W, K, pad, stride);
    if (s != WINO_OK) return s;
    if (ws_bytes < wino_host_workspace_bytes(N, C, H, W, K)) return WINO_ERR_INVALID_ARG;
    if (!aligned16(ws_dev)) return WINO_ERR_MISALIGNED;
    const size_t hwn = size_t(H) * W * N;
    const size_t xb = size_t(C) * hwn * 4, wb = size_t(9) * C * K * 4, ub = size_t(16) * C * K * 4,
                 yb = size_t(K) * hwn * 4;
    char* base = static_cast<char*>(ws_dev);
    float* x_dev = reinterpret_cast<float*>(base);
    float* w_dev = reinterpret_cast<float*>(base + round_up256(xb));
    float* u_dev = reinterpret_cast<float*>(base + round_up256(xb) + round_up256(wb));
    float* y_dev = reinterpret_cast<float*>(base + round_up256(xb) + round_up256(wb) + round_up256(ub));
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    cudaError_t e;
    if ((e = cudaMemcpyAsync(w_dev, w_host, wb, cudaMemcpyHostToDevice, st)) != cudaSuccess) return cuda_fail(e);
    if ((s = wino_filter_transform(w_dev, u_dev, C, K, stream)) != WINO_OK) return s;
    if ((e = cudaMemcpyAsync(x_dev, x_host, xb, cudaMemcpyHostToDevice, st)) != cudaSuccess) return cuda_fail(e);
    if ((s = wino_conv2d_f2x3_fwd(x_dev, u_dev, y_dev, N, C, H, W, K, pad, stride, stream)) != WINO_OK) return s;
    if ((e = cudaMemcpyAsync(y_host, y_dev, yb, cudaMemcpyDeviceToHost, st)) != cudaSuccess) return cuda_fail(e);
    return WINO_OK;
}

size_t wino_host_multi_workspace_bytes(const wino_host_layer_t* layers, int n_layers) {
    if (!layers || n_layers <= 0) return 0;
    size_t total = 0;
    for (int i = 0; i < n_layers; ++i) {
        const wino_host_layer_t& L = layers[i];
        const size_t b = wino_host_workspace_bytes(L.N, L.C, L.H, L.W, L.K);
        if (b == 0) return 0;
        total += b;
    }
    return total;
}

wino_status_t wino_conv2d_f2x3_fwd_host_multi(const wino_host_layer_t* layers, int n_layers, void* ws_dev,
                                              size_t ws_bytes, wino_stream_t stream) {
    if (!layers || n_layers <= 0 || !ws_dev) return WINO_ERR_INVALID_ARG;
    // per layer: slice along K (contiguous copies) when K >= 128, else along the batch (2-D copies)
    auto slices = [](const wino_host_layer_t& L, bool* kslice) {
        *kslice = L.K >= 128;
        return *kslice ? (L.K >= 256 ? 4 : 2) : (L.N >= 128 && L.N % 64 == 0 ? L.N / 64 : 1);
    };
    int64_t n_events = 1 + 1 + 2;  // fork, final join, error-path joins (s_in, s_out)
    for (int i = 0; i < n_layers; ++i) {
        const wino_host_layer_t& L = layers[i];
        if (!L.x_host || !L.w_host || !L.y_host) return WINO_ERR_INVALID_ARG;
        wino_status_t s = check_shape(L.N, L.C, L.H, L.W, L.K, 1, 1);
        if (s != WINO_OK) return s;
        bool ks;
        const int ns = slices(L, &ks);
        n_events += 1 + ((ks || ns == 1) ? 1 + ns : 2 * ns);
    }
    if (n_events > 65536) return WINO_ERR_TOO_LARGE;
    if (ws_bytes < wino_host_multi_workspace_bytes(layers, n_layers)) return WINO_ERR_INVALID_ARG;
    if (!aligned16(ws_dev)) return WINO_ERR_MISALIGNED;
    int dev;
    wino_status_t s = check_device(&dev);
    if (s != WINO_OK) return s;
    cudaStream_t s_in, s_out;
    if ((s = helper_streams(dev, &s_in, &s_out)) != WINO_OK) return s;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    EventPool ev;  // every event this call needs, created before anything is queued
    cudaError_t e = ev.reserve(static_cast<int>(n_events));
    if (e != cudaSuccess) return cuda_fail(e);
    cudaEvent_t j_in = ev.get(), j_out = ev.get();
    // Error after work was queued: the caller's stream must still not run ahead of the copies
    // already queued on the helper streams (they read / write the caller's host buffers).
    auto fail = [&](wino_status_t status) {
        if (cudaEventRecord(j_in, s_in) == cudaSuccess) cudaStreamWaitEvent(st, j_in, 0);
        if (cudaEventRecord(j_out, s_out) == cudaSuccess) cudaStreamWaitEvent(st, j_out, 0);
        return status;
    };
#define WINO_TRY(expr)                                        \
    do {                                                      \
        if ((e = (expr)) != cudaSuccess) return fail(cuda_fail(e)); \
    } while (0)
    cudaEvent_t e0 = ev.get();
    WINO_TRY(cudaEventRecord(e0, st));
    WINO_TRY(cudaStreamWaitEvent(s_in, e0, 0));
    WINO_TRY(cudaStreamWaitEvent(s_out, e0, 0));
    char* base = static_cast<char*>(ws_dev);
    for (int i = 0; i < n_layers; ++i) {
        const wino_host_layer_t& L = layers[i];
        const size_t hw = size_t(L.H) * L.W, hwn = hw * L.N;
        const size_t xb = size_t(L.C) * hwn * 4, wb = size_t(9) * L.C * L.K * 4, ub = size_t(16) * L.C * L.K * 4,
                     yb = size_t(L.K) * hwn * 4;
        float* x_dev = reinterpret_cast<float*>(base);
        float* w_dev = reinterpret_cast<float*>(base + round_up256(xb));
        float* u_dev = reinterpret_cast<float*>(base + round_up256(xb) + round_up256(wb));
        float* y_dev = reinterpret_cast<float*>(base + round_up256(xb) + round_up256(wb) + round_up256(ub));
        base += round_up256(xb) + round_up256(wb) + round_up256(ub) + round_up256(yb);
        // weights in, FTF on the compute stream
        WINO_TRY(cudaMemcpyAsync(w_dev, L.w_host, wb, cudaMemcpyHostToDevice, s_in));
        cudaEvent_t ew = ev.get();
        WINO_TRY(cudaEventRecord(ew, s_in));
        WINO_TRY(cudaStreamWaitEvent(st, ew, 0));
        if ((s = wino_filter_transform(w_dev, u_dev, L.C, L.K, stream)) != WINO_OK) return fail(s);
        bool kslice;
        const int nslice = slices(L, &kslice);
        if (kslice || nslice == 1) {
            WINO_TRY(cudaMemcpyAsync(x_dev, L.x_host, xb, cudaMemcpyHostToDevice, s_in));
            cudaEvent_t ex = ev.get();
            WINO_TRY(cudaEventRecord(ex, s_in));
            WINO_TRY(cudaStreamWaitEvent(st, ex, 0));
            const int kc = ((L.K + nslice - 1) / nslice + 63) / 64 * 64;
            for (int k0 = 0; k0 < L.K; k0 += kc) {
                const int k1 = k0 + kc < L.K ? k0 + kc : L.K;
                if ((s = launch_fwd_fp32(x_dev, u_dev + k0, L.K, y_dev + size_t(k0) * hwn, L.N, L.C, L.H, L.W,
                                         k1 - k0, dev, st)) != WINO_OK)
                    return fail(s);
                cudaEvent_t ec = ev.get();
                WINO_TRY(cudaEventRecord(ec, st));
                WINO_TRY(cudaStreamWaitEvent(s_out, ec, 0));
                WINO_TRY(cudaMemcpyAsync(L.y_host + size_t(k0) * hwn, y_dev + size_t(k0) * hwn,
                                         size_t(k1 - k0) * hwn * 4, cudaMemcpyDeviceToHost, s_out));
            }
        } else {
            const int nc = L.N / nslice;  // batch slice, rows of nc*4 = 256 B
            const size_t xs_elems = size_t(L.C) * hw * nc, ys_elems = size_t(L.K) * hw * nc;
            for (int j = 0; j < nslice; ++j) {
                float* xj = x_dev + j * xs_elems;
                float* yj = y_dev + j * ys_elems;
                WINO_TRY(cudaMemcpy2DAsync(xj, size_t(nc) * 4, L.x_host + size_t(j) * nc, size_t(L.N) * 4,
                                           size_t(nc) * 4, size_t(L.C) * hw, cudaMemcpyHostToDevice, s_in));
                cudaEvent_t ex = ev.get();
                WINO_TRY(cudaEventRecord(ex, s_in));
                WINO_TRY(cudaStreamWaitEvent(st, ex, 0));
                if ((s = launch_fwd_fp32(xj, u_dev, L.K, yj, nc, L.C, L.H, L.W, L.K, dev, st)) != WINO_OK)
                    return fail(s);
                cudaEvent_t ec = ev.get();
                WINO_TRY(cudaEventRecord(ec, st));
                WINO_TRY(cudaStreamWaitEvent(s_out, ec, 0));
                WINO_TRY(cudaMemcpy2DAsync(L.y_host + size_t(j) * nc, size_t(L.N) * 4, yj, size_t(nc) * 4,
                                           size_t(nc) * 4, size_t(L.K) * hw, cudaMemcpyDeviceToHost, s_out));
            }
        }
    }
    cudaEvent_t eo = ev.get();
    WINO_TRY(cudaEventRecord(eo, s_out));
    WINO_TRY(cudaStreamWaitEvent(st, eo, 0));  // caller's stream completes after every copy
#undef WINO_TRY
    return WINO_OK;
}

size_t wino_filter_workspace_bytes_f4(int C, int K) {
    if (C <= 0 || K <= 0) return 0;
    return size_t(36) * size_t(C) * size_t(K) * sizeof(float);
}

wino_status_t wino_filter_transform_f4(const float* w_dev, float* u4_dev, int C, int K, wino_stream_t stream) {
    if (!w_dev || !u4_dev || C <= 0 || K <= 0) return WINO_ERR_INVALID_ARG;
    if (int64_t(36) * C * K > kMaxElems) return WINO_ERR_TOO_LARGE;
    if (!aligned16(w_dev) || !aligned16(u4_dev)) return WINO_ERR_MISALIGNED;
    if (overlaps(w_dev, size_t(9) * C * K * 4, u4_dev, size_t(36) * C * K * 4)) return WINO_ERR_INVALID_ARG;
    int dev;
    wino_status_t s = check_device(&dev);
    if (s != WINO_OK) return s;
    const unsigned blocks = static_cast<unsigned>((int64_t(C) * K + 255) / 256);
    wino::f4::ftf4_kernel<<<blocks, 256, 0, reinterpret_cast<cudaStream_t>(stream)>>>(w_dev, u4_dev, C, K);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}

extern "C++" {
namespace {
std::atomic<uint64_t> g_attr_f4_sk[2];
// sk: 0 = never, 1 = planner's choice, 2 = always (needs ws >= f4 workspace bytes)
wino_status_t conv_f4(const float* x_dev, const float* u4_dev, float* y_dev, int N, int C, int H, int W, int K,
                      int pad, int stride, int sk, void* ws_dev, size_t ws_bytes, wino_stream_t stream) {
    if (!x_dev || !u4_dev || !y_dev) return WINO_ERR_INVALID_ARG;
    wino_status_t s = check_shape(N, C, H, W, K, pad, stride);
    if (s != WINO_OK) return s;
    if (int64_t(36) * C * K > kMaxElems) return WINO_ERR_TOO_LARGE;
    if (!aligned16(x_dev) || !aligned16(u4_dev) || !aligned16(y_dev) || (ws_dev && !aligned16(ws_dev)))
        return WINO_ERR_MISALIGNED;
    const size_t hwn = size_t(H) * W * N;
    const size_t yb = size_t(K) * hwn * 4;
    if (overlaps(y_dev, yb, x_dev, size_t(C) * hwn * 4) || overlaps(y_dev, yb, u4_dev, size_t(36) * C * K * 4))
        return WINO_ERR_INVALID_ARG;
    int dev;
    if ((s = check_device(&dev)) != WINO_OK) return s;
    using namespace wino::f4;
    Params prm;
    std::memset(&prm, 0, sizeof(prm));
    prm.y = y_dev;
    prm.x = x_dev;
    prm.u4 = u4_dev;
    prm.u_vec = K % 4 == 0 ? 1 : 0;
    prm.N = N;
    prm.C = C;
    prm.H = H;
    prm.W = W;
    prm.K = K;
    prm.TW = (W + 3) / 4;
    prm.NV = N * ((H + 3) / 4) * prm.TW;
    prm.num_kb = (K + BK - 1) / BK;
    prm.num_it = (C + BC - 1) / BC;
    prm.num_tiles = ((prm.NV + BN - 1) / BN) * prm.num_kb;
    // TMA boxes need the tile's 16 nu to be 16 consecutive n (N % 16) and 16-byte u rows (K % 4);
    // any other shape gathers with cp.async (generic path, same arithmetic)
    const bool gen = N % 16 != 0 || K % 4 != 0;
    if (!gen) {
        {
            const cuuint64_t dims[4] = {cuuint64_t(N), cuuint64_t(W), cuuint64_t(H), cuuint64_t(C)};
            const cuuint32_t box[4] = {BN, 6, 6, BC};
            if (!encode_map(&prm.tmx, x_dev, 4, dims, box)) return cuda_fail(cudaErrorInvalidValue);
        }
        {
            const cuuint64_t dims[3] = {cuuint64_t(K), 36, cuuint64_t(C)};
            const cuuint32_t box[3] = {BK, 36, BC};
            if (!encode_map(&prm.tmu, u4_dev, 3, dims, box)) return cuda_fail(cudaErrorInvalidValue);
        }
    }
    if (ws_dev && (overlaps(ws_dev, ws_bytes, x_dev, size_t(C) * hwn * 4) || overlaps(ws_dev, ws_bytes, y_dev, yb) ||
                   overlaps(ws_dev, ws_bytes, u4_dev, size_t(36) * C * K * 4)))
        return WINO_ERR_INVALID_ARG;
    const int sms = sm_count(dev) < 256 ? sm_count(dev) : 256;
    int grid = prm.num_tiles < sms ? prm.num_tiles : sms;
    // stream-K (as the F(2x2) kernel): estimates in 4-channel-block times, tile epilogue ~2 blocks
    const double units = double(prm.num_tiles) * prm.num_it;
    const bool sk_ok = ws_dev && ws_bytes >= f4_sk_bytes(sms) && units < 2147483647.0;
    if (sk == 2 && !sk_ok) return WINO_ERR_INVALID_ARG;
    bool use_sk = sk == 2;
    if (sk == 1 && sk_ok) {
        const double reg = std::ceil(double(prm.num_tiles) / sms) * (prm.num_it + 2.0);
        use_sk = std::ceil(units / sms) + 2.0 * (double(prm.num_tiles) / sms + 1.0) + 4.0 < 0.97 * reg;
    }
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    cudaError_t e;
    if (use_sk) {
        grid = sms;
        prm.sk_ws = static_cast<float*>(ws_dev);
        prm.sk_q = static_cast<int>(int64_t(units) / sms);
        prm.sk_r = static_cast<int>(int64_t(units) % sms);
        auto kern = gen ? fused_f4_kernel<true, true> : fused_f4_kernel<true, false>;
        if ((s = ensure_smem_attr(kern, dev, Smem::bytes, g_attr_f4_sk[gen])) != WINO_OK) return s;
        kern<<<grid, NT, Smem::bytes, st>>>(prm);
        e = cudaGetLastError();
        if (e == cudaSuccess && grid > 1) {
            f4_fixup_kernel<<<FIX_PARTS * (grid - 1), 256, 0, st>>>(prm, grid);
            e = cudaGetLastError();
        }
    } else {
        auto kern = gen ? fused_f4_kernel<false, true> : fused_f4_kernel<false, false>;
        if ((s = ensure_smem_attr(kern, dev, Smem::bytes, g_attr_f4[gen])) != WINO_OK) return s;
        kern<<<grid, NT, Smem::bytes, st>>>(prm);
        e = cudaGetLastError();
    }
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}
}  // namespace
}  // extern "C++"

wino_status_t wino_conv2d_f4x3_fwd(const float* x_dev, const float* u4_dev, float* y_dev, int N, int C, int H,
                                   int W, int K, int pad, int stride, wino_stream_t stream) {
    return conv_f4(x_dev, u4_dev, y_dev, N, C, H, W, K, pad, stride, 0, nullptr, 0, stream);
}

size_t wino_f4_workspace_bytes(int N, int C, int H, int W, int K) {
    if (check_shape(N, C, H, W, K, 1, 1) != WINO_OK) return 0;
    int dev = -1, sms = 148;
    if (check_device(&dev) == WINO_OK) sms = sm_count(dev);
    else cudaGetLastError();
    return f4_sk_bytes(sms < 256 ? sms : 256);
}

wino_status_t wino_conv2d_f4x3_fwd_ws(const float* x_dev, const float* u4_dev, float* y_dev, int N, int C, int H,
                                      int W, int K, int pad, int stride, int sk, void* ws_dev, size_t ws_bytes,
                                      wino_stream_t stream) {
    if (sk < 0 || sk > 2 || (ws_bytes > 0 && !ws_dev)) return WINO_ERR_INVALID_ARG;
    const int m = sk == 0 ? 1 : (sk == 1 ? 0 : 2);  // API 0 auto / 1 off / 2 force
    return conv_f4(x_dev, u4_dev, y_dev, N, C, H, W, K, pad, stride, m, ws_dev, ws_bytes, stream);
}

}  // extern "C"

// ---------------------------------------------------------------------------
// NEXT row N3: non-fused Winograd (u arrangement, ITF kernel -> V workspace, 16 batched
// tcgen05 GEMMs -> M workspace, OTF kernel); nonfused_tc.cuh
// ---------------------------------------------------------------------------
namespace {
// workspace carve-up for P planes (P = 2: 3xTF32, the FP32-accuracy variant; P = 1: TF32)
struct NfLayout {
    size_t v_off, u_off, m_off, total;
};
NfLayout nf_layout(int N, int C, int H, int W, int K, int P) {
    const size_t nv = size_t(N) * ((H + 1) / 2) * ((W + 1) / 2), c4 = size_t(wino::nftc::cp4(C));
    NfLayout L;
    L.v_off = 0;
    L.u_off = round_up256(size_t(16) * P * nv * c4 * 4);
    L.m_off = L.u_off + round_up256(size_t(16) * P * K * c4 * 4);
    L.total = L.m_off + round_up256(size_t(16) * K * nv * 4);
    return L;
}
std::atomic<uint64_t> g_attr_nf_gemm[2], g_attr_nf_itf[2];

template <int P>
wino_status_t nonfused_launch(const float* x_dev, const float* u_dev, float* y_dev, int N, int C, int H, int W, int K,
                              char* ws, int dev, cudaStream_t st) {
    using namespace wino::nftc;
    const NfLayout L = nf_layout(N, C, H, W, K, P);
    float* v = reinterpret_cast<float*>(ws + L.v_off);
    float* ug = reinterpret_cast<float*>(ws + L.u_off);
    float* m = reinterpret_cast<float*>(ws + L.m_off);
    const int TW = (W + 1) / 2;
    const int NV = N * ((H + 1) / 2) * TW;
    const int C4 = cp4(C), bnk = gemm_bnk(K);
    GemmParams gp;
    std::memset(&gp, 0, sizeof(gp));
    {
        const cuuint64_t dims[3] = {cuuint64_t(C), cuuint64_t(NV), cuuint64_t(16 * P)};
        const cuuint64_t strides[2] = {cuuint64_t(C4) * 4, cuuint64_t(NV) * C4 * 4};
        const cuuint32_t box[3] = {BKC, BM, 1};
        if (!encode_map(&gp.tmv, v, 3, dims, box, strides, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4,
                        CU_TENSOR_MAP_SWIZZLE_128B))
            return cuda_fail(cudaErrorInvalidValue);
    }
    {
        const cuuint64_t dims[3] = {cuuint64_t(C), cuuint64_t(K), cuuint64_t(16 * P)};
        const cuuint64_t strides[2] = {cuuint64_t(C4) * 4, cuuint64_t(K) * C4 * 4};
        const cuuint32_t box[3] = {BKC, cuuint32_t(bnk), 1};
        if (!encode_map(&gp.tmu, ug, 3, dims, box, strides, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4,
                        CU_TENSOR_MAP_SWIZZLE_128B))
            return cuda_fail(cudaErrorInvalidValue);
    }
    gp.m = m;
    gp.K = K;
    gp.NV = NV;
    gp.C = C;
    gp.bnk = bnk;
    gp.nchunks = (C + BKC - 1) / BKC;
    gp.stages = gemm_stages_for<P>(bnk, gp.nchunks);
    wino_status_t s;
    // 1. transformed filter -> GEMM operand layout (TF32 planes)
    nf_arrange_u_kernel<P><<<dim3(unsigned((K + 31) / 32), unsigned((C4 + 31) / 32), 16), 256, 0, st>>>(u_dev, ug, C,
                                                                                                       K);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e);
    // 2. ITF -> V [16 P][NV][C4]
    if ((s = ensure_smem_attr(nf_itf_kernel<P>, dev, ITF_SMEM, g_attr_nf_itf[P - 1])) != WINO_OK) return s;
    nf_itf_kernel<P><<<dim3(unsigned((NV + 31) / 32), unsigned((C4 + 31) / 32)), 256, ITF_SMEM, st>>>(x_dev, v, N, C,
                                                                                                     H, W, TW, NV);
    if ((e = cudaGetLastError()) != cudaSuccess) return cuda_fail(e);
    // 3. the 16 batched GEMMs on tcgen05: M[xi][k][nu]
    const int smem = gemm_smem_bytes<P>(bnk, gp.stages);
    if ((s = ensure_smem_attr(nf_gemm_kernel<P>, dev, gemm_smem_bytes<P>(256, gemm_stages<P>(256)),
                              g_attr_nf_gemm[P - 1])) != WINO_OK)
        return s;
    nf_gemm_kernel<P><<<dim3(unsigned((NV + BM - 1) / BM), unsigned((K + bnk - 1) / bnk), 16), GEMM_THREADS, smem,
                        st>>>(gp);
    if ((e = cudaGetLastError()) != cudaSuccess) return cuda_fail(e);
    // 4. OTF -> y
    wino::nf::otf_nf_kernel<<<unsigned((int64_t(K) * NV + wino::nf::THREADS - 1) / wino::nf::THREADS),
                              wino::nf::THREADS, 0, st>>>(m, y_dev, N, K, H, W, TW, NV);
    e = cudaGetLastError();
    return e == cudaSuccess ? WINO_OK : cuda_fail(e);
}
}  // namespace

extern "C" {

size_t wino_nonfused_workspace_bytes(int N, int C, int H, int W, int K) {
    if (check_shape(N, C, H, W, K, 1, 1) != WINO_OK) return 0;
    return nf_layout(N, C, H, W, K, 2).total;  // the 3xTF32 (two-plane) layout; TF32 uses a prefix of it
}

int wino_nonfused_launches(void) { return 4; }

extern "C++" {
namespace {
wino_status_t conv_nonfused(const float* x_dev, const float* u_dev, float* y_dev, int N, int C, int H, int W, int K,
                            int pad, int stride, void* ws_dev, size_t ws_bytes, bool tf32, wino_stream_t stream) {
    if (!x_dev || !u_dev || !y_dev || !ws_dev) return WINO_ERR_INVALID_ARG;
    wino_status_t s = check_shape(N, C, H, W, K, pad, stride);
    if (s != WINO_OK) return s;
    if (!aligned16(x_dev) || !aligned16(u_dev) || !aligned16(y_dev) || !aligned16(ws_dev)) return WINO_ERR_MISALIGNED;
    const int P = tf32 ? 1 : 2;
    const NfLayout L = nf_layout(N, C, H, W, K, P);
    if (ws_bytes < L.total) return WINO_ERR_INVALID_ARG;
    const long long nv = (long long)N * ((H + 1) / 2) * ((W + 1) / 2);
    const long long c4 = wino::nftc::cp4(C);
    if ((long long)16 * 2 * c4 * nv > kMaxElems || (long long)16 * K * nv > kMaxElems) return WINO_ERR_TOO_LARGE;
    const size_t hwn = size_t(H) * W * N, yb = size_t(K) * hwn * 4;
    if (overlaps(y_dev, yb, x_dev, size_t(C) * hwn * 4) || overlaps(y_dev, yb, u_dev, size_t(16) * C * K * 4) ||
        overlaps(ws_dev, L.total, x_dev, size_t(C) * hwn * 4) || overlaps(ws_dev, L.total, u_dev, size_t(16) * C * K * 4) ||
        overlaps(ws_dev, L.total, y_dev, yb))
        return WINO_ERR_INVALID_ARG;
    int dev;
    if ((s = check_device(&dev)) != WINO_OK) return s;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    return tf32 ? nonfused_launch<1>(x_dev, u_dev, y_dev, N, C, H, W, K, static_cast<char*>(ws_dev), dev, st)
                : nonfused_launch<2>(x_dev, u_dev, y_dev, N, C, H, W, K, static_cast<char*>(ws_dev), dev, st);
}
}  // namespace
}  // extern "C++"

wino_status_t wino_conv2d_f2x3_fwd_nonfused(const float* x_dev, const float* u_dev, float* y_dev, int N, int C,
                                            int H, int W, int K, int pad, int stride, void* ws_dev, size_t ws_bytes,
                                            wino_stream_t stream) {
    return conv_nonfused(x_dev, u_dev, y_dev, N, C, H, W, K, pad, stride, ws_dev, ws_bytes, false, stream);
}

wino_status_t wino_conv2d_f2x3_fwd_nonfused_tf32(const float* x_dev, const float* u_dev, float* y_dev, int N, int C,
                                                 int H, int W, int K, int pad, int stride, void* ws_dev,
                                                 size_t ws_bytes, wino_stream_t stream) {
    return conv_nonfused(x_dev, u_dev, y_dev, N, C, H, W, K, pad, stride, ws_dev, ws_bytes, true, stream);
}

}  // extern "C"
