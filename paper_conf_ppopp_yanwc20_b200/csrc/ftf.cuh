// ftf.cuh -- filter-transform kernel (FTF), the separate kernel of Sec. 3.1
// (L209) / Sec. 4.1 (L345): u[c,:,:,k] = G w[c,:,:,k] G^T (Eq. 5).
//
// HBM-bound (Fig. 2): 36 B read + 64 B written per (c,k).  Threads run
// with k fastest, so each of the 9 loads and 16 stores is a fully coalesced warp
// access along K (the "CR'S'K" layout of Table 4).  wino_filter_transform is
// ftf_multi_kernel with one job.
#pragma once
#include "wino_transforms.cuh"

namespace wino {

constexpr int FTF_THREADS = 256;

// Same transform reading PyTorch's weight layout w (K,C,3,3) ("KCRS"), writing u
// (C,4,4,K): the NCHW front end (Sec. 8.4).  k fastest across threads, so the
// 16 stores stay coalesced; each thread's 9 loads are one contiguous 36 B run.
__global__ void __launch_bounds__(FTF_THREADS) ftf_kcrs_kernel(const float* __restrict__ w,
                                                               float* __restrict__ u, int C, int K) {
    const long idx = (long)blockIdx.x * FTF_THREADS + threadIdx.x;
    if (idx >= (long)C * K) return;
    const int c = (int)(idx / K), k = (int)(idx - (long)c * K);
    const float* wk = w + ((size_t)k * C + c) * 9;
    float g[9], t[16];
#pragma unroll
    for (int e = 0; e < 9; ++e) g[e] = __ldg(wk + e);
    ftf_4x4(g, t);
    float* uc = u + (size_t)c * 16 * K + k;
#pragma unroll
    for (int e = 0; e < 16; ++e) uc[(size_t)e * K] = t[e];
}

// Several filter transforms in one launch (the layers of a network step): block b belongs to the
// job whose block range [first[j], first[j+1]) holds it.  A job with K % 4 == 0 (vec[j]) gives each
// thread 4 consecutive k: 9 LDG.128 + 16 STG.128 per thread, so a quarter of the threads keep
// 4x the bytes in flight each (the transform is HBM-bound: 100 B per (c,k)); else one (c,k) per thread.
constexpr int FTF_MAX_JOBS = 8;
struct FtfJobs {
    const float* w[FTF_MAX_JOBS];
    float* u[FTF_MAX_JOBS];
    int C[FTF_MAX_JOBS], K[FTF_MAX_JOBS], vec[FTF_MAX_JOBS];
    unsigned first[FTF_MAX_JOBS + 1];
    int n;
};

__global__ void __launch_bounds__(FTF_THREADS) ftf_multi_kernel(const __grid_constant__ FtfJobs jobs) {
    int j = 0;
    while (j + 1 < jobs.n && blockIdx.x >= jobs.first[j + 1]) ++j;
    const int C = jobs.C[j], K = jobs.K[j];
    const long idx = (long)(blockIdx.x - jobs.first[j]) * FTF_THREADS + threadIdx.x;
    if (jobs.vec[j]) {
        const int K4 = K >> 2;
        if (idx >= (long)C * K4) return;
        const int c = (int)(idx / K4), k = 4 * (int)(idx - (long)c * K4);
        const float* wc = jobs.w[j] + (size_t)c * 9 * K + k;
        float4 g4[9];
#pragma unroll
        for (int e = 0; e < 9; ++e) g4[e] = __ldg(reinterpret_cast<const float4*>(wc + (size_t)e * K));
        float t[4][16];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            float g[9];
#pragma unroll
            for (int e = 0; e < 9; ++e) g[e] = q == 0 ? g4[e].x : q == 1 ? g4[e].y : q == 2 ? g4[e].z : g4[e].w;
            ftf_4x4(g, t[q]);
        }
        float* uc = jobs.u[j] + (size_t)c * 16 * K + k;
#pragma unroll
        for (int e = 0; e < 16; ++e)
            *reinterpret_cast<float4*>(uc + (size_t)e * K) = make_float4(t[0][e], t[1][e], t[2][e], t[3][e]);
        return;
    }
    if (idx >= (long)C * K) return;
    const int c = (int)(idx / K), k = (int)(idx - (long)c * K);
    const float* wc = jobs.w[j] + (size_t)c * 9 * K + k;
    float g[9], t[16];
#pragma unroll
    for (int e = 0; e < 9; ++e) g[e] = __ldg(wc + (size_t)e * K);
    ftf_4x4(g, t);
    float* uc = jobs.u[j] + (size_t)c * 16 * K + k;
#pragma unroll
    for (int e = 0; e < 16; ++e) uc[(size_t)e * K] = t[e];
}

}  // namespace wino
