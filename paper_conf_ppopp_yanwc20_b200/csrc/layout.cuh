// layout.cuh -- dense 2-D transpose out[s][r] = in[r][s] (fp32), used by the NCHW
// front end with a workspace (NEXT row N2): x (N, C*H*W) -> (C*H*W, N) = CHWN before
// the fused kernel, y (K*H*W, N) -> (N, K*H*W) = NKHW after it.  HBM-bound: 8 B per
// element; 32 x 32 tiles through padded shared memory so both the loads and the
// stores are 128 B rows.  The grid is 1-D over all (row tile, column tile) pairs (row tiles
// fastest), so neither dimension meets the 65535 limit of gridDim.y.
#pragma once
#include <cstdint>

namespace wino {

constexpr int TR_TILE = 32, TR_ROWS = 8;  // 32 x 8 threads, 4 elements each

__global__ void __launch_bounds__(TR_TILE* TR_ROWS) transpose2d_kernel(const float* __restrict__ in,
                                                                      float* __restrict__ out, int R, long long S) {
    __shared__ float t[TR_TILE][TR_TILE + 1];
    const int nrt = (R + TR_TILE - 1) / TR_TILE;
    const int r0 = static_cast<int>(blockIdx.x % nrt) * TR_TILE;
    const long long s0 = (long long)(blockIdx.x / nrt) * TR_TILE;
    const int tx = threadIdx.x, ty = threadIdx.y;
#pragma unroll
    for (int j = 0; j < TR_TILE; j += TR_ROWS) {
        const int r = r0 + ty + j;
        const long long s = s0 + tx;
        if (r < R && s < S) t[ty + j][tx] = in[(size_t)r * S + s];
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < TR_TILE; j += TR_ROWS) {
        const long long s = s0 + ty + j;
        const int r = r0 + tx;
        if (r < R && s < S) out[(size_t)s * R + r] = t[tx][ty + j];
    }
}

}  // namespace wino
