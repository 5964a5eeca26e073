// wino_transforms.cuh -- the three F(2x2,3x3) tile transforms in FP32 registers.
//
// Yan, Wang & Chu (PPoPP'20), Sec. 2.1 Eq. 1-3 (L85-113) and Sec. 3.1 Eq. 5-8
// (L191-207).  Operation counts follow L115: FTF 28 float instructions,
// ITF 32 FADD, OTF 24 FADD.  Rounding: FP32 round-to-nearest; FMA contraction
// allowed (reading R7).
#pragma once

namespace wino {

// Eq. 5: U = G g G^T, G = [[1,0,0],[1/2,1/2,1/2],[1/2,-1/2,1/2],[0,0,1]].
// Per 3-vector (a,b,c): t = 0.5*(a+c); row1 = t + 0.5*b; row2 = t - 0.5*b
// (4 instructions; 7 vectors -> 28, L115).  g[r][s], u[r'][s'] row-major.
__device__ __forceinline__ void ftf_4x4(const float g[9], float u[16]) {
    float t[4][3];
#pragma unroll
    for (int s = 0; s < 3; ++s) {
        const float a = g[s], b = g[3 + s], c = g[6 + s];
        const float h = 0.5f * (a + c);
        t[0][s] = a;
        t[1][s] = fmaf(0.5f, b, h);
        t[2][s] = fmaf(-0.5f, b, h);
        t[3][s] = c;
    }
#pragma unroll
    for (int r = 0; r < 4; ++r) {
        const float a = t[r][0], b = t[r][1], c = t[r][2];
        const float h = 0.5f * (a + c);
        u[4 * r + 0] = a;
        u[4 * r + 1] = fmaf(0.5f, b, h);
        u[4 * r + 2] = fmaf(-0.5f, b, h);
        u[4 * r + 3] = c;
    }
}

// Eq. 6: V = B^T d B, B^T = [[1,0,-1,0],[0,1,1,0],[0,-1,1,0],[0,1,0,-1]]; 32 FADD.
__device__ __forceinline__ void itf_4x4(const float d[16], float v[16]) {
    float t[16];
#pragma unroll
    for (int c = 0; c < 4; ++c) {  // columns: B^T d
        t[0 + c] = d[0 + c] - d[8 + c];
        t[4 + c] = d[4 + c] + d[8 + c];
        t[8 + c] = d[8 + c] - d[4 + c];
        t[12 + c] = d[4 + c] - d[12 + c];
    }
#pragma unroll
    for (int r = 0; r < 4; ++r) {  // rows: (B^T d) B
        v[4 * r + 0] = t[4 * r + 0] - t[4 * r + 2];
        v[4 * r + 1] = t[4 * r + 1] + t[4 * r + 2];
        v[4 * r + 2] = t[4 * r + 2] - t[4 * r + 1];
        v[4 * r + 3] = t[4 * r + 1] - t[4 * r + 3];
    }
}

// Eq. 8: Y = A^T M A, A^T = [[1,1,1,0],[0,1,-1,-1]]; 24 FADD.  y[a][b] row-major 2x2.
__device__ __forceinline__ void otf_2x2(const float m[16], float y[4]) {
    float t[8];
#pragma unroll
    for (int c = 0; c < 4; ++c) {
        t[c] = m[c] + m[4 + c] + m[8 + c];
        t[4 + c] = m[4 + c] - m[8 + c] - m[12 + c];
    }
#pragma unroll
    for (int r = 0; r < 2; ++r) {
        y[2 * r + 0] = t[4 * r + 0] + t[4 * r + 1] + t[4 * r + 2];
        y[2 * r + 1] = t[4 * r + 1] - t[4 * r + 2] - t[4 * r + 3];
    }
}

}  // namespace wino
