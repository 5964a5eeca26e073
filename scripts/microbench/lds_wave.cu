// LDS.128 broadcast patterns: shared-memory cycles per warp-level LDS.128 on sm_100a.
// Each pattern maps lane -> float4 index; 12 warps / SM issue back-to-back loads
// (asm volatile, immediate offsets, no other work).  Result: cycles / warp-LDS / SM.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void __launch_bounds__(384, 1) k(const int* pat, int iters, float* out) {
    __shared__ float4 s[2048];
    for (int i = threadIdx.x; i < 2048; i += blockDim.x) s[i] = make_float4(i, i + 1, i + 2, i + 3);
    __syncthreads();
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const unsigned a = (unsigned)__cvta_generic_to_shared(&s[pat[lane] + 64 * w]);
    float x = 0.f;
    for (int it = 0; it < iters; ++it) {
#define L(off) { float p, q, r, t; asm volatile("ld.volatile.shared.v4.f32 {%0,%1,%2,%3}, [%4+" #off "];" : "=f"(p), "=f"(q), "=f"(r), "=f"(t) : "r"(a)); asm volatile("" :: "f"(p), "f"(q), "f"(r), "f"(t)); x += p; }
        L(0) L(1024) L(2048) L(3072) L(4096) L(5120) L(6144) L(7168)
        L(8192) L(9216) L(10240) L(11264) L(12288) L(13312) L(14336) L(15360)
    }
    if (x == 1234.5f) out[threadIdx.x] = x;
}
int main() {
    float* out; cudaMalloc(&out, 4096);
    int* dp; cudaMalloc(&dp, 32 * 4);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    const int iters = 8192;
    const char* names[] = {"same", "lane>>2", "lane&3", "(lane>>1)&3", "((lane>>3)<<1)|(lane&1)", "lane>>1",
                           "lane&7", "lane", "lane>>3", "lane&1", "(lane>>2)&1", "(lane&1)+2*(lane>>3)", "lane>>4",
                           "(lane&3)+4*(lane>>4)", "((lane>>2)&1)+2*(lane>>4)", "(lane>>1)&1", "(lane>>2)&3",
                           "(lane>>2)&7 + 8*(lane&1)?"};
    const int NP = 18;
    for (int p = 0; p < NP; ++p) {
        int h[32];
        for (int l = 0; l < 32; ++l) {
            int v = 0;
            switch (p) {
                case 0: v = 0; break;
                case 1: v = l >> 2; break;
                case 2: v = l & 3; break;
                case 3: v = (l >> 1) & 3; break;
                case 4: v = ((l >> 3) << 1) | (l & 1); break;
                case 5: v = l >> 1; break;
                case 6: v = l & 7; break;
                case 7: v = l; break;
                case 8: v = l >> 3; break;
                case 9: v = l & 1; break;
                case 10: v = (l >> 2) & 1; break;
                case 11: v = (l & 1) + 2 * (l >> 3); break;
                case 12: v = l >> 4; break;
                case 13: v = (l & 3) + 4 * (l >> 4); break;
                case 14: v = ((l >> 2) & 1) + 2 * (l >> 4); break;
                case 15: v = (l >> 1) & 1; break;
                case 16: v = (l >> 2) & 3; break;
                case 17: v = ((l >> 2) & 7) + 8 * (l & 1); break;
            }
            h[l] = v;
        }
        cudaMemcpy(dp, h, sizeof(h), cudaMemcpyHostToDevice);
        k<<<sms, 384>>>(dp, 16, out);
        cudaEventRecord(a);
        k<<<sms, 384>>>(dp, iters, out);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        double lds_per_sm = 12.0 * iters * 16;
        printf("%-30s %.3f cycles per warp LDS.128 per SM (at 1965 MHz)\n", names[p], ms * 1e-3 * 1965e6 / lds_per_sm);
    }
    return 0;
}
