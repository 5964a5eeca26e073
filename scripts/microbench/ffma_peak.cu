// FP32 FFMA throughput microbenchmark for B200 (sm_100a): establishes the
// measured CUDA-core FP32 ceiling used beside the nominal 148*128*2*f peak.
// Variants differ only in operand form; SASS register parity is inspected with
// scripts/sass_bank.py.
#include <cstdio>
#include <cuda_runtime.h>

#define CHAINS 16
template <int MODE>
__global__ void __launch_bounds__(256) ffma_kernel(float* out, float a, int iters) {
    float acc[CHAINS], b[CHAINS];
#pragma unroll
    for (int i = 0; i < CHAINS; ++i) { acc[i] = threadIdx.x * 1e-3f + i; b[i] = 1.0f + i * 1e-4f; }
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < CHAINS; ++i) {
            if (MODE == 0) acc[i] = fmaf(a, b[i], acc[i]);              // 3 registers (a reused)
            else if (MODE == 1) acc[i] = fmaf(acc[i], 0.9999f, a);       // register, immediate, register
            else if (MODE == 2) acc[i] = fmaf(b[i], acc[i], b[(i + 1) % CHAINS]);  // 3 distinct, no reuse
        }
    }
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < CHAINS; ++i) s += acc[i];
    if (s == 12345.678f) out[0] = s;
}

template <int MODE>
float run(float* out, int blocks, int iters) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    ffma_kernel<MODE><<<blocks, 256>>>(out, 1.0001f, iters);
    cudaEventRecord(e0);
    ffma_kernel<MODE><<<blocks, 256>>>(out, 1.0001f, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double flops = 2.0 * CHAINS * (double)iters * blocks * 256;
    return (float)(flops / (ms * 1e-3) / 1e12);
}

int main() {
    float* out; cudaMalloc(&out, 4);
    int dev; cudaGetDevice(&dev);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
    for (int occ : {4, 8}) {
        int blocks = sms * occ;
        printf("{\"sms\": %d, \"clock_khz\": %d, \"blocks\": %d, \"mode0_3reg_tflops\": %.2f, \"mode1_imm_tflops\": %.2f, \"mode2_noreuse_tflops\": %.2f}\n",
               sms, clk, blocks, run<0>(out, blocks, 20000), run<1>(out, blocks, 20000), run<2>(out, blocks, 20000));
    }
    return 0;
}
