// tmem_ld.cu -- TMEM -> register read throughput (tcgen05.ld.32x32b) per SM, 4 or 8 warps.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
template <int NW>
__global__ void k(float* out, int reps, unsigned long long* cyc) {
    __shared__ uint32_t tb;
    int warp = threadIdx.x / 32;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tb)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    uint32_t base = tb + ((uint32_t)((warp & 3) * 32) << 16);
    int col0 = (warp >> 2) * 256;  // 8 warps: second half of the columns
    float acc = 0;
    long long t0 = clock64();
    for (int r = 0; r < reps; ++r) {
        for (int c = col0; c < col0 + 512 / (NW / 4); c += 32) {
            uint32_t v[32];
            asm volatile(
                "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                  "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]),
                  "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]),
                  "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]),
                  "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
                : "r"(base + c));
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
            for (int j = 0; j < 32; ++j) acc += __uint_as_float(v[j]);
        }
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tb));
}
int main() {
    float* out; cudaMalloc(&out, 148 * 256 * 4);
    unsigned long long* cyc; cudaMalloc(&cyc, 148 * 8);
    unsigned long long h[148];
    int reps = 200;
    k<4><<<148, 128>>>(out, reps, cyc);
    cudaDeviceSynchronize();
    cudaMemcpy(h, cyc, 148 * 8, cudaMemcpyDeviceToHost);
    printf("{\"warps\": 4, \"bytes_per_clk_per_sm\": %.1f, \"err\": \"%s\"}\n", 512.0 * 128 * 4 * reps / h[0],
           cudaGetErrorString(cudaGetLastError()));
    k<8><<<148, 256>>>(out, reps, cyc);
    cudaDeviceSynchronize();
    cudaMemcpy(h, cyc, 148 * 8, cudaMemcpyDeviceToHost);
    printf("{\"warps\": 8, \"bytes_per_clk_per_sm\": %.1f, \"err\": \"%s\"}\n", 512.0 * 128 * 4 * reps / h[0],
           cudaGetErrorString(cudaGetLastError()));
    return 0;
}
