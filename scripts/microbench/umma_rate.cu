// umma_rate.cu -- cycles per tcgen05.mma.kind::f16 (SS operands, SWIZZLE_NONE K-major, K = 16)
// for M in {64, 128} x N in {16..256}: one thread issues R rounds of 16 MMAs (distinct TMEM
// columns) either back to back (one commit at the end) or with a commit + wait after every
// round of 16 (the fused kernels' pattern).  grid = 1 or 148 CTAs.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o umma_rate umma_rate.cu
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t make_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    return uint64_t((saddr >> 4) & 0x3FFF) | (uint64_t((lbo >> 4) & 0x3FFF) << 16) |
           (uint64_t((sbo >> 4) & 0x3FFF) << 32) | (uint64_t(1) << 46);
}
__device__ __forceinline__ void wait_bar(uint64_t* bar, uint32_t ph) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                     : "=r"(ok) : "r"(smem_u32(bar)), "r"(ph) : "memory");
}
template <int M, int N, bool SYNC>
__global__ void k(unsigned long long* out, int R) {
    extern __shared__ __align__(1024) uint8_t sm[];
    uint8_t* sa = sm;                 // 16 A tiles of M x 16 fp16
    uint8_t* sb = sm + 16 * M * 32;   // 16 B tiles of N x 16 fp16
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tb;
    int tid = threadIdx.x, warp = tid / 32;
    for (int e = tid; e < (16 * M * 32 + 16 * N * 32) / 4; e += blockDim.x) reinterpret_cast<uint32_t*>(sm)[e] = 0;
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tb)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (tid == 0) {
        const uint32_t idesc = (1u << 4) | (uint32_t(N >> 3) << 17) | (uint32_t(M >> 4) << 24);
        unsigned long long t0 = clock64();
        uint32_t ph = 0;
        for (int r = 0; r < R; ++r) {
#pragma unroll
            for (int xi = 0; xi < 16; ++xi) {
                uint64_t ad = make_desc(smem_u32(sa + xi * M * 32), 128, 256);
                uint64_t bd = make_desc(smem_u32(sb + xi * N * 32), 128, 256);
                uint32_t d = tb + ((xi * N) % 512);
                asm volatile("{.reg .pred p; setp.ne.b32 p, %4, 0; tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;}"
                             ::"r"(d), "l"(ad), "l"(bd), "r"(idesc), "r"(1));
            }
            if (SYNC) {
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar)) : "memory");
                wait_bar(&bar, ph);
                ph ^= 1;
            }
        }
        if (!SYNC) {
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar)) : "memory");
            wait_bar(&bar, 0);
        }
        unsigned long long t1 = clock64();
        if (blockIdx.x == 0) out[0] = t1 - t0;
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tb));
}
template <int M, int N, bool SYNC>
void run(int grid, unsigned long long* d) {
    const int R = 256;
    const int smem = 16 * (M + N) * 32;
    cudaFuncSetAttribute(k<M, N, SYNC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    k<M, N, SYNC><<<grid, 128, smem>>>(d, R);
    k<M, N, SYNC><<<grid, 128, smem>>>(d, R);
    cudaDeviceSynchronize();
    unsigned long long c;
    cudaMemcpy(&c, d, 8, cudaMemcpyDeviceToHost);
    double per = double(c) / (R * 16);
    printf("M=%3d N=%3d %s grid=%3d: %7.1f cyc/MMA  (floor %d)  %6.1f MAC/clk\n", M, N, SYNC ? "commit/16" : "stream   ", grid,
           per, (M < 128 ? 128 : M) * N / 256, double(M) * N * 16 / per);
}
int main() {
    unsigned long long* d;
    cudaMalloc(&d, 8);
    for (int grid : {1, 148}) {
        run<128, 16, false>(grid, d); run<128, 32, false>(grid, d); run<128, 64, false>(grid, d);
        run<128, 128, false>(grid, d); run<128, 256, false>(grid, d);
        run<64, 32, false>(grid, d); run<64, 64, false>(grid, d);
        run<128, 32, true>(grid, d); run<128, 64, true>(grid, d); run<64, 32, true>(grid, d);
    }
    cudaError_t e = cudaGetLastError();
    printf("%s\n", cudaGetErrorString(e));
    return 0;
}
