// umma_m64.cu -- where does D land in TMEM for tcgen05.mma kind::tf32 with M = 64?
// A[m][k] = m + 1 (K-major interleave), B = ones  ->  D[m][n] = 8 (m + 1).
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t make_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    return uint64_t((saddr >> 4) & 0x3FFF) | (uint64_t((lbo >> 4) & 0x3FFF) << 16) |
           (uint64_t((sbo >> 4) & 0x3FFF) << 32) | (uint64_t(1) << 46);
}
__global__ void k(float* D) {
    __shared__ __align__(1024) float sa[64 * 8];
    __shared__ __align__(1024) float sb[2 * 32 * 8];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tb;
    int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
    for (int e = tid; e < 64 * 8; e += 128) {
        int m = e / 8, kk = e % 8;
        sa[((m / 8) * 256 + (kk / 4) * 128 + (m % 8) * 16 + (kk % 4) * 4) / 4] = float(m + 1);
    }
    for (int e = tid; e < 2 * 32 * 8; e += 128) sb[e] = e < 256 ? 1.f : 2.f;
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"(smem_u32(&tb)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    // zero TMEM columns 0..31 of all lanes first
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    uint32_t base = tb + ((uint32_t)(32 * warp) << 16);
    for (int c = 0; c < 32; c += 4) {
        asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1,%1,%1,%1};" ::"r"(base + c), "r"(0));
    }
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (tid == 0) {
        uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((32u >> 3) << 17) | ((64u >> 4) << 24);
        uint64_t ad = make_desc(smem_u32(sa), 128, 256), bd = make_desc(smem_u32(sb), 128, 256);
        asm volatile("{.reg .pred p; setp.ne.b32 p, %4, 0; tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;}"
                     ::"r"(tb), "l"(ad), "l"(bd), "r"(idesc), "r"(0));
        // second accumulator at TMEM lane offset 16, B scaled by 2 (second half of sb holds 2s)
        uint64_t bd2 = make_desc(smem_u32(sb) + 1024, 128, 256);
        asm volatile("{.reg .pred p; setp.ne.b32 p, %4, 0; tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;}"
                     ::"r"(tb + (16u << 16)), "l"(ad), "l"(bd2), "r"(idesc), "r"(0));
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar)) : "memory");
    }
    uint32_t ok = 0;
    while (!ok) asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0,1,0,p;}" : "=r"(ok) : "r"(smem_u32(&bar)) : "memory");
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    for (int c = 0; c < 32; c += 4) {
        uint32_t r[4];
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(base + c));
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        for (int j = 0; j < 4; ++j) D[(32 * warp + lane) * 32 + c + j] = __uint_as_float(r[j]);
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(tb));
}
int main() {
    float* D; cudaMallocManaged(&D, 128 * 32 * 4);
    k<<<1, 128>>>(D);
    printf("err %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    for (int lane = 0; lane < 128; ++lane) {
        printf("lane %3d: ", lane);
        for (int c = 0; c < 32; ++c) printf("%g ", D[lane * 32 + c] / 8.f);
        printf("\n");
    }
    return 0;
}
