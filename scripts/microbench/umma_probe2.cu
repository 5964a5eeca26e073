// umma_probe2.cu -- bisect tcgen05.mma execution: layout-agnostic all-ones operands.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ uint64_t make_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo, int version) {
    uint64_t d = 0;
    d |= uint64_t((saddr >> 4) & 0x3FFF);
    d |= uint64_t((lbo >> 4) & 0x3FFF) << 16;
    d |= uint64_t((sbo >> 4) & 0x3FFF) << 32;
    d |= uint64_t(version) << 46;
    return d;
}
// MODE 0: tf32 5-op form; 1: tf32 with mask vector; 2: f16(bf16) 5-op form
template <int MODE>
__global__ void k(float* D, int version, int bmajor) {
    __shared__ __align__(1024) uint32_t sa[2048];
    __shared__ __align__(1024) uint32_t sb[2048];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tmem_base;
    const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
    const uint32_t one = (MODE == 2) ? 0x3F803F80u : 0x3F800000u;  // bf16x2 ones or fp32 one
    for (int e = tid; e < 2048; e += blockDim.x) { sa[e] = one; sb[e] = one; }
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(smem_u32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;\n" ::"r"(smem_u32(&tmem_base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
    }
    asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
    const uint32_t tbase = tmem_base;
    if (tid == 0) {
        uint32_t idesc = (1u << 4) | ((MODE == 2 ? 1u : 2u) << 7) | ((MODE == 2 ? 1u : 2u) << 10) |
                         (uint32_t(bmajor) << 16) | ((32u >> 3) << 17) | ((128u >> 4) << 24);
        uint64_t adesc = make_desc(smem_u32(sa), 128, 256, version);
        uint64_t bdesc = make_desc(smem_u32(sb), 128, 256, version);
        if (MODE == 0)
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                         "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tbase),
                         "l"(adesc), "l"(bdesc), "r"(idesc), "r"(0));
        else if (MODE == 1)
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                         "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, {%5, %5, %5, %5}, p;\n\t}\n" ::"r"(tbase),
                         "l"(adesc), "l"(bdesc), "r"(idesc), "r"(0), "r"(0));
        else
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                         "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tbase),
                         "l"(adesc), "l"(bdesc), "r"(idesc), "r"(0));
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(smem_u32(&bar)) : "memory");
    }
    uint32_t ok = 0;
    while (!ok) {
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
                     : "=r"(ok) : "r"(smem_u32(&bar)) : "memory");
    }
    asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
    uint32_t r[8];
    uint32_t taddr = tbase + ((uint32_t)(32 * warp) << 16);
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];\n"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]) : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
    for (int j = 0; j < 8; ++j) D[tid * 8 + j] = __uint_as_float(r[j]);
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;\n" ::"r"(tbase));
    (void)lane;
}
template <int MODE>
void run(const char* name, int version, int bmajor) {
    float* D; cudaMallocManaged(&D, 1024 * 4);
    for (int i = 0; i < 1024; ++i) D[i] = -1;
    k<MODE><<<1, 128>>>(D, version, bmajor);
    cudaError_t e = cudaDeviceSynchronize();
    printf("%-26s v%d bmaj%d: %s D[0]=%g D[7]=%g D[1000]=%g\n", name, version, bmajor, cudaGetErrorString(e), D[0], D[7], D[1000]);
    cudaFree(D);
}
int main() {
    for (int v = 0; v < 2; ++v) for (int bm = 0; bm < 2; ++bm) {
        run<0>("tf32 5-op", v, bm);
        run<1>("tf32 mask", v, bm);
        run<2>("bf16 5-op", v, bm);
    }
    return 0;
}
