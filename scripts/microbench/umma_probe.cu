// umma_probe.cu -- layout probe for tcgen05.mma kind::tf32 on sm_100a.
//
// Verifies, on the GPU, the shared-memory operand layouts and descriptors used
// by the tensor-core Winograd kernel before they are used there:
//   A (M=128 x K=8)  K-major, SWIZZLE_NONE: byte(m,k) = (m/8)*256 + (k/4)*128 + (m%8)*16 + (k%4)*4
//                    -> LBO = 128 B (K chunk), SBO = 256 B (8-row group)
//   B (N=32  x K=8)  MN-major, SWIZZLE_NONE: byte(n,k) = (n/4)*SBO_B + k*16 + (n%4)*4, SBO_B = 144 B
//                    (padded so ITF stores along n are bank-conflict free)
// D (128 x 32 fp32) lands in TMEM lanes 0..127, columns 0..31; read back with
// tcgen05.ld.32x32b.x8.  Integer-valued operands make the TF32 product exact.
// Also exercises accumulate (2nd MMA with enable_input_d = 1).
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
static unsigned __float_as_uint_host(float f) { unsigned u; memcpy(&u, &f, 4); return u; }

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ uint64_t make_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = 0;
    d |= uint64_t((saddr >> 4) & 0x3FFF);
    d |= uint64_t((lbo >> 4) & 0x3FFF) << 16;
    d |= uint64_t((sbo >> 4) & 0x3FFF) << 32;
    d |= uint64_t(1) << 46;  // version = 1 (Blackwell)
    // base_offset = 0, lbo_mode = 0, layout_type (bits 61..63) = 0 = SWIZZLE_NONE
    return d;
}

template <int SBO_B, int A_MAJOR_MN>
__global__ void probe(const float* A, const float* B, float* D, int accumulate_twice) {
    __shared__ __align__(1024) float sa[128 * 8];
    __shared__ __align__(1024) float sb[1024];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tmem_base;
    const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
    // fill A (M=128 x K=8)
    for (int e = tid; e < 128 * 8; e += blockDim.x) {
        int m = e / 8, k = e % 8;
        int byte;
        if (A_MAJOR_MN) byte = (m / 4) * 128 + k * 16 + (m % 4) * 4;  // MN-major interleave, SBO=128
        else byte = (m / 8) * 256 + (k / 4) * 128 + (m % 8) * 16 + (k % 4) * 4;
        sa[byte / 4] = A[e];
    }
    for (int e = tid; e < 32 * 8; e += blockDim.x) {
        int n = e / 8, k = e % 8;
        int byte = (n / 4) * SBO_B + k * 16 + (n % 4) * 4;
        sb[byte / 4] = B[k * 32 + n];  // B given as (K=8, N=32) row-major
    }
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(smem_u32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;\n" ::"r"(smem_u32(&tmem_base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
    }
    asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");  // generic smem writes -> async proxy
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
    const uint32_t tbase = tmem_base;
    if (tid == 0) {
        // instruction descriptor: F32 accum, TF32 A/B, majors, N=32, M=128
        uint32_t idesc = 0;
        idesc |= 1u << 4;            // c_format F32
        idesc |= 2u << 7;            // a_format TF32
        idesc |= 2u << 10;           // b_format TF32
        idesc |= uint32_t(A_MAJOR_MN) << 15;  // a_major
        idesc |= 1u << 16;           // b_major = MN
        idesc |= (32u >> 3) << 17;   // N
        idesc |= (128u >> 4) << 24;  // M
        uint64_t adesc = A_MAJOR_MN ? make_desc(smem_u32(sa), 1024 /*LBO unused*/, 128)
                                    : make_desc(smem_u32(sa), 128, 256);
        uint64_t bdesc = make_desc(smem_u32(sb), 1024 /*LBO unused: one K group*/, SBO_B);
        for (int r = 0; r < 1 + accumulate_twice; ++r) {
            uint32_t acc = r > 0;
            asm volatile(
                "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tbase),
                "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc));
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                         smem_u32(&bar))
                     : "memory");
    }
    // wait for MMA completion
    {
        uint32_t ok = 0;
        while (!ok) {
            asm volatile(
                "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
                : "=r"(ok)
                : "r"(smem_u32(&bar))
                : "memory");
        }
    }
    asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
    // warp w (0..3) reads lanes 32w..32w+31, columns 0..31 in 4 chunks of 8
    for (int c0 = 0; c0 < 32; c0 += 8) {
        uint32_t r[8];
        uint32_t taddr = tbase + ((uint32_t)(32 * warp) << 16) + c0;
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];\n"
            : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
            : "r"(taddr));
        asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
        for (int j = 0; j < 8; ++j) D[(32 * warp + lane) * 32 + c0 + j] = __uint_as_float(r[j]);
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;\n" ::"r"(tbase));
}


__global__ void tmem_roundtrip(float* out) {
    __shared__ uint32_t tmem_base;
    const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;\n" ::"r"(smem_u32(&tmem_base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
    uint32_t tbase = tmem_base;
    uint32_t taddr = tbase + ((uint32_t)(32 * warp) << 16);
    uint32_t v[8];
    for (int j = 0; j < 8; ++j) v[j] = __float_as_uint(float(tid * 100 + j));
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};\n" ::"r"(taddr),
                 "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]));
    asm volatile("tcgen05.wait::st.sync.aligned;\n" ::: "memory");
    uint32_t r[8];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];\n"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                 : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
    for (int j = 0; j < 8; ++j) out[tid * 8 + j] = __uint_as_float(r[j]);
    if (tid == 0) out[1024] = __uint_as_float(tbase);
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;\n" ::"r"(tbase));
}
template <int SBO_B, int A_MN>
int run_case(const char* name, void (*fill)(float*, float*), int twice, bool verbose) {
    float *A, *B, *D;
    cudaMallocManaged(&A, 128 * 8 * 4);
    cudaMallocManaged(&B, 8 * 32 * 4);
    cudaMallocManaged(&D, 128 * 32 * 4);
    fill(A, B);
    for (int i = 0; i < 128 * 32; ++i) D[i] = -999.f;
    probe<SBO_B, A_MN><<<1, 128>>>(A, B, D, twice);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
        printf("{\"probe\": \"%s\", \"error\": \"%s\"}\n", name, cudaGetErrorString(e));
        return 1;
    }
    int bad = 0;
    for (int m = 0; m < 128; ++m)
        for (int n = 0; n < 32; ++n) {
            double ref = 0;
            for (int k = 0; k < 8; ++k) ref += double(A[m * 8 + k]) * B[k * 32 + n];
            ref *= (1 + twice);
            if (ref != D[m * 32 + n]) ++bad;
        }
    printf("%-44s mismatches %4d", name, bad);
    if (verbose || bad) {
        printf("\n   D[0][0..15]:");
        for (int n = 0; n < 16; ++n) printf(" %g", D[n]);
        printf("\n   D[0..15][0]:");
        for (int m = 0; m < 16; ++m) printf(" %g", D[m * 32]);
        printf("\n   D[8][0..7]:");
        for (int n = 0; n < 8; ++n) printf(" %g", D[8 * 32 + n]);
    }
    printf("\n");
    cudaFree(A); cudaFree(B); cudaFree(D);
    return bad != 0;
}
void f_ones(float* A, float* B) { for (int i = 0; i < 1024; ++i) A[i] = 1; for (int i = 0; i < 256; ++i) B[i] = 1; }
void f_bn(float* A, float* B) { for (int i = 0; i < 1024; ++i) A[i] = 1; for (int i = 0; i < 256; ++i) B[i] = i % 32; }
void f_am(float* A, float* B) { for (int i = 0; i < 1024; ++i) A[i] = i / 8; for (int i = 0; i < 256; ++i) B[i] = 1; }
void f_k0(float* A, float* B) { for (int i = 0; i < 1024; ++i) A[i] = (i % 8) == 0; for (int i = 0; i < 256; ++i) B[i] = (i / 32) * 100 + i % 32; }
void f_k5(float* A, float* B) { for (int i = 0; i < 1024; ++i) A[i] = (i % 8) == 5; for (int i = 0; i < 256; ++i) B[i] = (i / 32) * 100 + i % 32; }
void f_rand(float* A, float* B) { for (int i = 0; i < 1024; ++i) A[i] = float((i * 7 + 3) % 11 - 5); for (int i = 0; i < 256; ++i) B[i] = float((i * 5 + 1) % 9 - 4); }

int main() {
    int fails = 0;
    {
        float* o; cudaMallocManaged(&o, 1025 * 4);
        tmem_roundtrip<<<1, 128>>>(o);
        cudaError_t e = cudaDeviceSynchronize();
        int bad = 0;
        for (int t = 0; t < 128; ++t) for (int j = 0; j < 8; ++j) bad += o[t * 8 + j] != float(t * 100 + j);
        printf("tmem roundtrip: %s bad=%d tbase=0x%x o[0..3]=%g %g %g %g o[8]=%g\n", cudaGetErrorString(e), bad,
               __float_as_uint_host(o[1024]), o[0], o[1], o[2], o[3], o[8]);
    }
    fails += run_case<144, 0>("ones", f_ones, 0, true);
    fails += run_case<144, 0>("B=n", f_bn, 0, false);
    fails += run_case<144, 0>("A=m", f_am, 0, false);
    fails += run_case<144, 0>("A=onehot k0, B=100k+n", f_k0, 0, false);
    fails += run_case<144, 0>("A=onehot k5, B=100k+n", f_k5, 0, false);
    fails += run_case<144, 0>("rand", f_rand, 0, false);
    fails += run_case<144, 0>("rand acc2", f_rand, 1, false);
    fails += run_case<144, 1>("A MN-major: rand", f_rand, 0, false);
    fails += run_case<128, 0>("B SBO128: rand", f_rand, 0, false);
    return fails;
}
