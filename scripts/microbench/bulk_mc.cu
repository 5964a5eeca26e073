// bulk_mc.cu -- does TMA/bulk multicast across a 2-CTA cluster raise the per-SM fill rate?
// Each CTA of a pair issues half of every chunk with .multicast::cluster to both CTAs;
// each CTA's mbarrier expects the whole chunk.  Compare with unicast (each CTA loads the
// whole chunk itself).  Reports received B/clk per SM.
#include <cuda_runtime.h>
#include <cooperative_groups.h>
#include <cstdint>
#include <cstdio>
namespace cg = cooperative_groups;
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ bool try_wait(uint64_t* b, uint32_t ph) {
    uint32_t ok;
    asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                 : "=r"(ok) : "r"(smem_u32(b)), "r"(ph) : "memory");
    return ok;
}
template <int S, bool MC>
__global__ void __cluster_dims__(2, 1, 1) kern(const uint8_t* src, int chunk, int iters, unsigned long long* clk) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ __align__(8) uint64_t full[S], empty[S];
    cg::cluster_group cl = cg::this_cluster();
    const uint32_t rank = cl.block_rank();
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full[s])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 2;" ::"r"(smem_u32(&empty[s])));
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    cl.sync();
    if (threadIdx.x != 0) { cl.sync(); return; }
    long long t0 = clock64();
    auto issue = [&](int i) {
        int s = i % S;
        if (i >= S) {  // both CTAs released slot s
            while (!try_wait(&empty[s], ((i / S) - 1) & 1)) {}
        }
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&full[s])), "r"(chunk) : "memory");
        const uint8_t* g = src + (size_t)(i % 64) * chunk;
        if (MC) {
            int half = chunk / 2;
            asm volatile(
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1], %2, [%3], %4;" ::"r"(
                    smem_u32(smem + s * chunk + rank * half)), "l"(g + rank * half), "r"(half), "r"(smem_u32(&full[s])), "h"((uint16_t)3)
                : "memory");
        } else {
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                             smem_u32(smem + s * chunk)), "l"(g), "r"(chunk), "r"(smem_u32(&full[s]))
                         : "memory");
        }
    };
    for (int i = 0; i < S; ++i) issue(i);
    for (int i = 0; i < iters; ++i) {
        int s = i % S;
        while (!try_wait(&full[s], (i / S) & 1)) {}
        for (uint32_t r = 0; r < 2; ++r) {  // release slot s in both CTAs
            uint32_t remote;
            asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(smem_u32(&empty[s])), "r"(r));
            asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(remote) : "memory");
        }
        if (i + S < iters) issue(i + S);
    }
    clk[blockIdx.x] = clock64() - t0;
    cl.sync();
}
template <int S, bool MC>
void run(const uint8_t* src, unsigned long long* clk, int chunk) {
    int smem = S * chunk;
    cudaFuncSetAttribute(kern<S, MC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    int iters = 60 * S;
    kern<S, MC><<<148, 32, smem>>>(src, chunk, iters, clk);
    kern<S, MC><<<148, 32, smem>>>(src, chunk, iters, clk);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long h[148];
    cudaMemcpy(h, clk, 148 * 8, cudaMemcpyDeviceToHost);
    double avg = 0; for (int i = 0; i < 148; ++i) avg += h[i]; avg /= 148;
    printf("{\"multicast\": %d, \"slots\": %d, \"chunk\": %d, \"recv_B_per_clk_per_sm\": %.1f, \"err\": \"%s\"}\n", MC, S, chunk,
           double(chunk) * iters / avg, cudaGetErrorString(e));
}
int main() {
    uint8_t* src; cudaMalloc(&src, 64u << 20); cudaMemset(src, 1, 64u << 20);
    unsigned long long* clk; cudaMalloc(&clk, 148 * 8);
    run<2, false>(src, clk, 65536);
    run<2, true>(src, clk, 65536);
    run<3, false>(src, clk, 65536);
    run<3, true>(src, clk, 65536);
    run<4, false>(src, clk, 32768);
    run<4, true>(src, clk, 32768);
    return 0;
}
