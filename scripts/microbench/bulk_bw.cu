// bulk_bw.cu -- per-SM global->shared fill bandwidth with cp.async.bulk (L2-resident source).
// Each CTA streams `iters` chunks of `chunk` bytes into an S-slot smem ring, one
// elected thread issuing, mbarrier completion, no consumer work.  Reports B/clk/SM
// for all-CTAs-read-the-same-data (like the transformed filter) and for
// per-CTA-distinct data, at 64 and 148 CTAs.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int S>
__global__ void bulk_kernel(const uint8_t* src, size_t src_bytes, int chunk, int iters, int distinct,
                            unsigned long long* clk) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ __align__(8) uint64_t bar[S];
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar[s])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x != 0) return;
    long long t0 = clock64();
    size_t base = distinct ? (size_t)blockIdx.x * 4096 * 37 : 0;
    for (int i = 0; i < iters; ++i) {
        int s = i % S;
        if (i >= S) {
            uint32_t ph = ((i / S) - 1) & 1, ok = 0;
            while (!ok)
                asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                             : "=r"(ok) : "r"(smem_u32(&bar[s])), "r"(ph) : "memory");
        }
        size_t off = (base + (size_t)i * chunk) % (src_bytes - chunk);
        off &= ~size_t(15);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[s])), "r"(chunk) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         smem_u32(smem + s * chunk)), "l"(src + off), "r"(chunk), "r"(smem_u32(&bar[s]))
                     : "memory");
    }
    for (int i = iters; i < iters + S; ++i) {
        int s = i % S;
        uint32_t ph = ((i / S) - 1) & 1, ok = 0;
        while (!ok)
            asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                         : "=r"(ok) : "r"(smem_u32(&bar[s])), "r"(ph) : "memory");
    }
    clk[blockIdx.x] = clock64() - t0;
}

template <int S>
void sweep(const uint8_t* src, size_t src_bytes, unsigned long long* clk, int chunk, int ctas) {
    unsigned long long h[148];
    int smem = S * chunk;
    if (smem > 200 * 1024) return;
    cudaFuncSetAttribute(bulk_kernel<S>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    int iters = 50 * S;
    bulk_kernel<S><<<ctas, 32, smem>>>(src, src_bytes, chunk, iters, 0, clk);
    bulk_kernel<S><<<ctas, 32, smem>>>(src, src_bytes, chunk, iters, 0, clk);
    cudaDeviceSynchronize();
    cudaMemcpy(h, clk, ctas * 8, cudaMemcpyDeviceToHost);
    double avg = 0; for (int i = 0; i < ctas; ++i) avg += h[i]; avg /= ctas;
    double bpc = double(chunk) * iters / avg;
    printf("{\"slots\": %d, \"chunk\": %d, \"inflight_KB\": %d, \"ctas\": %d, \"B_per_clk_per_sm\": %.1f, \"latency_cyc\": %.0f}\n",
           S, chunk, S * chunk / 1024, ctas, bpc, S * chunk / bpc);
}
int main() {
    const size_t src_bytes = 16u << 20;
    uint8_t* src; cudaMalloc(&src, src_bytes); cudaMemset(src, 1, src_bytes);
    unsigned long long* clk; cudaMalloc(&clk, 148 * 8);
    for (int ctas : {148}) {
        sweep<1>(src, src_bytes, clk, 32768, ctas);
        sweep<2>(src, src_bytes, clk, 32768, ctas);
        sweep<4>(src, src_bytes, clk, 32768, ctas);
        sweep<6>(src, src_bytes, clk, 32768, ctas);
        sweep<3>(src, src_bytes, clk, 65536, ctas);
        sweep<2>(src, src_bytes, clk, 65536, ctas);
        sweep<12>(src, src_bytes, clk, 16384, ctas);
        sweep<24>(src, src_bytes, clk, 8192, ctas);
        sweep<48>(src, src_bytes, clk, 4096, ctas);
        sweep<8>(src, src_bytes, clk, 4096, ctas);
    }
    return 0;
}
