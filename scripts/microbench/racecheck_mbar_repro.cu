// racecheck on the mbarrier hand-off the kernels use: warp 0's lanes write shared memory,
// __syncwarp(), ONE elected lane arrives (release) on an mbarrier; warp 1 waits (acquire) and
// reads.  PER_LANE = 0: the kernels' pattern (one arrival per warp, count 1); PER_LANE = 1:
// every lane arrives (count 32).  Both are ordered by the PTX memory model (bar.warp.sync orders
// the lanes' writes before the elected lane's release).  Build + run:
//   nvcc -gencode arch=compute_100a,code=sm_100a -DPER_LANE=0 racecheck_mbar_repro.cu -o r0
//   compute-sanitizer --tool racecheck ./r0      (reports RAW hazards for PER_LANE=0 only)
#include <cstdio>
#include <cstdint>
#ifndef PER_LANE
#define PER_LANE 0
#endif
__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__global__ void k(float* out) {
    __shared__ float buf[32];
    __shared__ __align__(8) uint64_t bar;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(&bar)), "r"(PER_LANE ? 32 : 1));
    __syncthreads();
    if (warp == 0) {
        buf[lane] = float(lane);  // producer writes
        __syncwarp();
        if (PER_LANE || lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sa(&bar)) : "memory");
    } else {
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0,1,0,p; }"
                         : "=r"(ok) : "r"(sa(&bar)) : "memory");
        out[lane] = buf[(lane + 1) & 31];  // consumer reads another lane's value
    }
}
int main() {
    float* d;
    cudaMalloc(&d, 32 * sizeof(float));
    k<<<1, 64>>>(d);
    float h[32];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    int bad = 0;
    for (int i = 0; i < 32; ++i) bad += h[i] != float((i + 1) & 31);
    printf("PER_LANE=%d values %s\n", PER_LANE, bad ? "WRONG" : "ok");
    return bad != 0;
}
