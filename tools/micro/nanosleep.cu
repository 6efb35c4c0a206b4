// Measures what __nanosleep(t) actually sleeps on this GPU (globaltimer ns), one warp
// per SM and 6 warps per SM.
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ unsigned long long gt() { unsigned long long t; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)); return t; }
__global__ void k(unsigned t, int reps, unsigned long long* out) {
    unsigned long long t0 = gt();
    for (int i = 0; i < reps; ++i) __nanosleep(t);
    unsigned long long t1 = gt();
    if ((threadIdx.x & 31) == 0) out[blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32] = (t1 - t0) / reps;
}
int main() {
    unsigned long long* d; cudaMalloc(&d, 1 << 20);
    unsigned long long h[4096];
    for (int warps : {1, 6}) for (unsigned t : {100u, 500u, 1000u, 1500u, 3000u, 10000u, 100000u, 1000000u}) {
        int reps = t >= 100000 ? 20 : 200;
        k<<<148, 32 * warps>>>(t, reps, d);
        cudaMemcpy(h, d, 148 * warps * 8, cudaMemcpyDeviceToHost);
        unsigned long long mn = ~0ull, mx = 0, s = 0;
        for (int i = 0; i < 148 * warps; ++i) { mn = h[i] < mn ? h[i] : mn; mx = h[i] > mx ? h[i] : mx; s += h[i]; }
        printf("warps/SM %d  nanosleep(%7u): actual ns per call min %llu avg %llu max %llu\n", warps, t, mn, s / (148 * warps), mx);
    }
    return 0;
}
