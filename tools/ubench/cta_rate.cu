// CTA launch-rate probe: how long does a grid of short single-warp CTAs take
// against the same warps packed 2/4/8 per CTA?  Each warp spins `work` clocks
// (0 = empty).  Diagnostics only.
#include <cstdio>
#include <cuda_runtime.h>

__global__ void spin(long long work, int *sink)
{
    long long t0 = clock64();
    if (work) while (clock64() - t0 < work) {}
    if (threadIdx.x == 0 && blockIdx.x == 0x7fffffff) *sink = 1;
}

int main()
{
    int *sink;
    cudaMalloc(&sink, 4);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int warps_total = 6663;
    for (long long work : {0LL, 2000LL, 20000LL}) {
        for (int wpc : {1, 2, 4, 8}) {
            int grid = (warps_total + wpc - 1) / wpc;
            for (int i = 0; i < 3; i++) spin<<<grid, 32 * wpc>>>(work, sink);
            cudaEventRecord(a);
            const int reps = 50;
            for (int i = 0; i < reps; i++) spin<<<grid, 32 * wpc>>>(work, sink);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            printf("work %6lld clk  warps/CTA %d  grid %5d  %.2f us per launch\n", work, wpc, grid, ms * 1e3 / reps);
        }
    }
    return 0;
}
