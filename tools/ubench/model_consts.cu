// Microbenchmark of the hardware-model constants of the fusion benefit model
// (Eqs. 3-7): tg = cycles to access a pixel in global
// memory ("the global memory access latency (typically 400-800 cycles)"), ts =
// cycles to access a pixel in shared memory ("typically in a few cycles"),
// cALU / cSFU = average cost in cycles of an ALU / SFU operation.  The paper
// says these "can be adapted for new architectures": this
// program measures them on the B200 it runs on.
//
// Method: one thread, dependent chains timed with clock64 (latency, as the
// paper's conservative estimate uses latency):
//   tg      pointer chase over a 1 GiB buffer, a random line per hop (DRAM)
//   tg_l2   pointer chase over 16 MiB (L2 hits)
//   ts      pointer chase in 32 KiB of shared memory
//   c_alu   FFMA chain;  c_alu_int  IMAD chain
//   c_sfu   MUFU.EX2 chain (exp2f approx)
// Prints one JSON object.
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <random>
#include <cuda_runtime.h>

__global__ void chase_global(const unsigned *__restrict__ next, int hops, unsigned start, long long *cyc, unsigned *sink)
{
    unsigned p = start;
    for (int i = 0; i < 64; i++) p = next[p];   // warm the TLB path a little
    const long long t0 = clock64();
    for (int i = 0; i < hops; i++) p = next[p];
    const long long t1 = clock64();
    *cyc = t1 - t0;
    *sink = p;
}

__global__ void chase_shared(int hops, long long *cyc, unsigned *sink)
{
    __shared__ unsigned s[8192];
    for (int i = 0; i < 8192; i++) s[i] = (i * 2897u + 1u) & 8191u;   // a permutation (2897 odd)
    __syncthreads();
    unsigned p = 0;
    const long long t0 = clock64();
    for (int i = 0; i < hops; i++) p = s[p];
    const long long t1 = clock64();
    *cyc = t1 - t0;
    *sink = p;
}

template <int KIND>
__global__ void chain(int n, float x, long long *cyc, float *sink)
{
    float a = x;
    unsigned u = __float_as_uint(x);
    const long long t0 = clock64();
    for (int i = 0; i < n; i++) {
#pragma unroll
        for (int j = 0; j < 16; j++) {
            if (KIND == 0) a = fmaf(a, 1.0001f, 0.25f);
            if (KIND == 1) u = u * u + 7u;           // IMAD (not foldable)
            if (KIND == 2) a = exp2f(a) * 0.5f;   // MUFU.EX2 + FMUL
        }
    }
    const long long t1 = clock64();
    *cyc = t1 - t0;
    *sink = a + (float)u;
}

int main()
{
    long long *dcyc;
    unsigned *dsink;
    float *fsink;
    cudaMalloc(&dcyc, sizeof(long long));
    cudaMalloc(&dsink, 4);
    cudaMalloc(&fsink, 4);
    long long cyc;
    auto chase = [&](size_t bytes, int hops) {
        const size_t n = bytes / 4, line = 32;           // one hop per 128-byte line
        const size_t nl = n / line;
        std::vector<unsigned> order(nl);
        for (size_t i = 0; i < nl; i++) order[i] = (unsigned)i;
        std::mt19937_64 rng(12345);
        std::shuffle(order.begin(), order.end(), rng);
        std::vector<unsigned> next(n, 0);
        for (size_t i = 0; i < nl; i++) next[(size_t)order[i] * line] = order[(i + 1) % nl] * (unsigned)line;
        unsigned *d;
        cudaMalloc(&d, n * 4);
        cudaMemcpy(d, next.data(), n * 4, cudaMemcpyHostToDevice);
        chase_global<<<1, 1>>>(d, hops, order[0] * (unsigned)line, dcyc, dsink);
        cudaMemcpy(&cyc, dcyc, 8, cudaMemcpyDeviceToHost);
        cudaFree(d);
        return (double)cyc / hops;
    };
    const double tg = chase((size_t)1 << 30, 20000);
    const double tg_l2 = chase((size_t)16 << 20, 20000);
    chase_shared<<<1, 1>>>(100000, dcyc, dsink);
    cudaMemcpy(&cyc, dcyc, 8, cudaMemcpyDeviceToHost);
    const double ts = (double)cyc / 100000;
    const int n = 20000;
    chain<0><<<1, 1>>>(n, 1.0f, dcyc, fsink);
    cudaMemcpy(&cyc, dcyc, 8, cudaMemcpyDeviceToHost);
    const double c_alu = (double)cyc / (n * 16.0);
    chain<1><<<1, 1>>>(n, 1.0f, dcyc, fsink);
    cudaMemcpy(&cyc, dcyc, 8, cudaMemcpyDeviceToHost);
    const double c_alu_int = (double)cyc / (n * 16.0);
    chain<2><<<1, 1>>>(n, 1.0f, dcyc, fsink);
    cudaMemcpy(&cyc, dcyc, 8, cudaMemcpyDeviceToHost);
    const double c_sfu = (double)cyc / (n * 16.0) - c_alu;   // minus the FMUL of the chain
    cudaError_t e = cudaDeviceSynchronize();
    printf("{\"tg\": %.1f, \"tg_l2\": %.1f, \"ts\": %.1f, \"c_alu\": %.2f, \"c_alu_int\": %.2f, \"c_sfu\": %.2f, "
           "\"unit\": \"cycles (latency, one thread, clock64)\", \"status\": \"%s\"}\n",
           tg, tg_l2, ts, c_alu, c_alu_int, c_sfu, cudaGetErrorString(e));
    return e == cudaSuccess ? 0 : 1;
}
