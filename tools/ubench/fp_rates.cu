// Microbenchmark: per-SM issue throughput of FP32 scalar vs packed (f32x2)
// instructions on sm_100a (used to calibrate the streaming kernel's FP mix,
// DESIGN.md §5.2).  Each thread runs 8 independent dependency chains.
#include <cstdio>
#include <cuda_runtime.h>

#define N_ITER 4096
template <int KIND>
__global__ void k(float *out, float s)
{
    float a[8];
    float2 p[8];
    for (int i = 0; i < 8; i++) { a[i] = threadIdx.x * 0.001f + i; p[i] = make_float2(a[i], a[i] + 1.f); }
    const float b = s * 1.0001f, c = s * 0.9999f;
    const float2 b2 = make_float2(b, c), c2 = make_float2(c, b);
    for (int it = 0; it < N_ITER; it++) {
#pragma unroll
        for (int i = 0; i < 8; i++) {
            if (KIND == 0) a[i] = fmaf(a[i], b, c);               // FFMA reg,reg,reg
            if (KIND == 1) a[i] = fmaf(a[i], 1.0001f, 0.5f);      // FFMA imm
            if (KIND == 2) a[i] = a[i] + b;                       // FADD
            if (KIND == 3) a[i] = a[i] * b;                       // FMUL
            if (KIND == 4) p[i] = __ffma2_rn(p[i], b2, c2);       // FFMA2
            if (KIND == 5) p[i] = __fadd2_rn(p[i], b2);           // FADD2
            if (KIND == 6) p[i] = __fmul2_rn(p[i], b2);           // FMUL2
            if (KIND == 7) p[i] = __ffma2_rn(p[i], make_float2(1.0001f, 1.0001f), make_float2(0.5f, 0.5f)); // FFMA2 imm
        }
    }
    float r = 0;
    for (int i = 0; i < 8; i++) r += a[i] + p[i].x + p[i].y;
    if (r == 12345.f) out[0] = r;
}

int main()
{
    float *d;
    cudaMalloc(&d, 4);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const char *names[] = {"FFMA r,r,r", "FFMA imm", "FADD", "FMUL", "FFMA2", "FADD2", "FMUL2", "FFMA2 imm"};
    void (*fns[])(float *, float) = {k<0>, k<1>, k<2>, k<3>, k<4>, k<5>, k<6>, k<7>};
    for (int warps = 4; warps <= 32; warps *= 2) {
        for (int f = 0; f < 8; f++) {
            cudaEvent_t e0, e1;
            cudaEventCreate(&e0); cudaEventCreate(&e1);
            fns[f]<<<sms, warps * 32>>>(d, 1.0f);
            cudaEventRecord(e0);
            fns[f]<<<sms, warps * 32>>>(d, 1.0f);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            int clk;
            cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
            double instr = (double)sms * warps * N_ITER * 8;          // warp-instructions
            double cyc = ms * 1e-3 * clk * 1e3;                       // at max clock
            printf("warps/SM %2d  %-10s  %.3f warp-instr/clk/SM  (%.2f us)\n", warps, names[f], instr / cyc / sms, ms * 1e3);
        }
    }
    return 0;
}
