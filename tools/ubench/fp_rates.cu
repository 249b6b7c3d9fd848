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
    unsigned q[8];
    for (int i = 0; i < 8; i++) q[i] = threadIdx.x * 7u + i;
    const unsigned qb = __float_as_uint(s) ^ 0x1234567u, qc = qb * 3u + 1u;
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
            if (KIND == 8) q[i] = q[i] + qb + qc;                        // IADD3 r,r,r
            if (KIND == 9) q[i] = q[i] * qb + qc;                        // IMAD r,r,r
            if (KIND == 10) q[i] = (q[i] & qb) ^ (q[i] >> 1);           // LOP3 + SHF
            if (KIND == 11) q[i] = __byte_perm(q[i], qb, 0x6420);        // PRMT
            if (KIND == 12) q[i] = __vminu2(q[i] + qc, qb);              // VIADD? + VIMNMX.U16x2
            if (KIND == 13) q[i] = (q[i] >> 3) | qb;                     // SHF + LOP (alu)
            if (KIND == 14) { p[i] = __ffma2_rn(p[i], b2, c2); q[i] = q[i] + qb + qc; }   // FFMA2 + IADD3 mix
            if (KIND == 15) { a[i] = fmaf(a[i], b, c); q[i] = q[i] + qb + qc; }           // FFMA + IADD3 mix
        }
    }
    float r = 0;
    for (int i = 0; i < 8; i++) r += a[i] + p[i].x + p[i].y + (float)q[i];
    if (r == 12345.f) out[0] = r;
}

int main()
{
    float *d;
    cudaMalloc(&d, 4);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const char *names[] = {"FFMA r,r,r", "FFMA imm", "FADD", "FMUL", "FFMA2", "FADD2", "FMUL2", "FFMA2 imm",
                           "IADD3", "IMAD", "LOP3", "PRMT", "VIMNMX16x2", "SHF|LOP", "FFMA2+IADD3", "FFMA+IADD3"};
    void (*fns[])(float *, float) = {k<0>, k<1>, k<2>, k<3>, k<4>, k<5>, k<6>, k<7>,
                                     k<8>, k<9>, k<10>, k<11>, k<12>, k<13>, k<14>, k<15>};
    for (int warps = 4; warps <= 32; warps *= 2) {
        for (int f = 0; f < 16; f++) {
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
