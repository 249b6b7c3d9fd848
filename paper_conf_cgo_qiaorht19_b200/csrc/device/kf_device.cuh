// kf_device.cuh -- device-side library included by every generated fused
// kernel (compiled by NVRTC for sm_100a).  Hand-written; the code generator
// (codegen.cpp) only emits the per-block glue that calls into it.
//
// Value types: KF_F32 pipelines compute in float; KF_U8X4 pipelines compute per
// channel in int32 (struct I4) and store saturated uchar4 (PAPER.md:1051-1053:
// the intermediate becomes a register; narrowing at every kernel
// boundary, kept in the fused kernel).
#pragma once

#define KF_MAX_IMG 16
#define KF_MAX_RECT 4

// A border-frame rectangle of the slow (index-exchange) path, tiled by one of
// two tile shapes (0: 32 x 8 for the top/bottom frame, 1: 8 x 32 for the
// left/right frame).  CTAs [cta0, cta0 + ntx * nty) of the launch cover it.
struct KfRect {
    int x0, x1, y0, y1;
    int shape, ntx, nty, cta0;
};

// Launch arguments of one fused block kernel (__grid_constant__).  Mirrors the
// geometry computed by runtime.cu.
struct KfArgs {
    const void *img[KF_MAX_IMG];   // external images of the block (slot order)
    int base[KF_MAX_IMG];          // global row held by row 0 of each buffer
    int rlast[KF_MAX_IMG];         // last global row held by each buffer
    void *out;                     // block output image
    int out_base;                  // global row held by row 0 of `out`
    int W, H;                      // image size (global)
    int r0, r1;                    // output rows computed by this launch
#ifdef KF_BOUNDS
    // bounds-checking build only (libkfuse_bounds.so): every
    // global access is checked against these spans before it is made
    unsigned long long span_lo[KF_MAX_IMG], span_hi[KF_MAX_IMG];   // readable: the external image buffers
    unsigned long long out_lo, out_hi;                            // writable: this launch's output rows
    int n_span;
    unsigned *viol;                                               // [count, first addr lo, hi, is_write]
#endif
    int indep;                     // 1: independent of the previous kernel on the stream (kf_run_batch
                                   // frames after the first): griddepcontrol.wait moves to the kernel's end
    // border frame: slow path, CTAs [0, frame_ctas)
    KfRect rect[KF_MAX_RECT];
    int n_rect, frame_ctas;
    // interior: streaming fast path, one warp per item, CTAs [frame_ctas, ...)
    int fx0, fx1, fy0, fy1;        // interior output rectangle (x multiple of 4)
    int strip;                     // output rows per item
    int n_chunks;                  // column chunks of (32 - 2*HL) * 4 columns
    int n_strips;                  // row strips (the last one takes the remainder)
    int n_items;                   // n_chunks * n_strips
    int edge_l, edge_r, edge_t, edge_b;   // image edges handled by the edge chunks / strips
    int n_long;                    // strips [0, n_long) are two units tall, the rest one unit
};

// ------------------------------------------------------------ border map
// Per-axis index map of PAPER.md:1050-1052 (clamp / mirror / repeat) plus
// mirror101 and constant, folded until in range.  -1 = use the constant.
enum { KF_B_CLAMP = 0, KF_B_MIRROR = 1, KF_B_MIRROR101 = 2, KF_B_REPEAT = 3, KF_B_CONSTANT = 4 };

template <int MODE>
__device__ __forceinline__ int kf_border(int p, int n)
{
    if (MODE == KF_B_CLAMP) return min(max(p, 0), n - 1);
    if (MODE == KF_B_CONSTANT) return (p >= 0 && p < n) ? p : -1;
    if (MODE == KF_B_REPEAT) { int r = p % n; return r < 0 ? r + n : r; }
    if (MODE == KF_B_MIRROR) {
        while (p < 0 || p >= n) p = (p < 0) ? -p - 1 : 2 * n - p - 1;
        return p;
    }
    // MIRROR101
    if (n == 1) return 0;
    while (p < 0 || p >= n) p = (p < 0) ? -p : 2 * n - p - 2;
    return p;
}

__device__ __forceinline__ int kf_wrap(int p, int n) { int r = p % n; return r < 0 ? r + n : r; }

// ------------------------------------------------------------- I4 (u8x4)
struct I4 { int x, y, z, w; };

__device__ __forceinline__ I4 kf_i4(int v) { return I4{v, v, v, v}; }
__device__ __forceinline__ I4 kf_unpack(unsigned u)
{
    return I4{(int)(u & 0xffu), (int)((u >> 8) & 0xffu), (int)((u >> 16) & 0xffu), (int)(u >> 24)};
}
// a pixel in SWAR form (two channels per 16-bit lane pair, bias 0) -> I4
__device__ __forceinline__ I4 kf_unpack_sw(unsigned lo, unsigned hi)
{
    return I4{(int)(lo & 0xffffu), (int)(lo >> 16), (int)(hi & 0xffffu), (int)(hi >> 16)};
}
__device__ __forceinline__ int kf_sat(int v) { return min(max(v, 0), 255); }
__device__ __forceinline__ unsigned kf_pack(I4 a)
{
    return (unsigned)kf_sat(a.x) | ((unsigned)kf_sat(a.y) << 8) | ((unsigned)kf_sat(a.z) << 16) |
           ((unsigned)kf_sat(a.w) << 24);
}

#define KF_I4_BIN(name, expr)                                                              \
    __device__ __forceinline__ I4 name(I4 a, I4 b)                                         \
    {                                                                                      \
        I4 r;                                                                              \
        { int A = a.x, B = b.x; r.x = (expr); }                                            \
        { int A = a.y, B = b.y; r.y = (expr); }                                            \
        { int A = a.z, B = b.z; r.z = (expr); }                                            \
        { int A = a.w, B = b.w; r.w = (expr); }                                            \
        return r;                                                                          \
    }
#define KF_I4_UN(name, expr)                                                               \
    __device__ __forceinline__ I4 name(I4 a)                                               \
    {                                                                                      \
        I4 r;                                                                              \
        { int A = a.x; r.x = (expr); }                                                     \
        { int A = a.y; r.y = (expr); }                                                     \
        { int A = a.z; r.z = (expr); }                                                     \
        { int A = a.w; r.w = (expr); }                                                     \
        return r;                                                                          \
    }

KF_I4_BIN(kf_add, A + B)
KF_I4_BIN(kf_sub, A - B)
KF_I4_BIN(kf_mul, A * B)
KF_I4_BIN(kf_div, B == 0 ? 0 : A / B)
KF_I4_BIN(kf_min, min(A, B))
KF_I4_BIN(kf_max, max(A, B))
KF_I4_UN(kf_abs, abs(A))
KF_I4_UN(kf_neg, -A)
KF_I4_UN(kf_satu8, kf_sat(A))

template <int N> __device__ __forceinline__ I4 kf_shr(I4 a) { return I4{a.x >> N, a.y >> N, a.z >> N, a.w >> N}; }
template <int N> __device__ __forceinline__ I4 kf_shl(I4 a)
{
    return I4{(int)((unsigned)a.x << N), (int)((unsigned)a.y << N), (int)((unsigned)a.z << N),
              (int)((unsigned)a.w << N)};
}
__device__ __forceinline__ I4 kf_clamp(I4 a, I4 lo, I4 hi) { return kf_min(kf_max(a, lo), hi); }
__device__ __forceinline__ I4 kf_sel_gt(I4 a, I4 b, I4 c, I4 d)
{
    return I4{a.x > b.x ? c.x : d.x, a.y > b.y ? c.y : d.y, a.z > b.z ? c.z : d.z, a.w > b.w ? c.w : d.w};
}
__device__ __forceinline__ I4 kf_lut(I4 a, const int *__restrict__ t, int n)
{
    return I4{__ldg(t + min(max(a.x, 0), n - 1)), __ldg(t + min(max(a.y, 0), n - 1)),
              __ldg(t + min(max(a.z, 0), n - 1)), __ldg(t + min(max(a.w, 0), n - 1))};
}
// multiply-accumulate with an integer mask coefficient
__device__ __forceinline__ I4 kf_mac(I4 acc, int m, I4 v)
{
    return I4{acc.x + m * v.x, acc.y + m * v.y, acc.z + m * v.z, acc.w + m * v.w};
}

// -------------------------------------------------------------- float
// Explicitly rounded forms: the compiler never contracts a product into a
// later addition, so every code variant of a fused kernel (edge strips, peeled
// warm-up iterations, steady-state loop) rounds the same operations the same
// way and band / strip decompositions stay bit-identical.
__device__ __forceinline__ float kf_add(float a, float b) { return __fadd_rn(a, b); }
__device__ __forceinline__ float kf_sub(float a, float b) { return __fsub_rn(a, b); }
__device__ __forceinline__ float kf_mul(float a, float b) { return __fmul_rn(a, b); }
__device__ __forceinline__ float kf_div(float a, float b) { return a / b; }
__device__ __forceinline__ float kf_min(float a, float b) { return fminf(a, b); }
__device__ __forceinline__ float kf_max(float a, float b) { return fmaxf(a, b); }
__device__ __forceinline__ float kf_abs(float a) { return fabsf(a); }
__device__ __forceinline__ float kf_neg(float a) { return -a; }
// SQRT is the hardware square root (MUFU.SQRT, sqrt.approx.f32): measured on
// B200 over every positive normal float, it is within 1 ulp of the correctly
// rounded result (tools/ubench/sqrt_approx.cu; R-19).  One
// instruction instead of the ~10-instruction IEEE sequence with a slow path.
__device__ __forceinline__ float kf_sqrt(float a)
{
    float r;
    asm("sqrt.approx.f32 %0, %1;" : "=f"(r) : "f"(a));
    return r;
}
__device__ __forceinline__ float kf_exp(float a) { return expf(a); }
__device__ __forceinline__ float kf_log(float a) { return logf(a); }
__device__ __forceinline__ float kf_pow(float a, float b) { return powf(a, b); }
__device__ __forceinline__ float kf_clamp(float a, float lo, float hi) { return fminf(fmaxf(a, lo), hi); }
__device__ __forceinline__ float kf_sel_gt(float a, float b, float c, float d) { return a > b ? c : d; }
__device__ __forceinline__ float kf_mac(float acc, float m, float v) { return fmaf(m, v, acc); }

// ------------------------------------------------------ global image access
__device__ __forceinline__ float kf_ldf_r(const void *p, int base, int W, int y, int x)
{
    return __ldg((const float *)p + (size_t)(y - base) * W + x);
}
__device__ __forceinline__ I4 kf_ldi_r(const void *p, int base, int W, int y, int x)
{
    return kf_unpack(__ldg((const unsigned *)p + (size_t)(y - base) * W + x));
}
__device__ __forceinline__ void kf_stf_r(void *p, int base, int W, int y, int x, float v)
{
    ((float *)p)[(size_t)(y - base) * W + x] = v;
}
__device__ __forceinline__ void kf_sti_r(void *p, int base, int W, int y, int x, I4 v)
{
    ((unsigned *)p)[(size_t)(y - base) * W + x] = kf_pack(v);
}

// 128-bit accesses of the streaming path (4 pixels per lane)
__device__ __forceinline__ float4 kf_ld4f_r(const float *p) { return __ldg((const float4 *)p); }
__device__ __forceinline__ uint4 kf_ld4u_r(const unsigned *p) { return __ldg((const uint4 *)p); }
__device__ __forceinline__ void kf_st4f_r(float *p, float a, float b, float c, float d)
{
    *(float4 *)p = make_float4(a, b, c, d);
}
__device__ __forceinline__ void kf_st4u_r(unsigned *p, unsigned a, unsigned b, unsigned c, unsigned d)
{
    *(uint4 *)p = make_uint4(a, b, c, d);
}

// Access macros used by the generated code.  In the bounds-checking build
// (KF_BOUNDS, libkfuse_bounds.so -- our stand-in for compute-sanitizer's
// memcheck) every global read must fall inside one of the
// launch's external image buffers and every write inside the launch's own
// output rows; an access outside is skipped and counted (the first address is
// kept) instead of faulting.  They expand where the launch arguments `a` are in
// scope (every generated function).  Otherwise they are the plain accesses.
#ifdef KF_BOUNDS
__device__ __noinline__ bool kf_bchk(const KfArgs &a, const void *p, unsigned n, int wr)
{
    const unsigned long long x = (unsigned long long)p;
    if (wr) {
        if (x >= a.out_lo && x + n <= a.out_hi) return true;
    } else {
        for (int i = 0; i < a.n_span; i++)
            if (x >= a.span_lo[i] && x + n <= a.span_hi[i]) return true;
    }
    if (atomicAdd(a.viol, 1u) == 0u) {
        a.viol[1] = (unsigned)x;
        a.viol[2] = (unsigned)(x >> 32);
        a.viol[3] = (unsigned)wr;
    }
    return false;
}
__device__ __noinline__ int kf_bidx(const KfArgs &a, int i, int n)   // table index (LUT) in [0, n)
{
    if (i >= 0 && i < n) return i;
    if (atomicAdd(a.viol, 1u) == 0u) { a.viol[1] = (unsigned)i; a.viol[2] = 0xffffffffu; a.viol[3] = 2u; }
    return 0;
}
#define kf_ldf(p, base, W, y, x) \
    (kf_bchk(a, (const float *)(p) + (size_t)((y) - (base)) * (W) + (x), 4, 0) ? kf_ldf_r(p, base, W, y, x) : 0.0f)
#define kf_ldi(p, base, W, y, x) \
    (kf_bchk(a, (const unsigned *)(p) + (size_t)((y) - (base)) * (W) + (x), 4, 0) ? kf_ldi_r(p, base, W, y, x) : kf_i4(0))
#define kf_stf(p, base, W, y, x, v) \
    do { if (kf_bchk(a, (float *)(p) + (size_t)((y) - (base)) * (W) + (x), 4, 1)) kf_stf_r(p, base, W, y, x, v); } while (0)
#define kf_sti(p, base, W, y, x, v) \
    do { if (kf_bchk(a, (unsigned *)(p) + (size_t)((y) - (base)) * (W) + (x), 4, 1)) kf_sti_r(p, base, W, y, x, v); } while (0)
#define kf_ld4f(p) (kf_bchk(a, (p), 16, 0) ? kf_ld4f_r(p) : make_float4(0.f, 0.f, 0.f, 0.f))
#define kf_ld4u(p) (kf_bchk(a, (p), 16, 0) ? kf_ld4u_r(p) : make_uint4(0u, 0u, 0u, 0u))
#define kf_st4f(p, x0, x1, x2, x3) do { if (kf_bchk(a, (p), 16, 1)) kf_st4f_r((p), x0, x1, x2, x3); } while (0)
#define kf_st4u(p, x0, x1, x2, x3) do { if (kf_bchk(a, (p), 16, 1)) kf_st4u_r((p), x0, x1, x2, x3); } while (0)
#define KF_LDG(p) (kf_bchk(a, (p), (unsigned)sizeof(*(p)), 0) ? __ldg(p) : 0)
#define KF_WOK(p, n) kf_bchk(a, (p), (n), 1)
#define KF_IDX(i, n) kf_bidx(a, (int)(i), (n))
#define KF_RCHK(p, n) ((void)kf_bchk(a, (p), (n), 0))
#else
#define kf_ldf kf_ldf_r
#define kf_ldi kf_ldi_r
#define kf_stf kf_stf_r
#define kf_sti kf_sti_r
#define kf_ld4f kf_ld4f_r
#define kf_ld4u kf_ld4u_r
#define kf_st4f kf_st4f_r
#define kf_st4u kf_st4u_r
#define KF_LDG(p) __ldg(p)
#define KF_WOK(p, n) true
#define KF_IDX(i, n) (i)
#define KF_RCHK(p, n) ((void)0)
#endif
#define KF_FULL 0xffffffffu
__device__ __forceinline__ float kf_shup(float v, int d) { return __shfl_up_sync(KF_FULL, v, d); }
__device__ __forceinline__ float kf_shdn(float v, int d) { return __shfl_down_sync(KF_FULL, v, d); }
__device__ __forceinline__ I4 kf_shup(I4 v, int d)
{
    return I4{__shfl_up_sync(KF_FULL, v.x, d), __shfl_up_sync(KF_FULL, v.y, d), __shfl_up_sync(KF_FULL, v.z, d),
              __shfl_up_sync(KF_FULL, v.w, d)};
}
__device__ __forceinline__ I4 kf_shdn(I4 v, int d)
{
    return I4{__shfl_down_sync(KF_FULL, v.x, d), __shfl_down_sync(KF_FULL, v.y, d),
              __shfl_down_sync(KF_FULL, v.z, d), __shfl_down_sync(KF_FULL, v.w, d)};
}
// first product of an accumulation (mask coefficient m)
__device__ __forceinline__ float kf_mul1(float m, float v) { return __fmul_rn(m, v); }
__device__ __forceinline__ I4 kf_mul1(int m, I4 v) { return I4{m * v.x, m * v.y, m * v.z, m * v.w}; }

// ------------------------------------------------ packed f32x2 (sm_100a)
// Two adjacent pixels of a lane as one 64-bit register pair: FFMA2 / FADD2 /
// FMUL2 issue one instruction for both.  Operations without a
// packed form run per component.
//
// ptxas contracts a packed FMUL2 into a following FADD2 (one FFMA2, one
// rounding) even for mul.rn/add.rn.f32x2, and only where the product has a
// single use -- so the same expression rounded differently in the peeled
// warm-up iterations than in the loop (measured: band runs differed from the
// whole-image run by a few ulps).  A packed product whose rounding matters is
// therefore an FFMA2 with an addend of -0.0 the compiler cannot see
// (a * b + (-0) == a * b exactly, signed zeros included): there is no multiply
// left to contract.  Multiplies by a power of two are exact and stay FMUL2.
typedef float2 F2;
#ifdef KF_NVRTC
__constant__ float kf_nz = -0.0f;   // never written; opaque to the compiler
#define KF_NZ2 make_float2(kf_nz, kf_nz)
#else
#define KF_NZ2 make_float2(-0.0f, -0.0f)
#endif
__device__ __forceinline__ bool kf_pow2f(float m) { return (__float_as_uint(m) & 0x007fffffu) == 0u && m != 0.0f; }
__device__ __forceinline__ F2 kf2(float a) { return make_float2(a, a); }
__device__ __forceinline__ F2 kf2_add(F2 a, F2 b) { return __fadd2_rn(a, b); }
__device__ __forceinline__ F2 kf2_sub(F2 a, F2 b) { return __fadd2_rn(a, make_float2(-b.x, -b.y)); }
__device__ __forceinline__ F2 kf2_mul(F2 a, F2 b) { return __ffma2_rn(a, b, KF_NZ2); }
__device__ __forceinline__ F2 kf2_fma(F2 a, F2 b, F2 c) { return __ffma2_rn(a, b, c); }          // a*b + c
__device__ __forceinline__ F2 kf2_fms(F2 a, F2 b, F2 c) { return __ffma2_rn(a, b, make_float2(-c.x, -c.y)); }  // a*b - c
__device__ __forceinline__ F2 kf2_nfma(F2 a, F2 b, F2 c) { return __ffma2_rn(make_float2(-a.x, -a.y), b, c); }  // c - a*b
__device__ __forceinline__ F2 kf2_mac(F2 acc, float m, F2 v) { return __ffma2_rn(v, make_float2(m, m), acc); }
__device__ __forceinline__ F2 kf2_mul1(float m, F2 v)
{
    return kf_pow2f(m) ? __fmul2_rn(v, make_float2(m, m)) : __ffma2_rn(v, make_float2(m, m), KF_NZ2);
}
__device__ __forceinline__ F2 kf2_div(F2 a, F2 b) { return make_float2(a.x / b.x, a.y / b.y); }
__device__ __forceinline__ F2 kf2_min(F2 a, F2 b) { return make_float2(fminf(a.x, b.x), fminf(a.y, b.y)); }
__device__ __forceinline__ F2 kf2_max(F2 a, F2 b) { return make_float2(fmaxf(a.x, b.x), fmaxf(a.y, b.y)); }
__device__ __forceinline__ F2 kf2_abs(F2 a) { return make_float2(fabsf(a.x), fabsf(a.y)); }
__device__ __forceinline__ F2 kf2_neg(F2 a) { return make_float2(-a.x, -a.y); }
__device__ __forceinline__ F2 kf2_sqrt(F2 a) { return make_float2(kf_sqrt(a.x), kf_sqrt(a.y)); }
__device__ __forceinline__ F2 kf2_exp(F2 a) { return make_float2(expf(a.x), expf(a.y)); }
__device__ __forceinline__ F2 kf2_log(F2 a) { return make_float2(logf(a.x), logf(a.y)); }
__device__ __forceinline__ F2 kf2_pow(F2 a, F2 b) { return make_float2(powf(a.x, b.x), powf(a.y, b.y)); }
__device__ __forceinline__ F2 kf2_clamp(F2 a, F2 lo, F2 hi)
{
    return make_float2(fminf(fmaxf(a.x, lo.x), hi.x), fminf(fmaxf(a.y, lo.y), hi.y));
}
__device__ __forceinline__ F2 kf2_sel_gt(F2 a, F2 b, F2 c, F2 d)
{
    return make_float2(a.x > b.x ? c.x : d.x, a.y > b.y ? c.y : d.y);
}

// ------------------------------------------- asynchronous row ring (cp.async)
// Each streaming warp keeps DS input rows (512 B each) in flight in a shared
// memory ring: 16 B per lane per row via cp.async (LDGSTS), one commit group
// per row, consumed DS-1 groups later.
__device__ __forceinline__ void kf_cp16_r(void *smem, const void *gmem)
{
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem) : "memory");
}
#ifdef KF_BOUNDS
#define kf_cp16(d, g) do { if (kf_bchk(a, (g), 16, 0)) kf_cp16_r((d), (g)); } while (0)
#else
#define kf_cp16 kf_cp16_r
#endif
__device__ __forceinline__ void kf_cp_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N> __device__ __forceinline__ void kf_cp_wait()
{
    asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory");
}

// ------------------------------------- TMA row feed (option tma)
// The same ring, filled by the Tensor Memory Accelerator instead: one elected
// lane issues ONE bulk copy (cp.async.bulk, SASS UBLKCP) of the warp's whole
// contiguous row segment (32 lanes x 16 B) per row, completing on an mbarrier
// per ring slot (expect_tx / complete_tx); the lanes wait on the slot's phase
// parity instead of a cp.async group count.  Before a slot is refilled the
// warp synchronises (every lane has read it) and the issuing lane orders those
// generic-proxy reads before the async-proxy write (fence.proxy.async).
__device__ __forceinline__ unsigned kf_smem_addr(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void kf_mbar_init(unsigned long long *bar, unsigned count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(kf_smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void kf_mbar_init_fence() { asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory"); }
__device__ __forceinline__ void kf_proxy_fence() { asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory"); }
__device__ __forceinline__ void kf_bulk_row(void *smem, const void *gmem, unsigned bytes, unsigned long long *bar)
{
    const unsigned b = kf_smem_addr(bar);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(b), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n"
                 ::"r"(kf_smem_addr(smem)), "l"(gmem), "r"(bytes), "r"(b) : "memory");
}
__device__ __forceinline__ void kf_mbar_wait(unsigned long long *bar, unsigned parity)
{
    const unsigned b = kf_smem_addr(bar);
    unsigned done;
    do {
        asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
                     : "=r"(done) : "r"(b), "r"(parity) : "memory");
    } while (!done);
}
__device__ __forceinline__ int kf_wrap_lt(int x, int n) { return x >= n ? x - n : x; }
