/*
 * kf_oracle.c -- TEST INFRASTRUCTURE ONLY.  Plain, slow, obviously-correct CPU
 * executor of an image-pipeline DAG, UNFUSED: every kernel runs separately over
 * the whole image and every intermediate image is materialised.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  It shares no code, header or
 * constant with the CUDA path (paper_conf_cgo_qiaorht19_b200/); the op-IR
 * opcode numbers are restated here from the interface (include/kfuse.h), not
 * included.
 *
 * What it computes (the definition the fused GPU path must reproduce):
 *   - "fusion preserves the original order of execution ... only the input of
 *     the source kernel and the output of the destination kernel are
 *     preserved" (§II-B, Listing 1): the fused result IS
 *     the unfused result, so this executor is the oracle.
 *   - Fig. 4c is "correct" because it equals "clamp+conv+clamp+conv"
 *     (§IV-A): every local kernel applies ITS OWN border
 *     handling to the materialised intermediate image.
 *   - point operator: out(y,x) = f(in_1(y,x), ..., in_n(y,x))
 *   - local operator: acc(y,x) = sum_j sum_i m[j][i] * B(in, y+j-mh/2, x+i-mw/2),
 *     out = post(acc)  (correlation)
 *   - border map B per axis (PAPER.md:1050-1052 clamp, mirror, repeat; constant
 *     and mirror101 are extra modes), folded repeatedly when the
 *     mask is wider than the image.
 *
 * Precision: f32 pipelines are evaluated in fp64 and intermediates are kept in
 * fp64 (the paper fixes no precision); u8x4 pipelines are
 * evaluated per channel in exact integer arithmetic (int64, checked to stay in
 * int32, the GPU's accumulator width) and every kernel output is saturated to
 * [0,255] when it is stored (narrowing at every kernel boundary).
 *
 * Built with -O2 -ffp-contract=off -fopenmp.  Threads: or_set_threads(n) (1 =
 * the plain serial loop).  With n > 1 the ROWS of one kernel are split over
 * threads (each pixel is still computed by exactly the code below, in the same
 * order of taps); kernels still run one after another.  This is the SURVEY
 * §8(d) "OpenMP over rows on all cores" baseline mode and makes full-size
 * element-by-element parity affordable; it changes no arithmetic.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* ---- op-IR opcodes (restated from include/kfuse.h kf_opcode) ---------- */
enum {
    OR_LOAD = 0, OR_CONST = 1, OR_ADD = 2, OR_SUB = 3, OR_MUL = 4, OR_DIV = 5,
    OR_MIN = 6, OR_MAX = 7, OR_ABS = 8, OR_NEG = 9, OR_SQRT = 10, OR_EXP = 11,
    OR_LOG = 12, OR_POW = 13, OR_SHR = 14, OR_SHL = 15, OR_SAT_U8 = 16,
    OR_CLAMP = 17, OR_SELECT_GT = 18, OR_LUT = 19
};
enum { OR_CLAMP_MODE = 0, OR_MIRROR = 1, OR_MIRROR101 = 2, OR_REPEAT = 3, OR_CONSTANT = 4 };
enum { OR_F32 = 0, OR_U8X4 = 1 };
enum { OR_POINT = 0, OR_LOCAL = 1 };

typedef struct {
    int kind;                 /* OR_POINT / OR_LOCAL */
    int n_inputs;
    const int *inputs;        /* image ids (a local op has exactly one) */
    int n_prog;               /* point: body; local: post program on ACC (0 = identity) */
    const int *prog_op;
    const int *prog_arg;
    const double *prog_imm;
    const int *lut;
    int lut_len;
    int mw, mh;               /* local only */
    const double *mask;       /* mh rows of mw, row-major */
    int mode;
    double constant;
} or_op;

static int g_err;            /* sticky: 1 = int32 overflow, 2 = bad program */
static int g_threads = 1;

static void set_err(int e) { __atomic_store_n(&g_err, e, __ATOMIC_RELAXED); }

/* Number of threads for or_run / or_eval_points (<= 0: all cores). Returns it. */
int or_set_threads(int n)
{
#ifdef _OPENMP
    g_threads = n > 0 ? n : omp_get_num_procs();
#else
    g_threads = 1;
    (void)n;
#endif
    return g_threads;
}

/* ---- border map, -1 = constant ---------------------- */
int or_border(int p, int n, int mode)
{
    if (p >= 0 && p < n) return p;
    switch (mode) {
    case OR_CLAMP_MODE:
        return p < 0 ? 0 : n - 1;
    case OR_MIRROR:          /* symmetric: -1 -> 0, n -> n-1 */
        while (p < 0 || p >= n) p = (p < 0) ? -p - 1 : 2 * n - p - 1;
        return p;
    case OR_MIRROR101:       /* reflect-101: -1 -> 1, n -> n-2 */
        if (n == 1) return 0;
        while (p < 0 || p >= n) p = (p < 0) ? -p : 2 * n - p - 2;
        return p;
    case OR_REPEAT:
        return ((p % n) + n) % n;
    default:
        return -1;
    }
}

/* ---- program interpreter ------------------------------------------------ */
typedef double (*fload_fn)(void *ctx, int k);
typedef int64_t (*iload_fn)(void *ctx, int k);

static double run_f(const or_op *o, int n, const int *op, const int *arg, const double *imm,
                    fload_fn load, void *ctx)
{
    double st[64];
    int sp = 0;
    for (int i = 0; i < n; i++) {
        double a, b, c;
        switch (op[i]) {
        case OR_LOAD: st[sp++] = load(ctx, arg[i]); break;
        case OR_CONST: st[sp++] = imm[i]; break;
        case OR_ADD: b = st[--sp]; a = st[--sp]; st[sp++] = a + b; break;
        case OR_SUB: b = st[--sp]; a = st[--sp]; st[sp++] = a - b; break;
        case OR_MUL: b = st[--sp]; a = st[--sp]; st[sp++] = a * b; break;
        case OR_DIV: b = st[--sp]; a = st[--sp]; st[sp++] = a / b; break;
        case OR_MIN: b = st[--sp]; a = st[--sp]; st[sp++] = a < b ? a : b; break;
        case OR_MAX: b = st[--sp]; a = st[--sp]; st[sp++] = a > b ? a : b; break;
        case OR_ABS: a = st[--sp]; st[sp++] = fabs(a); break;
        case OR_NEG: a = st[--sp]; st[sp++] = -a; break;
        case OR_SQRT: a = st[--sp]; st[sp++] = sqrt(a); break;
        case OR_EXP: a = st[--sp]; st[sp++] = exp(a); break;
        case OR_LOG: a = st[--sp]; st[sp++] = log(a); break;
        case OR_POW: b = st[--sp]; a = st[--sp]; st[sp++] = pow(a, b); break;
        case OR_CLAMP: c = st[--sp]; b = st[--sp]; a = st[--sp];
            st[sp++] = a < b ? b : (a > c ? c : a); break;
        case OR_SELECT_GT: { double d = st[--sp]; c = st[--sp]; b = st[--sp]; a = st[--sp];
            st[sp++] = a > b ? c : d; break; }
        default: set_err(2); return 0.0;   /* SHR/SHL/SAT/LUT are integer-only */
        }
    }
    (void)o;
    if (sp != 1) set_err(2);
    return sp == 1 ? st[0] : 0.0;
}

static int64_t chk(int64_t v)
{
    if (v > INT32_MAX || v < INT32_MIN) set_err(1);
    return v;
}

static int64_t floor_shr(int64_t v, int n)
{
    int64_t d = (int64_t)1 << n;     /* arithmetic shift == floor division by 2^n */
    return v >= 0 ? v / d : -((-v + d - 1) / d);
}

static int64_t run_i(const or_op *o, int n, const int *op, const int *arg, const double *imm,
                     iload_fn load, void *ctx)
{
    int64_t st[64];
    int sp = 0;
    for (int i = 0; i < n; i++) {
        int64_t a, b, c;
        switch (op[i]) {
        case OR_LOAD: st[sp++] = load(ctx, arg[i]); break;
        case OR_CONST: st[sp++] = (int64_t)imm[i]; break;
        case OR_ADD: b = st[--sp]; a = st[--sp]; st[sp++] = chk(a + b); break;
        case OR_SUB: b = st[--sp]; a = st[--sp]; st[sp++] = chk(a - b); break;
        case OR_MUL: b = st[--sp]; a = st[--sp]; st[sp++] = chk(a * b); break;
        case OR_DIV: b = st[--sp]; a = st[--sp]; st[sp++] = b == 0 ? 0 : a / b; break;
        case OR_MIN: b = st[--sp]; a = st[--sp]; st[sp++] = a < b ? a : b; break;
        case OR_MAX: b = st[--sp]; a = st[--sp]; st[sp++] = a > b ? a : b; break;
        case OR_ABS: a = st[--sp]; st[sp++] = chk(a < 0 ? -a : a); break;
        case OR_NEG: a = st[--sp]; st[sp++] = chk(-a); break;
        case OR_SHR: a = st[--sp]; st[sp++] = floor_shr(a, arg[i]); break;
        case OR_SHL: a = st[--sp]; st[sp++] = chk(a * ((int64_t)1 << arg[i])); break;
        case OR_SAT_U8: a = st[--sp]; st[sp++] = a < 0 ? 0 : (a > 255 ? 255 : a); break;
        case OR_CLAMP: c = st[--sp]; b = st[--sp]; a = st[--sp];
            st[sp++] = a < b ? b : (a > c ? c : a); break;
        case OR_SELECT_GT: { int64_t d = st[--sp]; c = st[--sp]; b = st[--sp]; a = st[--sp];
            st[sp++] = a > b ? c : d; break; }
        case OR_LUT: a = st[--sp];
            if (a < 0) a = 0;
            if (a >= o->lut_len) a = o->lut_len - 1;
            st[sp++] = o->lut[a]; break;
        default: set_err(2); return 0;
        }
    }
    if (sp != 1) set_err(2);
    return sp == 1 ? st[0] : 0;
}

static int64_t sat_u8(int64_t v) { return v < 0 ? 0 : (v > 255 ? 255 : v); }

/* ======================= 1. materialising executor ======================= */
/* images: f32 pipelines -> double[H*W]; u8x4 -> int64[H*W*4] (already saturated) */

typedef struct { void **img; int x, y, c, W; const or_op *o; double acc_f; int64_t acc_i; } pctx;

static double pload_f(void *vc, int k)
{
    pctx *p = (pctx *)vc;
    if (p->o->kind == OR_LOCAL) return p->acc_f;          /* post program: ACC */
    return ((double *)p->img[p->o->inputs[k]])[(size_t)p->y * p->W + p->x];
}
static int64_t pload_i(void *vc, int k)
{
    pctx *p = (pctx *)vc;
    if (p->o->kind == OR_LOCAL) return p->acc_i;
    return ((int64_t *)p->img[p->o->inputs[k]])[((size_t)p->y * p->W + p->x) * 4 + p->c];
}

static void exec_op(int W, int H, int dtype, void **img, const or_op *o, void *out)
{
    int nc = dtype == OR_F32 ? 1 : 4;
#pragma omp parallel for schedule(static) num_threads(g_threads) if (g_threads > 1)
    for (int y = 0; y < H; y++) {
        pctx ctx;
        ctx.img = img; ctx.W = W; ctx.o = o;
        for (int x = 0; x < W; x++)
            for (int c = 0; c < nc; c++) {
                ctx.x = x; ctx.y = y; ctx.c = c;
                if (o->kind == OR_LOCAL) {
                    int cy = o->mh / 2, cx = o->mw / 2;
                    const void *in = img[o->inputs[0]];
                    double af = 0.0;
                    int64_t ai = 0;
                    for (int j = 0; j < o->mh; j++)
                        for (int i = 0; i < o->mw; i++) {
                            double m = o->mask[j * o->mw + i];
                            int yy = or_border(y + j - cy, H, o->mode);
                            int xx = or_border(x + i - cx, W, o->mode);
                            if (dtype == OR_F32) {
                                double v = (yy < 0 || xx < 0) ? o->constant
                                         : ((const double *)in)[(size_t)yy * W + xx];
                                af += m * v;
                            } else {
                                int64_t v = (yy < 0 || xx < 0) ? (int64_t)o->constant
                                          : ((const int64_t *)in)[((size_t)yy * W + xx) * 4 + c];
                                ai = chk(ai + (int64_t)m * v);
                            }
                        }
                    ctx.acc_f = af; ctx.acc_i = ai;
                    if (dtype == OR_F32)
                        ((double *)out)[(size_t)y * W + x] = o->n_prog
                            ? run_f(o, o->n_prog, o->prog_op, o->prog_arg, o->prog_imm, pload_f, &ctx) : af;
                    else
                        ((int64_t *)out)[((size_t)y * W + x) * 4 + c] = sat_u8(o->n_prog
                            ? run_i(o, o->n_prog, o->prog_op, o->prog_arg, o->prog_imm, pload_i, &ctx) : ai);
                } else {
                    if (dtype == OR_F32)
                        ((double *)out)[(size_t)y * W + x] =
                            run_f(o, o->n_prog, o->prog_op, o->prog_arg, o->prog_imm, pload_f, &ctx);
                    else
                        ((int64_t *)out)[((size_t)y * W + x) * 4 + c] =
                            sat_u8(run_i(o, o->n_prog, o->prog_op, o->prog_arg, o->prog_imm, pload_i, &ctx));
                }
            }
    }
}

/*
 * or_run: execute all kernels in declaration order.
 * inputs[i]: f32 -> float[H*W]; u8x4 -> uint8[H*W*4].
 * For each requested image id req_ids[r], writes req_out[r]:
 *   f32 -> double[H*W] (exact fp64 value); u8x4 -> uint8[H*W*4].
 * Intermediates are freed after their last use.  Returns 0, or the sticky error.
 */
int or_run(int W, int H, int dtype, int n_inputs, const void *const *inputs,
           int n_ops, const or_op *ops, int n_req, const int *req_ids, void *const *req_out)
{
    int n_img = n_inputs + n_ops, nc = dtype == OR_F32 ? 1 : 4;
    size_t npx = (size_t)W * H, esz = dtype == OR_F32 ? sizeof(double) : sizeof(int64_t);
    void **img = (void **)calloc((size_t)n_img, sizeof(void *));
    int *last = (int *)malloc(sizeof(int) * (size_t)n_img);
    g_err = 0;
    for (int i = 0; i < n_img; i++) last[i] = i < n_inputs ? -1 : i - n_inputs;
    for (int k = 0; k < n_ops; k++)
        for (int j = 0; j < ops[k].n_inputs; j++) last[ops[k].inputs[j]] = k;
    for (int r = 0; r < n_req; r++) last[req_ids[r]] = n_ops;     /* keep requested ones */
    for (int i = 0; i < n_inputs; i++) {
        img[i] = malloc(npx * nc * esz);
        for (size_t p = 0; p < npx * nc; p++) {
            if (dtype == OR_F32) ((double *)img[i])[p] = ((const float *)inputs[i])[p];
            else ((int64_t *)img[i])[p] = ((const uint8_t *)inputs[i])[p];
        }
    }
    for (int k = 0; k < n_ops; k++) {
        int id = n_inputs + k;
        img[id] = malloc(npx * nc * esz);
        exec_op(W, H, dtype, img, &ops[k], img[id]);
        for (int j = 0; j < id; j++)
            if (img[j] && last[j] == k) { free(img[j]); img[j] = NULL; }
    }
    for (int r = 0; r < n_req; r++) {
        const void *src = img[req_ids[r]];
        if (dtype == OR_F32) memcpy(req_out[r], src, npx * sizeof(double));
        else for (size_t p = 0; p < npx * 4; p++) ((uint8_t *)req_out[r])[p] = (uint8_t)((const int64_t *)src)[p];
    }
    for (int i = 0; i < n_img; i++) free(img[i]);
    free(img);
    free(last);
    return g_err;
}

/* ================== 2. pointwise (recursive) evaluator =================== */
/*
 * The same definition evaluated at one pixel by recursion over the DAG: the
 * value of image I at an in-image position q is the producer evaluated at q
 * with ITS OWN accessor on its inputs; a local consumer reads I at B_c(p)
 * (index exchange semantics, §IV-B).  Used for
 * sampled parity at full BASELINE sizes.  Exponential in depth, no memo.
 */
typedef struct { int W, H, dtype, n_inputs; const void *const *inputs; const or_op *ops; } ectx;
typedef struct { const ectx *e; const or_op *o; int y, x, c; double acc_f; int64_t acc_i; } eload;

static double ev_f(const ectx *e, int id, int y, int x);
static int64_t ev_i(const ectx *e, int id, int y, int x, int c);

static double eload_f(void *vc, int k)
{
    eload *l = (eload *)vc;
    if (l->o->kind == OR_LOCAL) return l->acc_f;
    return ev_f(l->e, l->o->inputs[k], l->y, l->x);
}
static int64_t eload_i(void *vc, int k)
{
    eload *l = (eload *)vc;
    if (l->o->kind == OR_LOCAL) return l->acc_i;
    return ev_i(l->e, l->o->inputs[k], l->y, l->x, l->c);
}

static double ev_f(const ectx *e, int id, int y, int x)
{
    if (id < e->n_inputs) return ((const float *)e->inputs[id])[(size_t)y * e->W + x];
    const or_op *o = &e->ops[id - e->n_inputs];
    eload l = {e, o, y, x, 0, 0.0, 0};
    if (o->kind == OR_LOCAL) {
        int cy = o->mh / 2, cx = o->mw / 2;
        double af = 0.0;
        for (int j = 0; j < o->mh; j++)
            for (int i = 0; i < o->mw; i++) {
                int yy = or_border(y + j - cy, e->H, o->mode);
                int xx = or_border(x + i - cx, e->W, o->mode);
                double v = (yy < 0 || xx < 0) ? o->constant : ev_f(e, o->inputs[0], yy, xx);
                af += o->mask[j * o->mw + i] * v;
            }
        if (!o->n_prog) return af;
        l.acc_f = af;
    }
    return run_f(o, o->n_prog, o->prog_op, o->prog_arg, o->prog_imm, eload_f, &l);
}

static int64_t ev_i(const ectx *e, int id, int y, int x, int c)
{
    if (id < e->n_inputs) return ((const uint8_t *)e->inputs[id])[((size_t)y * e->W + x) * 4 + c];
    const or_op *o = &e->ops[id - e->n_inputs];
    eload l = {e, o, y, x, c, 0.0, 0};
    if (o->kind == OR_LOCAL) {
        int cy = o->mh / 2, cx = o->mw / 2;
        int64_t ai = 0;
        for (int j = 0; j < o->mh; j++)
            for (int i = 0; i < o->mw; i++) {
                int yy = or_border(y + j - cy, e->H, o->mode);
                int xx = or_border(x + i - cx, e->W, o->mode);
                int64_t v = (yy < 0 || xx < 0) ? (int64_t)o->constant : ev_i(e, o->inputs[0], yy, xx, c);
                ai = chk(ai + (int64_t)o->mask[j * o->mw + i] * v);
            }
        if (!o->n_prog) return sat_u8(ai);
        l.acc_i = ai;
    }
    return sat_u8(run_i(o, o->n_prog, o->prog_op, o->prog_arg, o->prog_imm, eload_i, &l));
}

/* or_eval_points: value of image `id` at n points (ys[i], xs[i]).
 * f32 -> out is double[n]; u8x4 -> out is uint8[n*4]. */
int or_eval_points(int W, int H, int dtype, int n_inputs, const void *const *inputs,
                   int n_ops, const or_op *ops, int id, int n, const int *ys, const int *xs, void *out)
{
    ectx e = {W, H, dtype, n_inputs, inputs, ops};
    (void)n_ops;
    g_err = 0;
#pragma omp parallel for schedule(dynamic, 16) num_threads(g_threads) if (g_threads > 1)
    for (int i = 0; i < n; i++) {
        if (dtype == OR_F32) ((double *)out)[i] = ev_f(&e, id, ys[i], xs[i]);
        else for (int c = 0; c < 4; c++) ((uint8_t *)out)[i * 4 + c] = (uint8_t)ev_i(&e, id, ys[i], xs[i], c);
    }
    return g_err;
}
