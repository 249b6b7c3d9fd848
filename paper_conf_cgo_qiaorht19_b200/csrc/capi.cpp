// capi.cpp -- extern "C" boundary of libkfuse (include/kfuse.h).  Every entry
// point converts kf::Error into a kf_status and a thread-local message.
#include <cmath>
#include <cstring>

#include "kf_internal.h"

namespace kf {

static thread_local std::string g_last_error;

void set_error(const std::string &msg) { g_last_error = msg; }

[[noreturn]] void fail(kf_status st, const std::string &msg) { throw Error{st, msg}; }

template <class F>
static kf_status guard(F &&f)
{
    try {
        f();
        return KF_OK;
    } catch (const Error &e) {
        g_last_error = e.msg;
        return e.st;
    } catch (const std::bad_alloc &) {
        g_last_error = "host allocation failed";
        return KF_ERR_OOM;
    } catch (const std::exception &e) {
        g_last_error = e.what();
        return KF_ERR_ARG;
    }
}

static void check_id(const kf_pipeline *p, int id)
{
    if (id < 0 || id >= p->n_images()) fail(KF_ERR_BAD_ID, "image id " + std::to_string(id) + " does not exist");
}

static void check_mutable(const kf_pipeline *p)
{
    if (!p) fail(KF_ERR_ARG, "null pipeline");
    if (p->frozen) fail(KF_ERR_FROZEN, "pipeline is frozen: a plan already exists");
}

static std::vector<Instr> copy_prog(const kf_instr *prog, int n)
{
    if (n < 0 || (n > 0 && !prog)) fail(KF_ERR_ARG, "bad program pointer/size");
    if (n > 4096) fail(KF_ERR_PROGRAM, "program longer than 4096 instructions");
    std::vector<Instr> v(n);
    for (int i = 0; i < n; i++) v[i] = Instr{prog[i].op, prog[i].arg, prog[i].imm};
    return v;
}

}  // namespace kf

using namespace kf;


extern "C" {

void kf_model_params_paper(kf_model_params *m)
{
    if (!m) return;
    m->tg = 400.0;
    m->ts = 4.0;       // "a few cycles", PAPER.md:421-424 (R-5)
    m->c_alu = 4.0;
    m->c_sfu = 16.0;   // not given (R-5)
    m->gamma = 0.0;    // omitted
    m->c_mshared = 2.0;// PAPER.md:708-712
    m->phi_mode = 0;
    m->tile_w = 32;
    m->tile_h = 32;
    m->eq3_mode = 0;
    m->bw_bytes_clk = 0.0;
    m->issue_lanes_clk = 0.0;
    m->overlap = 0.0;
}

void kf_model_params_b200(kf_model_params *m)
{
    kf_model_params_paper(m);
    if (!m) return;
    m->c_mshared = 5.0;
    m->phi_mode = 1;
}

void kf_model_params_b200_roofline(kf_model_params *m)
{
    kf_model_params_paper(m);
    if (!m) return;
    m->phi_mode = 2;          // DESIGN.md R-20
    m->c_mshared = 5.0;
    m->tile_w = 120;          // streaming column chunk (32 - 2 halo lanes) x 4 pixels ...
    m->tile_h = 32;           // ... by a strip of rows
    m->bw_bytes_clk = 22.45;  // 6528.4 GB/s / (148 SMs x 1.965 GHz)
    m->issue_lanes_clk = 115.0;   // 3.6 FFMA warp-instr / clk / SM (profiles/r01_fp_int_issue_rates.txt)
    m->overlap = 1.0;             // fitted (profiles/r02_calibration.md)
}

kf_status kf_pipeline_create(int32_t width, int32_t height, kf_dtype dtype, kf_pipeline **out)
{
    return guard([&] {
        if (!out) fail(KF_ERR_ARG, "null out");
        if (width <= 0 || height <= 0 || (int64_t)width * height >= (int64_t)1 << 31)
            fail(KF_ERR_ARG, "image size must be positive with width*height < 2^31");
        if (dtype != KF_F32 && dtype != KF_U8X4) fail(KF_ERR_ARG, "unknown dtype");
        auto p = new kf_pipeline();
        p->W = width;
        p->H = height;
        p->dtype = dtype;
        *out = p;
    });
}

void kf_pipeline_destroy(kf_pipeline *p) { delete p; }

kf_status kf_add_input(kf_pipeline *p, int32_t *image_id)
{
    return guard([&] {
        check_mutable(p);
        if (!image_id) fail(KF_ERR_ARG, "null image_id");
        if (!p->ops.empty()) fail(KF_ERR_ARG, "inputs must be declared before kernels");
        if (p->n_inputs >= 8) fail(KF_ERR_ARG, "at most 8 pipeline inputs");
        *image_id = p->n_inputs++;
    });
}

kf_status kf_add_point_op(kf_pipeline *p, const int32_t *inputs, int32_t n_inputs, const kf_instr *prog,
                          int32_t n_instr, const kf_cost *cost, const int32_t *lut, int32_t lut_len,
                          int32_t *out_image)
{
    return guard([&] {
        check_mutable(p);
        if (!out_image || !inputs || n_inputs < 1 || n_inputs > 8) fail(KF_ERR_ARG, "point op needs 1..8 inputs");
        if ((lut && lut_len < 1) || lut_len < 0 || lut_len > 65536) fail(KF_ERR_ARG, "bad lut size");
        if ((int)p->ops.size() >= 64) fail(KF_ERR_ARG, "at most 64 kernels per pipeline");
        Op op;
        op.kind = POINT;
        for (int i = 0; i < n_inputs; i++) {
            check_id(p, inputs[i]);
            op.inputs.push_back(inputs[i]);
        }
        op.prog = copy_prog(prog, n_instr);
        if (lut) op.lut.assign(lut, lut + lut_len);
        validate_program(p, op.prog, n_inputs, lut != nullptr);
        if (cost) {
            if (cost->n_alu < 0 || cost->n_sfu < 0) fail(KF_ERR_ARG, "negative cost");
            op.n_alu = cost->n_alu;
            op.n_sfu = cost->n_sfu;
        } else {
            default_cost(p, op);
        }
        p->ops.push_back(std::move(op));
        *out_image = p->n_images() - 1;
    });
}

kf_status kf_add_local_op(kf_pipeline *p, int32_t input, const double *mask, int32_t mask_w, int32_t mask_h,
                          kf_boundary mode, double constant, const kf_instr *post, int32_t n_post,
                          const kf_cost *cost, int32_t *out_image)
{
    return guard([&] {
        check_mutable(p);
        if (!out_image || !mask) fail(KF_ERR_ARG, "null pointer");
        check_id(p, input);
        if (mask_w < 1 || mask_h < 1 || mask_w % 2 == 0 || mask_h % 2 == 0 || mask_w > 31 || mask_h > 31)
            fail(KF_ERR_MASK, "mask must be odd-sized, at most 31x31");
        if (mode < KF_CLAMP || mode > KF_CONSTANT) fail(KF_ERR_ARG, "unknown boundary mode");
        if ((int)p->ops.size() >= 64) fail(KF_ERR_ARG, "at most 64 kernels per pipeline");
        Op op;
        op.kind = LOCAL;
        op.inputs = {input};
        op.mw = mask_w;
        op.mh = mask_h;
        op.mask.assign(mask, mask + (size_t)mask_w * mask_h);
        for (double v : op.mask) {
            if (!std::isfinite(v)) fail(KF_ERR_MASK, "mask coefficients must be finite");
            if (p->dtype == KF_U8X4 && (v != std::floor(v) || std::fabs(v) > 65536))
                fail(KF_ERR_MASK, "KF_U8X4 masks must hold integers in [-65536, 65536]");
        }
        op.mode = mode;
        op.constant = constant;
        if (p->dtype == KF_U8X4 && (constant != std::floor(constant) || constant < 0 || constant > 255))
            fail(KF_ERR_ARG, "KF_U8X4 border constant must be an integer in [0,255]");
        op.prog = copy_prog(post, n_post);
        if (!op.prog.empty()) validate_program(p, op.prog, 1, false);
        if (cost) {
            if (cost->n_alu < 0 || cost->n_sfu < 0) fail(KF_ERR_ARG, "negative cost");
            op.n_alu = cost->n_alu;
            op.n_sfu = cost->n_sfu;
        } else {
            default_cost(p, op);
        }
        p->ops.push_back(std::move(op));
        *out_image = p->n_images() - 1;
    });
}

kf_status kf_mark_output(kf_pipeline *p, int32_t image_id)
{
    return guard([&] {
        check_mutable(p);
        check_id(p, image_id);
        if (image_id < p->n_inputs) fail(KF_ERR_ARG, "a pipeline input cannot be an output");
        for (int o : p->outputs)
            if (o == image_id) fail(KF_ERR_ARG, "image already marked as output");
        p->outputs.push_back(image_id);
    });
}

kf_status kf_plan_fusion(kf_pipeline *p, const kf_model_params *m, kf_plan **out)
{
    return guard([&] {
        if (!p || !m || !out) fail(KF_ERR_ARG, "null pointer");
        *out = plan_fusion(p, *m);
    });
}

kf_status kf_plan_basic(kf_pipeline *p, const kf_model_params *m, kf_plan **out)
{
    return guard([&] {
        if (!p || !m || !out) fail(KF_ERR_ARG, "null pointer");
        *out = plan_basic(p, *m);
    });
}

kf_status kf_plan_exact(kf_pipeline *p, const kf_model_params *m, kf_plan **out)
{
    return guard([&] {
        if (!p || !m || !out) fail(KF_ERR_ARG, "null pointer");
        *out = plan_exact(p, *m);
    });
}

kf_status kf_plan_unfused(kf_pipeline *p, kf_plan **out)
{
    return guard([&] {
        if (!p || !out) fail(KF_ERR_ARG, "null pointer");
        if (p->ops.empty()) fail(KF_ERR_ARG, "pipeline has no kernels");
        std::vector<std::vector<int>> b;
        for (int k = 0; k < (int)p->ops.size(); k++) b.push_back({k});
        *out = plan_from_blocks(p, b, false);
    });
}

kf_status kf_plan_from_blocks(kf_pipeline *p, const int32_t *block_of_kernel, kf_plan **out)
{
    return guard([&] {
        if (!p || !block_of_kernel || !out) fail(KF_ERR_ARG, "null pointer");
        if (p->ops.empty()) fail(KF_ERR_ARG, "pipeline has no kernels");
        std::map<int, std::vector<int>> m;
        for (int k = 0; k < (int)p->ops.size(); k++) m[block_of_kernel[k]].push_back(k);
        std::vector<std::vector<int>> b;
        for (auto &kv : m) b.push_back(kv.second);
        *out = plan_from_blocks(p, b, true);
    });
}

void kf_plan_destroy(kf_plan *plan) { delete plan; }

int32_t kf_plan_num_blocks(const kf_plan *plan) { return plan ? (int32_t)plan->blocks.size() : -1; }
int32_t kf_plan_num_launches(const kf_plan *plan) { return plan ? (int32_t)plan->blocks.size() : -1; }
int32_t kf_plan_halo_rows(const kf_plan *plan) { return plan ? plan->halo_rows : -1; }
int32_t kf_plan_num_cuts(const kf_plan *plan) { return plan ? (int32_t)plan->cuts.size() : -1; }

kf_status kf_plan_block(const kf_plan *plan, int32_t i, int32_t *kernels, int32_t *n)
{
    return guard([&] {
        if (!plan || !n) fail(KF_ERR_ARG, "null pointer");
        if (i < 0 || i >= (int)plan->blocks.size()) fail(KF_ERR_ARG, "block index out of range");
        const auto &b = plan->blocks[i];
        *n = (int32_t)b.size();
        if (kernels)
            for (size_t j = 0; j < b.size(); j++) kernels[j] = b[j];
    });
}

kf_status kf_plan_objective(const kf_plan *plan, int64_t *beta_q, int64_t *beta_eps)
{
    return guard([&] {
        if (!plan || !beta_q || !beta_eps) fail(KF_ERR_ARG, "null pointer");
        *beta_q = plan->beta_q;
        *beta_eps = plan->beta_eps;
    });
}

kf_status kf_plan_edge(const kf_plan *plan, int32_t src, int32_t dst, double *w, int32_t *is_eps,
                       int32_t *ctx_legal, int32_t *profitable)
{
    return guard([&] {
        if (!plan) fail(KF_ERR_ARG, "null plan");
        for (const EdgeInfo &e : plan->edges)
            if (e.ks == src && e.kd == dst) {
                if (w) *w = e.w;
                if (is_eps) *is_eps = e.eps > 0;
                if (ctx_legal) *ctx_legal = e.ctx_legal;
                if (profitable) *profitable = e.profitable;
                return;
            }
        fail(KF_ERR_BAD_ID, "no such edge");
    });
}

kf_status kf_plan_cut(const kf_plan *plan, int32_t i, int32_t *side, int32_t *n_side, int64_t *w_q,
                      int64_t *w_eps, int32_t *phases)
{
    return guard([&] {
        if (!plan) fail(KF_ERR_ARG, "null plan");
        if (i < 0 || i >= (int)plan->cuts.size()) fail(KF_ERR_ARG, "cut index out of range");
        const CutInfo &c = plan->cuts[i];
        if (n_side) *n_side = (int32_t)c.side.size();
        if (side)
            for (size_t j = 0; j < c.side.size(); j++) side[j] = c.side[j];
        if (w_q) *w_q = c.q;
        if (w_eps) *w_eps = c.eps;
        if (phases) *phases = c.phases;
    });
}

kf_status kf_plan_kernel_source(kf_pipeline *p, const kf_plan *plan, int32_t block, char *buf, size_t cap,
                                size_t *len)
{
    return guard([&] {
        if (!p || !plan || plan->pipe != p) fail(KF_ERR_ARG, "plan does not belong to pipeline");
        if (block < 0 || block >= (int)plan->blocks.size()) fail(KF_ERR_ARG, "block index out of range");
        std::string s = generate_block(p, plan->info[block], block);
        if (len) *len = s.size();
        if (buf && cap) {
            size_t n = std::min(cap - 1, s.size());
            std::memcpy(buf, s.data(), n);
            buf[n] = 0;
        }
    });
}

kf_status kf_prepare(kf_pipeline *p, const kf_plan *plan)
{
    return guard([&] {
        if (!p || !plan || plan->pipe != p) fail(KF_ERR_ARG, "plan does not belong to pipeline");
        prepare(p, const_cast<kf_plan *>(plan));
    });
}

kf_status kf_run(kf_pipeline *p, const kf_plan *plan, const void *const *d_inputs, int32_t n_in,
                 void *const *d_outputs, int32_t n_out, void *stream)
{
    return guard([&] {
        if (!p || !plan || plan->pipe != p) fail(KF_ERR_ARG, "plan does not belong to pipeline");
        run(p, const_cast<kf_plan *>(plan), d_inputs, n_in, d_outputs, n_out, stream, 0, p->H, 0, p->H);
    });
}

kf_status kf_run_batch(kf_pipeline *p, const kf_plan *plan, int32_t n_frames, const void *const *d_inputs,
                       int32_t n_in, void *const *d_outputs, int32_t n_out, void *stream)
{
    return guard([&] {
        if (!p || !plan || plan->pipe != p) fail(KF_ERR_ARG, "plan does not belong to pipeline");
        run_batch(p, const_cast<kf_plan *>(plan), n_frames, d_inputs, n_in, d_outputs, n_out, stream);
    });
}

kf_status kf_bounds_report(kf_pipeline *p, int64_t *violations, uint64_t *first_addr, int32_t *first_kind)
{
    return guard([&] {
        if (!p || !violations || !first_addr || !first_kind) fail(KF_ERR_ARG, "null argument");
        long long c = 0;
        unsigned long long ad = 0;
        int k = 0;
        bounds_report(p, &c, &ad, &k);
        *violations = c;
        *first_addr = ad;
        *first_kind = k;
    });
}

kf_status kf_run_host(kf_pipeline *p, const kf_plan *plan, const void *const *h_inputs, int32_t n_in,
                      void *const *h_outputs, int32_t n_out, void *stream)
{
    return guard([&] {
        if (!p || !plan || plan->pipe != p) fail(KF_ERR_ARG, "plan does not belong to pipeline");
        run_host(p, const_cast<kf_plan *>(plan), h_inputs, n_in, h_outputs, n_out, stream);
    });
}

kf_status kf_run_host_async(kf_pipeline *p, const kf_plan *plan, const void *const *h_inputs, int32_t n_in,
                            void *const *h_outputs, int32_t n_out, void *stream)
{
    return guard([&] {
        if (!p || !plan || plan->pipe != p) fail(KF_ERR_ARG, "plan does not belong to pipeline");
        run_host(p, const_cast<kf_plan *>(plan), h_inputs, n_in, h_outputs, n_out, stream, true);
    });
}

kf_status kf_run_band(kf_pipeline *p, const kf_plan *plan, int32_t row0, int32_t row1,
                      const void *const *d_in_band, int32_t in_row0, int32_t in_row1, void *const *d_out_band,
                      void *stream)
{
    return guard([&] {
        if (!p || !plan || plan->pipe != p) fail(KF_ERR_ARG, "plan does not belong to pipeline");
        if (row0 < 0 || row1 > p->H || row0 >= row1) fail(KF_ERR_ARG, "bad output row band");
        int need0 = std::max(0, row0 - plan->halo_rows), need1 = std::min(p->H, row1 + plan->halo_rows);
        if (in_row0 > need0 || in_row1 < need1)
            fail(KF_ERR_ARG, "input band must cover rows [" + std::to_string(need0) + ", " +
                                 std::to_string(need1) + ")");
        for (const auto &op : p->ops)
            if (op.kind == LOCAL && op.mode == KF_REPEAT)
                fail(KF_ERR_ARG, "REPEAT border mode is not supported in band mode (needs a ring exchange)");
        run(p, const_cast<kf_plan *>(plan), d_in_band, p->n_inputs, d_out_band, (int)p->outputs.size(), stream,
            row0, row1, in_row0, in_row1);
    });
}

const char *kf_last_error(void) { return g_last_error.c_str(); }
kf_status kf_set_option(kf_pipeline *p, const char *name, int64_t value)
{
    return guard([&] {
        if (!p) fail(KF_ERR_ARG, "null pipeline");
        set_option(p, name, (long long)value);
    });
}

kf_status kf_get_option(const kf_pipeline *p, const char *name, int64_t *value)
{
    return guard([&] {
        if (!p || !value) fail(KF_ERR_ARG, "null pipeline or value");
        *value = (int64_t)get_option(p, name);
    });
}

const char *kf_version(void)
{
#if defined(KF_TEST_HOOKS)
    return "kfuse 0.2 (sm_100a) TEST HOOKS BUILD -- negative controls, not the product library";
#elif defined(KF_BOUNDS)
    return "kfuse 0.2 (sm_100a) BOUNDS-CHECKING BUILD -- checked global accesses, not the product library";
#else
    return "kfuse 0.2 (sm_100a)";
#endif
}

}  // extern "C"
