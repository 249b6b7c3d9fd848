// codegen.cpp -- emits the CUDA C++ of ONE fused kernel per partition block.
//
// Fusion techniques of the paper, B200 re-design:
//   * point-based fusion: the producer body is inlined and the intermediate
//     lives in a register (Listing 1 :225-252);
//   * point-to-local / local-to-local: a producer consumed by an in-block local
//     kernel ("staged") is computed ONCE per position of the tile plus its halo
//     into shared memory; only the halo is recomputed by neighbouring tiles
//     (instead of the paper's per-tap recompute);
//   * border fusion + index exchange (§IV): staged values
//     are indexed by in-image coordinates; a local consumer remaps an
//     out-of-image tap with ITS OWN border mode before reading, so the fused
//     result equals "clamp+conv+clamp+conv" (Fig. 4c), never "pad once".
//     Tiles whose whole footprint is inside the image (the interior region,
//     PAPER.md:1089-1093) run a variant without any remapping.
//   * blocks whose local kernels all use REPEAT use a torus slot model: slot p
//     holds the value at p mod n, which is exact because wrap needs no exchange.
#include <algorithm>
#include <cstdio>
#include <functional>
#include <sstream>

#include "kf_internal.h"

namespace kf {

std::string kernel_name(int block) { return "kf_b" + std::to_string(block); }

namespace {

std::string fconst(double v)
{
    char buf[64];
    std::snprintf(buf, sizeof buf, "%af", (double)(float)v);
    std::string s(buf);
    if (s[0] == '-') return "(" + s + ")";
    return s;
}

struct Gen {
    const kf_pipeline *p;
    const BlockInfo &b;
    int block;
    int TW, TH;
    bool f32;
    std::map<int, int> slot;             // external image -> slot
    std::vector<std::vector<int>> groups;  // staged kernels grouped by halo, topological
    std::ostringstream o;
    int tmp = 0;

    Gen(const kf_pipeline *p_, const BlockInfo &b_, int block_, int tw, int th)
        : p(p_), b(b_), block(block_), TW(tw), TH(th), f32(p_->dtype == KF_F32) {}

    std::string KV() const { return f32 ? "float" : "I4"; }
    std::string var() { return "v" + std::to_string(tmp++); }
    bool in_block(int img) const
    {
        return img >= p->n_inputs && std::binary_search(b.kernels.begin(), b.kernels.end(), img - p->n_inputs);
    }
    std::string smem_name(int k) const { return "s_" + std::to_string(k); }
    int RW(int k) const { return TW + 2 * b.hx.at(k); }
    int RH(int k) const { return TH + 2 * b.hy.at(k); }

    // global load of an external image at in-image (or, torus: wrapped) coordinates
    std::string ext_load(int img, const std::string &Y, const std::string &X) const
    {
        int s = slot.at(img);
        return std::string(f32 ? "kf_ldf" : "kf_ldi") + "(a.img[" + std::to_string(s) + "], a.base[" +
               std::to_string(s) + "], W, " + Y + ", " + X + ")";
    }
    std::string smem_load(int k, const std::string &Y, const std::string &X) const
    {
        std::string idx = "((" + Y + ") - (oy - " + std::to_string(b.hy.at(k)) + ")) * " + std::to_string(RW(k)) +
                          " + ((" + X + ") - (ox - " + std::to_string(b.hx.at(k)) + "))";
        return f32 ? smem_name(k) + "[" + idx + "]" : "kf_unpack(" + smem_name(k) + "[" + idx + "])";
    }

    // Emits code computing kernel/image `img` at position (y, x); returns the variable.
    // memo: values already computed at this position; group: staged kernels computed
    // in the current loop (read from memo, not smem).
    std::string eval(int img, std::map<int, std::string> &memo, const std::set<int> &group, bool border,
                     const std::string &ind)
    {
        auto it = memo.find(img);
        if (it != memo.end()) return it->second;
        std::string v = var();
        if (!in_block(img)) {
            std::string Y = "y", X = "x";
            if (border && b.torus) { Y = "kf_wrap(y, H)"; X = "kf_wrap(x, W)"; }
            o << ind << "const " << KV() << " " << v << " = " << ext_load(img, Y, X) << ";\n";
            memo[img] = v;
            return v;
        }
        int k = img - p->n_inputs;
        if (b.staged.count(k) && !group.count(k)) {
            o << ind << "const " << KV() << " " << v << " = " << smem_load(k, "y", "x") << ";\n";
            memo[img] = v;
            return v;
        }
        const Op &op = p->ops[k];
        std::vector<std::string> loads;
        std::string acc;
        if (op.kind == POINT) {
            for (int in : op.inputs) loads.push_back(eval(in, memo, group, border, ind));
        } else {
            acc = var();
            o << ind << KV() << " " << acc << " = " << (f32 ? "0.0f" : "kf_i4(0)") << ";\n";
            const int in = op.inputs[0];
            const bool staged_in = in_block(in);
            const int cy = op.mh / 2, cx = op.mw / 2;
            for (int j = 0; j < op.mh; j++)
                for (int i = 0; i < op.mw; i++) {
                    double m = op.mask[(size_t)j * op.mw + i];
                    if (m == 0.0) continue;
                    const int dy = j - cy, dx = i - cx;
                    std::string Y = "y + (" + std::to_string(dy) + ")", X = "x + (" + std::to_string(dx) + ")";
                    std::string val;
                    if (!border || (b.torus && staged_in)) {
                        val = staged_in ? smem_load(in - p->n_inputs, Y, X) : ext_load(in, Y, X);
                    } else if (b.torus) {
                        val = ext_load(in, "kf_wrap(" + Y + ", H)", "kf_wrap(" + X + ", W)");
                    } else {
                        // index exchange: remap with THIS (consumer) kernel's border mode
                        std::string mode = std::to_string(op.mode);
                        std::string yy = var(), xx = var();
                        o << ind << "const int " << yy << " = kf_border<" << mode << ">(" << Y << ", H);\n";
                        o << ind << "const int " << xx << " = kf_border<" << mode << ">(" << X << ", W);\n";
                        std::string rd = staged_in ? smem_load(in - p->n_inputs, yy, xx) : ext_load(in, yy, xx);
                        if (op.mode == KF_CONSTANT) {
                            std::string c = f32 ? fconst(op.constant) : "kf_i4(" + std::to_string((int)op.constant) + ")";
                            val = "((" + yy + " < 0 || " + xx + " < 0) ? " + c + " : " + rd + ")";
                        } else {
                            val = rd;
                        }
                    }
                    std::string mc = f32 ? fconst(m) : std::to_string((long long)m);
                    o << ind << acc << " = kf_mac(" << acc << ", " << mc << ", " << val << ");\n";
                }
            loads.push_back(acc);
        }
        std::string r = program(op, k, loads, ind, op.kind == LOCAL && op.prog.empty() ? acc : "");
        if (!f32) {
            o << ind << "const I4 " << v << " = kf_satu8(" << r << ");\n";   // narrowing at the kernel boundary
        } else {
            o << ind << "const float " << v << " = " << r << ";\n";
        }
        memo[img] = v;
        return v;
    }

    // postfix op-IR -> straight-line code; returns the result expression
    std::string program(const Op &op, int k, const std::vector<std::string> &loads, const std::string &ind,
                        const std::string &identity)
    {
        if (!identity.empty()) return identity;
        std::vector<std::string> st;
        auto pop = [&] { std::string s = st.back(); st.pop_back(); return s; };
        for (const Instr &in : op.prog) {
            std::string t = var(), e;
            switch (in.op) {
            case KF_OP_LOAD: st.push_back(loads[op.kind == LOCAL ? 0 : in.arg]); continue;
            case KF_OP_CONST:
                e = f32 ? fconst(in.imm) : "kf_i4(" + std::to_string((long long)(int64_t)in.imm) + ")";
                break;
            case KF_OP_ADD: case KF_OP_SUB: case KF_OP_MUL: case KF_OP_DIV: case KF_OP_MIN: case KF_OP_MAX:
            case KF_OP_POW: {
                std::string bb = pop(), aa = pop();
                const char *fn = in.op == KF_OP_ADD ? "kf_add" : in.op == KF_OP_SUB ? "kf_sub"
                               : in.op == KF_OP_MUL ? "kf_mul" : in.op == KF_OP_DIV ? "kf_div"
                               : in.op == KF_OP_MIN ? "kf_min" : in.op == KF_OP_MAX ? "kf_max" : "kf_pow";
                e = std::string(fn) + "(" + aa + ", " + bb + ")";
                break;
            }
            case KF_OP_ABS: e = "kf_abs(" + pop() + ")"; break;
            case KF_OP_NEG: e = "kf_neg(" + pop() + ")"; break;
            case KF_OP_SQRT: e = "kf_sqrt(" + pop() + ")"; break;
            case KF_OP_EXP: e = "kf_exp(" + pop() + ")"; break;
            case KF_OP_LOG: e = "kf_log(" + pop() + ")"; break;
            case KF_OP_SHR: e = "kf_shr<" + std::to_string(in.arg) + ">(" + pop() + ")"; break;
            case KF_OP_SHL: e = "kf_shl<" + std::to_string(in.arg) + ">(" + pop() + ")"; break;
            case KF_OP_SAT_U8: e = "kf_satu8(" + pop() + ")"; break;
            case KF_OP_CLAMP: {
                std::string hi = pop(), lo = pop(), x = pop();
                e = "kf_clamp(" + x + ", " + lo + ", " + hi + ")";
                break;
            }
            case KF_OP_SELECT_GT: {
                std::string d = pop(), c = pop(), bb = pop(), aa = pop();
                e = "kf_sel_gt(" + aa + ", " + bb + ", " + c + ", " + d + ")";
                break;
            }
            case KF_OP_LUT:
                e = "kf_lut(" + pop() + ", kf_lut_" + std::to_string(block) + "_" + std::to_string(k) + ", " +
                    std::to_string(op.lut.size()) + ")";
                break;
            default: fail(KF_ERR_PROGRAM, "codegen: bad opcode");
            }
            o << ind << "const " << KV() << " " << t << " = " << e << ";\n";
            st.push_back(t);
        }
        return st.back();
    }

    void body(bool border)
    {
        const std::string ind = "        ";
        o << "template <> __device__ __forceinline__ void " << kernel_name(block) << "_body<" << (border ? "true" : "false")
          << ">(const KfArgs &a, const int ox, const int oy";
        for (auto &g : groups)
            for (int k : g) o << ", " << (f32 ? "float" : "unsigned") << " *__restrict__ " << smem_name(k);
        o << ")\n{\n    const int W = a.W, H = a.H;\n    (void)H;\n";
        for (auto &g : groups) {
            const int k0 = g[0];
            const int hx = b.hx.at(k0), hy = b.hy.at(k0);
            const int rw = RW(k0), rh = RH(k0);
            std::set<int> gs(g.begin(), g.end());
            o << "    // stage: kernels";
            for (int k : g) o << " " << k;
            o << " over the tile + halo (" << hx << "," << hy << ")\n";
            o << "    for (int i = threadIdx.x; i < " << rw * rh << "; i += blockDim.x) {\n";
            o << "        const int y = oy - " << hy << " + i / " << rw << ", x = ox - " << hx << " + i % " << rw << ";\n";
            if (border && !b.torus)
                o << "        if (y < 0 || y >= H || x < 0 || x >= W || y < a.r0 - " << hy << " || y >= a.r1 + " << hy
                  << ") continue;\n";
            std::map<int, std::string> memo;
            for (int k : g) {
                std::string v = eval(p->n_inputs + k, memo, gs, border, ind);
                o << ind << smem_name(k) << "[i] = " << (f32 ? v : "kf_pack(" + v + ")") << ";\n";
            }
            o << "    }\n    __syncthreads();\n";
        }
        // sink
        o << "    for (int i = threadIdx.x; i < " << TW * TH << "; i += blockDim.x) {\n";
        o << "        const int y = oy + i / " << TW << ", x = ox + i % " << TW << ";\n";
        o << "        if (y >= a.r1 || x >= W) continue;\n";
        std::map<int, std::string> memo;
        std::string v = eval(p->n_inputs + b.sink, memo, {}, border, ind);
        o << ind << (f32 ? "kf_stf" : "kf_sti") << "(a.out, a.out_base, W, y, x, " << v << ");\n";
        o << "    }\n}\n\n";
    }

    std::string run()
    {
        for (size_t i = 0; i < b.ext.size(); i++) slot[b.ext[i]] = (int)i;
        if (b.ext.size() > 16) fail(KF_ERR_ARG, "block reads more than 16 external images");
        // staged kernels grouped by (hx, hy), descending hx+hy (topological)
        std::map<std::pair<int, int>, std::vector<int>> byhalo;
        for (int k : b.staged) byhalo[{b.hx.at(k), b.hy.at(k)}].push_back(k);
        std::vector<std::pair<int, int>> keys;
        for (auto &kv : byhalo) keys.push_back(kv.first);
        std::stable_sort(keys.begin(), keys.end(), [](auto &l, auto &r) {
            return l.first + l.second > r.first + r.second;
        });
        for (auto &kk : keys) groups.push_back(byhalo[kk]);

        o << "// generated by libkfuse codegen: block " << block << " kernels {";
        for (int k : b.kernels) o << " " << k;
        o << " } sink " << b.sink << (b.torus ? " (torus)" : "") << "\n";
        o << "#include \"kf_device.cuh\"\n\n";
        for (int k : b.kernels)
            if (!p->ops[k].lut.empty()) {
                o << "__device__ const int kf_lut_" << block << "_" << k << "[" << p->ops[k].lut.size() << "] = {";
                for (size_t i = 0; i < p->ops[k].lut.size(); i++) o << (i ? "," : "") << p->ops[k].lut[i];
                o << "};\n";
            }
        o << "template <bool BORDER> __device__ void " << kernel_name(block) << "_body(const KfArgs &a, int ox, int oy";
        for (auto &g : groups)
            for (size_t j = 0; j < g.size(); j++) o << ", " << (f32 ? "float" : "unsigned") << " *__restrict__";
        o << ");\n";
        body(false);
        body(true);
        int smem = 0;
        for (auto &g : groups)
            for (int k : g) smem += RW(k) * RH(k) * 4;
        if (smem > 48 * 1024) fail(KF_ERR_ARG, "fused block needs more than 48 KB of shared memory");
        o << "extern \"C\" __global__ void __launch_bounds__(256) " << kernel_name(block)
          << "(const __grid_constant__ KfArgs a)\n{\n";
        for (auto &g : groups)
            for (int k : g)
                o << "    __shared__ " << (f32 ? "float " : "unsigned ") << smem_name(k) << "[" << RW(k) * RH(k)
                  << "];\n";
        o << "    const int ox = blockIdx.x * " << TW << ";\n";
        o << "    const int oy = a.r0 + blockIdx.y * " << TH << ";\n";
        o << "    const bool interior = ox >= " << b.Rx << " && ox + " << TW + b.Rx << " <= a.W && oy >= " << b.Ry
          << " && oy + " << TH + b.Ry << " <= a.H && oy + " << TH << " <= a.r1;\n";
        std::string args = "a, ox, oy";
        for (auto &g : groups)
            for (int k : g) args += ", " + smem_name(k);
        o << "    if (interior) " << kernel_name(block) << "_body<false>(" << args << ");\n";
        o << "    else " << kernel_name(block) << "_body<true>(" << args << ");\n}\n";
        return o.str();
    }
};

}  // namespace

std::string generate_block(const kf_pipeline *p, const BlockInfo &b, int block, int tile_w, int tile_h)
{
    Gen g(p, b, block, tile_w > 0 ? tile_w : 32, tile_h > 0 ? tile_h : 8);
    return g.run();
}

}  // namespace kf
