// codegen.cpp -- emits the CUDA C++ of ONE fused kernel per partition block.
//
// Fusion techniques of the paper, B200 re-design:
//   * point-based fusion: the producer body is inlined and the intermediate
//     lives in a register (Listing 1 :225-252);
//   * point-to-local / local-to-local: the producer is computed once per pixel
//     of the consumer's footprint and kept on chip; only the halo is
//     recomputed by neighbouring tiles (instead of the paper's per-tap
//     recompute);
//   * the image is split into the paper's interior and border regions
//     (§IV-B):
//       - INTERIOR (fast path): every output pixel whose whole input footprint
//         is inside the image.  One warp streams a 4-pixel-wide column chunk
//         down a strip of rows: each kernel of the block is evaluated once per
//         (row, pixel) in registers, vertical taps read per-image register
//         ring buffers of past rows, horizontal taps come from the lane's own
//         registers or warp shuffles, separable (rank-1) masks run
//         vertical-then-horizontal.  No border logic at all.
//       - BORDER FRAME (slow path): 2-D tiles whose producers are staged in
//         shared memory over tile + halo.  Border fusion + index exchange
//         (PAPER.md:1061-1133): staged values are indexed by in-image
//         coordinates; a local consumer remaps an out-of-image tap with ITS OWN
//         border mode before reading, so the fused result equals
//         "clamp+conv+clamp+conv" (Fig. 4c), never "pad once".
//   * blocks whose local kernels all use REPEAT use a torus slot model in the
//     frame: slot p holds the value at p mod n (wrap needs no exchange).
#include <algorithm>
#include <climits>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <numeric>
#include <sstream>

#include "kf_internal.h"

namespace kf {

// Entry-point name: block index, sink kernel and block size, so that launch
// lists of different plans of one pipeline tell their kernels apart.
std::string kernel_name(const BlockInfo &b, int block)
{
    return "kf_b" + std::to_string(block) + "_k" + std::to_string(b.sink) + "n" + std::to_string(b.kernels.size());
}

namespace {
std::string kernel_name(int block) { return "kf_b" + std::to_string(block); }   // prefix of the device helpers
}  // namespace

namespace {

std::string fconst(double v)
{
    char buf[64];
    std::snprintf(buf, sizeof buf, "%af", (double)(float)v);
    std::string s(buf);
    if (s[0] == '-') return "(" + s + ")";
    return s;
}

std::string iconst(long long v)
{
    if (v < 0) return "(" + std::to_string(v) + ")";
    return std::to_string(v);
}

// postfix op-IR -> straight-line code, shared by both paths.  `loads` are the
// values of LOAD k (a local op's post program: LOAD 0 = the accumulator).
struct ProgEmitter {
    bool f32;
    int block;
    int *tmp;
    std::string KV() const { return f32 ? "float" : "I4"; }
    std::string var() { return "v" + std::to_string((*tmp)++); }

    std::string emit(std::ostringstream &o, const Op &op, int k, const std::vector<std::string> &loads,
                     const std::string &ind)
    {
        std::vector<std::string> st;
        auto pop = [&] { std::string s = st.back(); st.pop_back(); return s; };
        for (const Instr &in : op.prog) {
            std::string t = var(), e;
            switch (in.op) {
            case KF_OP_LOAD: st.push_back(loads[op.kind == LOCAL ? 0 : in.arg]); continue;
            case KF_OP_CONST:
                e = f32 ? fconst(in.imm) : "kf_i4(" + iconst((long long)(int64_t)in.imm) + ")";
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

    // Packed f32x2 form of a float program (two adjacent pixels per value).
    // The postfix program is rebuilt as a tree (each value is consumed once)
    // so that a MUL feeding an ADD/SUB becomes one FFMA2 -- the contraction
    // nvcc performs on scalar code but not across the _rn pair intrinsics.
    struct Node {
        int op, arg;
        double imm;
        std::vector<int> ch;
    };
    std::string emit2(std::ostringstream &o, const Op &op, const std::vector<std::string> &loads,
                      const std::string &ind)
    {
        std::vector<Node> nodes;
        std::vector<int> st;
        for (const Instr &in : op.prog) {
            Node n{in.op, in.arg, in.imm, {}};
            int arity = 0;
            switch (in.op) {
            case KF_OP_LOAD: case KF_OP_CONST: arity = 0; break;
            case KF_OP_ABS: case KF_OP_NEG: case KF_OP_SQRT: case KF_OP_EXP: case KF_OP_LOG: arity = 1; break;
            case KF_OP_CLAMP: arity = 3; break;
            case KF_OP_SELECT_GT: arity = 4; break;
            case KF_OP_SHR: case KF_OP_SHL: case KF_OP_SAT_U8: case KF_OP_LUT:
                fail(KF_ERR_PROGRAM, "codegen: integer opcode in a float program");
            default: arity = 2;
            }
            n.ch.assign(st.end() - arity, st.end());
            st.resize(st.size() - arity);
            nodes.push_back(n);
            st.push_back((int)nodes.size() - 1);
        }
        std::function<std::string(int)> ev = [&](int i) -> std::string {
            const Node &n = nodes[i];
            auto is = [&](int c, int opc) { return nodes[c].op == opc; };
            auto cst = [&](int c) { return fconst(nodes[c].imm); };
            std::string e;
            if (n.op == KF_OP_LOAD) return loads[op.kind == LOCAL ? 0 : n.arg];
            if (n.op == KF_OP_CONST) return "kf2(" + fconst(n.imm) + ")";
            if (n.op == KF_OP_ADD || n.op == KF_OP_SUB) {
                const int a = n.ch[0], b = n.ch[1];
                const bool add = n.op == KF_OP_ADD;
                if (is(b, KF_OP_MUL)) {
                    std::string x = ev(a), m0 = ev(nodes[b].ch[0]), m1 = ev(nodes[b].ch[1]);
                    e = std::string(add ? "kf2_fma(" : "kf2_nfma(") + m0 + ", " + m1 + ", " + x + ")";
                } else if (is(a, KF_OP_MUL)) {
                    std::string m0 = ev(nodes[a].ch[0]), m1 = ev(nodes[a].ch[1]), y = ev(b);
                    e = std::string(add ? "kf2_fma(" : "kf2_fms(") + m0 + ", " + m1 + ", " + y + ")";
                } else {
                    e = std::string(add ? "kf2_add(" : "kf2_sub(") + ev(a) + ", " + ev(b) + ")";
                }
            } else if (n.op == KF_OP_MUL && is(n.ch[1], KF_OP_CONST)) {
                e = "kf2_mul1(" + cst(n.ch[1]) + ", " + ev(n.ch[0]) + ")";
            } else if (n.op == KF_OP_MUL && is(n.ch[0], KF_OP_CONST)) {
                e = "kf2_mul1(" + cst(n.ch[0]) + ", " + ev(n.ch[1]) + ")";
            } else {
                static const std::map<int, const char *> fn = {
                    {KF_OP_MUL, "kf2_mul"}, {KF_OP_DIV, "kf2_div"}, {KF_OP_MIN, "kf2_min"}, {KF_OP_MAX, "kf2_max"},
                    {KF_OP_POW, "kf2_pow"}, {KF_OP_ABS, "kf2_abs"}, {KF_OP_NEG, "kf2_neg"}, {KF_OP_SQRT, "kf2_sqrt"},
                    {KF_OP_EXP, "kf2_exp"}, {KF_OP_LOG, "kf2_log"}, {KF_OP_CLAMP, "kf2_clamp"},
                    {KF_OP_SELECT_GT, "kf2_sel_gt"}};
                auto it = fn.find(n.op);
                if (it == fn.end()) fail(KF_ERR_PROGRAM, "codegen: bad opcode");
                e = std::string(it->second) + "(";
                for (size_t c = 0; c < n.ch.size(); c++) e += (c ? ", " : "") + ev(n.ch[c]);
                e += ")";
            }
            std::string t = var();
            o << ind << "const F2 " << t << " = " << e << ";\n";
            return t;
        };
        return ev(st.back());
    }

    // Deferred power-of-two scaling: a packed value may be held
    // as `stored` with true value = stored x 2^e, e a compile-time exponent.
    // Scaling by a power of two is exact in binary floating point (away from
    // overflow and subnormals), so (a 2^e)(b 2^f) = ab 2^(e+f) and
    // a 2^e + b 2^e = (a + b) 2^e hold bit for bit: a normalised mask's 1/16
    // is applied once at the end of the chain instead of at every stage.
    struct Val {
        std::string x;      // F2 expression (empty for a constant)
        int e = 0;
        bool isc = false;
        double c = 0.0;
    };
    static std::string lit2(double c, int e) { return "kf2(" + fconst(std::ldexp((double)(float)c, -e)) + ")"; }
    static bool pow2(double c, int &k)
    {
        if (c <= 0.0) return false;
        int ex = 0;
        const double m = std::frexp(c, &ex);
        if (m != 0.5) return false;
        k = ex - 1;
        return k >= -60 && k <= 60;
    }
    std::string tmp2(std::ostringstream &o, const std::string &e, const std::string &ind)
    {
        std::string t = var();
        o << ind << "const F2 " << t << " = " << e << ";\n";
        return t;
    }
    // v as an F2 expression at exponent e
    std::string at(std::ostringstream &o, const Val &v, int e, const std::string &ind)
    {
        if (v.isc) return lit2(v.c, e);
        if (v.e == e) return v.x;
        return tmp2(o, "kf2_mul1(" + fconst(std::ldexp(1.0, v.e - e)) + ", " + v.x + ")", ind);
    }
    Val emit2e(std::ostringstream &o, const Op &op, const std::vector<Val> &loads, const std::string &ind)
    {
        std::vector<Node> nodes;
        std::vector<int> st;
        for (const Instr &in : op.prog) {
            Node n{in.op, in.arg, in.imm, {}};
            int arity = 0;
            switch (in.op) {
            case KF_OP_LOAD: case KF_OP_CONST: arity = 0; break;
            case KF_OP_ABS: case KF_OP_NEG: case KF_OP_SQRT: case KF_OP_EXP: case KF_OP_LOG: arity = 1; break;
            case KF_OP_CLAMP: arity = 3; break;
            case KF_OP_SELECT_GT: arity = 4; break;
            case KF_OP_SHR: case KF_OP_SHL: case KF_OP_SAT_U8: case KF_OP_LUT:
                fail(KF_ERR_PROGRAM, "codegen: integer opcode in a float program");
            default: arity = 2;
            }
            n.ch.assign(st.end() - arity, st.end());
            st.resize(st.size() - arity);
            nodes.push_back(n);
            st.push_back((int)nodes.size() - 1);
        }
        auto mk = [&](const std::string &e, int ex) { Val v; v.x = tmp2(o, e, ind); v.e = ex; return v; };
        std::function<Val(int)> ev = [&](int i) -> Val {
            const Node &n = nodes[i];
            if (n.op == KF_OP_LOAD) return loads[op.kind == LOCAL ? 0 : n.arg];
            if (n.op == KF_OP_CONST) { Val v; v.isc = true; v.c = (double)(float)n.imm; return v; }
            if (n.op == KF_OP_ADD || n.op == KF_OP_SUB) {
                const bool add = n.op == KF_OP_ADD;
                const int a = n.ch[0], b = n.ch[1];
                // a MUL child contracts into one FFMA2 (as emit2)
                const int mi = nodes[b].op == KF_OP_MUL ? b : nodes[a].op == KF_OP_MUL ? a : -1;
                if (mi >= 0) {
                    Val m0 = ev(nodes[mi].ch[0]), m1 = ev(nodes[mi].ch[1]);
                    Val x = ev(mi == b ? a : b);
                    if (!(m0.isc && m1.isc)) {
                        int ep;
                        std::string f0, f1;
                        if (m0.isc) { ep = m1.e; f0 = lit2(m0.c, 0); f1 = m1.x; }
                        else if (m1.isc) { ep = m0.e; f0 = m0.x; f1 = lit2(m1.c, 0); }
                        else { ep = m0.e + m1.e; f0 = m0.x; f1 = m1.x; }
                        if (x.isc || !m0.isc || !m1.isc) {
                            const std::string xs = at(o, x, ep, ind);
                            const char *fn = mi == b ? (add ? "kf2_fma(" : "kf2_nfma(") : (add ? "kf2_fma(" : "kf2_fms(");
                            return mk(std::string(fn) + f0 + ", " + f1 + ", " + xs + ")", ep);
                        }
                    }
                    // fall through: both multiplicands constant
                }
                Val va = ev(a), vb = ev(b);
                if (va.isc && vb.isc) {
                    Val v;
                    v.x = tmp2(o, std::string(add ? "kf2_add(" : "kf2_sub(") + lit2(va.c, 0) + ", " + lit2(vb.c, 0) + ")", ind);
                    return v;
                }
                const int e = va.isc ? vb.e : va.e;
                return mk(std::string(add ? "kf2_add(" : "kf2_sub(") + at(o, va, e, ind) + ", " + at(o, vb, e, ind) + ")", e);
            }
            if (n.op == KF_OP_MUL) {
                Val va = ev(n.ch[0]), vb = ev(n.ch[1]);
                int k = 0;
                if (va.isc && vb.isc) return mk("kf2_mul(" + lit2(va.c, 0) + ", " + lit2(vb.c, 0) + ")", 0);
                if (va.isc || vb.isc) {
                    const Val &c = va.isc ? va : vb, &x = va.isc ? vb : va;
                    if (pow2(c.c, k)) { Val r = x; r.e = x.e + k; return r; }   // free: the exponent moves
                    return mk("kf2_mul1(" + fconst(c.c) + ", " + x.x + ")", x.e);
                }
                return mk("kf2_mul(" + va.x + ", " + vb.x + ")", va.e + vb.e);
            }
            if (n.op == KF_OP_DIV) {
                Val va = ev(n.ch[0]), vb = ev(n.ch[1]);
                int k = 0;
                if (!va.isc && vb.isc && pow2(vb.c, k)) { Val r = va; r.e = va.e - k; return r; }
                if (va.isc && vb.isc) return mk("kf2_div(" + lit2(va.c, 0) + ", " + lit2(vb.c, 0) + ")", 0);
                if (vb.isc) return mk("kf2_div(" + va.x + ", " + lit2(vb.c, 0) + ")", va.e);
                if (va.isc) return mk("kf2_div(" + lit2(va.c, vb.e) + ", " + vb.x + ")", 0);   // c / (s 2^e) = (c 2^-e / s) 2^0
                return mk("kf2_div(" + va.x + ", " + vb.x + ")", va.e - vb.e);
            }
            if (n.op == KF_OP_MIN || n.op == KF_OP_MAX) {
                Val va = ev(n.ch[0]), vb = ev(n.ch[1]);
                const int e = va.isc ? vb.e : va.e;
                const char *fn = n.op == KF_OP_MIN ? "kf2_min(" : "kf2_max(";
                return mk(std::string(fn) + at(o, va, e, ind) + ", " + at(o, vb, e, ind) + ")", va.isc && vb.isc ? 0 : e);
            }
            if (n.op == KF_OP_ABS || n.op == KF_OP_NEG) {
                Val va = ev(n.ch[0]);
                const char *fn = n.op == KF_OP_ABS ? "kf2_abs(" : "kf2_neg(";
                return mk(std::string(fn) + at(o, va, va.isc ? 0 : va.e, ind) + ")", va.isc ? 0 : va.e);
            }
            if (n.op == KF_OP_SQRT) {
                Val va = ev(n.ch[0]);
                const int e = va.isc ? 0 : (va.e % 2 == 0 ? va.e : va.e - 1);
                return mk("kf2_sqrt(" + at(o, va, e, ind) + ")", e / 2);
            }
            if (n.op == KF_OP_CLAMP) {
                Val vx = ev(n.ch[0]), vl = ev(n.ch[1]), vh = ev(n.ch[2]);
                const int e = vx.isc ? 0 : vx.e;
                return mk("kf2_clamp(" + at(o, vx, e, ind) + ", " + at(o, vl, e, ind) + ", " + at(o, vh, e, ind) + ")", e);
            }
            if (n.op == KF_OP_SELECT_GT) {
                Val va = ev(n.ch[0]), vb = ev(n.ch[1]), vc = ev(n.ch[2]), vd = ev(n.ch[3]);
                const int ec = va.isc ? vb.e : va.e, er = vc.isc ? vd.e : vc.e;
                return mk("kf2_sel_gt(" + at(o, va, ec, ind) + ", " + at(o, vb, ec, ind) + ", " + at(o, vc, er, ind) + ", " +
                              at(o, vd, er, ind) + ")", vc.isc && vd.isc ? 0 : er);
            }
            // EXP, LOG, POW: on true values
            static const std::map<int, const char *> fn = {{KF_OP_EXP, "kf2_exp("}, {KF_OP_LOG, "kf2_log("}, {KF_OP_POW, "kf2_pow("}};
            auto it = fn.find(n.op);
            if (it == fn.end()) fail(KF_ERR_PROGRAM, "codegen: bad opcode");
            std::string e = it->second;
            for (size_t c = 0; c < n.ch.size(); c++) e += (c ? ", " : "") + at(o, ev(n.ch[c]), 0, ind);
            return mk(e + ")", 0);
        };
        Val r = ev(st.back());
        if (r.isc) { Val v; v.x = tmp2(o, lit2(r.c, 0), ind); return v; }
        return r;
    }
};

// ======================================================================= SWAR
// u8x4 pipelines in the interior path: two channels per 32-bit register, one
// per 16-bit lane ("SWAR").  A pixel is two registers, lo =
// (c0, c1) and hi = (c2, c3).  A value of the method (an integer per channel,
// int32 semantics, R-16) is held with a compile-time bias B >= 0 in every lane
// (lane = v + B) and a compile-time interval [vlo, vhi] of v, the same for all
// channels.  Interval analysis at code-generation time decides whether a
// kernel fits: every materialised lane must stay in [0, 65535].
//   * linear forms sum c_i x_i + k (ADD/SUB/NEG/SHL/MUL-by-constant and every
//     mask accumulation) are evaluated with plain 32-bit integer arithmetic on
//     both registers: arithmetic mod 2^32 is a ring, so whenever the final
//     lanes are in range the packed result is exact, whatever the order or the
//     intermediate wrap-arounds (IADD3 / LEA / IMAD serve two channels each);
//   * SHR n (arithmetic, floor): bias aligned to 2^n, then (x >> n) & mask;
//   * MIN / MAX / CLAMP / SAT: VIMNMX.U16x2 on equal biases;
//   * everything else (DIV, ABS, SELECT, LUT, variable products, overflowing
//     ranges) makes the kernel fall back to per-channel int32 (I4) code.
// Kernel outputs are saturated to [0, 255] (R-16), normalised to bias 0 and
// packed to uchar4 with one PRMT; ring rows are unpacked with two.
struct SwReg {
    std::string lo, hi;
    long long B = 0, vlo = 0, vhi = 255;
};
struct SwLin {
    std::vector<std::pair<long long, SwReg>> t;
    long long k = 0;
};
struct SwFail {};

// SWAR table gathers of the interior path read a shared-memory copy of the
// table (option lut_smem; filled once per CTA at kernel entry): a 32-bit LDS
// address instead of 64-bit global address arithmetic per gather.  Decided
// per block by stream_info (si.lut_smem), which keeps the CTA's static shared
// memory -- rings or frame tiles plus the tables -- within 48 KB.
static bool lut_in_smem(const StreamInfo &si, const Op &op)
{
    return si.lut_smem && !op.lut.empty() && op.lut.size() <= 1024;
}

static long long floordiv(long long a, long long b) { return a >= 0 ? a / b : -((-a + b - 1) / b); }

struct SwEmitter {
    std::ostringstream *o = nullptr;   // null: interval-only dry run (feasibility)
    int *tmp = nullptr;
    std::string ind;
    std::string lut_sym;               // table of the kernel being emitted (LUT ops)
    bool lut_shared = false;           // lut_sym is the CTA's shared-memory copy (plain indexing)
    std::string var() { return "w" + std::to_string((*tmp)++); }
    static std::string lit(long long v)   // v * 0x10001 as an unsigned literal (mod 2^32)
    {
        const unsigned long long u = (unsigned long long)(v * 65537LL) & 0xffffffffULL;
        char b[32];
        std::snprintf(b, sizeof b, "0x%llxu", u);
        return b;
    }
    static SwLin of(const SwReg &r) { return SwLin{{{1, r}}, 0}; }
    static SwLin cst(long long k) { return SwLin{{}, k}; }
    static SwLin add(SwLin a, const SwLin &b, long long sb = 1)
    {
        for (auto &t : b.t) a.t.push_back({sb * t.first, t.second});
        a.k += sb * b.k;
        return a;
    }
    static SwLin scale(SwLin a, long long c)
    {
        for (auto &t : a.t) t.first *= c;
        a.k *= c;
        return a;
    }
    static void interval(const SwLin &l, long long &lo, long long &hi)
    {
        lo = hi = l.k;
        for (auto &t : l.t) {
            const long long a = t.first * t.second.vlo, b = t.first * t.second.vhi;
            lo += std::min(a, b);
            hi += std::max(a, b);
        }
    }
    // materialise with a bias >= minB, multiple of `align`
    SwReg mat(const SwLin &l, long long align = 1, long long minB = 0)
    {
        long long lo, hi;
        interval(l, lo, hi);
        long long B = std::max(std::max(0LL, -lo), minB);
        B = (B + align - 1) / align * align;
        if (hi + B > 65535 || lo + B < 0) throw SwFail{};
        if (l.t.size() == 1 && l.t[0].first == 1 && l.k == 0 && l.t[0].second.B == B) return l.t[0].second;
        long long K = B + l.k;
        for (auto &t : l.t) {
            if (std::llabs(t.first) > 65535) throw SwFail{};
            K -= t.first * t.second.B;
        }
        SwReg r;
        r.B = B;
        r.vlo = lo;
        r.vhi = hi;
        if (o) {
            r.lo = var();
            r.hi = var();
            for (int h = 0; h < 2; h++) {
                std::string e;
                for (auto &t : l.t) {
                    const std::string &x = h ? t.second.hi : t.second.lo;
                    const long long c = t.first;
                    if (c == 0) continue;
                    if (c == 1) e += (e.empty() ? "" : " + ") + x;
                    else if (c == -1) e += (e.empty() ? "0u - " : " - ") + x;
                    else if (c > 0) e += (e.empty() ? "" : " + ") + std::to_string(c) + "u * " + x;
                    else e += (e.empty() ? "0u - " : " - ") + std::to_string(-c) + "u * " + x;
                }
                e += (e.empty() ? "" : " + ") + lit(K);
                *o << ind << "const unsigned " << (h ? r.hi : r.lo) << " = " << e << ";\n";
            }
        }
        return r;
    }
    SwReg shr(const SwReg &x, int n)
    {
        if (n <= 0) return x;
        if (n >= 16) throw SwFail{};
        SwReg a = mat(of(x), 1LL << n);
        SwReg r;
        r.B = a.B >> n;
        r.vlo = floordiv(a.vlo, 1LL << n);
        r.vhi = floordiv(a.vhi, 1LL << n);
        if (o) {
            r.lo = var();
            r.hi = var();
            if (n == 8) {   // each lane's high byte moved down: one PRMT instead of SHF + LOP3 (both ALU pipe)
                *o << ind << "const unsigned " << r.lo << " = __byte_perm(" << a.lo << ", 0u, 0x4341);\n";
                *o << ind << "const unsigned " << r.hi << " = __byte_perm(" << a.hi << ", 0u, 0x4341);\n";
            } else {
                const std::string m = lit(0xffff >> n);
                *o << ind << "const unsigned " << r.lo << " = (" << a.lo << " >> " << n << ") & " << m << ";\n";
                *o << ind << "const unsigned " << r.hi << " = (" << a.hi << " >> " << n << ") & " << m << ";\n";
            }
        }
        return r;
    }
    SwReg minmax(const SwReg &a0, const SwReg &b0, bool mx)
    {
        const long long B = std::max(a0.B, b0.B);
        SwReg a = mat(of(a0), 1, B), b = mat(of(b0), 1, B);
        if (a.B != b.B) throw SwFail{};
        SwReg r;
        r.B = a.B;
        r.vlo = mx ? std::max(a.vlo, b.vlo) : std::min(a.vlo, b.vlo);
        r.vhi = mx ? std::max(a.vhi, b.vhi) : std::min(a.vhi, b.vhi);
        if (o) {
            r.lo = var();
            r.hi = var();
            const char *fn = mx ? "__vmaxu2" : "__vminu2";
            *o << ind << "const unsigned " << r.lo << " = " << fn << "(" << a.lo << ", " << b.lo << ");\n";
            *o << ind << "const unsigned " << r.hi << " = " << fn << "(" << a.hi << ", " << b.hi << ");\n";
        }
        return r;
    }
    SwReg clamp(const SwReg &x0, long long lo, long long hi)
    {
        SwReg x = x0;
        if (lo > hi) throw SwFail{};
        if (x.vhi <= lo) return mat(cst(lo));   // constant results
        if (x.vlo >= hi) return mat(cst(hi));
        if (x.vlo < lo) {
            SwReg r = x;
            r.vlo = lo;
            if (o) {
                r.lo = var();
                r.hi = var();
                *o << ind << "const unsigned " << r.lo << " = __vmaxu2(" << x.lo << ", " << lit(lo + x.B) << ");\n";
                *o << ind << "const unsigned " << r.hi << " = __vmaxu2(" << x.hi << ", " << lit(lo + x.B) << ");\n";
            }
            x = r;
        }
        if (x.vhi > hi) {
            SwReg r = x;
            r.vhi = hi;
            r.vlo = std::min(x.vlo, hi);
            if (o) {
                r.lo = var();
                r.hi = var();
                *o << ind << "const unsigned " << r.lo << " = __vminu2(" << x.lo << ", " << lit(hi + x.B) << ");\n";
                *o << ind << "const unsigned " << r.hi << " = __vminu2(" << x.hi << ", " << lit(hi + x.B) << ");\n";
            }
            x = r;
        }
        return x;
    }
    // kernel boundary: saturate to [0, 255] and normalise to bias 0 (R-16)
    SwReg sat_norm(const SwLin &l) { return mat(of(clamp(mat(l), 0, 255))); }
    // table gather per channel (index clamped to the table, as kf_lut does);
    // entries must fit a lane: [0, 65535]
    SwReg lut(const SwReg &x0, const std::vector<int> &tab)
    {
        if (tab.empty()) throw SwFail{};
        const long long n = (long long)tab.size();
        const long long tmin = *std::min_element(tab.begin(), tab.end());
        const long long tmax = *std::max_element(tab.begin(), tab.end());
        if (tmin < 0 || tmax > 65535 || n > 65536) throw SwFail{};
        SwReg x = mat(of(clamp(x0, 0, n - 1)));   // bias 0 lanes = indices
        SwReg r;
        r.B = 0;
        r.vlo = tmin;
        r.vhi = tmax;
        if (o) {
            std::string t[4];
            for (int c = 0; c < 4; c++) {
                t[c] = var();
                const std::string &w = c < 2 ? x.lo : x.hi;
                const std::string idx = "KF_IDX(" + (c % 2 ? "(" + w + " >> 16)" : "(" + w + " & 0xffffu)") + ", " +
                                        std::to_string(n) + ")";
                *o << ind << "const unsigned " << t[c] << " = (unsigned)"
                   << (lut_shared ? lut_sym + "[" + idx + "]" : "__ldg(" + lut_sym + " + " + idx + ")") << ";\n";
            }
            r.lo = var();
            r.hi = var();
            *o << ind << "const unsigned " << r.lo << " = __byte_perm(" << t[0] << ", " << t[1] << ", 0x5410);\n";
            *o << ind << "const unsigned " << r.hi << " = __byte_perm(" << t[2] << ", " << t[3] << ", 0x5410);\n";
        }
        return r;
    }
    SwReg unpack(const std::string &u)
    {
        SwReg r;
        if (o) {
            r.lo = var();
            r.hi = var();
            *o << ind << "const unsigned " << r.lo << " = __byte_perm(" << u << ", 0u, 0x4140);\n";
            *o << ind << "const unsigned " << r.hi << " = __byte_perm(" << u << ", 0u, 0x4342);\n";
        }
        return r;
    }
    std::string pack(const SwReg &x)   // requires bias 0 and [0, 255]
    {
        if (x.B != 0 || x.vlo < 0 || x.vhi > 255) throw SwFail{};
        return "__byte_perm(" + x.lo + ", " + x.hi + ", 0x6420)";
    }
    // postfix op-IR over linear forms (LOAD k = loads[k]; a local op's post: LOAD 0 = acc)
    SwLin prog(const Op &op, const std::vector<SwLin> &loads)
    {
        std::vector<SwLin> st;
        auto pop = [&] { SwLin v = st.back(); st.pop_back(); return v; };
        auto isc = [](const SwLin &l) { return l.t.empty(); };
        for (const Instr &in : op.prog) {
            switch (in.op) {
            case KF_OP_LOAD: st.push_back(loads[op.kind == LOCAL ? 0 : in.arg]); break;
            case KF_OP_CONST: {
                const double c = in.imm;
                if (c != std::floor(c) || std::fabs(c) > 65535) throw SwFail{};
                st.push_back(cst((long long)c));
                break;
            }
            case KF_OP_ADD: { SwLin b = pop(), a = pop(); st.push_back(add(a, b)); break; }
            case KF_OP_SUB: { SwLin b = pop(), a = pop(); st.push_back(add(a, b, -1)); break; }
            case KF_OP_NEG: st.push_back(scale(pop(), -1)); break;
            case KF_OP_MUL: {
                SwLin b = pop(), a = pop();
                if (isc(b)) st.push_back(scale(a, b.k));
                else if (isc(a)) st.push_back(scale(b, a.k));
                else throw SwFail{};
                break;
            }
            case KF_OP_SHL:
                if (in.arg < 0 || in.arg > 15) throw SwFail{};
                st.push_back(scale(pop(), 1LL << in.arg));
                break;
            case KF_OP_SHR: {
                SwLin a = pop();
                if (isc(a)) { st.push_back(cst(a.k >> in.arg)); break; }
                st.push_back(of(shr(mat(a), in.arg)));
                break;
            }
            case KF_OP_MIN: case KF_OP_MAX: {
                SwLin b = pop(), a = pop();
                const bool mx = in.op == KF_OP_MAX;
                if (isc(a) && isc(b)) st.push_back(cst(mx ? std::max(a.k, b.k) : std::min(a.k, b.k)));
                else if (isc(b)) st.push_back(of(mx ? clamp(mat(a), b.k, LLONG_MAX / 4) : clamp(mat(a), LLONG_MIN / 4, b.k)));
                else if (isc(a)) st.push_back(of(mx ? clamp(mat(b), a.k, LLONG_MAX / 4) : clamp(mat(b), LLONG_MIN / 4, a.k)));
                else st.push_back(of(minmax(mat(a), mat(b), mx)));
                break;
            }
            case KF_OP_CLAMP: {
                SwLin hi = pop(), lo = pop(), x = pop();
                if (!isc(lo) || !isc(hi)) throw SwFail{};
                st.push_back(of(clamp(mat(x), lo.k, hi.k)));
                break;
            }
            case KF_OP_SAT_U8: st.push_back(of(clamp(mat(pop()), 0, 255))); break;
            case KF_OP_LUT: st.push_back(of(lut(mat(pop()), op.lut))); break;
            default: throw SwFail{};   // DIV, ABS, SELECT_GT, POW, ...
            }
        }
        return st.back();
    }
};

// Can kernel k run in SWAR form?  Interval-only dry run of the same emitter
// (its inputs are kernel outputs or input images: always [0, 255]).
static bool swar_feasible(const Op &op, const Separable &sp)
{
    int tmp = 0;
    SwEmitter e;
    e.tmp = &tmp;
    try {
        SwReg x;   // a [0, 255] value
        SwLin acc;
        if (op.kind == POINT) {
            std::vector<SwLin> loads(op.inputs.size(), SwEmitter::of(x));
            e.clamp(e.mat(e.prog(op, loads)), 0, 255);
            return true;
        }
        if (sp.ok) {
            SwLin v;
            for (double c : sp.col) if (c != 0.0) v = SwEmitter::add(v, SwEmitter::scale(SwEmitter::of(x), (long long)c));
            SwReg vr = e.mat(v);
            for (double c : sp.row) if (c != 0.0) acc = SwEmitter::add(acc, SwEmitter::scale(SwEmitter::of(vr), (long long)c));
        } else {
            for (double m : op.mask) if (m != 0.0) acc = SwEmitter::add(acc, SwEmitter::scale(SwEmitter::of(x), (long long)m));
        }
        SwLin r = op.prog.empty() ? acc : e.prog(op, {acc});
        e.clamp(e.mat(r), 0, 255);
        return true;
    } catch (const SwFail &) {
        return false;
    }
}

// ====================================================================== frame
// Slow path: 2-D tiles with shared-memory staging and index exchange.  Used
// for every output pixel outside the interior rectangle (and for the whole
// image when the interior is empty).
struct FrameGen {
    const kf_pipeline *p;
    const BlockInfo &b;
    int block;
    bool f32;
    std::map<int, int> slot;               // external image -> slot
    std::vector<std::vector<int>> groups;  // staged kernels grouped by halo, topological
    std::ostringstream &o;
    int tmp = 0;
    int TW = 32, TH = 8;
    ProgEmitter pe;
    bool naive = false;      // negative control only (option naive_border, KF_TEST_HOOKS build)
    int naive_mode = KF_CLAMP;
    double naive_const = 0.0;

    FrameGen(const kf_pipeline *p_, const BlockInfo &b_, int block_, std::ostringstream &o_)
        : p(p_), b(b_), block(block_), f32(p_->dtype == KF_F32), o(o_), pe{p_->dtype == KF_F32, block_, &tmp}
    {
        naive = !b.torus && opt(p, "naive_border");
        for (int k : b.kernels)
            if (p->ops[k].kind == LOCAL) {   // "pad once": the input is padded with the first local kernel's mode
                naive_mode = p->ops[k].mode;
                naive_const = p->ops[k].constant;
                break;
            }
    }

    std::string KV() const { return f32 ? "float" : "I4"; }
    std::string var() { return "v" + std::to_string(tmp++); }
    bool in_block(int img) const
    {
        return img >= p->n_inputs && std::binary_search(b.kernels.begin(), b.kernels.end(), img - p->n_inputs);
    }
    std::string smem_name(int k) const { return "s_" + std::to_string(k); }
    int RW(int k) const { return TW + 2 * b.hx.at(k); }
    int RH(int k) const { return TH + 2 * b.hy.at(k); }

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

    // Emits code computing image `img` at (y, x); returns the variable.
    std::string eval(int img, std::map<int, std::string> &memo, const std::set<int> &group, const std::string &ind)
    {
        auto it = memo.find(img);
        if (it != memo.end()) return it->second;
        std::string v = var();
        if (!in_block(img)) {
            std::string Y = "y", X = "x";
            if (b.torus) { Y = "kf_wrap(y, H)"; X = "kf_wrap(x, W)"; }
            if (naive) {   // negative control: the padded input plane at (y, x)
                const std::string md = std::to_string(naive_mode);
                std::string yy = var(), xx = var();
                o << ind << "const int " << yy << " = kf_border<" << md << ">(y, H);\n";
                o << ind << "const int " << xx << " = kf_border<" << md << ">(x, W);\n";
                std::string c = f32 ? fconst(naive_const) : "kf_i4(" + iconst((int)naive_const) + ")";
                o << ind << "const " << KV() << " " << v << " = (" << yy << " < 0 || " << xx << " < 0) ? " << c
                  << " : " << ext_load(img, yy, xx) << ";\n";
                memo[img] = v;
                return v;
            }
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
            for (int in : op.inputs) loads.push_back(eval(in, memo, group, ind));
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
                    if ((b.torus || naive) && staged_in) {   // naive: no index exchange (Fig. 4b)
                        val = smem_load(in - p->n_inputs, Y, X);
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
                            std::string c = f32 ? fconst(op.constant) : "kf_i4(" + iconst((int)op.constant) + ")";
                            val = "((" + yy + " < 0 || " + xx + " < 0) ? " + c + " : " + rd + ")";
                        } else {
                            val = rd;
                        }
                    }
                    std::string mc = f32 ? fconst(m) : iconst((long long)m);
                    o << ind << acc << " = kf_mac(" << acc << ", " << mc << ", " << val << ");\n";
                }
            loads.push_back(acc);
        }
        std::string r = (op.kind == LOCAL && op.prog.empty()) ? acc : pe.emit(o, op, k, loads, ind);
        if (!f32) {
            o << ind << "const I4 " << v << " = kf_satu8(" << r << ");\n";   // narrowing at the kernel boundary
        } else {
            o << ind << "const float " << v << " = " << r << ";\n";
        }
        memo[img] = v;
        return v;
    }

    // One tile shape: stage every staged kernel over tile + halo, then the sink
    // over the tile, writing only pixels inside the frame rectangle.
    void body(int shape)
    {
        const std::string ind = "        ";
        o << "__device__ __forceinline__ void " << kernel_name(block) << "_frame" << shape
          << "(const KfArgs &a, const int ox, const int oy, const KfRect &rc";
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
            o << "        const int y = oy - " << hy << " + i / " << rw << ", x = ox - " << hx << " + i % " << rw
              << ";\n";
            if (naive)
                o << "        if (y < a.r0 - " << hy << " || y >= a.r1 + " << hy << ") continue;\n";
            else if (!b.torus)
                o << "        if (y < 0 || y >= H || x < 0 || x >= W || y < a.r0 - " << hy << " || y >= a.r1 + "
                  << hy << ") continue;\n";
            std::map<int, std::string> memo;
            for (int k : g) {
                std::string v = eval(p->n_inputs + k, memo, gs, ind);
                o << ind << smem_name(k) << "[i] = " << (f32 ? v : "kf_pack(" + v + ")") << ";\n";
            }
            o << "    }\n    __syncthreads();\n";
        }
        o << "    for (int i = threadIdx.x; i < " << TW * TH << "; i += blockDim.x) {\n";
        o << "        const int y = oy + i / " << TW << ", x = ox + i % " << TW << ";\n";
        o << "        if (y >= rc.y1 || x >= rc.x1) continue;\n";
        std::map<int, std::string> memo;
        std::string v = eval(p->n_inputs + b.sink, memo, {}, ind);
        o << ind << (f32 ? "kf_stf" : "kf_sti") << "(a.out, a.out_base, W, y, x, " << v << ");\n";
        o << "    }\n}\n\n";
    }

    void run()
    {
        for (size_t i = 0; i < b.ext.size(); i++) slot[b.ext[i]] = (int)i;
        // staged kernels grouped by (hx, hy), descending hx+hy (topological)
        std::map<std::pair<int, int>, std::vector<int>> byhalo;
        for (int k : b.staged) byhalo[{b.hx.at(k), b.hy.at(k)}].push_back(k);
        std::vector<std::pair<int, int>> keys;
        for (auto &kv : byhalo) keys.push_back(kv.first);
        std::stable_sort(keys.begin(), keys.end(), [](auto &l, auto &r) {
            return l.first + l.second > r.first + r.second;
        });
        for (auto &kk : keys) groups.push_back(byhalo[kk]);
        int smem = 0;
        for (int shape = 0; shape < 2; shape++) {
            TW = shape == 0 ? kFrameTiles[0][0] : kFrameTiles[1][0];
            TH = shape == 0 ? kFrameTiles[0][1] : kFrameTiles[1][1];
            body(shape);
        }
        for (auto &g : groups)
            for (int k : g) {
                int n = 0;
                for (int s = 0; s < 2; s++)
                    n = std::max(n, (kFrameTiles[s][0] + 2 * b.hx.at(k)) * (kFrameTiles[s][1] + 2 * b.hy.at(k)));
                smem += n * 4;
            }
        if (smem > 48 * 1024) fail(KF_ERR_ARG, "fused block needs more than 48 KB of shared memory");
        // dispatcher for frame CTAs
        o << "__device__ __forceinline__ void " << kernel_name(block) << "_frame(const KfArgs &a, int cta)\n{\n";
        int off = 0;   // staged tiles live in the block's shared buffer (shared with the interior rings)
        for (auto &g : groups)
            for (int k : g) {
                int n = 0;
                for (int s = 0; s < 2; s++)
                    n = std::max(n, (kFrameTiles[s][0] + 2 * b.hx.at(k)) * (kFrameTiles[s][1] + 2 * b.hy.at(k)));
                o << "    " << (f32 ? "float" : "unsigned") << " *" << smem_name(k) << " = (" << (f32 ? "float" : "unsigned")
                  << " *)(" << kernel_name(block) << "_smem + " << off << ");\n";
                off += n * 4;
            }
        std::string sargs;
        for (auto &g : groups)
            for (int k : g) sargs += ", " + smem_name(k);
        o << "    int r = 0;\n";
        o << "    while (r + 1 < a.n_rect && cta >= a.rect[r + 1].cta0) r++;\n";
        o << "    const KfRect &rc = a.rect[r];\n";
        o << "    const int t = cta - rc.cta0;\n";
        o << "    if (rc.shape == 0) {\n";
        o << "        " << kernel_name(block) << "_frame0(a, rc.x0 + (t % rc.ntx) * " << kFrameTiles[0][0]
          << ", rc.y0 + (t / rc.ntx) * " << kFrameTiles[0][1] << ", rc" << sargs << ");\n";
        o << "    } else {\n";
        o << "        " << kernel_name(block) << "_frame1(a, rc.x0 + (t % rc.ntx) * " << kFrameTiles[1][0]
          << ", rc.y0 + (t / rc.ntx) * " << kFrameTiles[1][1] << ", rc" << sargs << ");\n";
        o << "    }\n}\n\n";
    }
};

// ================================================================== interior
// Streaming path: one warp streams a column chunk along a strip of rows.
//
// Schedule.  Let HY(i) be the rows of image i the block needs
// above/below the sink row (BlockInfo::hy for kernels, ext_hy for external
// images) and L = max HY over the external images.  Rows are counted in the
// strip's streaming direction (dir = +1 downward, -1 upward: r' = r or
// H-1-r).  At iteration t the warp
//   - has external image e at row  t - L + HY(e)  (prefetched D iterations ago),
//   - computes kernel k at row     t - L + HY(k)  (as late as possible),
// so the sink (HY = 0) emits row t - L.  A consumer k reads its producer i at
// iteration offset HY(k) - HY(i) + dy' <= 0: per-image register rings of P
// slots indexed by iteration mod P; the loop body is emitted P times so every
// ring index is a compile-time constant (no register moves).
//
// Image edges (index exchange, R-12): a consumer reads its
// producer at B(p) with ITS OWN border mode.
//   - vertical: the strip that starts at an image edge (top strip downward,
//     bottom strip upward) peels its first Q iterations, in which every tap row
//     r' + dy' < 0 is redirected statically to the ring slot of row B(r' + dy')
//     (always an already computed row) or to the constant;
//   - horizontal: in the first/last column chunk the lane holding columns
//     0..3 (W-4..W-1) replaces the taps that would come from the neighbour
//     lane by its own register at B(c) (or the constant): one select per tap.
struct StreamGen {
    const kf_pipeline *p;
    const BlockInfo &b;
    const StreamInfo &si;
    int block;
    bool f32;
    std::ostringstream &o;
    int tmp = 0;
    ProgEmitter pe;
    const int V;      // pixels per lane (si.V)
    const int NQ;     // float4 / uint4 vectors per lane per row (V / 4)
    std::map<int, int> slot;   // external image -> slot
    // per-iteration memo: (image, ring slot, column) -> unpacked value variable
    std::map<std::tuple<int, int, int>, std::string> val_memo;
    // (var, lane offset, edge key, border constant): the constant is part of the
    // key -- two CONSTANT-border consumers of the same row with different
    // constants must not share an edge substitution
    std::map<std::tuple<std::string, int, int, std::string>, std::string> shfl_memo;
    std::map<std::tuple<int, int, int>, SwReg> sw_memo;                     // SWAR values (image, slot, column)
    std::map<std::pair<int, int>, std::string> dl_memo;                      // delay-line rows read (image, age)
    std::string cur_it = "0";                                                // iteration index of the body being emitted
    std::map<int, int> xe;   // pair mode: deferred power-of-two exponent of each image's stored values
    int xe_of(int img) const { auto it = xe.find(img); return pm && it != xe.end() ? it->second : 0; }
    void set_xe(int img, int e)
    {
        auto it = xe.find(img);
        if (it != xe.end() && it->second != e) fail(KF_ERR_PROGRAM, "codegen: inconsistent deferred exponent");
        xe[img] = e;
    }
    std::string cvalx(const Op &op, int e) const { return f32 ? fconst(std::ldexp((double)(float)op.constant, -e)) : cval(op); }
    std::map<std::tuple<std::string, int, int, long long>, SwReg> swsh_memo;   // SWAR shuffles (same key)
    // variant being emitted
    int dir = 1;
    bool el = false, er = false;
    bool pm = false;   // f32 values kept as packed pixel pairs (F2) for column-local math
    bool runptr = false;   // steady-state loop uses running row pointers (set per variant)
    bool vedge = false;    // variant starts at an image edge (peeled iterations remap taps)
    bool defer_ok = true;  // pair mode: defer normalised masks' power-of-two scales (option "defer")
    std::set<int> prp;     // external images fed by running row pointers from the prologue on (interior strips)
    bool qptr = false;     // steady-state loop: ring slots addressed from per-trip base pointers
    bool tma = false;      // this variant feeds the ring with TMA bulk row copies (option tma)
    int peel_Q = 0;        // peeled iterations of the variant being emitted
    int loop_u0 = 0;       // first iteration of the steady-state loop of the variant being emitted

    StreamGen(const kf_pipeline *p_, const BlockInfo &b_, const StreamInfo &si_, int block_, std::ostringstream &o_)
        : p(p_), b(b_), si(si_), block(block_), f32(p_->dtype == KF_F32), o(o_), pe{p_->dtype == KF_F32, block_, &tmp},
          V(si_.V), NQ(si_.V / 4)
    {
    }

    std::string KV() const { return f32 ? "float" : "I4"; }
    std::string RT() const { return f32 ? "float" : "unsigned"; }   // ring storage type
    std::string var() { return "v" + std::to_string(tmp++); }
    int HY(int img) const { return si.hy.at(img); }
    int NR() const { return pm ? V / 2 : V; }                         // ring registers per row
    int NRi(int img) const { return si.swring.count(img) ? 2 * V : NR(); }   // SWAR rings: (lo, hi) per pixel
    std::string RDT() const { return pm ? "F2" : RT(); }               // ring register type
    static int md(int a, int m) { return ((a % m) + m) % m; }
    bool is_ext(int img) const { return std::binary_search(b.ext.begin(), b.ext.end(), img); }
    // Ring slot of image img at iteration offset `off` (<= 0: past rows; +D:
    // the prefetch of an external image) seen from loop-body copy j.  Unrolled:
    // slot = iteration mod P.  Rolled (one body copy, rings shifted by register
    // moves at the end of every iteration): slot = age (+D for external images).
    // Rolled trips of T rows (si.T): body copy j of a trip sees its newest row
    // at slot T-1-j, and the rings shift by T once per trip (peeled iterations
    // are copy T-1 and shift by one), halving the moves for T = 2.
    int sl(int img, int off, int j) const
    {
        if (!si.rolled) return md(j + off, si.P);
        return -off + (si.T - 1 - j) + (is_ext(img) && !si.sring ? si.D : 0);
    }
    int ring_len(int img) const
    {
        if (!si.rolled) return si.P;
        return si.depth.at(img) + si.T - 1 + (is_ext(img) && !si.sring ? si.D : 0);
    }
    std::string ring(int img, int s, int v) const
    {
        return "r" + std::to_string(img) + "_" + std::to_string(s) + "_" + std::to_string(v);
    }
    std::string cval(const Op &op) const
    {
        return f32 ? fconst(op.constant) : "kf_i4(" + iconst((int)op.constant) + ")";
    }

    // value of image img at ring slot s, column v of this lane (unpacked)
    std::string pval(int img, int s, int q) const { return ring(img, s, q); }
    std::string value(int img, int s, int v, const std::string &ind)
    {
        if (pm) return ring(img, s, v / 2) + (v % 2 ? ".y" : ".x");
        auto key = std::make_tuple(img, s, v);
        auto it = val_memo.find(key);
        if (it != val_memo.end()) return it->second;
        std::string r = ring(img, s, v);
        if (!f32) {
            std::string t = var();
            if (si.swring.count(img))
                o << ind << "const I4 " << t << " = kf_unpack_sw(" << ring(img, s, 2 * v) << ", " << ring(img, s, 2 * v + 1)
                  << ");\n";
            else
                o << ind << "const I4 " << t << " = kf_unpack(" << r << ");\n";
            r = t;
        }
        val_memo[key] = r;
        return r;
    }

    // Border map of one axis at an edge of an image of (large) size n, for the
    // columns/rows just outside: returns the in-image index relative to the
    // edge (0 = the edge pixel), or -1 for the constant.  c < 0 = outside.
    static int edge_map(int mode, int c)
    {
        switch (mode) {
        case KF_CLAMP: return 0;
        case KF_MIRROR: return -c - 1;
        case KF_MIRROR101: return -c;
        default: return -1;   // KF_CONSTANT
        }
    }

    // value at column offset q (relative to this lane's first column) of a row
    // whose V per-lane values are `row`: own register or a warp shuffle; in an
    // edge chunk the edge lane substitutes the border-mapped own register.
    std::string at_col(const std::vector<std::string> &row, int q, const Op &op, const std::string &csub,
                       const std::string &ind)
    {
        if (q >= 0 && q < V) return row[q];
        int lo = q >= 0 ? q / V : -((-q + V - 1) / V);
        int idx = q - lo * V;
        const bool edge = (q < 0 && el) || (q >= V && er);
        const int ekey = edge ? op.mode * 64 + q : -1000;
        auto key = std::make_tuple(row[idx], lo, ekey, edge ? csub : std::string());
        auto it = shfl_memo.find(key);
        if (it != shfl_memo.end()) return it->second;
        std::string t = var();
        o << ind << "const " << KV() << " " << t << " = " << (lo < 0 ? "kf_shup(" : "kf_shdn(") << row[idx] << ", "
          << std::abs(lo) << ");\n";
        if (edge) {
            std::string sub;
            if (q < 0) {
                int m = edge_map(op.mode, q);   // column q < 0 of the lane at x = 0
                sub = m < 0 ? csub : row[m];
            } else {
                int m = edge_map(op.mode, -(q - V) - 1);   // column W + (q - V) of the lane at x = W - V
                sub = m < 0 ? csub : row[V - 1 - m];
            }
            std::string t2 = var();
            o << ind << "const " << KV() << " " << t2 << " = (" << (q < 0 ? "x == 0" : "x == W - " + std::to_string(V)) << ") ? "
              << sub << " : " << t << ";\n";
            t = t2;
        }
        shfl_memo[key] = t;
        return t;
    }

    // acc = sum_i c_i * v_i over non-zero coefficients (emitted as FMA chain)
    std::string lincomb(std::vector<std::pair<double, std::string>> terms, const std::string &ind)
    {
        // start from a unit-coefficient term when there is one (no multiply)
        std::stable_partition(terms.begin(), terms.end(), [](const auto &t) { return t.first == 1.0; });
        std::string acc;
        for (auto &t : terms) {
            if (t.first == 0.0) continue;
            std::string c = f32 ? fconst(t.first) : iconst((long long)t.first);
            std::string nv = var();
            if (acc.empty()) {
                if (t.first == 1.0)
                    o << ind << "const " << KV() << " " << nv << " = " << t.second << ";\n";
                else
                    o << ind << "const " << KV() << " " << nv << " = kf_mul1(" << c << ", " << t.second << ");\n";
            } else if (t.first == 1.0) {
                o << ind << "const " << KV() << " " << nv << " = kf_add(" << acc << ", " << t.second << ");\n";
            } else if (t.first == -1.0) {
                o << ind << "const " << KV() << " " << nv << " = kf_sub(" << acc << ", " << t.second << ");\n";
            } else {
                o << ind << "const " << KV() << " " << nv << " = kf_mac(" << acc << ", " << c << ", " << t.second
                  << ");\n";
            }
            acc = nv;
        }
        if (acc.empty()) {
            acc = var();
            o << ind << "const " << KV() << " " << acc << " = " << (f32 ? "0.0f" : "kf_i4(0)") << ";\n";
        }
        return acc;
    }

    // packed form of lincomb over pixel pairs
    std::string lincomb2(std::vector<std::pair<double, std::string>> terms, const std::string &ind)
    {
        std::stable_partition(terms.begin(), terms.end(), [](const auto &t) { return t.first == 1.0; });
        std::string acc;
        for (auto &t : terms) {
            if (t.first == 0.0) continue;
            std::string c = fconst(t.first), nv = var();
            if (acc.empty())
                o << ind << "const F2 " << nv << " = " << (t.first == 1.0 ? t.second : "kf2_mul1(" + c + ", " + t.second + ")")
                  << ";\n";
            else if (t.first == 1.0)
                o << ind << "const F2 " << nv << " = kf2_add(" << acc << ", " << t.second << ");\n";
            else if (t.first == -1.0)
                o << ind << "const F2 " << nv << " = kf2_sub(" << acc << ", " << t.second << ");\n";
            else
                o << ind << "const F2 " << nv << " = kf2_mac(" << acc << ", " << c << ", " << t.second << ");\n";
            acc = nv;
        }
        if (acc.empty()) {
            acc = var();
            o << ind << "const F2 " << acc << " = kf2(0.0f);\n";
        }
        return acc;
    }

    // Row of producer `in` needed by consumer k (image kimg) at primed tap
    // offset dyp, in iteration slot j.  `u` >= 0: the iteration index is the
    // compile-time constant u of a peeled edge iteration (rows relative to the
    // strip start = the image edge), so taps outside the image are remapped;
    // u < 0: steady state, no remap.  Returns an empty vector for a constant row.
    int tap_slot(int kimg, const Op &op, int in, int dyp, int j, int u, bool &is_const) const
    {
        const int L = si.L;
        int s = sl(in, HY(kimg) - HY(in) + dyp, j);
        is_const = false;
        if (u >= 0 && vedge) {
            const int rk = u - 2 * L + HY(kimg);   // consumer row (primed, 0 = edge row)
            const int rr = rk + dyp;
            if (rr < 0 && rk >= 0) {
                const int m = edge_map(op.mode, rr);
                if (m < 0) {
                    is_const = true;
                    return -1;
                }
                s = sl(in, m + 2 * L - HY(in) - u, j);   // the iteration that computed row m of `in`
            }
        }
        return s;
    }
    std::vector<std::string> tap_row(int kimg, const Op &op, int in, int dyp, int j, int u, bool &is_const,
                                     const std::string &ind)
    {
        const int s = tap_slot(kimg, op, in, dyp, j, u, is_const);
        if (is_const) return {};
        last_slot = s;
        std::vector<std::string> row;
        for (int v = 0; v < V; v++) row.push_back(value(in, s, v, ind));
        return row;
    }
    int last_slot = 0;   // ring slot of the last tap_row (pair access in pair mode)

    // ---- SWAR form of u8x4 kernels
    SwEmitter swe(const std::string &ind) { SwEmitter e; e.o = &o; e.tmp = &tmp; e.ind = ind; return e; }
    std::string lut_sym(int k) const { return "kf_lut_" + std::to_string(block) + "_" + std::to_string(k); }
    // value of image img at ring slot s, column v (bias 0, [0, 255]): memo or unpack
    SwReg svalue(int img, int s, int v, const std::string &ind)
    {
        auto key = std::make_tuple(img, s, v);
        auto it = sw_memo.find(key);
        if (it != sw_memo.end()) return it->second;
        if (si.delay.count(img) && s >= si.depth.at(img)) {   // row older than the register ring: delay line
            auto dk = std::make_pair(img, s);
            if (!dl_memo.count(dk)) {
                const std::string t = var();
                o << ind << "const uint4 " << t << " = dl" << img << "[((" << cur_it << " - " << s << ") & "
                  << si.delay.at(img) - 1 << ") * 32];\n";
                dl_memo[dk] = t;
            }
            const char *c[4] = {"x", "y", "z", "w"};
            SwReg r = swe(ind).unpack(dl_memo[dk] + "." + c[v]);
            sw_memo[key] = r;
            return r;
        }
        if (si.swring.count(img)) {   // SWAR ring: already unpacked (bias 0, [0, 255])
            SwReg r;
            r.lo = ring(img, s, 2 * v);
            r.hi = ring(img, s, 2 * v + 1);
            sw_memo[key] = r;
            return r;
        }
        SwReg r = swe(ind).unpack(ring(img, s, v));
        sw_memo[key] = r;
        return r;
    }
    // SWAR twin of at_col: own register or warp shuffle (both halves); in an
    // edge chunk the edge lane substitutes its border-mapped own register or,
    // for CONSTANT, `csub` (a value with the row's bias)
    SwReg at_col_sw(const std::vector<SwReg> &row, int q, const Op &op, long long csub, const std::string &ind)
    {
        if (q >= 0 && q < V) return row[q];
        int lo = q >= 0 ? q / V : -((-q + V - 1) / V);
        int idx = q - lo * V;
        const bool edge = (q < 0 && el) || (q >= V && er);
        const int ekey = edge ? op.mode * 64 + q : -1000;
        auto key = std::make_tuple(row[idx].lo, lo, ekey, edge ? csub : 0LL);
        auto it = swsh_memo.find(key);
        if (it != swsh_memo.end()) return it->second;
        SwReg t = row[idx];
        t.lo = var();
        t.hi = var();
        const char *fn = lo < 0 ? "__shfl_up_sync" : "__shfl_down_sync";
        o << ind << "const unsigned " << t.lo << " = " << fn << "(KF_FULL, " << row[idx].lo << ", " << std::abs(lo) << ");\n";
        o << ind << "const unsigned " << t.hi << " = " << fn << "(KF_FULL, " << row[idx].hi << ", " << std::abs(lo) << ");\n";
        if (edge) {
            std::string slo, shi;
            int m;
            if (q < 0) m = edge_map(op.mode, q);
            else m = edge_map(op.mode, -(q - V) - 1);
            if (m < 0) {
                slo = shi = SwEmitter::lit(csub + row[0].B);
                // the border constant may lie outside the row's interval (a
                // producer whose values are provably >= 128, a constant 0):
                // the bias analysis downstream must see it, or a sum that goes
                // negative only at the image edge wraps a 16-bit lane
                t.vlo = std::min(t.vlo, csub);
                t.vhi = std::max(t.vhi, csub);
            } else {
                const SwReg &sr = q < 0 ? row[m] : row[V - 1 - m];
                slo = sr.lo;
                shi = sr.hi;
            }
            const std::string cond = q < 0 ? "x == 0" : "x == W - " + std::to_string(V);
            SwReg t2 = t;
            t2.lo = var();
            t2.hi = var();
            o << ind << "const unsigned " << t2.lo << " = (" << cond << ") ? " << slo << " : " << t.lo << ";\n";
            o << ind << "const unsigned " << t2.hi << " = (" << cond << ") ? " << shi << " : " << t.hi << ";\n";
            t = t2;
        }
        swsh_memo[key] = t;
        return t;
    }
    void kernel_sw(int k, int j, int u, const std::string &ind)
    {
        const Op &op = p->ops[k];
        const int img = p->n_inputs + k;
        SwEmitter e = swe(ind);
        e.lut_sym = lut_sym(k);
        if (lut_in_smem(si, op)) {
            e.lut_sym = "kf_lutsh_" + std::to_string(block) + "_" + std::to_string(k);
            e.lut_shared = true;
        }
        std::vector<SwLin> res(V);
        if (op.kind == POINT) {
            for (int v = 0; v < V; v++) {
                std::vector<SwLin> loads;
                for (int in : op.inputs) loads.push_back(SwEmitter::of(svalue(in, sl(in, HY(img) - HY(in), j), v, ind)));
                res[v] = e.prog(op, loads);
            }
        } else {
            const int in = op.inputs[0];
            const int rx = op.mw / 2, ry = op.mh / 2;
            auto mrow = [&](int dyp) { return ry + dir * dyp; };
            const long long c = (long long)op.constant;
            const Separable &sp = si.sep.at(k);
            std::vector<SwLin> acc(V);
            if (sp.ok) {
                std::vector<SwLin> vl(V);
                long long csum = 0;
                for (double cc : sp.col) csum += (long long)cc;
                for (int dy = -ry; dy <= ry; dy++) {   // mask-row order in both directions
                    const int dyp = dir * dy;
                    const long long cf = (long long)sp.col[mrow(dyp)];
                    if (cf == 0) continue;
                    bool isc = false;
                    const int s = tap_slot(img, op, in, dyp, j, u, isc);
                    for (int v = 0; v < V; v++)
                        vl[v] = isc ? SwEmitter::add(vl[v], SwEmitter::cst(cf * c))
                                    : SwEmitter::add(vl[v], SwEmitter::scale(SwEmitter::of(svalue(in, s, v, ind)), cf));
                }
                std::vector<SwReg> vs(V);
                for (int v = 0; v < V; v++) vs[v] = e.mat(vl[v]);
                for (int v = 0; v < V; v++)
                    for (int dx = -rx; dx <= rx; dx++) {
                        const long long rf = (long long)sp.row[dx + rx];
                        if (rf == 0) continue;
                        acc[v] = SwEmitter::add(acc[v], SwEmitter::scale(SwEmitter::of(at_col_sw(vs, v + dx, op, c * csum, ind)), rf));
                    }
            } else {
                for (int dy = -ry; dy <= ry; dy++) {
                    const int dyp = dir * dy;
                    const int mr = mrow(dyp);
                    bool any = false;
                    for (int dx = -rx; dx <= rx; dx++) any |= op.mask[(size_t)mr * op.mw + dx + rx] != 0.0;
                    if (!any) continue;
                    bool isc = false;
                    const int s = tap_slot(img, op, in, dyp, j, u, isc);
                    std::vector<SwReg> row(V);
                    if (!isc)
                        for (int v = 0; v < V; v++) row[v] = svalue(in, s, v, ind);
                    for (int dx = -rx; dx <= rx; dx++) {
                        const long long m = (long long)op.mask[(size_t)mr * op.mw + dx + rx];
                        if (m == 0) continue;
                        for (int v = 0; v < V; v++)
                            acc[v] = isc ? SwEmitter::add(acc[v], SwEmitter::cst(m * c))
                                         : SwEmitter::add(acc[v], SwEmitter::scale(SwEmitter::of(at_col_sw(row, v + dx, op, c, ind)), m));
                    }
                }
            }
            for (int v = 0; v < V; v++) res[v] = op.prog.empty() ? acc[v] : e.prog(op, {acc[v]});
        }
        const int ws = sl(img, 0, j);
        for (int v = 0; v < V; v++) {
            SwReg r = e.sat_norm(res[v]);   // narrowing at the kernel boundary (R-16)
            if (si.swring.count(img)) {
                o << ind << ring(img, ws, 2 * v) << " = " << r.lo << ";\n";
                o << ind << ring(img, ws, 2 * v + 1) << " = " << r.hi << ";\n";
            } else {
                o << ind << ring(img, ws, v) << " = " << e.pack(r) << ";\n";
            }
            sw_memo[std::make_tuple(img, ws, v)] = r;
        }
        if (si.delay.count(img)) {   // the packed row into the kernel's delay line, slot (iteration mod S)
            o << ind << "dl" << img << "[(" << cur_it << " & " << si.delay.at(img) - 1 << ") * 32] = make_uint4(";
            for (int v = 0; v < V; v++) o << (v ? ", " : "") << ring(img, ws, v);
            o << ");\n";
        }
    }

    // kernel k at iteration slot j: emits code, stores its V values into its
    // ring slot j, and memoises the unpacked values.
    void kernel(int k, int j, int u, const std::string &ind)
    {
        if (si.swk.count(k)) {
            kernel_sw(k, j, u, ind);
            return;
        }
        const Op &op = p->ops[k];
        const int img = p->n_inputs + k;
        std::vector<std::string> res(V);
        if (pm && op.kind == POINT) {
            const int ws = sl(img, 0, j);
            for (int q = 0; q < V / 2; q++) {
                std::vector<ProgEmitter::Val> loads;
                for (int in : op.inputs) {
                    ProgEmitter::Val v;
                    v.x = pval(in, sl(in, HY(img) - HY(in), j), q);
                    v.e = xe_of(in);
                    loads.push_back(v);
                }
                const ProgEmitter::Val r = pe.emit2e(o, op, loads, ind);
                set_xe(img, r.e);
                o << ind << ring(img, ws, q) << " = " << r.x << ";\n";
            }
            return;
        }
        if (op.kind == POINT) {
            std::vector<std::vector<std::string>> ins;
            for (int in : op.inputs) {
                int s = sl(in, HY(img) - HY(in), j);
                std::vector<std::string> row;
                for (int v = 0; v < V; v++) row.push_back(value(in, s, v, ind));
                ins.push_back(row);
            }
            for (int v = 0; v < V; v++) {
                std::vector<std::string> loads;
                for (auto &r : ins) loads.push_back(r[v]);
                res[v] = pe.emit(o, op, k, loads, ind);
            }
        } else {
            const int in = op.inputs[0];
            const int rx = op.mw / 2, ry = op.mh / 2;
            // mask row of primed tap offset dyp (upward strips flip the mask)
            auto mrow = [&](int dyp) { return ry + dir * dyp; };
            std::vector<std::string> acc(V);
            const Separable &sp = si.sep.at(k);
            // pair mode: integer column weights, the mask's power-of-two scale deferred
            const int ein = xe_of(in);
            int ks = 0;
            const bool defer = pm && defer_ok && sp.ok && ProgEmitter::pow2(sp.scale, ks);
            if (!defer) ks = 0;
            const double csc = defer ? sp.scale : 1.0;
            const int eacc = ein + ks;
            if (sp.ok) {
                // vertical pass in the lane's own columns, then horizontal taps
                std::vector<std::pair<double, std::vector<std::string>>> rows;
                std::vector<std::pair<double, int>> prow;   // pair mode: (coefficient, ring slot)
                std::vector<double> cterms;   // coefficients of constant (exterior) rows
                for (int dy = -ry; dy <= ry; dy++) {   // mask-row order in both directions (same rounding)
                    const int dyp = dir * dy;
                    const double c = sp.col[mrow(dyp)] / csc;
                    if (c == 0.0) continue;
                    bool isc = false;
                    auto r = tap_row(img, op, in, dyp, j, u, isc, ind);
                    if (isc) cterms.push_back(c);
                    else { rows.push_back({c, r}); prow.push_back({c, last_slot}); }
                }
                std::vector<std::string> vs(V);
                std::string cst;
                if (!cterms.empty()) {
                    double cs = 0.0;
                    for (double c : cterms) cs += c;
                    cst = var();
                    o << ind << "const " << KV() << " " << cst << " = kf_mul1(" << (f32 ? fconst(cs) : iconst((long long)cs))
                      << ", " << cvalx(op, ein) << ");\n";
                }
                if (pm) {
                    for (int q = 0; q < V / 2; q++) {
                        std::vector<std::pair<double, std::string>> terms;
                        for (auto &r : prow) terms.push_back({r.first, pval(in, r.second, q)});
                        if (!cst.empty()) terms.push_back({1.0, "kf2(" + cst + ")"});
                        std::string pv = lincomb2(terms, ind);
                        vs[2 * q] = pv + ".x";
                        vs[2 * q + 1] = pv + ".y";
                    }
                } else {
                    for (int v = 0; v < V; v++) {
                        std::vector<std::pair<double, std::string>> terms;
                        for (auto &r : rows) terms.push_back({r.first, r.second[v]});
                        if (!cst.empty()) terms.push_back({1.0, cst});
                        vs[v] = lincomb(terms, ind);
                    }
                }
                // an exterior column of a CONSTANT consumer is c in every row: c * sum(col)
                std::string csub;
                if (op.mode == KF_CONSTANT && (el || er)) {
                    double cs = 0.0;
                    for (double c : sp.col) cs += c / csc;
                    csub = var();
                    o << ind << "const " << KV() << " " << csub << " = kf_mul1("
                      << (f32 ? fconst(cs) : iconst((long long)cs)) << ", " << cvalx(op, ein) << ");\n";
                }
                for (int v = 0; v < V; v++) {
                    std::vector<std::pair<double, std::string>> terms;
                    for (int dx = -rx; dx <= rx; dx++)
                        if (sp.row[dx + rx] != 0.0)
                            terms.push_back({sp.row[dx + rx], at_col(vs, v + dx, op, csub, ind)});
                    acc[v] = lincomb(terms, ind);
                }
            } else {
                std::vector<std::vector<std::pair<double, std::string>>> terms(V);
                for (int dy = -ry; dy <= ry; dy++) {
                    const int dyp = dir * dy;
                    const int mr = mrow(dyp);
                    bool any = false;
                    for (int dx = -rx; dx <= rx; dx++) any |= op.mask[(size_t)mr * op.mw + dx + rx] != 0.0;
                    if (!any) continue;
                    bool isc = false;
                    std::vector<std::string> row = tap_row(img, op, in, dyp, j, u, isc, ind);
                    for (int dx = -rx; dx <= rx; dx++) {
                        double m = op.mask[(size_t)mr * op.mw + dx + rx];
                        if (m == 0.0) continue;
                        for (int v = 0; v < V; v++)
                            terms[v].push_back({m, isc ? cvalx(op, ein) : at_col(row, v + dx, op, cvalx(op, ein), ind)});
                    }
                }
                for (int v = 0; v < V; v++) acc[v] = lincomb(terms[v], ind);
            }
            if (pm) {
                const int ws = sl(img, 0, j);
                for (int q = 0; q < V / 2; q++) {
                    ProgEmitter::Val a;
                    a.x = "make_float2(" + acc[2 * q] + ", " + acc[2 * q + 1] + ")";
                    a.e = eacc;
                    if (!op.prog.empty()) a = pe.emit2e(o, op, std::vector<ProgEmitter::Val>{a}, ind);
                    set_xe(img, a.e);
                    o << ind << ring(img, ws, q) << " = " << a.x << ";\n";
                }
                return;
            }
            for (int v = 0; v < V; v++)
                res[v] = op.prog.empty() ? acc[v] : pe.emit(o, op, k, std::vector<std::string>{acc[v]}, ind);
        }
        const int ws = sl(img, 0, j);
        for (int v = 0; v < V; v++) {
            std::string r = res[v];
            if (!f32) {   // narrowing at the kernel boundary
                std::string t = var();
                o << ind << "const I4 " << t << " = kf_satu8(" << r << ");\n";
                r = t;
                if (img != p->n_inputs + b.sink || si.depth.at(img) > 1)
                    o << ind << ring(img, ws, v) << " = kf_pack(" << r << ");\n";
            } else {
                o << ind << ring(img, ws, v) << " = " << r << ";\n";
            }
            val_memo[std::make_tuple(img, ws, v)] = r;
        }
    }

    // ring slot rs of image img from the NQ 128-bit vectors q[0..NQ) of one row
    // (pixel v is component v % 4 of vector v / 4)
    void unpack_row(int img, int rs, const std::vector<std::string> &q, const std::string &ind)
    {
        const char *c[4] = {"x", "y", "z", "w"};
        auto comp = [&](int v) { return q[v / 4] + "." + c[v % 4]; };
        if (pm) {
            for (int k = 0; k < V / 2; k++)
                o << ind << ring(img, rs, k) << " = make_float2(" << comp(2 * k) << ", " << comp(2 * k + 1) << ");\n";
        } else if (si.swring.count(img)) {
            for (int v = 0; v < V; v++) {
                o << ind << ring(img, rs, 2 * v) << " = __byte_perm(" << comp(v) << ", 0u, 0x4140);\n";
                o << ind << ring(img, rs, 2 * v + 1) << " = __byte_perm(" << comp(v) << ", 0u, 0x4342);\n";
            }
        } else {
            for (int v = 0; v < V; v++) o << ind << ring(img, rs, v) << " = " << comp(v) << ";\n";
        }
    }

    // prefetch of external image `img` for iteration `it` into ring slot rs
    void load(int img, int rs, const std::string &it, const std::string &ind)
    {
        int s = slot.at(img);
        std::string rp = "(ys - " + std::to_string(2 * si.L - HY(img)) + " + (" + it + "))";   // primed row
        std::string row = var();
        o << ind << "const int " << row << " = min(max(" << (dir > 0 ? rp : "(H - 1 - " + rp + ")") << ", a.base["
          << s << "]), a.rlast[" << s << "]);\n";
        std::string ptr = "g" + std::to_string(s) + " + " + row + " * W";
        const char *c[4] = {"x", "y", "z", "w"};
        if (si.vec) {
            std::vector<std::string> q(NQ);
            for (int k = 0; k < NQ; k++) {
                q[k] = var();
                o << ind << "const " << (f32 ? "float4 " : "uint4 ") << q[k] << " = " << (f32 ? "kf_ld4f(" : "kf_ld4u(")
                  << ptr << " + " << 4 * k << ");\n";
            }
            unpack_row(img, rs, q, ind);
        } else if (pm) {
            for (int q = 0; q < V / 2; q++)
                o << ind << ring(img, rs, q) << " = make_float2(KF_LDG(" << ptr << " + cl" << 2 * q << "), KF_LDG(" << ptr
                  << " + cl" << 2 * q + 1 << "));\n";
        } else if (si.swring.count(img)) {
            for (int v = 0; v < V; v++) {
                o << ind << ring(img, rs, 2 * v) << " = __byte_perm(KF_LDG(" << ptr << " + cl" << v << "), 0u, 0x4140);\n";
                o << ind << ring(img, rs, 2 * v + 1) << " = __byte_perm(KF_LDG(" << ptr << " + cl" << v << "), 0u, 0x4342);\n";
            }
        } else {
            for (int v = 0; v < V; v++)
                o << ind << ring(img, rs, v) << " = KF_LDG(" << ptr << " + cl" << v << ");\n";
        }
    }

    // primed-row expression -> clamped actual row of external image slot s
    std::string row_of(int img, const std::string &it, const std::string &ind)
    {
        int s = slot.at(img);
        std::string rp = "(ys - " + std::to_string(2 * si.L - HY(img)) + " + (" + it + "))";
        std::string row = var();
        o << ind << "const int " << row << " = min(max(" << (dir > 0 ? rp : "(H - 1 - " + rp + ")") << ", a.base["
          << s << "]), a.rlast[" << s << "]);\n";
        return row;
    }
    // shared-memory ring: start the copy of iteration `it`'s row into ring slot `ss`
    // Address of ring slot `ss` of image slot s.  In the steady-state loop the
    // slots are addressed from per-trip base pointers (sq = slot qb, sp = qprev,
    // sn = qnext) so that the unrolled rows use immediate offsets.
    std::string slot_ptr(int s, const std::string &ss) const
    {
        if (qptr) {
            if (ss == "qprev") return "sp" + std::to_string(s);
            if (ss == "qnext") return "sn" + std::to_string(s);
            if (ss.rfind("qb + ", 0) == 0) return "sq" + std::to_string(s) + " + " + std::to_string(32 * NQ * std::stoi(ss.substr(5)));
        }
        return "sr" + std::to_string(s) + " + (" + ss + ") * " + std::to_string(32 * NQ);
    }
    // the NQ 16-byte copies of one lane's row segment (lane-contiguous: a warp row is 512 * NQ bytes)
    void cp_row(const std::string &dst, const std::string &src, const std::string &guard, const std::string &ind)
    {
        o << ind << "if (" << guard << ") {";
        for (int k = 0; k < NQ; k++) o << " kf_cp16(" << dst << (k ? " + " + std::to_string(k) : "") << ", " << src
                                       << (k ? " + " + std::to_string(4 * k) : "") << ");";
        o << " }\n";
    }
    // mbarrier of ring slot `ss` of image slot s (TMA feed)
    std::string bar(int s, const std::string &ss) const
    {
        return "(mb + " + std::to_string(s * si.DS) + " + (" + ss + "))";
    }
    // TMA feed: lane 0 copies the warp's whole row segment (tb bytes) with one bulk copy
    void bulk_row(const std::string &dst, const std::string &src, const std::string &guard, int s,
                  const std::string &ss, const std::string &ind)
    {
        o << ind << "if (lane == 0 && " << guard << ") { KF_RCHK(" << src << ", tb); kf_bulk_row((char *)(" << dst
          << ") + toff, " << src << ", tb, " << bar(s, ss) << "); }\n";
    }
    void issue(int img, const std::string &ss, const std::string &it, const std::string &ind)
    {
        int s = slot.at(img);
        if (runptr || prp.count(img)) {   // running row pointer (rows stay inside [base, rlast])
            if (tma)
                bulk_row(slot_ptr(s, ss), "ip" + std::to_string(s), "(" + it + ") < nit", s, ss, ind);
            else
                cp_row(slot_ptr(s, ss), "ip" + std::to_string(s), "(" + it + ") < nit", ind);
            o << ind << "ip" << s << " += dW;\n";
            return;
        }
        std::string row = row_of(img, it, ind);
        if (tma)
            bulk_row(slot_ptr(s, ss), "g" + std::to_string(s) + " + " + row + " * W", "(" + it + ") < nit", s, ss, ind);
        else
            cp_row(slot_ptr(s, ss), "g" + std::to_string(s) + " + " + row + " * W", "(" + it + ") < nit", ind);
    }
    // TMA feed: wait until the row of iteration `it` (ring slot ss, phase parity par) landed
    void wait_row(const std::string &ss, const std::string &par, const std::string &it, const std::string &ind)
    {
        o << ind << "if ((" << it << ") < nit) {";
        for (int img : b.ext) o << " kf_mbar_wait(" << bar(slot.at(img), ss) << ", " << par << ");";
        o << " }\n";
    }
    // shared-memory ring: read ring slot `ss` into register ring slot rs
    void fetch(int img, const std::string &ss, int rs, const std::string &ind)
    {
        int s = slot.at(img);
        std::vector<std::string> q(NQ);
        for (int k = 0; k < NQ; k++) {
            q[k] = var();
            if (si.lpf)   // the row was read from the ring one iteration ago
                o << ind << "const " << (f32 ? "float4 " : "uint4 ") << q[k] << " = pf" << s << "_" << k << ";\n";
            else
                o << ind << "const " << (f32 ? "float4 " : "uint4 ") << q[k] << " = *(" << slot_ptr(s, ss) << " + " << k << ");\n";
        }
        unpack_row(img, rs, q, ind);
        if (si.delay.count(img))   // the packed row into the image's delay line, slot (iteration mod S)
            o << ind << "dl" << img << "[(" << cur_it << " & " << si.delay.at(img) - 1 << ") * 32] = " << q[0] << ";\n";
    }

    // One iteration (slot j).  u >= 0: peeled edge iteration with index u.
    void iteration(int j, int u, const std::string &uexpr, const std::string &ind)
    {
        const int D = si.D, L = si.L;
        val_memo.clear();
        shfl_memo.clear();
        sw_memo.clear();
        dl_memo.clear();
        swsh_memo.clear();
        o << ind.substr(2) << "{   // iteration " << uexpr << " + " << j << "\n";
        cur_it = u >= 0 ? std::to_string(u) : "(" + uexpr + " + " + std::to_string(j) + ")";
        if (si.sring) {
            const int DS = si.DS;
            std::string s_iss, s_get;
            if (u >= 0) {   // peeled: static slots
                s_iss = std::to_string((u + DS - 1) % DS);
                s_get = std::to_string(u % DS);
            } else {
                s_iss = j == 0 ? "qprev" : "qb + " + std::to_string(j - 1);
                s_get = "qb + " + std::to_string(j);
            }
            const std::string row_get = uexpr + " + " + std::to_string(j);
            const std::string row_nxt = uexpr + " + " + std::to_string(j + 1);
            if (tma) {   // every lane has read the slot about to be refilled (read a row or two ago)
                o << ind << "__syncwarp();\n";
                o << ind << "if (lane == 0) kf_proxy_fence();\n";
            }
            for (int img : b.ext) issue(img, s_iss, uexpr + " + " + std::to_string(j + DS - 1), ind);
            if (!tma) o << ind << "kf_cp_commit();\n";
            // TMA: phase parity of the row's slot = (row / DS) & 1, tracked as `ph` (flips when qb wraps)
            const std::string p_get = u >= 0 ? std::to_string((u / DS) & 1) : "ph";
            if (si.lpf) {
                // this iteration's row is already in registers; wait for the next
                // row and read it now, a whole iteration before its use
                for (int img : b.ext) fetch(img, s_get, sl(img, 0, j), ind);
                const bool wrap = !(u >= 0) && !(j + 1 < (si.rolled ? si.T : si.P));
                const std::string s_nxt = u >= 0 ? std::to_string((u + 1) % DS)
                                                 : (!wrap ? "qb + " + std::to_string(j + 1) : "qnext");
                const std::string p_nxt = u >= 0 ? std::to_string(((u + 1) / DS) & 1) : wrap ? "(ph ^ (qnext == 0))" : "ph";
                if (tma)
                    wait_row(s_nxt, p_nxt, row_nxt, ind);
                else
                    o << ind << "kf_cp_wait<" << DS - 2 << ">();\n";
                for (int img : b.ext)
                    for (int k = 0; k < NQ; k++)
                        o << ind << "pf" << slot.at(img) << "_" << k << " = *(" << slot_ptr(slot.at(img), s_nxt) << " + " << k << ");\n";
            } else {
                if (tma)
                    wait_row(s_get, p_get, row_get, ind);
                else
                    o << ind << "kf_cp_wait<" << DS - 1 << ">();\n";
                for (int img : b.ext) fetch(img, s_get, sl(img, 0, j), ind);
            }
        } else {
            for (int img : b.ext) load(img, sl(img, D, j), uexpr + " + " + std::to_string(j + D), ind);
        }
        // Kernel k is first needed at iteration 2L - 2 HY(k): its row then is the
        // first of the rows [ys - HY(k), ye + HY(k)) the strip's outputs read.
        // A peeled iteration skips it statically.  In the loop (option
        // warm_skip), kernels first needed after the loop's first iteration run
        // under a warp-uniform guard, so the warm-up rows of a loop that starts
        // at iteration 0 (rolled bodies) compute only what later rows read.
        // Consumers never read a skipped row (HY(producer) >= HY(consumer) +
        // ry(consumer)).  Temporaries of a guarded group go out of scope with it,
        // so the value memos are cleared after each group.  An int32 (I4) sink
        // whose ring is not written is stored from its memoised temporaries,
        // so it stays unguarded.
        const bool i4_sink_memo = !f32 && !si.swk.count(b.sink) && si.depth.at(p->n_inputs + b.sink) <= 1;
        int group = -1;
        for (int k : b.kernels) {
            const int first = 2 * L - 2 * HY(p->n_inputs + k);
            if (u >= 0) {
                if (u < first) continue;
                kernel(k, j, u, ind);
                continue;
            }
            const bool guard = opt(p, "warm_skip") && first > loop_u0 + j && !(k == b.sink && i4_sink_memo);
            const int g = guard ? first : -1;
            if (g != group) {
                if (group >= 0) {
                    o << ind << "}\n";
                    val_memo.clear(); shfl_memo.clear(); sw_memo.clear(); swsh_memo.clear(); dl_memo.clear();
                }
                if (g >= 0) o << ind << "if (" << uexpr << " + " << j << " >= " << first << ") {\n";
                group = g;
            }
            kernel(k, j, u, group >= 0 ? ind + "    " : ind);
        }
        if (group >= 0) {
            o << ind << "}\n";
            val_memo.clear(); shfl_memo.clear(); sw_memo.clear(); swsh_memo.clear(); dl_memo.clear();
        }
        const int simg = p->n_inputs + b.sink;
        const int ss = sl(simg, 0, j);
        const bool store = !(u >= 0 && u < 2 * L);   // warm-up iterations store nothing
        std::string orow;   // output row pointer expression
        // pair mode: the sink's deferred power-of-two exponent is applied here, once
        std::vector<std::string> sk(V);
        if (store && f32 && pm) {
            const int e = xe_of(simg);
            for (int q = 0; q < V / 2; q++) {
                std::string pr = ring(simg, ss, q);
                if (e != 0) {
                    pr = var();
                    o << ind << "const F2 " << pr << " = kf2_mul1(" << fconst(std::ldexp(1.0, e)) << ", " << ring(simg, ss, q)
                      << ");\n";
                }
                sk[2 * q] = pr + ".x";
                sk[2 * q + 1] = pr + ".y";
            }
        }
        if (!store) {
            o << ind << "{\n";
        } else if (runptr) {
            o << ind << "if (xst && (unsigned)(" << uexpr << " + " << j - 2 * L << ") < (unsigned)(ye - ys)) {\n";
            orow = "op";
        } else {
            o << ind << "const int yp = ys - " << 2 * L << " + " << uexpr << " + " << j << ";\n";
            o << ind << "if (xst && yp >= ys && yp < ye) {\n";
            o << ind << "    const int yo = " << (dir > 0 ? "yp" : "H - 1 - yp") << ";\n";
            orow = "gout + yo * W";
        }
        if (!store) {
        } else if (!si.vec) {
            for (int v = 0; v < V; v++) {
                std::string val = f32 ? (pm ? sk[v] : ring(simg, ss, v))
                                      : si.swk.count(b.sink) ? ring(simg, ss, v)
                                                             : "kf_pack(" + val_memo[std::make_tuple(simg, ss, v)] + ")";
                o << ind << "    if (x + " << v << " < a.fx1 && KF_WOK(&(" << orow << ")[" << v << "], 4)) (" << orow << ")["
                  << v << "] = " << val << ";\n";
            }
        } else if (f32) {
            for (int k = 0; k < NQ; k++) {
                o << ind << "    kf_st4f(" << orow << (k ? " + " + std::to_string(4 * k) : "");
                for (int v = 4 * k; v < 4 * k + 4; v++) o << ", " << (pm ? sk[v] : ring(simg, ss, v));
                o << ");\n";
            }
        } else {
            for (int k = 0; k < NQ; k++) {
                o << ind << "    kf_st4u(" << orow << (k ? " + " + std::to_string(4 * k) : "");
                for (int v = 4 * k; v < 4 * k + 4; v++)
                    o << ", " << (si.swk.count(b.sink) ? ring(simg, ss, v) : "kf_pack(" + val_memo[std::make_tuple(simg, ss, v)] + ")");
                o << ");\n";
            }
        }
        o << ind << "}\n";
        if (runptr) o << ind << "op += dW;\n";
        // age every ring: by one row after a peeled iteration (by T after the
        // last one, which hands over to the first trip: there a row of age a sits
        // at slot a + T - 1), by T rows after the last body copy of a rolled trip
        const int shift = !si.rolled ? 0 : u >= 0 ? (u == peel_Q - 1 ? si.T : 1) : (j == si.T - 1 ? si.T : 0);
        if (shift) {
            std::set<int> imgs(b.ext.begin(), b.ext.end());
            for (int k : b.kernels) imgs.insert(p->n_inputs + k);
            for (int img : imgs)
                for (int a = ring_len(img) - 1; a >= shift; a--)
                    for (int v = 0; v < NRi(img); v++)
                        o << ind << ring(img, a, v) << " = " << ring(img, a - shift, v) << ";\n";
        }
        o << ind.substr(2) << "}\n";
    }

    static std::string vname(int dir, bool ve, bool l, bool r)
    {
        return std::string("_") + (dir > 0 ? "d" : "u") + (ve ? "e" : "i") + (l ? "L" : "") + (r ? "R" : "");
    }

    // One variant: direction, vertical edge at the strip start, left/right edge chunk.
    void variant(int dir_, bool ve, bool l, bool r)
    {
        dir = dir_;
        el = l;
        er = r;
        // TMA row feed (option tma): interior chunks only -- an edge chunk clamps
        // its lanes' columns, so its row segment is not one contiguous copy
        tma = si.sring && si.vec && si.tma && !l && !r;
        const int P = si.P, D = si.D, L = si.L, HL = si.HL;
        o << "__device__ __forceinline__ void " << kernel_name(block) << "_fast" << vname(dir, ve, l, r)
          << "(const KfArgs &a, const int chunk, const int strip)\n{\n";
        o << "    const int lane = threadIdx.x & 31;\n";
        // this warp's private ring (and TMA barriers) in the CTA's shared buffer (option cta_warps)
        if (si.sring) {
            if (si.nw > 1)
                o << "    const int wslot = (threadIdx.x >> 5) * " << si.warp_smem << ";\n";
            else
                o << "    constexpr int wslot = 0;\n";
        }
        // The image size is fixed per pipeline (one iteration space):
        // baked in, row strides become immediates and unrolled rows use address offsets.
        if (opt(p, "const_w"))
            o << "    constexpr int W = " << p->W << ", H = " << p->H << ";\n    (void)H;\n";
        else
            o << "    const int W = a.W, H = a.H;\n    (void)H;\n";
        o << "    const int x = a.fx0 + (chunk * " << 32 - 2 * HL << " + lane - " << HL << ") * " << V << ";\n";
        o << "    const bool xst = lane >= " << HL << " && lane < " << 32 - HL << " && x < a.fx1;\n";
        // strip bounds in primed (streaming-direction) rows
        // balanced strips: strip i covers rows [fy0 + i*Hf/ns, fy0 + (i+1)*Hf/ns)
        o << "    const int Hf = a.fy1 - a.fy0;\n";
        // two strip heights (tail split): strip s starts at unit u(s) = 2s for s <= n_long,
        // s + n_long after; Hf is spread over n_strips + n_long units (n_long = 0: balanced)
        o << "    const int nu = a.n_strips + a.n_long;\n";
        o << "    const int u0 = strip <= a.n_long ? 2 * strip : strip + a.n_long;\n";
        o << "    const int u1 = strip + 1 <= a.n_long ? 2 * strip + 2 : strip + 1 + a.n_long;\n";
        o << "    const int ys0 = a.fy0 + (int)((long long)u0 * Hf / nu);\n";
        o << "    const int ye0 = a.fy0 + (int)((long long)u1 * Hf / nu);\n";
        if (dir > 0) {
            o << "    const int ys = ys0, ye = ye0;\n";
        } else {
            o << "    const int ys = H - ye0, ye = H - ys0;\n";
        }
        o << "    const int nit = ye - ys + " << 2 * L << ";\n";
        if (si.vec) {
            o << "    const int xl = min(max(x, 0), W - " << V << ");\n";
        } else {
            o << "    const int xl = 0;\n";
            for (int v = 0; v < V; v++) o << "    const int cl" << v << " = min(max(x + " << v << ", 0), W - 1);\n";
        }
        for (int img : b.ext) {
            int s = slot.at(img);
            o << "    const " << RT() << " *__restrict__ g" << s << " = (const " << RT() << " *)a.img[" << s
              << "] + xl - a.base[" << s << "] * W;\n";
        }
        std::set<int> imgs(b.ext.begin(), b.ext.end());
        for (int k : b.kernels) imgs.insert(p->n_inputs + k);
        for (int img : imgs) {
            o << "    " << RDT();
            bool first = true;
            for (int s = 0; s < ring_len(img); s++)
                for (int v = 0; v < NRi(img); v++) {
                    o << (first ? " " : ", ") << ring(img, s, v) << (pm ? " = kf2(0.0f)" : " = 0");
                    first = false;
                }
            o << ";\n";
        }
        // Interior strips (downward, not at an image edge) read rows
        // [ys - L, ye + L) of an image needed with the full halo L, which the
        // launch geometry keeps inside [base, rlast]: no clamps, one running
        // pointer from the first prologue row on.
        prp.clear();
        if (si.sring && !ve && dir > 0 && opt(p, "pro_rp"))
            for (int img : b.ext)
                if (HY(img) == L) prp.insert(img);
        if (!prp.empty()) {
            o << "    const int dW = W;\n";
            for (int img : prp) {
                int s = slot.at(img);
                o << "    const " << RT() << " *__restrict__ ip" << s << " = g" << s << " + (ys - " << 2 * L - HY(img)
                  << ") * W;\n";
            }
        }
        if (si.sring) {
            for (int img : b.ext) {
                int s = slot.at(img);
                o << "    " << (f32 ? "float4" : "uint4") << " *sr" << s << " = (" << (f32 ? "float4" : "uint4")
                  << " *)(" << kernel_name(block) << "_smem + " << s * si.DS * 512 * NQ << " + wslot) + lane * " << NQ << ";\n";
            }
            for (auto &kv : si.delay)   // shared-memory delay lines (stream_info)
                o << "    uint4 *dl" << kv.first << " = (uint4 *)(" << kernel_name(block) << "_smem + "
                  << si.delay_off.at(kv.first) << " + wslot) + lane;\n";
            if (tma) {
                // one mbarrier per (image, ring slot) after the rings.  The warp's
                // row segment is lanes 0..31's columns [x0w, x0w + 32V) clipped to
                // the image (W % 4 == 0, x0w % 4 == 0: 16-B multiples); lane 0's row
                // pointer already starts at the clipped column max(x0w, 0), which
                // lands at byte toff of the slot.  Lanes wholly outside the image
                // keep stale ring data: they are halo lanes no stored pixel reads.
                o << "    unsigned long long *mb = (unsigned long long *)(" << kernel_name(block) << "_smem + wslot + "
                  << si.ring_bytes << ");\n";
                o << "    const int x0w = a.fx0 + (chunk * " << 32 - 2 * HL << " - " << HL << ") * " << V << ";\n";
                o << "    const unsigned toff = (unsigned)(max(x0w, 0) - x0w) * 4u;\n";
                o << "    const unsigned tb = (unsigned)(min(x0w + " << 32 * V << ", W) - max(x0w, 0)) * 4u;\n";
                o << "    if (lane == 0) {\n";
                o << "        for (int i = 0; i < " << (int)b.ext.size() * si.DS << "; i++) kf_mbar_init(mb + i, 1);\n";
                o << "        kf_mbar_init_fence();\n";
                o << "    }\n";
                o << "    __syncwarp();\n";
            }
            for (int it = 0; it < si.DS - 1; it++) {
                for (int img : b.ext) issue(img, std::to_string(it), std::to_string(it), "    ");
                if (!tma) o << "    kf_cp_commit();\n";
            }
            if (si.lpf) {
                if (tma)
                    wait_row("0", "0", "0", "    ");
                else
                    o << "    kf_cp_wait<" << si.DS - 2 << ">();\n";
                for (int img : b.ext) {
                    int s = slot.at(img);
                    for (int k = 0; k < NQ; k++)
                        o << "    " << (f32 ? "float4" : "uint4") << " pf" << s << "_" << k << " = sr" << s << "[" << k << "];\n";
                }
            }
            o << "    int qb = 0;   // ring slot of the current iteration's row (multiple of the unroll)\n";
            if (tma) o << "    unsigned ph = 0;   // phase parity of ring slot qb's current row\n";
        } else {
            for (int it = 0; it < D; it++)
                for (int img : b.ext) load(img, si.rolled ? D - it : it % P, std::to_string(it), "    ");
        }
        o << "    " << RT() << " *__restrict__ gout = (" << RT() << " *)a.out + x - a.out_base * W;\n";
        int u0 = 0;
        // peeled iterations: the 2L warm-up iterations (only the kernels whose rows
        // are needed run) and, at an image edge, those in which some tap row lies
        // beyond the edge (remapped statically)
        // option peel_warmup = 0: an unrolled body runs its 2L warm-up iterations
        // through the loop itself (every kernel computed, stores masked) instead
        // of a peeled prologue that computes only the kernels already needed --
        // more arithmetic, less straight-line code (edge strips still peel)
        int need = si.rolled || !opt(p, "peel_warmup") ? 0 : 2 * L;
        vedge = ve;
        if (ve)
            for (int k : b.kernels)
                if (p->ops[k].kind == LOCAL)
                    need = std::max(need, 2 * L - HY(p->n_inputs + k) + p->ops[k].ry());
        if (need > 0) {
            // rolled: a multiple of T, so that the ring slot qb + j of a trip stays below DS
            const int Q = si.rolled ? (need + si.T - 1) / si.T * si.T : (need + P - 1) / P * P;
            peel_Q = Q;
            for (int u = 0; u < Q; u++) {
                if (si.rolled)   // peeled rolled iterations are body copy T-1 (newest row at slot 0)
                    iteration(si.T - 1, u, std::to_string(u - (si.T - 1)), "      ");
                else
                    iteration(u % P, u, std::to_string(u - u % P), "      ");
            }
            u0 = Q;
            if (si.sring) o << "    qb = " << Q % si.DS << ";\n";
            if (tma) o << "    ph = " << ((Q / si.DS) & 1) << ";\n";
        }
        vedge = false;
        const int step = si.rolled ? si.T : P;
        // steady state: running pointers for the next row to fetch into the ring and
        // the next output row (valid when the ring is deep enough that every row it
        // fetches after the prologue lies inside [base, rlast])
        const bool rp_ok = si.sring && si.DS - 1 >= 2 * L;
        if (rp_ok) {
            if (prp.empty()) o << "    const int dW = " << (dir > 0 ? "W" : "-W") << ";\n";
            for (int img : b.ext) {
                if (prp.count(img)) continue;   // already positioned at row u0 + DS - 1
                int s = slot.at(img);
                std::string row = row_of(img, std::to_string(u0 + si.DS - 1), "    ");
                o << "    const " << RT() << " *__restrict__ ip" << s << " = g" << s << " + " << row << " * W;\n";
            }
            std::string yp0 = "(ys - " + std::to_string(2 * L - u0) + ")";
            o << "    " << RT() << " *__restrict__ op = gout + " << (dir > 0 ? yp0 : "(H - 1 - " + yp0 + ")") << " * W;\n";
            runptr = true;
        }
        loop_u0 = u0;
        if (si.rolled) {
            const int T = si.T;
            // warm_skip = 2: the iterations before every kernel is needed run in
            // a loop of their own (guarded groups), so the
            // steady-state loop carries no guards
            int wend = u0;
            if (opt(p, "warm_skip") == 2) {
                for (int k : b.kernels) wend = std::max(wend, 2 * L - 2 * HY(p->n_inputs + k));
                wend = u0 + (wend - u0 + T - 1) / T * T;
            }
            auto rolled_loop = [&](const std::string &hi, int guard_u0) {
                loop_u0 = guard_u0;
                o << "    #pragma unroll 1\n";
                o << "    for (; u < " << hi << "; u += " << T << ") {\n";
                if (si.sring) o << "        const int qprev = qb == 0 ? " << si.DS - 1 << " : qb - 1;\n";
                if (si.lpf) o << "        const int qnext = qb + " << T << " == " << si.DS << " ? 0 : qb + " << T << ";\n";
                for (int j = 0; j < T; j++) iteration(j, -1, "u", "        ");
                if (si.sring)
                    o << "        qb += " << T << ";\n        if (qb == " << si.DS << ") { qb = 0;" << (tma ? " ph ^= 1u;" : "")
                      << " }\n";
                o << "    }\n";
            };
            o << "    int u = " << u0 << ";\n";
            if (wend > u0) rolled_loop("min(nit, " + std::to_string(wend) + ")", u0);
            rolled_loop("nit", wend);
            o << "}\n\n";
            runptr = false;
            return;
        } else {
            o << "    for (int u = " << u0 << "; u < nit; u += " << P << ") {\n";
            if (si.sring) o << "        const int qprev = qb == 0 ? " << si.DS - 1 << " : qb - 1;\n";
            if (si.lpf) o << "        const int qnext = qb + " << P << " == " << si.DS << " ? 0 : qb + " << P << ";\n";
            qptr = si.sring && opt(p, "qptr");
            if (qptr)
                for (int img : b.ext) {
                    const int s = slot.at(img);
                    const char *T = f32 ? "float4" : "uint4";
                    o << "        " << T << " *const sq" << s << " = sr" << s << " + qb * " << 32 * NQ << ";\n";
                    o << "        " << T << " *const sp" << s << " = sr" << s << " + qprev * " << 32 * NQ << ";\n";
                    if (si.lpf) o << "        " << T << " *const sn" << s << " = sr" << s << " + qnext * " << 32 * NQ << ";\n";
                }
            for (int j = 0; j < P; j++) iteration(j, -1, "u", "        ");
            qptr = false;
        }
        if (si.sring)
            o << "        qb += " << step << ";\n        if (qb == " << si.DS << ") { qb = 0;" << (tma ? " ph ^= 1u;" : "")
              << " }\n";
        o << "    }\n}\n\n";
        runptr = false;
    }

    void run()
    {
        for (size_t i = 0; i < b.ext.size(); i++) slot[b.ext[i]] = (int)i;
        pm = f32 && opt(p, "pairs");
        defer_ok = opt(p, "defer");

        // Variants (the variant is CTA-uniform):
        //   interior strip, interior chunk   -- the hot loop, no border logic
        //   interior strip, edge chunk       -- + lane selects at x == 0 / x == W-4
        //   top edge strip (downward)        -- + peeled remapped prologue, selects
        //   bottom edge strip (upward)       -- same in flipped row order
        const bool hsel = si.edge_l || si.edge_r;
        variant(1, false, false, false);
        if (hsel) variant(1, false, si.edge_l, si.edge_r);
        if (si.edge_v) {
            variant(1, true, si.edge_l, si.edge_r);
            variant(-1, true, si.edge_l, si.edge_r);
        }
        o << "__device__ __forceinline__ void " << kernel_name(block) << "_fast(const KfArgs &a, const int item)\n{\n";
        if (opt(p, "heavy_first")) {
            // heavy items first: the edge strips (longer peeled prologues) and the
            // edge chunks (lane selects) start in the first wave instead of
            // forming the tail of the last one
            o << "    const int s0 = item / a.n_chunks, c0 = item % a.n_chunks;\n";
            o << "    const int strip = a.edge_b ? (a.edge_t ? (s0 == 0 ? 0 : s0 == 1 ? a.n_strips - 1 : s0 - 1)\n"
                 "                                      : (s0 == 0 ? a.n_strips - 1 : s0 - 1)) : s0;\n";
            o << "    const int chunk = a.edge_r ? (a.edge_l ? (c0 == 0 ? 0 : c0 == 1 ? a.n_chunks - 1 : c0 - 1)\n"
                 "                                      : (c0 == 0 ? a.n_chunks - 1 : c0 - 1)) : c0;\n";
        } else {
            o << "    const int chunk = item % a.n_chunks, strip = item / a.n_chunks;\n";
        }
        if (si.edge_v) {
            o << "    if (a.edge_t && strip == 0) { " << kernel_name(block) << "_fast" << vname(1, true, si.edge_l, si.edge_r)
              << "(a, chunk, strip); return; }\n";
            o << "    if (a.edge_b && strip == a.n_strips - 1) { " << kernel_name(block) << "_fast"
              << vname(-1, true, si.edge_l, si.edge_r) << "(a, chunk, strip); return; }\n";
        }
        if (hsel)
            o << "    if ((a.edge_l && chunk == 0) || (a.edge_r && chunk == a.n_chunks - 1)) { " << kernel_name(block)
              << "_fast" << vname(1, false, si.edge_l, si.edge_r) << "(a, chunk, strip); return; }\n";
        o << "    " << kernel_name(block) << "_fast" << vname(1, false, false, false) << "(a, chunk, strip);\n";
        o << "}\n\n";
    }
};

}  // namespace

// ------------------------------------------------------------ block analysis

// Rank-1 factorisation m[j][i] = col[j] * row[i], exact in double.  Integer
// masks (u8x4) get integer factors (primitive row vector), float masks that
// are integers times a power of two get the same factors with the scale folded
// into the row (e.g. Gaussian/16 = [1,2,1] (x) [1,2,1]/16, exact in float32).
static Separable factor(const Op &op, bool integer)
{
    Separable s;
    const int mw = op.mw, mh = op.mh;
    double scale = 1.0;
    bool ints = true;
    for (double v : op.mask) ints &= std::floor(v) == v && std::fabs(v) < 1e9;
    if (!ints && !integer) {
        for (int e = 1; e <= 24 && !ints; e++) {
            scale = std::ldexp(1.0, -e);
            ints = true;
            for (double v : op.mask) {
                double w = v / scale;
                ints &= std::floor(w) == w && std::fabs(w) < 1e9;
            }
        }
        if (!ints) scale = 1.0;
    }
    if (!ints) return s;   // general float masks: direct 2-D taps (exact float order not needed, but keep simple)
    std::vector<long long> A(op.mask.size());
    for (size_t q = 0; q < A.size(); q++) A[q] = (long long)(op.mask[q] / scale);
    int jr = -1;
    for (int j = 0; j < mh && jr < 0; j++)
        for (int i = 0; i < mw; i++)
            if (A[(size_t)j * mw + i] != 0) { jr = j; break; }
    if (jr < 0) return s;
    long long g = 0;
    for (int i = 0; i < mw; i++) g = std::gcd(g, std::llabs(A[(size_t)jr * mw + i]));
    std::vector<long long> row(mw), col(mh);
    int ip = -1;
    for (int i = 0; i < mw; i++) {
        row[i] = A[(size_t)jr * mw + i] / g;
        if (row[i] != 0 && ip < 0) ip = i;
    }
    if (row[ip] < 0)
        for (auto &r : row) r = -r;
    for (int j = 0; j < mh; j++) {
        long long a = A[(size_t)j * mw + ip];
        if (a % row[ip] != 0) return s;
        col[j] = a / row[ip];
    }
    for (int j = 0; j < mh; j++)
        for (int i = 0; i < mw; i++)
            if (col[j] * row[i] != A[(size_t)j * mw + i]) return s;
    // sign: prefer the factor with more positive coefficients in the column
    int neg = 0, pos = 0;
    for (long long c : col) { neg += c < 0; pos += c > 0; }
    if (neg > pos) {
        for (auto &c : col) c = -c;
        for (auto &r : row) r = -r;
    }
    s.ok = true;
    s.scale = scale;
    // the power-of-two scale goes to the column factor: the vertical pass runs
    // on packed pixel pairs, the horizontal one per pixel, so the horizontal
    // pass keeps its unit coefficients (one multiply fewer per pixel)
    for (int j = 0; j < mh; j++) s.col.push_back((double)col[j] * scale);
    for (int i = 0; i < mw; i++) s.row.push_back((double)row[i]);
    return s;
}

// Schedule options.  They change how the same arithmetic is
// scheduled -- code shape, feed, launch geometry -- never its result: every
// option is covered by a GPU test that checks the output is bit-identical to
// the default.  Set per pipeline through kf_set_option (no environment
// variable reaches the library).  The measured-and-rejected alternatives
// (v8, persist, persist_waves, nlong) exist only in the KF_EXPERIMENTAL build.
namespace {
struct OptDef { const char *name; long long dflt, lo, hi; bool experimental; };
const OptDef kOpts[] = {
    {"swar", 1, 0, 1, false},           // u8x4 kernels in SWAR form (§5.2b)
    {"swring", 1, 0, 1, false},         // unpacked SWAR rings
    {"swring_cap", 164, 0, 1024, false},
    {"pairs", 1, 0, 1, true},           // f32 packed pixel pairs (FFMA2/FADD2); off changes rounding
    {"defer", 1, 0, 1, true},           // deferred power-of-two mask scales; off changes rounding
    {"prefetch", 4, 1, 16, false},      // register prefetch distance (no smem ring)
    {"sring", 1, 0, 1, false},          // cp.async shared-memory row ring
    {"smem_rows", 12, 2, 64, false},    // rows of that ring
    {"lds_pf", 1, 0, 1, false},         // ring rows read one iteration ahead
    {"const_w", 1, 0, 1, false},        // image size baked into the kernel
    {"pro_rp", 1, 0, 1, false},         // running row pointer from the prologue on
    {"qptr", 1, 0, 1, false},           // per-trip ring slot base pointers
    {"heavy_first", 1, 0, 1, false},    // edge items first
    {"code_budget", 12000, 0, 1 << 30, false},   // unrolled vs rolled body
    {"peel_warmup", 1, 0, 1, false},    // unrolled bodies peel the 2L warm-up iterations
    {"rtrip", 1, 1, 2, false},          // rows per trip of a rolled body (2: half the ring moves, but
                                        // twice the loop code: measured slower, instruction fetch stalls)
    {"rolled_edge_v", 1, 0, 1, false},  // rolled bodies keep the edge strips
    {"minctas", kMinCtasPerSm, 1, 32, false},    // __launch_bounds__ min CTAs per SM
    {"nstrips", 0, 0, 1 << 20, false},  // force the strip count (0 = cost model)
    {"host_taper", 1, 0, 1, false},     // kf_run_host thin first/last bands
    {"host_bands", 8, 1, 32, false},    // kf_run_host row bands (pipeline depth)
    {"host_async_bands", 2, 1, 32, false},   // kf_run_host_async row bands
    {"host_direct", 0, 0, 1, false},    // kf_run_host: kernels access pinned+mapped host buffers directly
    {"tma", 0, 0, 1, false},            // interior rows fed by TMA bulk copies + mbarriers (§5.5)
    {"cta_warps", 1, 1, 8, false},      // interior warps (items) per CTA (frame tiles use all of them)
    {"delay_smem", 1, 0, 1, false},     // rolled u8x4 bodies: far point-read rows from shared-memory delay lines
    {"lut_smem", 1, 0, 1, false},       // SWAR table gathers from a shared-memory copy of the table
    {"warm_skip", 2, 0, 2, false},      // rolled bodies: warm-up rows skip kernels not yet needed (1: guards in the loop, 2: own loop)
    {"pdl", 2, 0, 2, false},            // kf_run kernels launched as programmatic dependents (the CTA
                                        // launch overlaps the previous kernel's tail): 0 off, 1 all,
                                        // 2 unrolled blocks (rolled C4 measured slower)
    {"v8", 0, 0, 1, true},              // 8 pixels per lane (rejected, §5.4)
    {"persist", 0, 0, 1, true},         // persistent CTAs (rejected)
    {"persist_waves", 1, 1, 1 << 20, true},
    {"nlong", 0, 0, 1 << 20, true},     // tail split (rejected)
    {"cluster", 1, 1, 8, true},         // thread-block clusters of this many CTAs (CTA-dispatch experiment)
    // NEGATIVE CONTROL ONLY: settable in libkfuse_testhooks.so (KF_TEST_HOOKS),
    // never in the product library, where it is always 0.  The frame path then
    // evaluates in-block producers on the padded plane instead of remapping each
    // consumer tap -- the "pad once" fusion of Fig. 4b, which is WRONG at the
    // border.  Tests assert it fails parity.
    {"naive_border", 0, 0, 1, true},
    // BOUNDS-CHECKING BUILD ONLY (libkfuse_bounds.so): the writable span of each
    // launch loses its last output row, so the checker must report writes --
    // its self-test.  The skipped row is then left unwritten.
    {"bounds_shrink", 0, 0, 1, true},
};
#ifdef KF_EXPERIMENTAL
constexpr bool kExperimental = true;
#else
constexpr bool kExperimental = false;
#endif
#ifdef KF_TEST_HOOKS
constexpr bool kTestHooks = true;
#else
constexpr bool kTestHooks = false;
#endif
#ifdef KF_BOUNDS
constexpr bool kBounds = true;
#else
constexpr bool kBounds = false;
#endif
const OptDef *find_opt(const char *name)   // settable options of this build
{
    for (const OptDef &d : kOpts)
        if (!std::strcmp(d.name, name)) {
            if (!std::strcmp(name, "naive_border")) return kTestHooks ? &d : nullptr;
            if (!std::strcmp(name, "bounds_shrink")) return kBounds ? &d : nullptr;
            return (d.experimental && !kExperimental) ? nullptr : &d;
        }
    return nullptr;
}
}  // namespace

long long opt(const kf_pipeline *p, const char *name)
{
    const OptDef *d = find_opt(name);
    if (!d) {
        for (const OptDef &e : kOpts)
            if (!std::strcmp(e.name, name)) return e.dflt;   // experimental option, not built in
        fail(KF_ERR_ARG, std::string("internal: unknown option ") + name);
    }
    auto it = p->options.find(name);
    return it == p->options.end() ? d->dflt : it->second;
}

void set_option(kf_pipeline *p, const char *name, long long value)
{
    const OptDef *d = name ? find_opt(name) : nullptr;
    if (!d) fail(KF_ERR_ARG, std::string("unknown option '") + (name ? name : "(null)") + "'");
    if (value < d->lo || value > d->hi)
        fail(KF_ERR_ARG, std::string("option '") + name + "' out of range [" + std::to_string(d->lo) + ", " +
                             std::to_string(d->hi) + "]");
    p->options[name] = value;
}

long long get_option(const kf_pipeline *p, const char *name)
{
    if (!name || !find_opt(name)) fail(KF_ERR_ARG, std::string("unknown option '") + (name ? name : "(null)") + "'");
    return opt(p, name);
}

// Code-size weight of a program: SASS instructions its opcodes expand to
// (accurate libdevice powf / logf / expf / sqrtf / division are inline
// sequences of tens of instructions; fitted to cuobjdump counts on sm_100a).
static int prog_size(const Op &op)
{
    int n = 0;
    for (const Instr &in : op.prog) n += std::max(1, op_issue_slots(in.op));   // LOAD/CONST count 1 here
    return n;
}

StreamInfo stream_info(const kf_pipeline *p, const BlockInfo &b)
{
    StreamInfo si;
    // f32 blocks may run 8 pixels per lane (two float4 per row per lane):
    // half the shuffles and per-row overhead per pixel, twice the ring registers
    si.V = (p->dtype == KF_F32 && opt(p, "v8")) ? 8 : kStreamV;
    const int kV_ = si.V;
    si.vec = p->W % kV_ == 0;
    for (int img : b.ext) si.hy[img] = b.ext_hy.at(img);
    for (int k : b.kernels) si.hy[p->n_inputs + k] = b.hy.at(k);
    si.L = b.Ry;
    si.HL = std::max(1, (b.Rx + kV_ - 1) / kV_);
    // history depth of every image, in iterations
    int maxdepth_ext = 1, maxdepth = 1;
    for (auto &kv : si.hy) si.depth[kv.first] = 1;
    for (int k : b.kernels) {
        const Op &op = p->ops[k];
        const int img = p->n_inputs + k;
        for (int in : op.inputs) {
            int d = si.hy[in] - si.hy[img] + op.ry() + 1;
            si.depth[in] = std::max(si.depth[in], d);
        }
        if (op.kind == LOCAL) si.sep[k] = factor(op, p->dtype != KF_F32);
        if (p->dtype == KF_U8X4 && opt(p, "swar") &&
            swar_feasible(op, op.kind == LOCAL ? si.sep[k] : Separable{}))
            si.swk.insert(k);
    }
    for (auto &kv : si.depth) {
        bool ext = std::binary_search(b.ext.begin(), b.ext.end(), kv.first);
        (ext ? maxdepth_ext : maxdepth) = std::max(ext ? maxdepth_ext : maxdepth, kv.second);
    }
    // input feed: a cp.async shared-memory ring of DS rows per external image
    // (128-bit rows), else register prefetch D iterations ahead.  Ring period
    // P >= every depth (+ D for register-prefetched external images).
    si.D = (int)opt(p, "prefetch");
    si.sring = si.vec && opt(p, "sring") && !b.ext.empty();
    if (si.sring) {
        si.P = std::max(maxdepth, maxdepth_ext);
        const int want = (int)opt(p, "smem_rows");
        const int cap = 32768 / (128 * kV_ * (int)b.ext.size());   // <= 32 KB of ring per warp
        int DS = std::max(want, si.P + 1);
        DS = (DS + si.P - 1) / si.P * si.P;
        while (DS > cap && DS - si.P >= si.P + 1) DS -= si.P;
        if (DS > cap || DS < 2) si.sring = false;
        si.DS = DS;
        si.ring_bytes = (int)b.ext.size() * DS * 128 * kV_;
        si.lpf = si.sring && DS >= 3 && opt(p, "lds_pf");
        si.tma = si.sring && opt(p, "tma");
    }
    if (!si.sring) si.P = std::max(maxdepth, maxdepth_ext + si.D);
    // code size: scalar operations of one iteration (one body copy)
    long long ops = 0;
    for (int k : b.kernels) {
        const Op &op = p->ops[k];
        const int ch = p->dtype == KF_F32 ? 1 : si.swk.count(k) ? 2 : 4;   // SWAR: two channels per op
        if (op.kind == LOCAL) {
            int nnz = 0;
            for (double m : op.mask) nnz += m != 0.0;
            const Separable &sp = si.sep.at(k);
            int taps = sp.ok ? (int)(std::count_if(sp.col.begin(), sp.col.end(), [](double c) { return c != 0.0; }) +
                                     std::count_if(sp.row.begin(), sp.row.end(), [](double c) { return c != 0.0; }))
                             : nnz;
            ops += (long long)(taps + 2 * op.rx() + prog_size(op)) * kV_ * ch;
        } else {
            ops += (long long)prog_size(op) * kV_ * ch;
        }
    }
    si.iter_ops = ops;
    // unrolled: ~P copies per variant (4 variants + 2 peeled prologues); too
    // much straight-line code for NVRTC/ptxas and the instruction cache ->
    // one rolled body copy
    const long long budget = opt(p, "code_budget");
    si.rolled = ops * si.P * 6 > budget;
    // rows per rolled trip (option rtrip): 2 halves the ring-shift moves; the
    // shared-memory ring then holds a multiple of T rows (slot qb + j < DS)
    si.T = si.rolled && si.sring ? (int)opt(p, "rtrip") : 1;
    if (si.T > 1) {
        while (si.DS % si.T) si.DS += si.P;
        if (si.DS % si.T) si.DS = si.DS * si.T;
        si.ring_bytes = (int)b.ext.size() * si.DS * 128 * kV_;
    }
    // Shared-memory delay lines (option delay_smem): in a rolled
    // body every ring row is a register shifted by a move each iteration.  An
    // image whose deepest rows are read only by SWAR point kernels (a value
    // carried to the sink row: deep10's input for k7/k9, k0 for k8) keeps only
    // the rows its local consumers' windows read in registers; the older rows
    // come from a per-warp shared-memory line of S rows (packed, 16 B per lane,
    // row of iteration t in slot t mod S).  Fewer moves and registers, which
    // lets the next ring stay unpacked under the register cap.
    if (p->dtype == KF_U8X4 && si.rolled && si.T == 1 && si.sring && !si.tma && opt(p, "delay_smem")) {
        int off = si.ring_bytes;
        for (auto &kv : si.depth) {
            const int img = kv.first, full = kv.second;
            if (img == p->n_inputs + b.sink) continue;
            const bool ext = std::binary_search(b.ext.begin(), b.ext.end(), img);
            if (!ext && !si.swk.count(img - p->n_inputs)) continue;   // SWAR producer (packed row at hand)
            int wdepth = 1;
            bool ok = true;
            for (int k : b.kernels) {
                const Op &op = p->ops[k];
                if (std::find(op.inputs.begin(), op.inputs.end(), img) == op.inputs.end()) continue;
                if (!si.swk.count(k)) ok = false;   // far rows are read through the SWAR path only
                if (op.kind == LOCAL) wdepth = std::max(wdepth, si.hy[img] - si.hy[p->n_inputs + k] + op.ry() + 1);
            }
            if (!ok || full - wdepth < 2) continue;
            int S = 1;
            while (S < full) S *= 2;
            si.delay[img] = S;
            si.delay_off[img] = off;
            off += S * 32 * 16;
            kv.second = wdepth;
        }
        si.ring_bytes = off;
    }
    // register estimate: live ring values (depth per image, D prefetched rows)
    int live = 0;
    for (auto &kv : si.depth) {
        bool ext = std::binary_search(b.ext.begin(), b.ext.end(), kv.first);
        live += (kv.second + (ext && !si.sring ? si.D : 0)) * kV_;
    }
    // SWAR rings: a u8x4 image read at several rows per
    // iteration by SWAR local kernels keeps its ring unpacked -- (lo, hi) per
    // pixel, written once -- instead of packed uchar4 re-unpacked (2 PRMT per
    // pixel) at every row use.  Costs depth x V more registers; deepest first,
    // under a cap on the live ring registers.
    const int live_packed = live;
    if (p->dtype == KF_U8X4 && opt(p, "swring")) {
        const int cap = (int)opt(p, "swring_cap");
        std::vector<std::pair<int, int>> cand;   // (depth, image)
        for (auto &kv : si.depth) {
            const int img = kv.first;
            if (img == p->n_inputs + b.sink || kv.second < 3) continue;
            const bool ext = std::binary_search(b.ext.begin(), b.ext.end(), img);
            if (!ext && si.delay.count(img)) continue;   // its delay line stores the packed row
            if (!ext && !si.swk.count(img - p->n_inputs)) continue;   // producer must be SWAR (or a load)
            bool vert = false;
            for (int k : b.kernels)
                if (si.swk.count(k) && p->ops[k].kind == LOCAL && p->ops[k].ry() >= 1 && p->ops[k].inputs[0] == img)
                    vert = true;
            if (vert) cand.push_back({kv.second, img});
        }
        std::sort(cand.begin(), cand.end(), [](auto &a, auto &b2) { return a.first != b2.first ? a.first > b2.first : a.second < b2.second; });
        for (auto &c : cand) {
            const int extra = c.first * kV_;
            if (live + extra > cap) continue;
            live += extra;
            si.swring.insert(c.second);
        }
    }
    si.live_regs = live;
    // image edges inside the streaming path: not for REPEAT
    // (wrap reads the opposite side), horizontal only when every exterior tap of
    // the edge lane maps into its own 4 pixels
    bool rep = b.torus, hfit = true;
    for (int k : b.kernels) {
        const Op &op = p->ops[k];
        if (op.kind != LOCAL) continue;
        rep |= op.mode == KF_REPEAT;
        hfit &= op.rx() <= (op.mode == KF_MIRROR101 ? kV_ - 1 : kV_);
    }
    si.edge_v = !rep && p->H >= 4 * si.L + 2 * si.P + 8;
    // rolled bodies keep the edge strips too (peeled remapped prologue, then
    // the rolled loop), unless option rolled_edge_v=0 leaves those rows to the
    // frame: for deep10 the frame's index-exchange tiles cost 12 % of the kernel
    if (si.rolled && !opt(p, "rolled_edge_v")) si.edge_v = false;
    si.edge_l = !rep && hfit && p->W >= 4 * kV_;
    si.edge_r = si.edge_l && si.vec;
    si.ok = b.Rx <= 2 * kV_ * 4 && live_packed <= 160 && b.ext.size() <= KF_MAX_IMG_HOST;
    si.warp_smem = (si.ring_bytes + (si.tma ? 8 * (int)b.ext.size() * si.DS : 0) + 15) / 16 * 16;
    // warps per CTA, capped so the CTA's static shared buffer stays within 48 KB
    // shared-memory copies of small tables (option lut_smem) share the CTA's
    // 48 KB of static shared memory with the rings (or the frame tiles)
    int lut_bytes = 0;
    if (opt(p, "lut_smem"))
        for (int k : b.kernels)
            if (!p->ops[k].lut.empty() && p->ops[k].lut.size() <= 1024) lut_bytes += 4 * (int)p->ops[k].lut.size();
    si.nw = std::max(1, std::min((int)opt(p, "cta_warps"), (49152 - lut_bytes) / std::max(si.warp_smem, 1)));
    int frame_bytes = 0;
    for (int k : b.staged) {
        int n = 0;
        for (int s2 = 0; s2 < 2; s2++)
            n = std::max(n, (kFrameTiles[s2][0] + 2 * b.hx.at(k)) * (kFrameTiles[s2][1] + 2 * b.hy.at(k)));
        frame_bytes += n * 4;
    }
    si.lut_smem = lut_bytes > 0 && std::max(frame_bytes, si.nw * si.warp_smem) + lut_bytes <= 49152;
    if (opt(p, "naive_border")) si.ok = false;   // negative control: everything through the (naive) frame
    return si;
}

std::string generate_block(const kf_pipeline *p, const BlockInfo &b, int block)
{
    if (b.ext.size() > KF_MAX_IMG_HOST) fail(KF_ERR_ARG, "block reads more than 16 external images");
    std::ostringstream o;
    StreamInfo si = stream_info(p, b);
    o << "// generated by libkfuse codegen: block " << block << " kernels {";
    for (int k : b.kernels) o << " " << k;
    o << " } sink " << b.sink << (b.torus ? " (torus)" : "") << "; interior path "
      << (si.ok ? "streaming" : "none") << " (P=" << si.P << " D=" << si.D << " HL=" << si.HL << " L=" << si.L
      << " live~" << si.live_regs << " ops~" << si.iter_ops << (si.rolled ? " rolled" : " unrolled") << ")\n";
    o << "#include \"kf_device.cuh\"\n\n";
    for (int k : b.kernels)
        if (!p->ops[k].lut.empty()) {
            o << "__device__ const int kf_lut_" << block << "_" << k << "[" << p->ops[k].lut.size() << "] = {";
            for (size_t i = 0; i < p->ops[k].lut.size(); i++) o << (i ? "," : "") << p->ops[k].lut[i];
            o << "};\n";
            if (lut_in_smem(si, p->ops[k]))
                o << "__shared__ int kf_lutsh_" << block << "_" << k << "[" << p->ops[k].lut.size() << "];\n";
        }
    // one shared buffer per CTA: the frame path's staged tiles OR the interior
    // warp's input row rings (a CTA runs exactly one of the two paths)
    int frame_bytes = 0;
    for (int k : b.staged) {
        int n = 0;
        for (int s = 0; s < 2; s++)
            n = std::max(n, (kFrameTiles[s][0] + 2 * b.hx.at(k)) * (kFrameTiles[s][1] + 2 * b.hy.at(k)));
        frame_bytes += n * 4;
    }
    const int NW = si.nw;   // interior warps per CTA (option cta_warps): one ring each
    const int smem_bytes = std::max(16, std::max(frame_bytes, si.ok && si.sring ? NW * si.warp_smem : 0));
    o << "__shared__ __align__(16) unsigned char " << kernel_name(block) << "_smem[" << smem_bytes << "];\n\n";
    FrameGen fg(p, b, block, o);
    fg.run();
    if (si.ok) {
        StreamGen sg(p, b, si, block, o);
        sg.run();
    }
    o << "extern \"C\" __global__ void __launch_bounds__(" << kThreads * NW << ", "
      << std::max(1, (int)opt(p, "minctas") / NW) << ") " << kernel_name(b, block)
      << "(const __grid_constant__ KfArgs a)\n{\n";
    // Persistent CTAs: the grid is at most one wave of resident CTAs, and each
    // loops over work items (frame tiles first, then interior items) with a
    // grid stride -- no per-item CTA launch.  One warp per CTA: the item index
    // and the trip count are CTA-uniform, so the warp shuffles of the interior
    // path need no convergence barriers.  No cp.async copy is in flight between
    // items (every issued row was waited for), so the shared ring is reused.
    // With NW > 1 warps per CTA a frame unit uses all of them (its loops stride
    // by blockDim), an interior unit gives each warp its own item and ring.
    // Programmatic dependent launch.  Without the launch
    // attribute both instructions are no-ops.  With it: a dependent kernel
    // (indep = 0: kf_run, the first frame of kf_run_batch, every block of a
    // multi-block plan) waits for the previous grid -- its completion and the
    // visibility of its writes -- before the first global access, then lets
    // the next kernel be scheduled.  An independent frame (indep = 1: frames
    // after the first of kf_run_batch, whose buffers the runtime checked to be
    // disjoint) lets the next kernel be scheduled at once and waits for the
    // previous grid only at its end, so its completion still implies the
    // completion of every earlier kernel on the stream.
    o << "    if (!a.indep) asm volatile(\"griddepcontrol.wait;\" ::: \"memory\");\n";
    o << "    asm volatile(\"griddepcontrol.launch_dependents;\");\n";
    bool lut_fill = false;
    for (int k : b.kernels)
        if (lut_in_smem(si, p->ops[k])) {
            const std::string n = std::to_string(p->ops[k].lut.size());
            const std::string kb = std::to_string(block) + "_" + std::to_string(k);
            o << "    for (int i = threadIdx.x; i < " << n << "; i += blockDim.x) kf_lutsh_" << kb << "[i] = kf_lut_" << kb
              << "[i];\n";
            lut_fill = true;
        }
    if (lut_fill) o << "    __syncthreads();\n";
    o << "    const int total = a.frame_ctas + (a.n_items + " << NW - 1 << ") / " << NW << ";\n";
    o << "    for (int cta = blockIdx.x; cta < total; cta += gridDim.x) {\n";
    o << "        if (cta < a.frame_ctas) " << kernel_name(block) << "_frame(a, cta);\n";
    if (si.ok) {
        if (NW == 1) {
            o << "        else " << kernel_name(block) << "_fast(a, cta - a.frame_ctas);\n";
        } else {
            o << "        else {\n";
            o << "            const int item = (cta - a.frame_ctas) * " << NW << " + (int)(threadIdx.x >> 5);\n";
            o << "            if (item < a.n_items) " << kernel_name(block) << "_fast(a, item);\n";
            o << "        }\n";
        }
    }
    o << (NW == 1 ? "        __syncwarp();\n" : "        __syncthreads();\n");
    o << "    }\n";
    o << "    if (a.indep) asm volatile(\"griddepcontrol.wait;\" ::: \"memory\");\n";
    o << "}\n";
    return o.str();
}

}  // namespace kf
