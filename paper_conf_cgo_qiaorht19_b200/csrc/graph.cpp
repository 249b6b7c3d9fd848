// graph.cpp -- the kernel DAG G = (V, E) (§II) and op-IR
// validation.  Vertices are kernels in declaration order; an edge (ks, kd)
// exists when kd reads ks's output image.
#include <cmath>

#include "kf_internal.h"

namespace kf {

static bool is_sfu(int op) { return op == KF_OP_SQRT || op == KF_OP_EXP || op == KF_OP_LOG || op == KF_OP_POW; }

void validate_program(const kf_pipeline *p, const std::vector<Instr> &prog, int n_loads, bool has_lut)
{
    int depth = 0;
    const bool f32 = p->dtype == KF_F32;
    for (size_t i = 0; i < prog.size(); i++) {
        const Instr &in = prog[i];
        int pops = 0, pushes = 1;
        switch (in.op) {
        case KF_OP_LOAD:
            if (in.arg < 0 || in.arg >= n_loads)
                fail(KF_ERR_PROGRAM, "LOAD index " + std::to_string(in.arg) + " out of range");
            break;
        case KF_OP_CONST:
            if (!std::isfinite(in.imm)) fail(KF_ERR_PROGRAM, "CONST must be finite");
            break;
        case KF_OP_ADD: case KF_OP_SUB: case KF_OP_MUL: case KF_OP_DIV: case KF_OP_MIN: case KF_OP_MAX:
            pops = 2; break;
        case KF_OP_ABS: case KF_OP_NEG:
            pops = 1; break;
        case KF_OP_SQRT: case KF_OP_EXP: case KF_OP_LOG:
            if (!f32) fail(KF_ERR_PROGRAM, "SQRT/EXP/LOG need a KF_F32 pipeline");
            pops = 1; break;
        case KF_OP_POW:
            if (!f32) fail(KF_ERR_PROGRAM, "POW needs a KF_F32 pipeline");
            pops = 2; break;
        case KF_OP_SHR: case KF_OP_SHL:
            if (f32) fail(KF_ERR_PROGRAM, "SHR/SHL need a KF_U8X4 pipeline");
            if (in.arg < 0 || in.arg > 30) fail(KF_ERR_PROGRAM, "shift amount out of [0,30]");
            pops = 1; break;
        case KF_OP_SAT_U8:
            if (f32) fail(KF_ERR_PROGRAM, "SAT_U8 needs a KF_U8X4 pipeline");
            pops = 1; break;
        case KF_OP_CLAMP: pops = 3; break;
        case KF_OP_SELECT_GT: pops = 4; break;
        case KF_OP_LUT:
            if (f32) fail(KF_ERR_PROGRAM, "LUT needs a KF_U8X4 pipeline");
            if (!has_lut) fail(KF_ERR_PROGRAM, "LUT used but no table given");
            pops = 1; break;
        default:
            fail(KF_ERR_PROGRAM, "unknown opcode " + std::to_string(in.op));
        }
        if (depth < pops) fail(KF_ERR_PROGRAM, "stack underflow at instruction " + std::to_string(i));
        depth += pushes - pops;
        if (depth > 48) fail(KF_ERR_PROGRAM, "stack deeper than 48");
    }
    if (depth != 1) fail(KF_ERR_PROGRAM, "program must leave exactly one value");
}

// nALU / nSFU default to an opcode count (R-3).
// Issue slots per pixel of one op-IR instruction on sm_100a: 1, except the
// accurate transcendental / division sequences (SASS expansion, fitted to
// cuobjdump counts).  Shared by the code-size estimate (codegen.cpp) and the
// ROOFLINE benefit (planner.cpp, R-20).
int op_issue_slots(int opcode)
{
    switch (opcode) {
    case KF_OP_LOAD: case KF_OP_CONST: return 0;
    case KF_OP_POW: return 80;
    case KF_OP_LOG: return 30;
    case KF_OP_EXP: return 25;
    case KF_OP_SQRT: return 2;   // MUFU.SQRT (kf_sqrt)
    case KF_OP_DIV: return 15;
    default: return 1;
    }
}

void default_cost(const kf_pipeline *, Op &op)
{
    int alu = 0, sfu = 0;
    for (const Instr &in : op.prog) {
        if (in.op == KF_OP_LOAD || in.op == KF_OP_CONST) continue;
        if (is_sfu(in.op)) sfu++;
        else alu++;
    }
    if (op.kind == LOCAL) {
        int nnz = 0;
        for (double v : op.mask) nnz += v != 0.0;
        alu += 2 * std::max(nnz, 1) - 1;
    }
    op.n_alu = alu;
    op.n_sfu = sfu;
}

std::vector<std::vector<int>> producers(const kf_pipeline *p)
{
    std::vector<std::vector<int>> pr(p->ops.size());
    for (size_t kd = 0; kd < p->ops.size(); kd++)
        for (int img : p->ops[kd].inputs)
            if (img >= p->n_inputs) {
                int ks = img - p->n_inputs;
                bool dup = false;
                for (int x : pr[kd]) dup |= x == ks;
                if (!dup) pr[kd].push_back(ks);
            }
    return pr;
}

std::vector<std::vector<int>> consumers(const kf_pipeline *p)
{
    auto pr = producers(p);
    std::vector<std::vector<int>> co(p->ops.size());
    for (size_t kd = 0; kd < p->ops.size(); kd++)
        for (int ks : pr[kd]) co[ks].push_back((int)kd);
    return co;
}

}  // namespace kf
