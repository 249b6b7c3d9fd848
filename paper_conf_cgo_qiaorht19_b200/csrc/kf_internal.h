// kf_internal.h -- host-side data structures of libkfuse (not part of the ABI).
#pragma once

#include <cstdint>
#include <map>
#include <memory>
#include <set>
#include <tuple>
#include <string>
#include <vector>

#include "../../include/kfuse.h"

namespace kf {

// ---- error plumbing: a thrown kf::Error becomes a kf_status at the C boundary
struct Error {
    kf_status st;
    std::string msg;
};
[[noreturn]] void fail(kf_status st, const std::string &msg);
void set_error(const std::string &msg);

struct Instr {
    int op, arg;
    double imm;
};

enum Kind { POINT = 0, LOCAL = 1 };

struct Op {
    Kind kind = POINT;
    std::vector<int> inputs;      // image ids; LOCAL: exactly one
    std::vector<Instr> prog;      // POINT: body; LOCAL: post program on ACC (empty = identity)
    std::vector<int> lut;
    int mw = 0, mh = 0;           // LOCAL mask size (odd)
    std::vector<double> mask;     // row-major mh x mw
    int mode = KF_CLAMP;
    double constant = 0.0;
    int n_alu = 0, n_sfu = 0;     // Eq. 6 costs
    int rx() const { return kind == LOCAL ? mw / 2 : 0; }
    int ry() const { return kind == LOCAL ? mh / 2 : 0; }
};

struct Runtime;   // runtime.cu

}  // namespace kf

struct kf_pipeline {
    int W = 0, H = 0, dtype = KF_F32;
    int n_inputs = 0;
    std::vector<kf::Op> ops;
    std::vector<int> outputs;     // marked output image ids, in marking order
    bool frozen = false;
    kf::Runtime *rt = nullptr;    // owned; created lazily by the runtime
    std::map<std::string, long long> options;   // kf_set_option (schedule options, codegen.cpp)
    ~kf_pipeline();
    int n_images() const { return n_inputs + (int)ops.size(); }
    bool is_kernel_image(int id) const { return id >= n_inputs; }
};

namespace kf {

struct EdgeInfo {
    int ks, kd;
    int scenario;                 // 0 point-based, 1 point-to-local, 2 local-to-local
    double w;                     // benefit incl. gamma, before clamping (Eq. 12)
    bool ctx_legal, profitable;
    int64_t q, eps;               // weight as lexicographic pair
};

struct CutInfo {
    std::vector<int> side;
    int64_t q, eps;
    int phases;
};

// Block analysis shared by code generation and the executor.
struct BlockInfo {
    std::vector<int> kernels;     // ascending kernel ids
    int sink = -1;                // kernel id
    std::vector<int> ext;         // external images read (ascending image ids)
    std::map<int, int> hx, hy;    // halo of each kernel's OUTPUT needed inside the block
    std::map<int, int> ext_hx, ext_hy;  // halo of each external image
    std::set<int> staged;         // kernels consumed by an in-block local kernel
    bool torus = false;           // all local kernels REPEAT: slot model
    int Rx = 0, Ry = 0;           // max external halo
};

struct CompiledBlock;             // runtime.cu
// Memoised launch geometry of one block launch (runtime.cu): the geometry tail
// of the kernel arguments (frame rectangles onward) and the grid size.
struct Geom {
    std::vector<unsigned char> tail;
    unsigned grid = 0;
};
using GeomKey = std::tuple<int, int, int, long long, long long>;   // block, rows [r0, r1), nstrips, nlong

}  // namespace kf

struct kf_plan {
    kf_pipeline *pipe = nullptr;
    std::vector<std::vector<int>> blocks;    // topological (by sink)
    int64_t beta_q = 0, beta_eps = 0;
    std::vector<kf::EdgeInfo> edges;
    std::vector<kf::CutInfo> cuts;
    std::vector<kf::BlockInfo> info;         // per block
    int halo_rows = 0;
    // runtime state (runtime.cu)
    std::vector<std::shared_ptr<kf::CompiledBlock>> compiled;
    std::map<int, void *> workspace;         // image id -> device buffer (cut edges)
    std::map<kf::GeomKey, kf::Geom> geom;    // memoised launch geometry (runtime.cu)
    bool prepared = false;
    ~kf_plan();
};

namespace kf {

// graph.cpp
void validate_program(const kf_pipeline *p, const std::vector<Instr> &prog, int n_loads, bool has_lut);
void default_cost(const kf_pipeline *p, Op &op);
int op_issue_slots(int opcode);                                   // sm_100a issue slots of one op-IR opcode
std::vector<std::vector<int>> consumers(const kf_pipeline *p);   // kernel -> consumer kernels
std::vector<std::vector<int>> producers(const kf_pipeline *p);   // kernel -> producer kernels

// planner.cpp
kf_plan *plan_fusion(kf_pipeline *p, const kf_model_params &m);
kf_plan *plan_basic(kf_pipeline *p, const kf_model_params &m);   // §8(f)3, [12]
kf_plan *plan_exact(kf_pipeline *p, const kf_model_params &m);   // §8(f)4, n <= 16
kf_plan *plan_from_blocks(kf_pipeline *p, std::vector<std::vector<int>> blocks, bool check);
bool dependence_legal(const kf_pipeline *p, const std::set<int> &P);
bool header_legal(const kf_pipeline *p, const std::set<int> &P);
BlockInfo analyse_block(const kf_pipeline *p, const std::vector<int> &kernels);

// codegen.cpp
constexpr int kStreamV = 4;                              // pixels per lane of the interior path
constexpr int kThreads = 32;                             // threads per CTA (both paths): one warp
constexpr int kMinCtasPerSm = 12;                        // __launch_bounds__ min blocks (<= 168 regs)
constexpr int KF_MAX_IMG_HOST = 16;                      // = KF_MAX_IMG of kf_device.cuh
constexpr int kFrameTiles[2][2] = {{32, 8}, {8, 32}};    // frame tile shapes (w, h)

struct Separable {                // rank-1 mask: m[j][i] = col[j] * row[i]
    bool ok = false;
    std::vector<double> col, row;
    double scale = 1.0;           // power-of-two factor folded into col (col / scale are integers)
};

// Interior streaming schedule of one block (codegen.cpp StreamGen)
struct StreamInfo {
    bool ok = false;              // the block has an interior fast path
    int V = 4;                    // pixels per lane of the interior path (4, or 8 for f32 with option v8)
    bool vec = false;             // W % V == 0: 128-bit loads/stores
    int L = 0;                    // rows of lag of the sink behind the newest input row
    int HL = 1;                   // halo lanes per warp side
    int P = 1;                    // ring period = loop body copies
    int D = 4;                    // prefetch distance (iterations)
    int live_regs = 0;            // estimate of ring registers
    bool rolled = false;          // one loop-body copy + ring shifts (big blocks)
    int T = 1;                    // rows per rolled trip (body copies per rolled loop trip)
    int nw = 1;                   // interior warps per CTA (option cta_warps)
    int warp_smem = 0;            // shared-memory bytes of one warp's ring (+ TMA barriers)
    bool sring = false;           // external rows fed by a cp.async shared-memory ring
    int DS = 0;                   // rows in that ring (multiple of P)
    bool lpf = false;             // ring rows read one iteration ahead (LDS latency off the critical path)
    bool tma = false;             // the ring is filled by TMA bulk row copies (option tma)
    int ring_bytes = 0;           // its shared memory per warp
    long long iter_ops = 0;       // scalar operations per iteration (code-size estimate)
    bool edge_v = false;          // top/bottom image edges handled by edge strips
    bool edge_l = false, edge_r = false;   // left/right image edges handled by edge chunks
    std::map<int, int> hy;        // image -> rows needed around the sink row
    std::map<int, int> depth;     // image -> history depth (iterations)
    std::map<int, Separable> sep; // local kernel -> factorisation
    std::set<int> swk;            // u8x4 kernels in SWAR form (two channels per 32-bit op)
    std::set<int> swring;         // u8x4 images whose ring holds the unpacked SWAR (lo, hi) pair
    std::map<int, int> delay;     // u8x4 image -> rows S of its shared-memory delay line (option delay_smem)
    std::map<int, int> delay_off; // image -> byte offset of that line within the warp's shared memory
    bool lut_smem = false;        // small tables gathered from shared-memory copies (option lut_smem)
};

std::string kernel_name(const BlockInfo &b, int block);
long long opt(const kf_pipeline *p, const char *name);          // option value or its default
void set_option(kf_pipeline *p, const char *name, long long value);
long long get_option(const kf_pipeline *p, const char *name);
StreamInfo stream_info(const kf_pipeline *p, const BlockInfo &b);
std::string generate_block(const kf_pipeline *p, const BlockInfo &b, int block);

// runtime.cu
void prepare(kf_pipeline *p, kf_plan *plan);
void run(kf_pipeline *p, kf_plan *plan, const void *const *din, int n_in, void *const *dout, int n_out,
         void *stream, int row0, int row1, int in_row0, int in_row1, bool out_full = false,
         bool indep = false);
void run_batch(kf_pipeline *p, kf_plan *plan, int n_frames, const void *const *din, int n_in,
               void *const *dout, int n_out, void *stream);
void run_host(kf_pipeline *p, kf_plan *plan, const void *const *hin, int n_in, void *const *hout, int n_out,
              void *stream, bool async = false);
void bounds_report(kf_pipeline *p, long long *count, unsigned long long *addr, int *kind);
void release_plan(kf_plan *plan);
void release_runtime(kf_pipeline *p);

}  // namespace kf
