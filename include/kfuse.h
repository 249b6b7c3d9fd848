/*
 * kfuse.h -- C-ABI of the B200 kernel-fusion library (libkfuse.so).
 *
 * Implements the data-parallel hot path of Qiao, Reiche, Hannig, Teich,
 * "From Loop Fusion to Kernel Fusion: A Domain-Specific Approach to Locality
 * Optimization", CGO 2019 (citations are PAPER.md line ranges):
 *
 *   - a pipeline is the paper's kernel DAG G = (V, E): vertices are kernels,
 *     an edge (vi, vj) means vj consumes vi's output; every kernel reads >= 1
 *     image and writes exactly one (PAPER.md:172-184, §II; :197-201 §II-B);
 *   - kernels are point or local operators (§II-C-1);
 *   - kf_plan_fusion runs Alg. 1 (recursive Stoer-Wagner min cut) over the
 *     benefit model of Eqs. 3-12 and the legality rules of §II-B
 *     (PAPER.md:111-510, 717-769);
 *   - kf_run executes every partition block as ONE fused sm_100a kernel whose
 *     result equals the unfused execution exactly (integer) or to float32
 *     rounding (border fusion + index exchange §IV-A/B,
 *     PAPER.md:1061-1133).
 *
 * Conventions (all functions):
 *   - No exceptions cross this boundary.  Every kf_status != KF_OK leaves a
 *     human-readable, thread-local message in kf_last_error().
 *   - Image ids are dense int32 in declaration order: inputs first, then each
 *     kernel's output image (kernel k writes image n_inputs + k).
 *   - Images are dense, row-major, pitch = width * 4 bytes.  Base pointers
 *     must be 16-byte aligned when width % 4 == 0 (128-bit row access), else
 *     4-byte aligned (any row offset of a larger image works):
 *       KF_F32  : one float32 per pixel (gray)
 *       KF_U8X4 : one uchar4 per pixel (interleaved RGBA; each channel is an
 *                 independent image with identical kernels, int32 arithmetic)
 *   - Device pointers passed to kf_run* are CALLER-OWNED and must stay valid
 *     until the stream work completes.  The pipeline owns plans' workspaces
 *     and compiled modules.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *   - Not thread-safe per pipeline; distinct pipelines may be used from
 *     distinct threads.  A plan with more than one block keeps its cut-edge
 *     intermediates in ONE workspace: two kf_run / kf_run_band calls of such a
 *     plan must not be in flight on different streams at the same time
 *     (single-block plans write only their outputs and may overlap on
 *     disjoint output rows).
 */
#ifndef KFUSE_H
#define KFUSE_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    KF_OK = 0,
    KF_ERR_ARG = 1,            /* invalid argument (null pointer, bad size, bad enum) */
    KF_ERR_BAD_ID = 2,         /* image id does not exist (yet) */
    KF_ERR_HEADER = 3,         /* header incompatibility */
    KF_ERR_MASK = 4,           /* mask not odd-sized / not integral for KF_U8X4 */
    KF_ERR_FROZEN = 5,         /* graph edited after a plan was created */
    KF_ERR_ILLEGAL_BLOCK = 6,  /* kf_plan_from_blocks: a block violates IsLegal */
    KF_ERR_NVRTC = 7,          /* runtime compilation of a fused kernel failed */
    KF_ERR_CUDA = 8,           /* CUDA runtime / driver error */
    KF_ERR_NCCL = 9,           /* reserved for the multi-GPU layer */
    KF_ERR_OOM = 10,           /* device or host allocation failed */
    KF_ERR_PROGRAM = 11        /* malformed op-IR program (stack, opcode, dtype) */
} kf_status;

typedef enum { KF_F32 = 0, KF_U8X4 = 1 } kf_dtype;

/* Border handling of a local operator (clamp worked
 * example, mirror and repeat supported; constant and mirror101 extra).
 * Index maps per axis, applied repeatedly until in range:
 *   CLAMP     p<0 -> 0, p>=n -> n-1
 *   MIRROR    p<0 -> -p-1, p>=n -> 2n-p-1        (edge pixel duplicated)
 *   MIRROR101 p<0 -> -p,   p>=n -> 2n-p-2        (edge pixel not duplicated)
 *   REPEAT    p mod n
 *   CONSTANT  out-of-image pixels read `constant` */
typedef enum { KF_CLAMP = 0, KF_MIRROR = 1, KF_MIRROR101 = 2, KF_REPEAT = 3, KF_CONSTANT = 4 } kf_boundary;

/* Postfix op-IR of point bodies and local epilogues.  Stack machine; each
 * program must leave exactly one value.  F32 pipelines compute in float32,
 * U8X4 pipelines per channel in int32.
 *   LOAD k     push input k of a point op (k < n_inputs) / the accumulator in
 *              a local op's post program (k = 0)
 *   CONST      push imm (rounded to float32, or truncated to int32)
 *   ADD SUB MUL DIV MIN MAX        pop b, pop a, push a op b
 *                                  (int DIV truncates, x/0 = 0)
 *   ABS NEG SQRT EXP LOG           pop a, push f(a)  (SQRT/EXP/LOG: F32 only)
 *   POW        pop b, pop a, push a^b (F32 only)
 *   SHR n, SHL n                   arithmetic shift by arg = n (U8X4 only)
 *   SAT_U8     clamp to [0, 255] (U8X4 only)
 *   CLAMP      pop hi, pop lo, pop x, push min(max(x, lo), hi)
 *   SELECT_GT  pop d, pop c, pop b, pop a, push (a > b) ? c : d
 *   LUT        pop i, push lut[clamp(i, 0, lut_len-1)]  (U8X4 only)
 * A U8X4 kernel's result is saturated to [0,255] when stored. */
typedef enum {
    KF_OP_LOAD = 0, KF_OP_CONST = 1, KF_OP_ADD = 2, KF_OP_SUB = 3, KF_OP_MUL = 4,
    KF_OP_DIV = 5, KF_OP_MIN = 6, KF_OP_MAX = 7, KF_OP_ABS = 8, KF_OP_NEG = 9,
    KF_OP_SQRT = 10, KF_OP_EXP = 11, KF_OP_LOG = 12, KF_OP_POW = 13, KF_OP_SHR = 14,
    KF_OP_SHL = 15, KF_OP_SAT_U8 = 16, KF_OP_CLAMP = 17, KF_OP_SELECT_GT = 18,
    KF_OP_LUT = 19
} kf_opcode;

typedef struct { int32_t op; int32_t arg; double imm; } kf_instr;

/* Arithmetic cost of a kernel for the benefit model, Eq. 6:
 * costop = c_alu * n_alu + c_sfu * n_sfu.  When NULL is passed, n_alu/n_sfu
 * default to an opcode count (SQRT/EXP/LOG/POW are SFU ops; a local op adds
 * 2*nnz(mask)-1 multiply-adds).  The paper's Harris uses n_alu = 2 for the
 * squares. */
typedef struct { int32_t n_alu; int32_t n_sfu; } kf_cost;

/* Hardware-model constants of §II-C-2 and planner knobs.
 *   tg, ts        cycles per pixel access, global / shared (Eqs. 3-4)
 *   c_alu, c_sfu  cycles per ALU / SFU op (Eq. 6)
 *   gamma         additive benefit, launch overhead / CSE (Eq. 12)
 *   c_mshared     Eq. 2 threshold
 *   phi_mode      0 = PAPER: phi = costop*IS_ks*sz(kd) (Eq. 7) or *g (Eqs. 9-10)
 *                 1 = STAGED: the producer is computed once per staged tile
 *                     point and recomputed only on the halo: factor
 *                     (tile_w+2rx)(tile_h+2ry)/(tile_w*tile_h)  (R-4)
 *   eq3_mode      0 = delta_Mshared = IS*tg/ts as printed (Eq. 3); 1 = IS*(tg-ts)
 *   phi_mode 2 = ROOFLINE (R-20, the B200 issue-rate extension): a
 *     kernel set S fused into one kernel takes, in SM-cycles per pixel,
 *       M(S) = bpp * (|external input images| + 1) / bw_bytes_clk     (DRAM)
 *       C(S) = sum_k slots(k) * ch * r_S(k) / issue_lanes_clk           (issue)
 *       T(S) = max(M, C) + overlap * min(M, C)
 *     (overlap 0: a perfect roofline, 1: no overlap, M + C).  slots(k) = issue
 *     slots per pixel of kernel k: every program opcode except LOAD/CONST
 *     counts 1, except POW 80, LOG 30, EXP 25, SQRT 2, DIV 15 (their SASS
 *     expansion on sm_100a), plus one per non-zero mask tap of a local kernel;
 *     ch = 2 for U8X4 (two SWAR channel pairs) else 1; r_S(k) is the staged
 *     halo recompute factor of the producer inside S, as in STAGED.  An edge's
 *     benefit is w = T({ks}) + T({kd}) - T({ks, kd}) + gamma.  tg, ts, c_alu,
 *     c_sfu and kf_cost are unused in this mode.
 * kf_model_params_paper(): tg=400 ts=4 c_alu=4 c_sfu=16 gamma=0 c_mshared=2
 *   phi PAPER, 32x32.  kf_model_params_b200(): same but
 *   c_mshared=5, phi STAGED. */
typedef struct {
    double tg, ts, c_alu, c_sfu, gamma, c_mshared;
    int32_t phi_mode, tile_w, tile_h, eq3_mode;
    double bw_bytes_clk, issue_lanes_clk, overlap;   /* phi_mode 2 only (see below) */
} kf_model_params;

typedef struct kf_pipeline kf_pipeline;
typedef struct kf_plan kf_plan;

void kf_model_params_paper(kf_model_params *p);
void kf_model_params_b200(kf_model_params *p);
/* kf_model_params_b200_roofline(): phi_mode 2 with B200 constants:
 * bw_bytes_clk = 22.45 (6528 GB/s measured copy / 148 SMs / 1965 MHz),
 * issue_lanes_clk = 115 (measured FFMA rate 3.6 warp-instr/clk/SM), overlap 1
 * (fitted: best rank correlation with measured plan times, R-20),
 * tile 120x32 (the streaming chunk), c_mshared = 5, gamma = 0. */
void kf_model_params_b200_roofline(kf_model_params *p);

/* One iteration space per pipeline: every image is width x height (header
 * compatibility).  width, height in [1, 65535*...]: any
 * positive size with width*height < 2^31. */
kf_status kf_pipeline_create(int32_t width, int32_t height, kf_dtype dtype, kf_pipeline **out);
void kf_pipeline_destroy(kf_pipeline *p);

/* Declares a pipeline input image; all inputs precede all kernels. */
kf_status kf_add_input(kf_pipeline *p, int32_t *image_id);

/* Point operator: out(y,x) = prog(inputs(y,x)).
 * inputs: n_inputs >= 1 existing image ids (order = LOAD index).
 * lut: 256-entry (lut_len >= 1) int table for KF_OP_LUT, copied; NULL if unused.
 * cost: nullable, see kf_cost.  *out_image receives the new image id. */
kf_status kf_add_point_op(kf_pipeline *p, const int32_t *inputs, int32_t n_inputs,
                          const kf_instr *prog, int32_t n_instr, const kf_cost *cost,
                          const int32_t *lut, int32_t lut_len, int32_t *out_image);

/* Local operator: correlation with an odd mask_w x mask_h
 * row-major mask anchored at its centre,
 *   acc(y,x) = sum_j sum_i mask[j*mask_w+i] * B(input, y+j-mask_h/2, x+i-mask_w/2)
 * then out = post(acc) (n_post = 0: identity).  KF_U8X4 masks must hold
 * integers and `constant` an integer in [0,255].  Masks are copied. */
kf_status kf_add_local_op(kf_pipeline *p, int32_t input, const double *mask, int32_t mask_w,
                          int32_t mask_h, kf_boundary mode, double constant,
                          const kf_instr *post, int32_t n_post, const kf_cost *cost,
                          int32_t *out_image);

/* Pipeline outputs are external outputs for legality (Fig. 2c). */
kf_status kf_mark_output(kf_pipeline *p, int32_t image_id);

/* ---- schedule options -------------------------------------------------------
 * Per-pipeline integer options that change how the fused kernels are
 * SCHEDULED (code shape, input feed, launch geometry), never what they
 * compute: for every option the output is bit-identical to the default (GPU
 * test test_schedule_options_bit_identical).  No environment variable reaches
 * the library; this is the only tuning interface (DESIGN.md §5.4 lists the
 * options and their measurements).  Code-generation options take effect for
 * plans prepared afterwards; run-time options (nstrips, host_taper) at the next
 * kf_run.  Names: swar swring swring_cap prefetch sring smem_rows lds_pf
 * const_w pro_rp qptr heavy_first code_budget rolled_edge_v minctas nstrips
 * host_taper host_bands host_async_bands host_direct tma rtrip cta_warps peel_warmup pdl
 * warm_skip lut_smem delay_smem.  Unknown names or out-of-range values:
 * KF_ERR_ARG.  (The measured-and-rejected v8 / persist / persist_waves / nlong
 * / cluster and the rounding-changing diagnostics pairs / defer exist only in
 * a KF_EXPERIMENTAL build, the naive_border negative control only in the
 * KF_TEST_HOOKS build libkfuse_testhooks.so, and the bounds_shrink self-test
 * only in the bounds-checking build libkfuse_bounds.so -- never in
 * libkfuse.so.) */
kf_status kf_set_option(kf_pipeline *p, const char *name, int64_t value);
kf_status kf_get_option(const kf_pipeline *p, const char *name, int64_t *value);

/* ---- planning (host only; freezes the graph) ---------------------------- */
/* Alg. 1 GetLegalPartitions with the benefit model. */
kf_status kf_plan_fusion(kf_pipeline *p, const kf_model_params *m, kf_plan **out);
/* The "basic" fusion of the authors' previous work [12], the paper's
 * comparison column: only
 * point-to-point, local-to-point and point-to-local fusion, shared inputs
 * (Fig. 2b) rejected as external.  Greedy pair-wise merging by decreasing
 * edge benefit under IsLegal plus the basic rules (R-18).  Same
 * weights, output and ownership as kf_plan_fusion. */
kf_status kf_plan_basic(kf_pipeline *p, const kf_model_params *m, kf_plan **out);
/* Exact planner: the partition into IsLegal blocks with the
 * maximum total weight of the edges inside blocks (Eq. 1, lexicographic
 * (q, eps)), by subset DP in O(3^n) -- the exhaustive search the paper rules
 * out for large graphs.  KF_ERR_ARG for more than 16
 * kernels.  Same output and ownership as kf_plan_fusion. */
kf_status kf_plan_exact(kf_pipeline *p, const kf_model_params *m, kf_plan **out);
/* Every kernel its own block: the unfused GPU baseline. */
kf_status kf_plan_unfused(kf_pipeline *p, kf_plan **out);
/* Caller-chosen partition: block_of_kernel[k] = block label (any ints).  Every
 * multi-kernel block must pass IsLegal under the paper profile's dependence,
 * header and repeat-compatibility rules (resources and profitability are NOT
 * checked here), else KF_ERR_ILLEGAL_BLOCK. */
kf_status kf_plan_from_blocks(kf_pipeline *p, const int32_t *block_of_kernel, kf_plan **out);
void kf_plan_destroy(kf_plan *plan);

int32_t kf_plan_num_blocks(const kf_plan *plan);
/* Kernels of block i (topological order of blocks, ascending kernel ids inside);
 * `kernels` must hold n_kernels entries; *n receives the count. */
kf_status kf_plan_block(const kf_plan *plan, int32_t i, int32_t *kernels, int32_t *n);
/* beta of Eq. 1 as a lexicographic pair: real part in units of 2^-20 cycles
 * (exact fixed point) and the number of eps terms (R-9). */
kf_status kf_plan_objective(const kf_plan *plan, int64_t *beta_q, int64_t *beta_eps);
/* Edge (src kernel -> dst kernel) diagnostics: w = benefit before clamping,
 * is_eps (weight is eps), ctx_legal (pair legal in context), profitable (w > 0). */
kf_status kf_plan_edge(const kf_plan *plan, int32_t src, int32_t dst, double *w, int32_t *is_eps,
                       int32_t *ctx_legal, int32_t *profitable);
/* Min cuts taken by Alg. 1 line 13 in processing order: the t-side kernels,
 * the cut weight (q, eps) and the number of Stoer-Wagner phases. */
int32_t kf_plan_num_cuts(const kf_plan *plan);
kf_status kf_plan_cut(const kf_plan *plan, int32_t i, int32_t *side, int32_t *n_side,
                      int64_t *w_q, int64_t *w_eps, int32_t *phases);
/* Kernel launches one kf_run performs (= blocks). */
int32_t kf_plan_num_launches(const kf_plan *plan);
/* Rows of input halo one output row band needs: max accumulated vertical
 * radius over every input->output path of the plan. */
int32_t kf_plan_halo_rows(const kf_plan *plan);
/* Generated CUDA source of block i (debug aid).  Writes up to cap bytes
 * (NUL-terminated when it fits); *len receives the full length. */
kf_status kf_plan_kernel_source(kf_pipeline *p, const kf_plan *plan, int32_t block, char *buf,
                                size_t cap, size_t *len);

/* ---- execution ------------------------------------------------------------ */
/* Compiles (NVRTC -> sm_100a cubin, cached in memory and under
 * $KFUSE_CACHE_DIR or the package's kcache/) and loads every block kernel,
 * and allocates the workspace for cut edges.  Called implicitly by kf_run. */
kf_status kf_prepare(kf_pipeline *p, const kf_plan *plan);

/* Compile-only (no GPU needed): generates and NVRTC-compiles every block of
 * the plan into the cubin cache, so a later kf_prepare on the GPU box only
 * loads modules. */
kf_status kf_compile_plan(kf_pipeline *p, const kf_plan *plan);

/* Runs the plan: d_inputs[i] is input image i, d_outputs[j] receives the j-th
 * marked output.  Launches exactly kf_plan_num_launches kernels, asynchronously
 * on `stream`, in topological block order.  No allocation after kf_prepare. */
kf_status kf_run(kf_pipeline *p, const kf_plan *plan, const void *const *d_inputs, int32_t n_in,
                 void *const *d_outputs, int32_t n_out, void *stream);

/* A batch of INDEPENDENT frames (e.g. consecutive video frames): frame f reads
 * d_inputs[f*n_in + i] and writes d_outputs[f*n_out + j], with kf_run's layout,
 * alignment and result for every frame (bit-identical to n_frames kf_run
 * calls).  Every output image must be disjoint from every other frame's input
 * and output images (inputs may be shared), else KF_ERR_ARG before any launch.
 * Single-block plans launch frames 1..n-1 as programmatic dependent launches
 * that do not wait for the previous frame (only for its completion at their
 * end): the next frame's CTAs fill the SM slots the previous frame's tail
 * leaves idle.  Frame 0 waits for all earlier work on `stream` as kf_run does,
 * and completion of the last frame implies completion of all of them.
 * Multi-block plans share one workspace and run the frames in order.
 * Same paper passage as kf_run (one kernel per block); the
 * frame overlap is a B200 scheduling choice. */
kf_status kf_run_batch(kf_pipeline *p, const kf_plan *plan, int32_t n_frames, const void *const *d_inputs,
                       int32_t n_in, void *const *d_outputs, int32_t n_out, void *stream);

/* Bounds-checking build (libkfuse_bounds.so, built from the same sources with
 * KF_BOUNDS; tests only): every global read of a generated kernel must fall
 * inside one of the launch's external image buffers and every write inside the
 * launch's own output rows; an access outside is skipped and counted instead of
 * faulting.  Returns, and clears, the pipeline's record: the
 * number of violations since the last call, the first offending address and
 * its kind (0 read, 1 write, 2 table index; the index is then in the low 32
 * bits).  Synchronises the device.  Every other build: KF_ERR_ARG. */
kf_status kf_bounds_report(kf_pipeline *p, int64_t *violations, uint64_t *first_addr, int32_t *first_kind);

/* End-to-end call with HOST buffers: copies inputs host->device, runs, copies
 * outputs device->host, synchronises `stream`.  The image is processed in up to
 * 8 row bands on three engines: the H2D copy of band k+1's input rows, the
 * kernels of band k (kf_run_band semantics: border modes act at the global
 * edges, so the result equals kf_run's bit for bit) and the D2H copy of band
 * k-1's output rows overlap.  REPEAT plans run as one band.  Host buffers
 * (same layout as kf_run's device buffers) should be pinned for full
 * host-link bandwidth and overlap; pageable buffers work but serialise the
 * copies.  Device staging buffers, the two copy streams and their events are
 * owned by the pipeline.  Work already queued on `stream` precedes the copies. */
kf_status kf_run_host(kf_pipeline *p, const kf_plan *plan, const void *const *h_inputs, int32_t n_in,
                      void *const *h_outputs, int32_t n_out, void *stream);

/* kf_run_host without the final synchronisation, for a stream of host images:
 * returns once the work is queued; the outputs are in host memory when
 * `stream`'s work completes (its later work is ordered after the downloads).
 * Consecutive calls alternate between two device staging sets, so call k+1's
 * uploads overlap call k's downloads (the copy engines run both directions at
 * once).  Unlike kf_run_host, the uploads are NOT ordered after work already
 * queued on `stream`: the host inputs must be ready at the call and must not
 * be written by pending work, and inputs and outputs must stay untouched until
 * the stream's work completes.  Host buffers must be pinned.  Results equal
 * kf_run's bit for bit. */
kf_status kf_run_host_async(kf_pipeline *p, const kf_plan *plan, const void *const *h_inputs, int32_t n_in,
                            void *const *h_outputs, int32_t n_out, void *stream);

/* Row-band execution for the multi-GPU layer: computes output rows
 * [row0, row1) of every marked output into d_out_band[j] (rows row0.. at
 * pitch width*4).  d_in_band[i] holds input rows [in_row0, in_row1) of image i,
 * which must cover [row0 - H, row1 + H) clipped to [0, height), H =
 * kf_plan_halo_rows.  Border modes act at the GLOBAL image edges, so banded
 * output is bit-identical to kf_run's rows.  REPEAT plans are rejected
 * (KF_ERR_ARG): they would need a ring exchange. */
kf_status kf_run_band(kf_pipeline *p, const kf_plan *plan, int32_t row0, int32_t row1,
                      const void *const *d_in_band, int32_t in_row0, int32_t in_row1,
                      void *const *d_out_band, void *stream);

/* ---- multi-GPU halo rows over peer memory (NVLink P2P) ------------------
 * The north star's "halo rows ... read from peer memory over NVLink"
 * (BASELINE.json), as three stream-ordered, CUDA-graph-capturable
 * kernels synchronised by monotonic uint32 counters in device memory (no host
 * collective per step).  Pointers may be peer mappings (CUDA IPC) of another
 * GPU's memory; the caller owns every buffer.  Counters compare wrap-safe.
 * Every wait polls at most spin_limit times (~0.1 us each), then sets *err = 1
 * and gives up (a missing neighbour is an error, not a hang).  Up to 4
 * counters / segments per call; KF_ERR_ARG otherwise, KF_ERR_CUDA if the
 * launch fails. */

/* Release-increments each counter flags[i] (typically in the neighbours'
 * memory: "my rows of this step are ready"), after everything queued before
 * it on `stream`; increments *sent (local, nullable). */
kf_status kf_peer_signal(uint32_t *const *flags, int32_t n, uint32_t *sent, void *stream);

/* For each segment i < n (one per neighbour): wait until *flag[i] passes
 * *seen[i], then for each copy c < m (one per pipeline input image) copy
 * bytes[i*m+c] bytes from src[i*m+c] (the neighbour's boundary rows) to
 * dst[i*m+c] (the local halo rows), set *seen[i] += 1, then release-increment
 * ack[i] (the neighbour's "consumed" counter; ack may be null).  Any
 * alignment is accepted (16-B vectors when both ends are 16-B aligned, else
 * 4-B words or bytes).  n <= 4, 1 <= m <= 8. */
kf_status kf_peer_pull(int32_t n, int32_t m, void *const *dst, const void *const *src, const int64_t *bytes,
                       uint32_t *const *flag, uint32_t *const *seen, uint32_t *const *ack, uint32_t *err,
                       int64_t spin_limit, void *stream);

/* Wait until every *counter[i] reaches *target[i] (e.g. both neighbours acked
 * every signal before the own rows are overwritten). */
kf_status kf_peer_wait(int32_t n, uint32_t *const *counter, uint32_t *const *target, uint32_t *err,
                       int64_t spin_limit, void *stream);

/* Enables peer access from `device` to `peer_device` (NVLink P2P) so that the
 * kf_peer_* kernels launched on `device` can use peer mappings of
 * `peer_device`'s memory.  Idempotent; KF_OK when device == peer_device;
 * KF_ERR_CUDA when the pair has no peer path. */
kf_status kf_peer_enable(int32_t device, int32_t peer_device);

/* Thread-local message of the last failing call on this thread. */
const char *kf_last_error(void);
/* Library version string. */
const char *kf_version(void);

#ifdef __cplusplus
}
#endif
#endif /* KFUSE_H */
