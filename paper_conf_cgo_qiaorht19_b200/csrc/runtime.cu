// runtime.cu -- executor of libkfuse: compiles each partition block's
// generated kernel with NVRTC for sm_100a (cached), loads it through the CUDA
// driver API (entry points obtained from the runtime, so libkfuse.so loads on
// a machine without a driver), owns the workspace of cut-edge images and
// launches one kernel per block in topological order on the caller's stream
// (Alg. 1 output: "each partition block in the ready set is fused into one
// kernel").
#include <cuda.h>
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nvrtc.h>
#include <nvtx3/nvToolsExt.h>
#include <sys/stat.h>
#include <utime.h>
#include <zlib.h>
#include <unistd.h>

#include <algorithm>
#include <cstddef>
#include <cstdio>
#include <cstring>
#include <fstream>
#include <mutex>
#include <sstream>
#include <thread>

#include "kf_internal.h"
#include "device/kf_device.cuh"

namespace kf {

// NVTX ranges around the host-side steps (prepare, run, run_host and its
// bands): visible in Nsight Systems / ncu range filters, free without a tool.
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

static const char *kDeviceHeader =
#include "kf_device_cuh.inc"
    ;

// --------------------------------------------------------------- helpers
#define KF_CUDA(call)                                                                         \
    do {                                                                                      \
        cudaError_t e_ = (call);                                                              \
        if (e_ != cudaSuccess)                                                                \
            fail(KF_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_));            \
    } while (0)

struct Driver {
    CUresult (*moduleLoadData)(CUmodule *, const void *) = nullptr;
    CUresult (*moduleGetFunction)(CUfunction *, CUmodule, const char *) = nullptr;
    CUresult (*moduleUnload)(CUmodule) = nullptr;
    CUresult (*launchKernel)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                             CUstream, void **, void **) = nullptr;
    CUresult (*launchKernelEx)(const CUlaunchConfig *, CUfunction, void **, void **) = nullptr;
    CUresult (*getErrorString)(CUresult, const char **) = nullptr;
    CUresult (*occupancy)(int *, CUfunction, int, size_t) = nullptr;
};

static Driver &driver()
{
    static Driver d;
    static std::once_flag once;
    static std::string err;
    std::call_once(once, [] {
        int ndev = 0;
        cudaError_t e = cudaGetDeviceCount(&ndev);
        if (e != cudaSuccess || ndev == 0) {
            err = std::string("no CUDA device: ") + cudaGetErrorString(e);
            return;
        }
        cudaFree(nullptr);   // initialise the primary context (shared with PyTorch)
        auto get = [](const char *name, void **fn) {
            cudaDriverEntryPointQueryResult q;
            cudaError_t r = cudaGetDriverEntryPoint(name, fn, cudaEnableDefault, &q);
            if (r != cudaSuccess || q != cudaDriverEntryPointSuccess || !*fn)
                err += std::string(" missing driver entry point ") + name;
        };
        get("cuModuleLoadData", (void **)&d.moduleLoadData);
        get("cuModuleGetFunction", (void **)&d.moduleGetFunction);
        get("cuModuleUnload", (void **)&d.moduleUnload);
        get("cuLaunchKernel", (void **)&d.launchKernel);
        get("cuLaunchKernelEx", (void **)&d.launchKernelEx);
        get("cuGetErrorString", (void **)&d.getErrorString);
        get("cuOccupancyMaxActiveBlocksPerMultiprocessor", (void **)&d.occupancy);
    });
    if (!err.empty() || !d.launchKernel) fail(KF_ERR_CUDA, "CUDA unavailable:" + err);
    return d;
}

static void cu_check(CUresult r, const char *what)
{
    if (r == CUDA_SUCCESS) return;
    const char *s = "unknown";
    if (driver().getErrorString) driver().getErrorString(r, &s);
    fail(KF_ERR_CUDA, std::string(what) + ": " + s);
}

static uint64_t fnv1a(const std::string &s, uint64_t h = 1469598103934665603ull)
{
    for (unsigned char c : s) { h ^= c; h *= 1099511628211ull; }
    return h;
}

// Directory of the cubin cache: $KFUSE_CACHE_DIR, else <dir of libkfuse.so>/kcache.
static std::string cache_dir()
{
    if (const char *e = getenv("KFUSE_CACHE_DIR")) return e;
    Dl_info info;
    if (dladdr((void *)&cache_dir, &info) && info.dli_fname) {
        std::string f = info.dli_fname;
        size_t pos = f.rfind('/');
        if (pos != std::string::npos) return f.substr(0, pos) + "/kcache";
    }
    return "./kcache";
}

static const char *kNvrtcOpts[] = {"--gpu-architecture=sm_100a", "-std=c++17", "-lineinfo", "-DKF_NVRTC=1",
                                   "--extra-device-vectorization"
#ifdef KF_BOUNDS
                                   , "-DKF_BOUNDS=1"   // bounds-checking build: checked global accesses
#endif
};

// NVRTC -> sm_100a cubin, cached on disk by hash(source, header, options).
static std::string compile_cubin(const std::string &src, const std::string &name)
{
    std::string key = src + kDeviceHeader;
    for (const char *o : kNvrtcOpts) key += o;
    char hex[32];
    std::snprintf(hex, sizeof hex, "%016llx", (unsigned long long)fnv1a(key));
    const std::string dir = cache_dir();
    // zlib-compressed on disk ("KFZ1", uint64 size, deflate stream): the
    // -lineinfo cubins of the unrolled kernels are 1-2.5 MB each and compress ~4x
    const std::string path = dir + "/" + name + "_" + hex + ".cubin.z";
    {
        std::ifstream f(path, std::ios::binary);
        if (f) {
            std::stringstream ss;
            ss << f.rdbuf();
            std::string s = ss.str();
            uint64_t n = 0;
            if (s.size() > 12 && !s.compare(0, 4, "KFZ1")) {
                std::memcpy(&n, s.data() + 4, 8);
                std::string out(n, '\0');
                uLongf got = (uLongf)n;
                if (n > 16 && uncompress((Bytef *)&out[0], &got, (const Bytef *)s.data() + 12, (uLong)(s.size() - 12)) == Z_OK &&
                    got == n) {
                    utime(path.c_str(), nullptr);   // mark as used (tools/warm_test_cache.py --prune keeps used cubins)
                    return out;
                }
            }
        }
    }
    nvrtcProgram prog;
    const char *hdr_src[] = {kDeviceHeader};
    const char *hdr_name[] = {"kf_device.cuh"};
    if (nvrtcCreateProgram(&prog, src.c_str(), (name + ".cu").c_str(), 1, hdr_src, hdr_name) != NVRTC_SUCCESS)
        fail(KF_ERR_NVRTC, "nvrtcCreateProgram failed");
    nvrtcResult r = nvrtcCompileProgram(prog, (int)(sizeof kNvrtcOpts / sizeof kNvrtcOpts[0]), kNvrtcOpts);
    if (r != NVRTC_SUCCESS) {
        size_t n = 0;
        nvrtcGetProgramLogSize(prog, &n);
        std::string log(n, '\0');
        nvrtcGetProgramLog(prog, &log[0]);
        nvrtcDestroyProgram(&prog);
        fail(KF_ERR_NVRTC, "NVRTC failed for " + name + ": " + log);
    }
    size_t n = 0;
    nvrtcGetCUBINSize(prog, &n);
    std::string cubin(n, '\0');
    nvrtcGetCUBIN(prog, &cubin[0]);
    nvrtcDestroyProgram(&prog);
    mkdir(dir.c_str(), 0775);
    // per process AND thread: concurrent compiles of the same block write distinct temporaries
    std::string tmp = path + "." + std::to_string(getpid()) + "." +
                      std::to_string(std::hash<std::thread::id>()(std::this_thread::get_id())) + ".tmp";
    {
        uLongf zn = compressBound((uLong)cubin.size());
        std::string z(12 + zn, '\0');
        const uint64_t n = cubin.size();
        std::memcpy(&z[0], "KFZ1", 4);
        std::memcpy(&z[4], &n, 8);
        if (compress2((Bytef *)&z[12], &zn, (const Bytef *)cubin.data(), (uLong)cubin.size(), 6) == Z_OK) {
            z.resize(12 + zn);
            std::ofstream f(tmp, std::ios::binary);
            if (f) f.write(z.data(), (std::streamsize)z.size());
        }
    }
    if (rename(tmp.c_str(), path.c_str()) != 0) unlink(tmp.c_str());
    return cubin;
}

struct CompiledBlock {
    CUmodule mod = nullptr;
    CUfunction fn = nullptr;
    StreamInfo si;               // interior schedule the kernel was generated with
    int ctas_per_sm = 1;         // occupancy of the kernel (cuOccupancy...)
    int num_sms = 148;
    std::string source;
    ~CompiledBlock()
    {
        if (mod && driver().moduleUnload) driver().moduleUnload(mod);
    }
};

constexpr int kHostBands = 32;  // kf_run_host: most row bands (option host_bands, default 8)

struct Runtime {
    std::map<uint64_t, std::shared_ptr<CompiledBlock>> modules;   // by source hash
    std::vector<void *> stage_in[2], stage_out[2];                // kf_run_host staging (2 sets: async calls alternate)
    size_t stage_bytes = 0;
    int device = -1;
    // kf_run_host copy engines: H2D and D2H streams + per-band events
    cudaStream_t s_h2d = nullptr, s_d2h = nullptr;
    cudaEvent_t ev_in[kHostBands] = {}, ev_out[kHostBands] = {}, ev_start = nullptr, ev_done = nullptr;
    cudaEvent_t ev_kern[2] = {};   // kf_run_host_async: the kernels that read staging set s are done
    size_t async_calls = 0;
    unsigned *viol = nullptr;   // bounds-checking build: violation record [count, addr lo, addr hi, kind]
    ~Runtime()
    {
        if (viol) cudaFree(viol);
        for (int k = 0; k < 2; k++) {
            for (void *q : stage_in[k]) cudaFree(q);
            for (void *q : stage_out[k]) cudaFree(q);
            if (ev_kern[k]) cudaEventDestroy(ev_kern[k]);
        }
        for (int i = 0; i < kHostBands; i++) {
            if (ev_in[i]) cudaEventDestroy(ev_in[i]);
            if (ev_out[i]) cudaEventDestroy(ev_out[i]);
        }
        if (ev_start) cudaEventDestroy(ev_start);
        if (ev_done) cudaEventDestroy(ev_done);
        if (s_h2d) cudaStreamDestroy(s_h2d);
        if (s_d2h) cudaStreamDestroy(s_d2h);
    }
};

// Compile-only path usable without a GPU (build() warms the in-tree cache).
std::string compile_block_cubin(const kf_pipeline *p, const kf_plan *plan, int i)
{
    return compile_cubin(generate_block(p, plan->info[i], i), kernel_name(plan->info[i], i));
}

void prepare(kf_pipeline *p, kf_plan *plan)
{
    if (plan->prepared) return;
    NvtxRange nvtx("kf_prepare");
    Driver &d = driver();
    if (!p->rt) p->rt = new Runtime();
    int dev = 0;
    KF_CUDA(cudaGetDevice(&dev));
    if (p->rt->device >= 0 && p->rt->device != dev) fail(KF_ERR_CUDA, "pipeline used on two devices");
    p->rt->device = dev;
    plan->compiled.clear();
    for (size_t i = 0; i < plan->blocks.size(); i++) {
        std::string src = generate_block(p, plan->info[i], (int)i);
        uint64_t h = fnv1a(src);
        auto it = p->rt->modules.find(h);
        if (it == p->rt->modules.end()) {
            auto cb = std::make_shared<CompiledBlock>();
            std::string cubin = compile_cubin(src, kernel_name(plan->info[i], (int)i));
            cu_check(d.moduleLoadData(&cb->mod, cubin.data()), "cuModuleLoadData");
            cu_check(d.moduleGetFunction(&cb->fn, cb->mod, kernel_name(plan->info[i], (int)i).c_str()), "cuModuleGetFunction");
            cb->source = src;
            cb->si = stream_info(p, plan->info[i]);
            cu_check(d.occupancy(&cb->ctas_per_sm, cb->fn, kThreads * cb->si.nw, 0),
                     "cuOccupancyMaxActiveBlocksPerMultiprocessor");
            cb->ctas_per_sm = std::max(1, cb->ctas_per_sm);
            KF_CUDA(cudaDeviceGetAttribute(&cb->num_sms, cudaDevAttrMultiProcessorCount, dev));
            it = p->rt->modules.emplace(h, cb).first;
        }
        plan->compiled.push_back(it->second);
    }
    // workspace: block sinks that are not marked outputs (cut edges), full height
    std::set<int> outs(p->outputs.begin(), p->outputs.end());
    for (auto &b : plan->info) {
        int img = p->n_inputs + b.sink;
        bool consumed = false;
        for (auto &b2 : plan->info)
            for (int e : b2.ext) consumed |= e == img;
        if (!outs.count(img) || consumed) {
            if (!plan->workspace.count(img)) {
                void *q = nullptr;
                if (cudaMalloc(&q, (size_t)p->W * p->H * 4) != cudaSuccess)
                    fail(KF_ERR_OOM, "workspace allocation failed");
                plan->workspace[img] = q;
            }
        }
    }
    plan->prepared = true;
}

// Executes rows [row0, row1) of every output.  Full-image run: row0 = 0,
// row1 = H, inputs hold all rows (in_row0 = 0).  Band run: inputs hold rows
// from in_row0; each block computes its sink over the rows its consumers need.
// Launch geometry of one block.  The streaming path covers
// the rectangle [fx0, fx1) x [fy0, fy1): the whole rows [r0, r1) when the
// block's image edges can be handled by edge strips/chunks (index exchange
// inside the streaming path), otherwise only the pixels whose whole input
// footprint is inside the image.  Whatever remains -- the border frame -- is
// tiled by the shared-memory index-exchange path.  One warp (= one CTA) per
// (column chunk, row strip) item; the strip height is chosen so the items fill
// whole waves of resident warps.  Returns the grid size.
static unsigned launch_geometry(const kf_pipeline *p, KfArgs &a, const BlockInfo &b, const CompiledBlock &cb)
{
    const int W = a.W, H = a.H, V = cb.si.V;
    const StreamInfo &si = cb.si;
    int fx0 = 0, fx1 = 0, fy0 = 0, fy1 = 0;
    bool fast = si.ok, top = false, bot = false;
    if (fast) {
        top = si.edge_v && a.r0 == 0;
        bot = si.edge_v && a.r1 == H;
        fy0 = top ? 0 : std::max(a.r0, b.Ry);
        fy1 = bot ? H : std::min(a.r1, H - b.Ry);
        fx0 = si.edge_l ? 0 : (si.vec ? (b.Rx + V - 1) / V * V : b.Rx);
        fx1 = si.edge_r ? W : (si.vec ? (W - b.Rx) / V * V : W - b.Rx);
        fast = fx1 > fx0 && fy1 - fy0 >= (top && bot ? 2 * std::max(1, si.L) : 1);
    }
    struct R { int x0, x1, y0, y1, shape; };
    std::vector<R> rects;
    if (fast) {
        rects = {{0, W, a.r0, fy0, 0}, {0, W, fy1, a.r1, 0}, {0, fx0, fy0, fy1, 1}, {fx1, W, fy0, fy1, 1}};
    } else {
        rects = {{0, W, a.r0, a.r1, 0}};
    }
    int cta = 0;
    a.n_rect = 0;
    for (const R &r : rects) {
        if (r.x1 <= r.x0 || r.y1 <= r.y0) continue;
        KfRect &k = a.rect[a.n_rect++];
        k.x0 = r.x0; k.x1 = r.x1; k.y0 = r.y0; k.y1 = r.y1; k.shape = r.shape;
        k.ntx = (r.x1 - r.x0 + kFrameTiles[r.shape][0] - 1) / kFrameTiles[r.shape][0];
        k.nty = (r.y1 - r.y0 + kFrameTiles[r.shape][1] - 1) / kFrameTiles[r.shape][1];
        k.cta0 = cta;
        cta += k.ntx * k.nty;
    }
    a.frame_ctas = cta;
    if (!fast) return (unsigned)cta;
    a.fx0 = fx0; a.fx1 = fx1; a.fy0 = fy0; a.fy1 = fy1;
    a.edge_l = si.edge_l; a.edge_r = si.edge_r; a.edge_t = top; a.edge_b = bot;
    const int chunk_w = (32 - 2 * si.HL) * V;
    a.n_chunks = (fx1 - fx0 + chunk_w - 1) / chunk_w;
    const int Hf = fy1 - fy0;
    const long long slots = (long long)cb.num_sms * cb.ctas_per_sm * si.nw;   // resident interior warps per wave
    // ns balanced strips of floor/ceil(Hf/ns) rows.  Edge strips must be at
    // least L rows so that no interior strip reads beyond the image; a top and
    // a bottom edge need two strips.  Cost (fitted to B200 sweeps, DESIGN.md
    // §5.4): (iterations of one item + 2) x (waves + 1/2), iterations = rows +
    // 2L warm-up rounded up to the unroll P.  Several waves of short items
    // beat one wave of long ones: the hardware refills freed CTA slots, which
    // desynchronises the warps' load bursts and shortens the tail.
    const int min_strips = top && bot ? 2 : 1;
    const int smin = top || bot ? std::max(1, si.L) : 1;
    auto iters = [&](int rows) { return (double)((rows + 2 * si.L + si.P - 1) / si.P * si.P + 2); };
    double best = -1.0;
    int best_ns = min_strips;
    for (int ns = min_strips; ns <= std::max(min_strips, Hf / smin); ns++) {
        const int S = (Hf + ns - 1) / ns;
        const long long items = (long long)a.n_chunks * ns;
        const double w = (double)items / (double)slots;
        const double cost = iters(S) * (w + 0.5);
        if (best < 0 || cost < best - 1e-9) { best = cost; best_ns = ns; }
        if (items > 64 * slots) break;
    }
    if (const int force = (int)opt(p, "nstrips"))   // schedule option (sweeps; results unchanged)
        best_ns = std::max(min_strips, std::min(force, std::max(min_strips, Hf / smin)));
    a.n_strips = best_ns;
    a.strip = (Hf + best_ns - 1) / best_ns;
    // Optional tail split (experimental option "nlong" = n): the first n strips
    // are two units tall and the rest one unit, so the last wave runs short
    // items.  Edge strips must still hold smin rows.  Measured slower, so only in
    // the KF_EXPERIMENTAL build.
    a.n_long = 0;
    if (const int nl = (int)opt(p, "nlong")) {
        int n = std::min(nl, best_ns - 1);
        if (n > 0 && Hf / (best_ns + n) >= smin) a.n_long = n;
    }
    a.n_items = a.n_chunks * a.n_strips;
    return (unsigned)(cta + (a.n_items + si.nw - 1) / si.nw);   // si.nw interior items per CTA
}

void run(kf_pipeline *p, kf_plan *plan, const void *const *din, int n_in, void *const *dout, int n_out,
         void *stream, int row0, int row1, int in_row0, int in_row1, bool out_full, bool indep)
{
    if (n_in != p->n_inputs || (n_in && !din)) fail(KF_ERR_ARG, "wrong number of inputs");
    if (n_out != (int)p->outputs.size() || (n_out && !dout)) fail(KF_ERR_ARG, "wrong number of outputs");
    // 128-bit row access (the interior path's vector loads/stores) needs 16-B
    // aligned rows, i.e. 16-B aligned base pointers when W % 4 == 0; otherwise
    // the kernels access single 4-B pixels and any 4-B aligned pointer works
    // (e.g. a row offset into a larger image).
    const uintptr_t amask = p->W % 4 == 0 ? 15 : 3;
    for (int i = 0; i < n_in; i++)
        if (!din[i] || ((uintptr_t)din[i] & amask))
            fail(KF_ERR_ARG, amask == 15 ? "input pointers must be non-null, 16-B aligned"
                                         : "input pointers must be non-null, 4-B aligned");
    for (int j = 0; j < n_out; j++)
        if (!dout[j] || ((uintptr_t)dout[j] & amask))
            fail(KF_ERR_ARG, amask == 15 ? "output pointers must be non-null, 16-B aligned"
                                         : "output pointers must be non-null, 4-B aligned");
    prepare(p, plan);
    Driver &d = driver();
    const bool band = !(row0 == 0 && row1 == p->H && in_row0 == 0);
    NvtxRange nvtx(band ? "kf_run_band" : "kf_run");
    const int nimg = p->n_images();
    // rows each image must be available over
    std::vector<int> lo(nimg, INT32_MAX), hi(nimg, INT32_MIN);
    std::vector<int> blo(plan->blocks.size()), bhi(plan->blocks.size());
    for (int o : p->outputs) { lo[o] = row0; hi[o] = row1; }
    for (int bi = (int)plan->blocks.size() - 1; bi >= 0; bi--) {
        const BlockInfo &b = plan->info[bi];
        int s = p->n_inputs + b.sink;
        if (lo[s] > hi[s]) { lo[s] = row0; hi[s] = row1; }      // dead kernel: same rows as outputs
        blo[bi] = lo[s];
        bhi[bi] = hi[s];
        for (int e : b.ext) {
            lo[e] = std::min(lo[e], std::max(0, lo[s] - b.ext_hy.at(e)));
            hi[e] = std::max(hi[e], std::min(p->H, hi[s] + b.ext_hy.at(e)));
        }
    }
    // where each image lives
    std::vector<void *> ptr(nimg, nullptr);
    std::vector<int> base(nimg, 0), rlast(nimg, p->H - 1);
    for (int i = 0; i < p->n_inputs; i++) {
        ptr[i] = const_cast<void *>(din[i]);
        base[i] = in_row0;
        rlast[i] = band ? in_row1 - 1 : p->H - 1;
    }
    for (auto &kv : plan->workspace) { ptr[kv.first] = kv.second; base[kv.first] = 0; }
    std::vector<std::pair<int, int>> band_copies;   // (image, output slot) copied at the end
    for (int j = 0; j < n_out; j++) {
        int o = p->outputs[j];
        if (plan->workspace.count(o) && band) {
            band_copies.push_back({o, j});
        } else {
            ptr[o] = dout[j];
            base[o] = band && !out_full ? row0 : 0;   // out_full: dout holds the whole image
        }
    }
    CUstream st = (CUstream)stream;
    for (size_t bi = 0; bi < plan->blocks.size(); bi++) {
        const BlockInfo &b = plan->info[bi];
        const CompiledBlock &cb = *plan->compiled[bi];
        KfArgs a;
        std::memset(&a, 0, sizeof a);
        for (size_t s = 0; s < b.ext.size(); s++) {
            const int e = b.ext[s];
            a.img[s] = ptr[e];
            a.base[s] = base[e];
            a.rlast[s] = rlast[e];
        }
        int sink = p->n_inputs + b.sink;
        a.out = ptr[sink];
        a.out_base = base[sink];
        a.W = p->W;
        a.H = p->H;
        a.r0 = blo[bi];
        a.r1 = bhi[bi];
        a.indep = indep ? 1 : 0;
        if (a.r1 <= a.r0) continue;
        // The geometry depends only on the block, its output rows and the
        // run-time schedule options: memoised per plan, so an eager kf_run (and
        // every band of kf_run_host) skips the strip-count search.
        const GeomKey gk{(int)bi, a.r0, a.r1, opt(p, "nstrips"), opt(p, "nlong")};
        unsigned grid;
        constexpr size_t kTail = offsetof(KfArgs, rect);   // geometry fields: rect[] .. n_long
        auto git = plan->geom.find(gk);
        if (git != plan->geom.end()) {
            std::memcpy((unsigned char *)&a + kTail, git->second.tail.data(), sizeof(KfArgs) - kTail);
            grid = git->second.grid;
        } else {
            grid = launch_geometry(p, a, b, cb);
            Geom g;
            g.tail.assign((const unsigned char *)&a + kTail, (const unsigned char *)&a + sizeof(KfArgs));
            g.grid = grid;
            plan->geom.emplace(gk, std::move(g));
        }
        if (!cb.si.ok) a.n_items = 0;   // frame-only block
        {   // Optional persistent CTAs (experimental option "persist"): at most one
            // wave, the kernel strides over the items.  Measured slower (C3 27.4 ->
            // 30.0 us, C4 327 -> 363; profiles/r01_sweep_persist.jsonl) -- the
            // hardware refilling freed CTA slots balances better than a static
            // stride -- so only in the KF_EXPERIMENTAL build.
            const long long slots = (long long)cb.num_sms * cb.ctas_per_sm * opt(p, "persist_waves");
            if (opt(p, "persist") && (long long)grid > slots) grid = (unsigned)slots;
        }
        if (grid == 0) continue;
#ifdef KF_BOUNDS
        {   // readable spans: each external image's buffer rows [base, rlast]; writable:
            // this launch's output rows [r0, r1) (option bounds_shrink: minus the
            // last row -- the checker's self-test, which must then report writes)
            if (!p->rt->viol) {
                KF_CUDA(cudaMalloc(&p->rt->viol, 4 * sizeof(unsigned)));
                KF_CUDA(cudaMemset(p->rt->viol, 0, 4 * sizeof(unsigned)));
            }
            const unsigned long long rb = (unsigned long long)a.W * 4;
            a.n_span = (int)b.ext.size();
            for (size_t s2 = 0; s2 < b.ext.size(); s2++) {
                a.span_lo[s2] = (unsigned long long)a.img[s2];
                a.span_hi[s2] = a.span_lo[s2] + (unsigned long long)(a.rlast[s2] - a.base[s2] + 1) * rb;
            }
            a.out_lo = (unsigned long long)a.out + (unsigned long long)(a.r0 - a.out_base) * rb;
            a.out_hi = (unsigned long long)a.out + (unsigned long long)(a.r1 - a.out_base - (opt(p, "bounds_shrink") ? 1 : 0)) * rb;
            a.viol = p->rt->viol;
        }
#endif
        void *params[] = {&a};
        // option pdl: 0 off, 1 every launch, 2 (default) every launch of an
        // unrolled block -- measured faster on every memory-bound config, but
        // slower on the compute-bound rolled C4 kernel
        const long long pdl_opt = opt(p, "pdl");
        const bool pdl = indep || pdl_opt == 1 || (pdl_opt == 2 && !cb.si.rolled);
        const int cluster = (int)opt(p, "cluster");   // experimental: thread-block clusters of this many CTAs
        if (pdl || cluster > 1) {
            // Programmatic dependent launch: this grid may be
            // scheduled once every CTA of the previous kernel on the stream has
            // triggered (this library's kernels trigger after their own wait).
            // A dependent kernel (indep = 0) executes griddepcontrol.wait before
            // its first global access: stream order is kept and only the CTA
            // launch overlaps the previous tail.  An independent frame of
            // kf_run_batch runs concurrently with the previous frame's tail and
            // waits for it at its end.
            CUlaunchAttribute attr[2];
            std::memset(attr, 0, sizeof attr);
            unsigned na = 0;
            if (pdl) {
                attr[na].id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
                attr[na++].value.programmaticStreamSerializationAllowed = 1;
            }
            if (cluster > 1) {   // grid rounded up to whole clusters; surplus CTAs find no work
                grid = (grid + cluster - 1) / cluster * cluster;
                attr[na].id = CU_LAUNCH_ATTRIBUTE_CLUSTER_DIMENSION;
                attr[na].value.clusterDim.x = (unsigned)cluster;
                attr[na].value.clusterDim.y = 1;
                attr[na++].value.clusterDim.z = 1;
            }
            CUlaunchConfig cfg;
            std::memset(&cfg, 0, sizeof cfg);
            cfg.gridDimX = grid; cfg.gridDimY = 1; cfg.gridDimZ = 1;
            cfg.blockDimX = kThreads * cb.si.nw; cfg.blockDimY = 1; cfg.blockDimZ = 1;
            cfg.sharedMemBytes = 0;
            cfg.hStream = st;
            cfg.attrs = attr;
            cfg.numAttrs = na;
            cu_check(d.launchKernelEx(&cfg, cb.fn, params, nullptr), "cuLaunchKernelEx");
        } else {
            cu_check(d.launchKernel(cb.fn, grid, 1, 1, kThreads * cb.si.nw, 1, 1, 0, st, params, nullptr),
                     "cuLaunchKernel");
        }
    }
    for (auto &c : band_copies) {
        const char *src = (const char *)plan->workspace[c.first] + (size_t)row0 * p->W * 4;
        char *dst = (char *)dout[c.second] + (out_full ? (size_t)row0 * p->W * 4 : 0);
        KF_CUDA(cudaMemcpyAsync(dst, src, (size_t)(row1 - row0) * p->W * 4, cudaMemcpyDeviceToDevice,
                                (cudaStream_t)stream));
    }
}

// Independent frames (kf_run_batch): frame f runs the plan on
// din[f*n_in ..], dout[f*n_out ..].  Single-block plans launch the frames
// after the first as programmatic dependents that need not wait (indep): the
// CTAs of frame f+1 fill the SM slots that frame f's tail leaves idle.  That is
// only correct when no frame writes memory another frame touches, so every
// output image is checked to be disjoint from every other frame's images.
// Multi-block plans share one workspace between frames and run them in order.
void run_batch(kf_pipeline *p, kf_plan *plan, int n_frames, const void *const *din, int n_in,
               void *const *dout, int n_out, void *stream)
{
    if (n_frames < 0) fail(KF_ERR_ARG, "negative frame count");
    if (n_frames == 0) return;
    if (n_in != p->n_inputs || n_out != (int)p->outputs.size()) fail(KF_ERR_ARG, "wrong number of buffers");
    if ((n_in && !din) || (n_out && !dout)) fail(KF_ERR_ARG, "null buffer array");
    const uintptr_t bytes = (uintptr_t)p->W * p->H * 4;
    struct Span { uintptr_t lo, hi; int frame; bool out; };
    std::vector<Span> spans;
    for (int f = 0; f < n_frames; f++) {
        for (int i = 0; i < n_in; i++) spans.push_back({(uintptr_t)din[f * n_in + i], (uintptr_t)din[f * n_in + i] + bytes, f, false});
        for (int j = 0; j < n_out; j++) spans.push_back({(uintptr_t)dout[f * n_out + j], (uintptr_t)dout[f * n_out + j] + bytes, f, true});
    }
    std::sort(spans.begin(), spans.end(), [](const Span &x, const Span &y) { return x.lo < y.lo; });
    // any overlap of two spans of different frames, one of them written, is a hazard
    for (size_t i = 0; i < spans.size(); i++)
        for (size_t j = i + 1; j < spans.size() && spans[j].lo < spans[i].hi; j++)
            if (spans[i].frame != spans[j].frame && (spans[i].out || spans[j].out))
                fail(KF_ERR_ARG, "kf_run_batch: frames " + std::to_string(spans[i].frame) + " and " +
                                     std::to_string(spans[j].frame) + " share memory that one of them writes");
    prepare(p, plan);
    const bool overlap = plan->blocks.size() == 1;
    for (int f = 0; f < n_frames; f++)
        run(p, plan, din + (size_t)f * n_in, n_in, dout + (size_t)f * n_out, n_out, stream, 0, p->H, 0, p->H,
            false, overlap && f > 0);
}

// End-to-end call with host buffers.  The image is cut into kHostBands row
// bands and the three engines overlap: the H2D copy engine
// uploads band k+1's input rows while the SMs compute band k (kf_run_band
// semantics: border modes act at the global edges, so the result is identical
// to one whole-image run) and the D2H engine downloads band k-1's output rows.
// Band k waits only for the input rows it reads, [row0 - R, row1 + R).
// REPEAT plans (no band mode) and tiny images run as one band.
void run_host(kf_pipeline *p, kf_plan *plan, const void *const *hin, int n_in, void *const *hout, int n_out,
              void *stream, bool async)
{
    if (n_in != p->n_inputs || n_out != (int)p->outputs.size()) fail(KF_ERR_ARG, "wrong number of buffers");
    prepare(p, plan);
    NvtxRange nvtx("kf_run_host");
    if (opt(p, "host_direct")) {
        // Zero-copy (option host_direct): when every host buffer is pinned and
        // mapped (UVA: cudaHostAlloc / torch pin_memory), the kernels read the
        // inputs and write the outputs over the host link directly -- no staging
        // copies, no band pipeline.  Otherwise the staged path below runs.
        std::vector<const void *> di(n_in);
        std::vector<void *> dq(n_out);
        bool ok = true;
        auto mapped = [&](const void *h, void **d) {
            cudaPointerAttributes at;
            if (cudaPointerGetAttributes(&at, h) != cudaSuccess) { cudaGetLastError(); return false; }
            if (at.type != cudaMemoryTypeHost || !at.devicePointer) return false;
            *d = at.devicePointer;
            return true;
        };
        for (int i = 0; i < n_in && ok; i++) {
            void *d = nullptr;
            ok = mapped(hin[i], &d);
            di[i] = d;
        }
        for (int j = 0; j < n_out && ok; j++) ok = mapped(hout[j], &dq[j]);
        if (ok) {
            run(p, plan, di.data(), n_in, dq.data(), n_out, stream, 0, p->H, 0, p->H);
            if (!async) KF_CUDA(cudaStreamSynchronize((cudaStream_t)stream));
            return;
        }
    }
    Runtime &rt = *p->rt;
    const size_t row_bytes = (size_t)p->W * 4, bytes = row_bytes * p->H;
    // Staging set: the synchronous call uses set 0; asynchronous calls alternate
    // between two sets, so call k+1 uploads into one set while call k's kernels
    // and download still use the other.
    const int set = async ? (int)(rt.async_calls++ % 2) : 0;
    if (rt.stage_bytes != bytes) {
        for (int k = 0; k < 2; k++) {
            for (void *q : rt.stage_in[k]) cudaFree(q);
            for (void *q : rt.stage_out[k]) cudaFree(q);
            rt.stage_in[k].clear();
            rt.stage_out[k].clear();
        }
        rt.stage_bytes = bytes;
    }
    if (rt.stage_in[set].size() != (size_t)n_in || rt.stage_out[set].size() != (size_t)n_out) {
        for (void *q : rt.stage_in[set]) cudaFree(q);
        for (void *q : rt.stage_out[set]) cudaFree(q);
        rt.stage_in[set].assign(n_in, nullptr);
        rt.stage_out[set].assign(n_out, nullptr);
        for (auto &q : rt.stage_in[set])
            if (cudaMalloc(&q, bytes) != cudaSuccess) fail(KF_ERR_OOM, "staging allocation failed");
        for (auto &q : rt.stage_out[set])
            if (cudaMalloc(&q, bytes) != cudaSuccess) fail(KF_ERR_OOM, "staging allocation failed");
    }
    std::vector<void *> &stage_in = rt.stage_in[set], &stage_out = rt.stage_out[set];
    if (!rt.s_h2d) {
        KF_CUDA(cudaStreamCreateWithFlags(&rt.s_h2d, cudaStreamNonBlocking));
        KF_CUDA(cudaStreamCreateWithFlags(&rt.s_d2h, cudaStreamNonBlocking));
        for (int i = 0; i < kHostBands; i++) {
            KF_CUDA(cudaEventCreateWithFlags(&rt.ev_in[i], cudaEventDisableTiming));
            KF_CUDA(cudaEventCreateWithFlags(&rt.ev_out[i], cudaEventDisableTiming));
        }
        KF_CUDA(cudaEventCreateWithFlags(&rt.ev_start, cudaEventDisableTiming));
        KF_CUDA(cudaEventCreateWithFlags(&rt.ev_done, cudaEventDisableTiming));
        for (int k = 0; k < 2; k++) KF_CUDA(cudaEventCreateWithFlags(&rt.ev_kern[k], cudaEventDisableTiming));
    }
    cudaStream_t s = (cudaStream_t)stream;
    bool repeat = false;
    for (const auto &op : p->ops) repeat |= op.kind == LOCAL && op.mode == KF_REPEAT;
    const int R = plan->halo_rows;
    // bands per call: 8 for a synchronous call (its first upload and last
    // download are exposed; thin end bands shorten them), 2 for an asynchronous
    // one (consecutive calls hide each other's ends; fewer, larger copies)
    const int want = std::min(kHostBands, (int)opt(p, async ? "host_async_bands" : "host_bands"));
    int nb = repeat ? 1 : std::max(1, std::min(want, p->H / std::max(64, 4 * R)));
    std::vector<const void *> din(stage_in.begin(), stage_in.end());
    if (!async) {
        // the copy streams start after everything already queued on the caller's stream
        KF_CUDA(cudaEventRecord(rt.ev_start, s));
        KF_CUDA(cudaStreamWaitEvent(rt.s_h2d, rt.ev_start, 0));
        KF_CUDA(cudaStreamWaitEvent(rt.s_d2h, rt.ev_start, 0));
    } else {
        // asynchronous: the upload into this set waits only for the kernels that
        // read it two calls ago (the caller guarantees the host inputs are ready);
        // its download buffers were released when the caller's stream waited for
        // that call's downloads
        KF_CUDA(cudaStreamWaitEvent(rt.s_h2d, rt.ev_kern[set], 0));
    }
    int copied = 0;   // input rows [0, copied) are queued on the H2D stream
    // Band boundaries.  Only the first band's upload and the last band's
    // download are exposed (everything else overlaps), so with 8 bands the
    // ends are thin: row shares 1,3,6,6,6,6,3,1 / 32 (uniform when fewer bands).
    // Tapered shares (option host_taper, nb >= 5): 1, 3, 6, ..., 6, 3, 1 units
    // (nb = 8: 1,3,6,6,6,6,3,1 / 32), else uniform.
    const bool taper = nb >= 5 && opt(p, "host_taper");
    auto units = [&](int k) { return !taper ? 1 : (k == 0 || k == nb - 1) ? 1 : (k == 1 || k == nb - 2) ? 3 : 6; };
    long long tot_units = 0;
    for (int k = 0; k < nb; k++) tot_units += units(k);
    auto cut = [&](int k) {
        long long u = 0;
        for (int i = 0; i < k; i++) u += units(i);
        return (int)((long long)p->H * u / tot_units);
    };
    for (int k = 0; k < nb; k++) {
        const int r0 = cut(k), r1 = cut(k + 1);
        const int need = k == nb - 1 ? p->H : std::min(p->H, r1 + R);
        if (need > copied) {
            for (int i = 0; i < n_in; i++)
                KF_CUDA(cudaMemcpyAsync((char *)stage_in[i] + copied * row_bytes,
                                        (const char *)hin[i] + copied * row_bytes, (need - copied) * row_bytes,
                                        cudaMemcpyHostToDevice, rt.s_h2d));
            copied = need;
        }
        KF_CUDA(cudaEventRecord(rt.ev_in[k], rt.s_h2d));
        KF_CUDA(cudaStreamWaitEvent(s, rt.ev_in[k], 0));
        // the band writes rows [r0, r1) of the whole staging image (out_full): a
        // pointer offset to row r0 would not be 16-B aligned when W % 4 != 0
        std::vector<void *> dout(stage_out.begin(), stage_out.end());
        if (nb == 1)
            run(p, plan, din.data(), n_in, dout.data(), n_out, stream, 0, p->H, 0, p->H);
        else
            run(p, plan, din.data(), n_in, dout.data(), n_out, stream, r0, r1, 0, p->H, true);
        KF_CUDA(cudaEventRecord(rt.ev_out[k], s));
        KF_CUDA(cudaStreamWaitEvent(rt.s_d2h, rt.ev_out[k], 0));
        for (int j = 0; j < n_out; j++)
            KF_CUDA(cudaMemcpyAsync((char *)hout[j] + r0 * row_bytes, (const char *)stage_out[j] + r0 * row_bytes,
                                    (r1 - r0) * row_bytes, cudaMemcpyDeviceToHost, rt.s_d2h));
    }
    KF_CUDA(cudaEventRecord(rt.ev_kern[set], s));
    KF_CUDA(cudaEventRecord(rt.ev_done, rt.s_d2h));
    KF_CUDA(cudaStreamWaitEvent(s, rt.ev_done, 0));
    if (!async) KF_CUDA(cudaStreamSynchronize(s));
}

// Bounds-checking build: the pipeline's violation record (synchronises the
// device).  Other builds have no checks: KF_ERR_ARG.
void bounds_report(kf_pipeline *p, long long *count, unsigned long long *addr, int *kind)
{
#ifdef KF_BOUNDS
    unsigned h[4] = {0, 0, 0, 0};
    if (p->rt && p->rt->viol) {
        KF_CUDA(cudaDeviceSynchronize());
        KF_CUDA(cudaMemcpy(h, p->rt->viol, sizeof h, cudaMemcpyDeviceToHost));
        KF_CUDA(cudaMemset(p->rt->viol, 0, sizeof h));
    }
    *count = h[0];
    *addr = (unsigned long long)h[1] | ((unsigned long long)h[2] << 32);
    *kind = (int)h[3];
#else
    (void)p; (void)count; (void)addr; (void)kind;
    fail(KF_ERR_ARG, "bounds checks are compiled only into libkfuse_bounds.so");
#endif
}

void release_plan(kf_plan *plan)
{
    for (auto &kv : plan->workspace) cudaFree(kv.second);
    plan->workspace.clear();
    plan->compiled.clear();
}

void release_runtime(kf_pipeline *p) { delete p->rt; p->rt = nullptr; }

}  // namespace kf

kf_pipeline::~kf_pipeline() { kf::release_runtime(this); }
kf_plan::~kf_plan() { kf::release_plan(this); }

// Compile-only entry point (no GPU needed): warms the cubin cache for every
// block of a plan.  Used by __graft_entry__.build() and tests.
extern "C" kf_status kf_compile_plan(kf_pipeline *p, const kf_plan *plan)
{
    try {
        for (size_t i = 0; i < plan->blocks.size(); i++) kf::compile_block_cubin(p, plan, (int)i);
        return KF_OK;
    } catch (const kf::Error &e) {
        kf::set_error(e.msg);
        return e.st;
    }
}
