// peer.cu -- multi-GPU halo rows over peer memory (NVLink P2P), the north
// star's "extra halo rows that fused stencils need are read from peer memory
// over NVLink" (BASELINE.json).  Three tiny kernels, all
// stream-ordered and CUDA-graph-capturable, synchronised by monotonic counters
// in device memory instead of a host-side collective:
//
//   kf_peer_signal  release-increments counters that live in the NEIGHBOURS'
//                   memory ("my rows of this step are ready")
//   kf_peer_pull    waits (acquire) until a local counter passes its local
//                   `seen` count, copies the neighbour's boundary rows from
//                   its buffer into the local halo rows, bumps `seen`, and
//                   release-increments the neighbour's ack counter
//   kf_peer_wait    waits until local counters reach local targets (e.g. both
//                   neighbours acked every signal before the own rows are
//                   overwritten)
//
// Counters are compared wrap-safe ((int32)(a - b) >= 0).  Every spin is
// bounded: after `spin_limit` polls the kernel sets *err and gives up, so a
// missing neighbour turns into an error, never a hang.
#include <cuda_runtime.h>

#include <cstdint>

#include "kf_internal.h"

namespace kf {
namespace {

constexpr int kMaxSeg = 4;

struct SigArgs {
    unsigned *flag[kMaxSeg];   // peer (or local) counters
    unsigned *sent;            // local count of signals (nullable)
    int n;
};
constexpr int kMaxCopy = 8;   // copies per segment (one per pipeline input)

struct PullArgs {
    void *dst[kMaxSeg][kMaxCopy];
    const void *src[kMaxSeg][kMaxCopy];   // peer rows
    long long bytes[kMaxSeg][kMaxCopy];
    int m;                     // copies per segment
    unsigned *flag[kMaxSeg];   // local counter written by the neighbour
    unsigned *seen[kMaxSeg];   // local count of pulls done
    unsigned *ack[kMaxSeg];    // neighbour's ack counter (peer, nullable)
    unsigned *err;
    long long spin_limit;
    int n;
};
struct WaitArgs {
    unsigned *counter[kMaxSeg];
    unsigned *target[kMaxSeg];
    unsigned *err;
    long long spin_limit;
    int n;
};

__device__ __forceinline__ unsigned ld_acquire_sys(const unsigned *p)
{
    unsigned v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void red_release_sys(unsigned *p, unsigned v)
{
    asm volatile("red.release.sys.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ bool spin_until(const unsigned *p, unsigned want, long long limit, unsigned *err)
{
    for (long long it = 0; (int)(ld_acquire_sys(p) - want) < 0; it++) {
        if (it >= limit) {
            atomicExch(err, 1u);
            return false;
        }
        __nanosleep(128);
    }
    return true;
}

__global__ void peer_signal_k(const __grid_constant__ SigArgs a)
{
    const int i = threadIdx.x;
    __threadfence_system();   // the rows written before this kernel, ordered before the counters
    if (i < a.n) red_release_sys(a.flag[i], 1u);
    if (i == 0 && a.sent) *a.sent += 1u;
}

// one CTA per segment
__global__ void __launch_bounds__(512) peer_pull_k(const __grid_constant__ PullArgs a)
{
    const int s = blockIdx.x;
    __shared__ int ok;
    __shared__ unsigned want;
    if (threadIdx.x == 0) {
        want = *a.seen[s] + 1u;
        ok = spin_until(a.flag[s], want, a.spin_limit, a.err);
    }
    __syncthreads();   // the acquire of thread 0 orders the copies below (causality via bar.sync)
    if (!ok) return;
    for (int c = 0; c < a.m; c++) {
        // 16-B vectors when both ends are 16-B aligned (rows of a W % 4 == 0
        // image), else 4-B words (any f32 / uchar4 row offset), else bytes;
        // then the tail.
        const uintptr_t al = (uintptr_t)a.src[s][c] | (uintptr_t)a.dst[s][c];
        const char *sb = (const char *)a.src[s][c];
        char *db = (char *)a.dst[s][c];
        const long long nb = a.bytes[s][c];
        long long done = 0;
        if ((al & 15) == 0) {
            const long long n16 = nb >> 4;
            const int4 *src = (const int4 *)sb;
            int4 *dst = (int4 *)db;
            for (long long i = threadIdx.x; i < n16; i += blockDim.x) dst[i] = __ldcv(src + i);   // NVLink P2P loads
            done = n16 << 4;
        } else if ((al & 3) == 0) {
            const long long n4 = nb >> 2;
            const unsigned *src = (const unsigned *)sb;
            unsigned *dst = (unsigned *)db;
            for (long long i = threadIdx.x; i < n4; i += blockDim.x) dst[i] = __ldcv(src + i);
            done = n4 << 2;
        }
        for (long long i = done + threadIdx.x; i < nb; i += blockDim.x) db[i] = sb[i];
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        *a.seen[s] = want;
        if (a.ack[s]) red_release_sys(a.ack[s], 1u);   // the neighbour may now overwrite those rows
    }
}

__global__ void peer_wait_k(const __grid_constant__ WaitArgs a)
{
    const int i = threadIdx.x;
    if (i < a.n) spin_until(a.counter[i], *a.target[i], a.spin_limit, a.err);
}

}  // namespace
}  // namespace kf

using namespace kf;

#define KF_GUARD(...)                                                                          \
    do {                                                                                       \
        __VA_ARGS__;                                                                           \
        cudaError_t e_ = cudaGetLastError();                                                   \
        if (e_ != cudaSuccess) {                                                               \
            set_error(std::string("peer kernel launch: ") + cudaGetErrorString(e_));          \
            return KF_ERR_CUDA;                                                                \
        }                                                                                      \
        return KF_OK;                                                                          \
    } while (0)

extern "C" kf_status kf_peer_signal(uint32_t *const *flags, int32_t n, uint32_t *sent, void *stream)
{
    if (n < 0 || n > kMaxSeg || (n && !flags)) {
        set_error("kf_peer_signal: 0..4 counters");
        return KF_ERR_ARG;
    }
    SigArgs a{};
    for (int i = 0; i < n; i++) a.flag[i] = flags[i];
    a.sent = sent;
    a.n = n;
    KF_GUARD(peer_signal_k<<<1, 32, 0, (cudaStream_t)stream>>>(a));
}

extern "C" kf_status kf_peer_pull(int32_t n, int32_t m, void *const *dst, const void *const *src,
                                  const int64_t *bytes, uint32_t *const *flag, uint32_t *const *seen,
                                  uint32_t *const *ack, uint32_t *err, int64_t spin_limit, void *stream)
{
    if (n < 0 || n > kMaxSeg || m < 1 || m > kMaxCopy || !err || (n && (!dst || !src || !bytes || !flag || !seen))) {
        set_error("kf_peer_pull: bad arguments (0..4 segments of 1..8 copies)");
        return KF_ERR_ARG;
    }
    if (n == 0) return KF_OK;
    PullArgs a{};
    a.m = m;
    for (int i = 0; i < n; i++) {
        if (!flag[i] || !seen[i]) {
            set_error("kf_peer_pull: null counter");
            return KF_ERR_ARG;
        }
        for (int c = 0; c < m; c++) {
            const int j = i * m + c;
            if (!dst[j] || !src[j] || bytes[j] < 0) {
                set_error("kf_peer_pull: null copy");
                return KF_ERR_ARG;
            }
            a.dst[i][c] = dst[j];
            a.src[i][c] = src[j];
            a.bytes[i][c] = bytes[j];
        }
        a.flag[i] = flag[i];
        a.seen[i] = seen[i];
        a.ack[i] = ack ? ack[i] : nullptr;
    }
    a.err = err;
    a.spin_limit = spin_limit;
    a.n = n;
    KF_GUARD(peer_pull_k<<<n, 512, 0, (cudaStream_t)stream>>>(a));
}

extern "C" kf_status kf_peer_wait(int32_t n, uint32_t *const *counter, uint32_t *const *target, uint32_t *err,
                                  int64_t spin_limit, void *stream)
{
    if (n < 0 || n > kMaxSeg || !err || (n && (!counter || !target))) {
        set_error("kf_peer_wait: bad arguments");
        return KF_ERR_ARG;
    }
    if (n == 0) return KF_OK;
    WaitArgs a{};
    for (int i = 0; i < n; i++) {
        a.counter[i] = counter[i];
        a.target[i] = target[i];
    }
    a.err = err;
    a.spin_limit = spin_limit;
    a.n = n;
    KF_GUARD(peer_wait_k<<<1, 32, 0, (cudaStream_t)stream>>>(a));
}

// Lets kernels on `device` read and write `peer_device`'s memory (NVLink P2P),
// in the primary context every runtime in the process shares.  Idempotent.
extern "C" kf_status kf_peer_enable(int32_t device, int32_t peer_device)
{
    if (device == peer_device) return KF_OK;
    int can = 0;
    if (cudaDeviceCanAccessPeer(&can, device, peer_device) != cudaSuccess || !can) {
        set_error("kf_peer_enable: device " + std::to_string(device) + " cannot access device " +
                  std::to_string(peer_device));
        return KF_ERR_CUDA;
    }
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(device);
    cudaError_t e = cudaDeviceEnablePeerAccess(peer_device, 0);
    cudaSetDevice(cur);
    if (e == cudaErrorPeerAccessAlreadyEnabled) {
        cudaGetLastError();   // clear the sticky-free "already enabled" status
        return KF_OK;
    }
    if (e != cudaSuccess) {
        set_error(std::string("kf_peer_enable: ") + cudaGetErrorString(e));
        return KF_ERR_CUDA;
    }
    return KF_OK;
}
