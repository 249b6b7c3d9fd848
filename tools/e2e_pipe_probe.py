"""Is kf_run_host's e2e limited by the copies themselves?  Replays its copy
schedule (8 row bands: H2D of band k on one stream, D2H of band k on another
after band k's H2D) with no kernels, for 4096^2 f32, and compares with one
H2D + one D2H of the whole image running concurrently."""
import json
import time
import torch

W = H = 4096
rb = W * 4
hin = torch.empty(H * W, dtype=torch.float32).pin_memory()
hout = torch.empty(H * W, dtype=torch.float32).pin_memory()
din = torch.empty(H * W, dtype=torch.float32, device="cuda")
dout = torch.empty(H * W, dtype=torch.float32, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def banded(cuts):
    evs = []
    for k in range(len(cuts) - 1):
        r0, r1 = cuts[k], cuts[k + 1]
        with torch.cuda.stream(s1):
            din[r0 * W:r1 * W].copy_(hin[r0 * W:r1 * W], non_blocking=True)
            e = torch.cuda.Event()
            e.record(s1)
        s2.wait_event(e)
        with torch.cuda.stream(s2):
            hout[r0 * W:r1 * W].copy_(dout[r0 * W:r1 * W], non_blocking=True)
    torch.cuda.synchronize()


def whole():
    with torch.cuda.stream(s1):
        din.copy_(hin, non_blocking=True)
    with torch.cuda.stream(s2):
        hout.copy_(dout, non_blocking=True)
    torch.cuda.synchronize()


def t(fn, n=10):
    fn()
    t0 = time.perf_counter()
    for _ in range(n):
        fn()
    return (time.perf_counter() - t0) / n * 1e3


uni = [H * k // 8 for k in range(9)]
tap = [H * c // 32 for c in (0, 1, 4, 10, 16, 22, 28, 31, 32)]
b16 = [H * k // 16 for k in range(17)]
print(json.dumps({"whole_concurrent_ms": round(t(whole), 3), "bands8_uniform_ms": round(t(lambda: banded(uni)), 3),
                  "bands8_taper_ms": round(t(lambda: banded(tap)), 3), "bands16_ms": round(t(lambda: banded(b16)), 3)}))
