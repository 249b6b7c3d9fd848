"""Where does the banded host<->device copy schedule lose against two whole
concurrent copies?  Variants on 4096^2 f32 (64 MiB each way), pinned buffers:
  whole      one H2D and one D2H, concurrent, no dependency
  dep8       8 bands: D2H of band k waits for H2D of band k (kf_run_host's shape)
  nodep8     8 bands each way, no cross-stream dependency (chunking cost only)
  dep8_2s    as dep8, H2D bands alternate over two streams
  dep8_big   as dep8 but the D2H of bands 0-6 is one copy after band 6, then band 7
Diagnostics only."""
import json
import time
import torch

W = H = 4096
hin = torch.empty(H * W, dtype=torch.float32).pin_memory()
hout = torch.empty(H * W, dtype=torch.float32).pin_memory()
din = torch.empty(H * W, dtype=torch.float32, device="cuda")
dout = torch.empty(H * W, dtype=torch.float32, device="cuda")
a1, a2, b1 = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()
cuts = [H * k // 8 for k in range(9)]


def sl(t, k):
    return t[cuts[k] * W:cuts[k + 1] * W]


def whole():
    with torch.cuda.stream(a1):
        din.copy_(hin, non_blocking=True)
    with torch.cuda.stream(b1):
        hout.copy_(dout, non_blocking=True)
    torch.cuda.synchronize()


def dep8(two=False, dep=True):
    for k in range(8):
        s = a2 if (two and k % 2) else a1
        with torch.cuda.stream(s):
            sl(din, k).copy_(sl(hin, k), non_blocking=True)
            e = torch.cuda.Event()
            e.record(s)
        if dep:
            b1.wait_event(e)
        with torch.cuda.stream(b1):
            sl(hout, k).copy_(sl(dout, k), non_blocking=True)
    torch.cuda.synchronize()


def dep8_big():
    evs = []
    for k in range(8):
        with torch.cuda.stream(a1):
            sl(din, k).copy_(sl(hin, k), non_blocking=True)
            e = torch.cuda.Event()
            e.record(a1)
            evs.append(e)
    b1.wait_event(evs[6])
    with torch.cuda.stream(b1):
        hout[:cuts[7] * W].copy_(dout[:cuts[7] * W], non_blocking=True)
    b1.wait_event(evs[7])
    with torch.cuda.stream(b1):
        sl(hout, 7).copy_(sl(dout, 7), non_blocking=True)
    torch.cuda.synchronize()


def t(fn, n=10):
    fn()
    v = []
    for _ in range(5):
        t0 = time.perf_counter()
        for _ in range(n):
            fn()
        v.append((time.perf_counter() - t0) / n * 1e3)
    return round(sorted(v)[2], 3)


print(json.dumps({"whole": t(whole), "dep8": t(dep8), "nodep8": t(lambda: dep8(dep=False)),
                  "dep8_2s": t(lambda: dep8(two=True)), "dep8_big": t(dep8_big),
                  "h2d_only_whole": t(lambda: (din.copy_(hin, non_blocking=True), torch.cuda.synchronize())),
                  "d2h_only_whole": t(lambda: (hout.copy_(dout, non_blocking=True), torch.cuda.synchronize()))}))
