"""Diagnostic: device-to-device copy bandwidth of torch (cudaMemcpy-class) at the
benchmark image sizes, the practical HBM ceiling for a read+write stream."""
import torch

for n in (4096, 8192, 16384):
    xs = [torch.rand(n, n, device="cuda") for _ in range(4)]
    ys = [torch.empty_like(x) for x in xs]
    for i in range(8):
        ys[i % 4].copy_(xs[i % 4])
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    with torch.cuda.graph(g, stream=s):
        for i in range(200):
            ys[i % 4].copy_(xs[i % 4])
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        g.replay()
        torch.cuda.synchronize()
        e0.record(s)
        g.replay()
        e1.record(s)
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) / 200 * 1e3
    print(f"{n}x{n} f32 copy: {us:.2f} us  {2 * 4 * n * n / us / 1e3:.1f} GB/s")
