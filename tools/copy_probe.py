"""torch's own device copy at the bench sizes, timed like bench.py (graph replay,
4 rotating buffer sets): is the framework's copy kernel at the practical floor?"""
import json
import torch

for (W, H) in ((2048, 2048), (4096, 4096)):
    ins = [torch.rand(H, W, device="cuda") for _ in range(4)]
    outs = [torch.empty_like(x) for x in ins]
    s = torch.cuda.Stream()
    steps = 200
    with torch.cuda.stream(s):
        for i in range(3):
            outs[i % 4].copy_(ins[i % 4])
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for i in range(steps):
            outs[i % 4].copy_(ins[i % 4])
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        g.replay()
        torch.cuda.synchronize()
        e0.record(s)
        g.replay()
        e1.record(s)
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) / steps * 1e3
    print(json.dumps({"W": W, "H": H, "torch_copy_us": round(us, 2), "gbs": round(8 * W * H / us / 1e3, 1)}))
