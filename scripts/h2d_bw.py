"""Measured host->device copy bandwidth from pinned memory (the ceiling of the e2e number): one
stream with copies of several sizes, and 14 MB copies spread over 2 and 4 streams."""
import torch
h = torch.empty(448 * (1 << 20) // 4, dtype=torch.float32).pin_memory()
d = torch.empty_like(h, device="cuda")


def run(mb, nstreams, total_mb=448):
    n = mb * (1 << 20) // 4
    ss = [torch.cuda.Stream() for _ in range(nstreams)]
    k = total_mb // mb
    for rep in range(2):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for s in ss:
            s.wait_event(a)
        evs = []
        for i in range(k):
            s = ss[i % nstreams]
            with torch.cuda.stream(s):
                d[i * n:(i + 1) * n].copy_(h[i * n:(i + 1) * n], non_blocking=True)
        for s in ss:
            e = torch.cuda.Event()
            e.record(s)
            torch.cuda.current_stream().wait_event(e)
        b.record()
        torch.cuda.synchronize()
    return k * n * 4 / (a.elapsed_time(b) / 1e3) / 1e9


for mb, ns in ((14, 1), (28, 1), (56, 1), (112, 1), (14, 2), (14, 4), (7, 4), (28, 2)):
    print(f"H2D {mb} MB copies on {ns} stream(s): {run(mb, ns):.1f} GB/s", flush=True)
