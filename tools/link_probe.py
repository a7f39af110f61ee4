"""Host link bandwidth probe: pinned H2D / D2H of 8 GiB split over 1, 2 or 4 concurrent streams,
and both directions at once (the e2e link floor)."""
import json, sys
import torch

n = 1 << 30
h = torch.empty(n, dtype=torch.float64).pin_memory()
h2 = torch.empty(n, dtype=torch.float64).pin_memory()
d = torch.empty(n, dtype=torch.float64, device="cuda")
d2 = torch.empty(n, dtype=torch.float64, device="cuda")
h.fill_(1.0); h2.fill_(2.0)


def run(kind, ns):
    streams = [torch.cuda.Stream() for _ in range(ns)]
    step = n // ns
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for i, s in enumerate(streams):
        s.wait_event(e0)
        with torch.cuda.stream(s):
            sl = slice(i * step, (i + 1) * step)
            if kind in ("h2d", "both"):
                d[sl].copy_(h[sl], non_blocking=True)
            if kind in ("d2h", "both"):
                h2[sl].copy_(d2[sl], non_blocking=True)
    for s in streams:
        e1.wait_stream(s) if hasattr(e1, "wait_stream") else torch.cuda.current_stream().wait_stream(s)
    torch.cuda.current_stream().wait_stream(streams[0])
    for s in streams:
        torch.cuda.current_stream().wait_stream(s)
    e1.record()
    e1.synchronize()
    ms = e0.elapsed_time(e1)
    by = n * 8 * (2 if kind == "both" else 1)
    return by / ms / 1e6


for kind in ("h2d", "d2h", "both"):
    for ns in (1, 2, 4):
        best = max(run(kind, ns) for _ in range(3))
        print(json.dumps({"kind": kind, "streams": ns, "GBps": round(best, 2)}), flush=True)
