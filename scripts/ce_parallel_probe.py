"""Development helper: D2H / H2D copy-engine rate with 1, 2 and 4 concurrent streams
(1 GiB total per direction), and D2H + H2D at the same time."""
import torch

dev = torch.device("cuda", 0)
N = 1 << 30
h = torch.empty(N, dtype=torch.uint8).pin_memory()
h2 = torch.empty(N, dtype=torch.uint8).pin_memory()
d = torch.empty(N, dtype=torch.uint8, device=dev)
d2 = torch.empty(N, dtype=torch.uint8, device=dev)


def run(k, direction, reps=5):
    ss = [torch.cuda.Stream(dev) for _ in range(k)]
    part = N // k
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        for i, s in enumerate(ss):
            s.wait_event(e0) if False else None
            with torch.cuda.stream(s):
                sl = slice(i * part, (i + 1) * part)
                if direction in ("d2h", "both"):
                    h[sl].copy_(d[sl], non_blocking=True)
                if direction in ("h2d", "both"):
                    d2[sl].copy_(h2[sl], non_blocking=True)
    for s in ss:
        torch.cuda.current_stream().wait_stream(s)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    mult = 2 if direction == "both" else 1
    return round(N * reps * mult / ms / 1e6, 1)


for direction in ("d2h", "h2d", "both"):
    for k in (1, 2, 4):
        run(k, direction, 1)
        print(direction, k, "streams:", run(k, direction), "GB/s", flush=True)
