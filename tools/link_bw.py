"""Pinned host <-> device copy bandwidth on this box (CUDA events, 256 MiB, best of 5)."""
import json
import torch

n = 256 << 20
h = torch.empty(n, dtype=torch.uint8).pin_memory()
d = torch.empty(n, dtype=torch.uint8, device="cuda")
res = {}
for name, fn in (("h2d", lambda: d.copy_(h, non_blocking=True)), ("d2h", lambda: h.copy_(d, non_blocking=True))):
    best = 0.0
    for _ in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        best = max(best, n / (e0.elapsed_time(e1) / 1e3) / 1e9)
    res[name + "_gbs"] = round(best, 1)
s = torch.cuda.Stream()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
h2 = torch.empty(n, dtype=torch.uint8).pin_memory()
d2 = torch.empty(n, dtype=torch.uint8, device="cuda")
torch.cuda.synchronize()
e0.record()
d.copy_(h, non_blocking=True)
with torch.cuda.stream(s):
    h2.copy_(d2, non_blocking=True)
torch.cuda.current_stream().wait_stream(s)
e1.record(); torch.cuda.synchronize()
res["duplex_total_gbs"] = round(2 * n / (e0.elapsed_time(e1) / 1e3) / 1e9, 1)
print(json.dumps(res))
