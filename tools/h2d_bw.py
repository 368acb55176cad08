import torch, time
n = 1_800_000_000
h = torch.empty(n, dtype=torch.uint8).pin_memory()
d = torch.empty(n, dtype=torch.uint8, device="cuda")
for it in range(3):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); d.copy_(h, non_blocking=True); e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1); print("h2d GB/s", n / ms / 1e6)
    e0.record(); h.copy_(d, non_blocking=True); e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1); print("d2h GB/s", n / ms / 1e6)
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
h2 = torch.empty(n, dtype=torch.uint8).pin_memory(); d2 = torch.empty(n, dtype=torch.uint8, device="cuda")
torch.cuda.synchronize(); t = time.perf_counter()
with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
torch.cuda.synchronize(); print("duplex GB/s each", n / (time.perf_counter() - t) / 1e9)
