import torch, time
n = 109 * 2**20 // 4
h = torch.empty(n, dtype=torch.float32).pin_memory(); d = torch.empty(n, device='cuda')
h2 = torch.empty(n, dtype=torch.float32).pin_memory(); d2 = torch.empty(n, device='cuda')
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
for _ in range(3): d.copy_(h, non_blocking=True); h2.copy_(d2, non_blocking=True)
torch.cuda.synchronize()
def t(f, k=10):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    for _ in range(k): f()
    torch.cuda.synchronize(); return (time.perf_counter() - t0) / k
def both():
    with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
print("H2D GB/s", n*4/t(lambda: d.copy_(h, non_blocking=True))/1e9)
print("D2H GB/s", n*4/t(lambda: h2.copy_(d2, non_blocking=True))/1e9)
print("both ms", t(both)*1e3)
