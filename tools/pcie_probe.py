"""PCIe copy ceiling: 800 MB pinned host <-> device, each direction alone and both at once."""
import torch, time
n = 800_000_000 // 8
h1 = torch.empty(n, dtype=torch.float64).pin_memory(); h2 = torch.empty(n, dtype=torch.float64).pin_memory()
d1 = torch.empty(n, dtype=torch.float64, device="cuda"); d2 = torch.empty(n, dtype=torch.float64, device="cuda")
s1 = torch.cuda.Stream(); s2 = torch.cuda.Stream()
for it in range(3):
    torch.cuda.synchronize(); t = time.perf_counter()
    with torch.cuda.stream(s1): d1.copy_(h1, non_blocking=True)
    torch.cuda.synchronize(); a = time.perf_counter() - t
    t = time.perf_counter()
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
    torch.cuda.synchronize(); b = time.perf_counter() - t
    t = time.perf_counter()
    with torch.cuda.stream(s1): d1.copy_(h1, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
    torch.cuda.synchronize(); c = time.perf_counter() - t
    print(f"H2D {0.8/a:.1f} GB/s  D2H {0.8/b:.1f} GB/s  both {1.6/c:.1f} GB/s total ({c*1e3:.1f} ms for 800+800 MB)")
