"""H2D copy throughput vs size from pinned host memory (torch copies, CUDA events):
small separately pinned tensors vs slices of one large pinned arena."""
import torch
dev = torch.device("cuda", 0)
s = torch.cuda.current_stream()
big = torch.empty(256 << 20, dtype=torch.uint8).pin_memory()
dst = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
for nb in (16 << 10, 256 << 10, 2 << 20, 16 << 20, 128 << 20):
    own = torch.empty(nb, dtype=torch.uint8).pin_memory()
    for name, src in (("own pinned", own), ("arena slice", big[:nb])):
        ts = []
        for r in range(6):
            a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize(); a.record(s)
            dst[:nb].copy_(src, non_blocking=True)
            b.record(s); b.synchronize()
            ts.append(a.elapsed_time(b))
        t = sorted(ts)[len(ts) // 2]
        print("%9d B %-12s %8.1f us %7.1f GB/s" % (nb, name, t * 1000, nb / t / 1e6))
