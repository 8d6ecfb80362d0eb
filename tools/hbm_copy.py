"""Copy bandwidth of this box (read + write bytes / time, best of 10): normalises A/B runs across boxes."""
import torch
a = torch.empty(1 << 30, dtype=torch.bfloat16, device="cuda")
b = torch.empty_like(a)
best = 1e9
for _ in range(10):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); b.copy_(a); e1.record(); torch.cuda.synchronize()
    best = min(best, e0.elapsed_time(e1))
print(f"copy GB/s {2 * a.numel() * 2 / best / 1e6:.1f}")
