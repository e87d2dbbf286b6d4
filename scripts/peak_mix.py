#!/usr/bin/env python
"""HBM ceiling for C5's traffic mix (2 reads : 1 write, bf16) measured with
torch's own elementwise kernel: z = x + y over C5's 1,073,741,824 elements."""
import torch

n = 1 << 30
x = torch.randn(n, device="cuda", dtype=torch.bfloat16)
y = torch.randn(n, device="cuda", dtype=torch.bfloat16)
z = torch.empty_like(x)
for _ in range(3):
    torch.add(x, y, out=z)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
best = 1e9
for _ in range(10):
    e0.record()
    torch.add(x, y, out=z)
    e1.record()
    torch.cuda.synchronize()
    best = min(best, e0.elapsed_time(e1))
gbs = 3 * 2 * n / (best * 1e-3) / 1e9
print(f"torch add bf16 2R:1W over {n} elements: {best * 1e3:.1f} us, {gbs:.1f} GB/s")
a = torch.empty(n, device="cuda", dtype=torch.bfloat16)
for _ in range(3):
    a.copy_(x)
best = 1e9
for _ in range(10):
    e0.record()
    a.copy_(x)
    e1.record()
    torch.cuda.synchronize()
    best = min(best, e0.elapsed_time(e1))
print(f"torch copy bf16 1R:1W: {best * 1e3:.1f} us, {2 * 2 * n / (best * 1e-3) / 1e9:.1f} GB/s")
s = torch.empty(1, device="cuda", dtype=torch.float32)
best = 1e9
for _ in range(10):
    e0.record()
    s = x.sum(dtype=torch.float32)
    e1.record()
    torch.cuda.synchronize()
    best = min(best, e0.elapsed_time(e1))
print(f"torch sum bf16 read-only: {best * 1e3:.1f} us, {2 * n / (best * 1e-3) / 1e9:.1f} GB/s")
