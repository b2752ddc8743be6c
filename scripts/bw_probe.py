#!/usr/bin/env python
"""Achievable HBM bandwidth by access pattern (GPU box): pure write (fill), read+write (copy),
pure read (sum), 2 GiB buffers, CUDA events, best of 10.  The ceiling for the write-dominated
unfused entries (A1 writes 32 B per det-sample and reads ~0)."""
import json

import torch

n = (2 << 30) // 8
a = torch.empty(n, dtype=torch.float64, device="cuda")
b = torch.empty(n, dtype=torch.float64, device="cuda")
a.fill_(1.0)


def best(fn, nbytes):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(10):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return nbytes / (min(ts) * 1e-3) / 1e9


out = {"write_gbs": best(lambda: b.fill_(2.0), 8 * n), "copy_gbs": best(lambda: b.copy_(a), 16 * n),
       "read_gbs": best(lambda: a.sum(), 8 * n)}
print(json.dumps(out))
