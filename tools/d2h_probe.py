#!/usr/bin/env python3
"""Probe pinned D2H bandwidth vs buffer size and chunking (context for the e2e leg)."""
import torch

torch.cuda.set_device(0)
for gb in (1, 4, 12):
    n = gb << 30
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(n, dtype=torch.uint8, device="cuda")
    h.copy_(d, non_blocking=True)
    torch.cuda.synchronize()
    for chunks in (1, 8):
        s = torch.cuda.Stream()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            a.record()
            step = n // chunks
            for c in range(chunks):
                h[c * step:(c + 1) * step].copy_(d[c * step:(c + 1) * step], non_blocking=True)
            b.record()
        torch.cuda.synchronize()
        print(f"{gb} GiB pinned, {chunks} chunks: {n / (a.elapsed_time(b) / 1000) / 1e9:.1f} GB/s")
    del h, d
