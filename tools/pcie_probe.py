"""PCIe ceiling for the H0 staging path (run under gpurun): pinned host -> HBM copy
bandwidth on 1 and 2 streams (copy engines), and device -> host.  Not part of the product."""
import json
import sys

import torch

GB = 4 << 30
src = torch.empty(GB, dtype=torch.uint8).pin_memory()
src.fill_(7)
dst = torch.empty(GB, dtype=torch.uint8, device="cuda")
out = {}


def timed(fn, reps=3):
    best = 1e9
    for _ in range(reps):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) / 1e3)
    return best


def one():
    dst.copy_(src, non_blocking=True)


s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
h = GB // 2


def two():
    cur = torch.cuda.current_stream()
    s1.wait_stream(cur)
    s2.wait_stream(cur)
    with torch.cuda.stream(s1):
        dst[:h].copy_(src[:h], non_blocking=True)
    with torch.cuda.stream(s2):
        dst[h:].copy_(src[h:], non_blocking=True)
    cur.wait_stream(s1)
    cur.wait_stream(s2)


def d2h():
    src.copy_(dst, non_blocking=True)


out["h2d_1stream_GBps"] = GB / timed(one) / 1e9
out["h2d_2streams_GBps"] = GB / timed(two) / 1e9
out["d2h_1stream_GBps"] = GB / timed(d2h) / 1e9
print(json.dumps(out))
