"""Device -> pinned-host copy bandwidth on this box (the e2e leg's bound): one 238 MB copy, the same
bytes as K chunks on one stream, and split over 2 / 4 concurrent streams.  Usage: python tools/pcie_bw.py"""
import json
import torch

MB = 238 * 2**20
dev = torch.empty(MB // 8, dtype=torch.float64, device="cuda").normal_()
host = torch.empty(MB // 8, dtype=torch.float64).pin_memory()
res = {}


def timed(fn, reps=5):
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(reps):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b))
    return best


for nstreams in (1, 2, 4):
    streams = [torch.cuda.Stream() for _ in range(nstreams)]

    def go():
        cur = torch.cuda.current_stream()
        n = dev.numel()
        for k, s in enumerate(streams):
            s.wait_stream(cur)
            with torch.cuda.stream(s):
                lo, hi = n * k // nstreams, n * (k + 1) // nstreams
                host[lo:hi].copy_(dev[lo:hi], non_blocking=True)
        for s in streams:
            cur.wait_stream(s)

    ms = timed(go)
    res[f"d2h_streams{nstreams}_GBps"] = round(MB / ms / 1e6, 2)
for k in (8, 32):
    def go():
        n = dev.numel()
        for c in range(k):
            lo, hi = n * c // k, n * (c + 1) // k
            host[lo:hi].copy_(dev[lo:hi], non_blocking=True)
    ms = timed(go)
    res[f"d2h_chunks{k}_GBps"] = round(MB / ms / 1e6, 2)


def h2d():
    dev.copy_(host, non_blocking=True)


res["h2d_GBps"] = round(MB / timed(h2d) / 1e6, 2)
print(json.dumps(res))
