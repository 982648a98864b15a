"""Host-link probe for the e2e path: 200 MB pinned H2D alone, D2H alone, and both at once on
two streams (full duplex?), CUDA events; prints one JSON line."""
import json
import torch


def main():
    n = 50_000_000
    xh = torch.empty(n, dtype=torch.float32).pin_memory()
    yh = torch.empty(n, dtype=torch.float32).pin_memory()
    xd = torch.empty(n, dtype=torch.float32, device="cuda")
    yd = torch.empty(n, dtype=torch.float32, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    out = {}
    def timeit(fn, k=10):
        fn(); torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(k):
            fn()
        b.record(); torch.cuda.synchronize()
        return a.elapsed_time(b) / k
    def h2d():
        with torch.cuda.stream(s1):
            xd.copy_(xh, non_blocking=True)
        torch.cuda.current_stream().wait_stream(s1)
    def d2h():
        with torch.cuda.stream(s2):
            yh.copy_(yd, non_blocking=True)
        torch.cuda.current_stream().wait_stream(s2)
    def both():
        with torch.cuda.stream(s1):
            xd.copy_(xh, non_blocking=True)
        with torch.cuda.stream(s2):
            yh.copy_(yd, non_blocking=True)
        torch.cuda.current_stream().wait_stream(s1)
        torch.cuda.current_stream().wait_stream(s2)
    for name, f in (("h2d", h2d), ("d2h", d2h), ("both", both)):
        ms = timeit(f)
        out[name] = {"ms": ms, "GBps_per_direction": n * 4 / (ms * 1e-3) / 1e9}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
