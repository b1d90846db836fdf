#!/usr/bin/env python
"""Host<->device copy rates with pinned buffers: H2D alone, D2H alone, both at
once on two streams (the ceiling of the pipelined host-buffer SpMV call)."""
import sys
import torch


def timed(fn, reps=20):
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for r in range(reps + 3):
        torch.cuda.synchronize()
        s.record()
        fn()
        e.record()
        torch.cuda.synchronize()
        if r >= 3:
            ts.append(s.elapsed_time(e) * 1e-3)
    ts.sort()
    return ts[len(ts) // 2]


def main():
    dev = torch.device("cuda:0")
    for mb in [float(a) for a in sys.argv[1:]] or [8.0, 64.0]:
        n = int(mb * (1 << 20)) // 4
        hx = torch.ones(n, dtype=torch.float32).pin_memory()
        hy = torch.empty(n, dtype=torch.float32).pin_memory()
        dx = torch.empty(n, dtype=torch.float32, device=dev)
        dy = torch.ones(n, dtype=torch.float32, device=dev)
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
        cur = torch.cuda.current_stream()

        def both():
            s1.wait_stream(cur)
            s2.wait_stream(cur)
            with torch.cuda.stream(s1):
                dx.copy_(hx, non_blocking=True)
            with torch.cuda.stream(s2):
                hy.copy_(dy, non_blocking=True)
            cur.wait_stream(s1)
            cur.wait_stream(s2)

        th = timed(lambda: dx.copy_(hx, non_blocking=True))
        td = timed(lambda: hy.copy_(dy, non_blocking=True))
        tb = timed(both)
        B = n * 4
        print(f"{mb:g} MB: H2D {th*1e6:.0f} us ({B/th/1e9:.1f} GB/s)  D2H {td*1e6:.0f} us ({B/td/1e9:.1f} GB/s)  "
              f"both {tb*1e6:.0f} us ({2*B/tb/1e9:.1f} GB/s total)", flush=True)


if __name__ == "__main__":
    main()
