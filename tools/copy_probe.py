#!/usr/bin/env python
"""Device copy bandwidth vs size (L2 flushed before each rep, median of 20):
the practical ceiling for a kernel moving the same number of bytes."""
import sys
import torch

def main():
    dev = torch.device("cuda:0")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for mb in [int(a) for a in sys.argv[1:]] or [64, 128, 242, 470, 1000, 4000]:
        n = (mb << 20) // 8          # half read, half write
        a = torch.ones(n, dtype=torch.float32, device=dev)
        b = torch.empty_like(a)
        ts = []
        for r in range(23):
            flush.fill_(r & 255)
            s.record(); b.copy_(a); e.record(); torch.cuda.synchronize()
            if r >= 3:
                ts.append(s.elapsed_time(e) * 1e-3)
        ts.sort()
        t = ts[len(ts) // 2]
        print(f"copy {mb} MB moved: {t*1e6:.1f} us  {(mb << 20) / t / 1e9:.0f} GB/s", flush=True)
        c = torch.ones((mb << 20) // 4, dtype=torch.float32, device=dev)   # read-only: a sum over mb MB
        ts = []
        for r in range(23):
            flush.fill_(r & 255)
            s.record(); c.sum(); e.record(); torch.cuda.synchronize()
            if r >= 3:
                ts.append(s.elapsed_time(e) * 1e-3)
        ts.sort()
        t = ts[len(ts) // 2]
        print(f"read {mb} MB (torch sum): {t*1e6:.1f} us  {(mb << 20) / t / 1e9:.0f} GB/s", flush=True)
        del c
        del a, b

if __name__ == "__main__":
    main()
