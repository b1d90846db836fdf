#!/usr/bin/env python
"""Host-buffer call (nitro_spmv_run_host) on configs[4] (3D 27-pt 512^3, DIA):
time per call against the number of row chunks of the copy/multiply pipeline
(NITRO_RUN_HOST_CHUNKS is read once per process, so each count runs in its own
process).  usage: python tools/e2e_chunks.py [counts...]"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import sys, json, torch
sys.path.insert(0, sys.argv[1])
import paper_conf_ipps_muralidharanshgc14_b200 as nitro, synth
dev = torch.device("cuda:0")
A = synth.stencil("3d27", 512, mode=1, seed=1, device=dev)
M = nitro.SpMV.from_csr(A)
hx = torch.empty(A.cols, dtype=torch.float32).pin_memory(); hx.uniform_(-1, 1)
hy = torch.empty(A.rows, dtype=torch.float32).pin_memory()
M.prepare(nitro.DIA)
ts = []
for r in range(8):
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record(); M.run_host(nitro.DIA, hx.numpy(), hy.numpy()); e.record(); e.synchronize()
    if r >= 2: ts.append(s.elapsed_time(e))
ts.sort()
print(json.dumps({"ms": ts[len(ts) // 2], "GBps_h2d_d2h": 2 * A.rows * 4 / (ts[len(ts) // 2] * 1e-3) / 1e9}))
"""


def main():
    counts = [int(c) for c in sys.argv[1:]] or [1, 4, 8, 16, 32]
    out = {}
    for c in counts:
        env = dict(os.environ, NITRO_RUN_HOST_CHUNKS=str(c))
        r = subprocess.run([sys.executable, "-c", CHILD, ROOT], env=env, capture_output=True, text=True, timeout=600)
        line = [l for l in r.stdout.splitlines() if l.startswith("{")]
        out[c] = json.loads(line[-1]) if line else {"error": r.stderr[-500:]}
        print(c, out[c], flush=True)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
