"""bench.py on the GPU, small and quick: the single-GPU path and the
multi-rank path (nitro_dist_*, NCCL all-gather, max-over-ranks reductions)
with a one-rank communicator (--dist), on configs[1]; the line carries the
contract keys (roofline, e2e with host copies, clocks, gpu_launches)."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("extra", [[], ["--dist"]], ids=["single", "dist1"])
def test_bench_quick_line(extra):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--workload", "c1", "--quick", "--no-cpu",
                        "--steps", "4", "--warmup", "3"] + extra, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [json.loads(l) for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = lines[0]
    assert d["n_gpus"] == 1 and d["steps"] == 4 and d["value"] > 0 and d["unit"] == "GB/s"
    assert d["config"]["workload"].startswith("3d27pt_stencil_128^3")
    assert d["selected_variant"] in d["exhaustive"] and d["gpu_launches"] >= 4
    assert 0 < d["roofline"]["frac"] < 1.2 and d["roofline"]["bound"] == "hbm"
    assert d["e2e"]["h2d_bytes_per_step"] == 128 ** 3 * 4 and d["e2e"]["value"] > 0
    assert "sm_mhz" in d["clocks"]
    if extra:
        assert "nccl_all_gather_floor_ms" in d and "row-partitioned" in d["config"]["parallelism"]
        assert d["e2e"]["api"].startswith("pinned H2D x + nitro_dist_spmv_run")
