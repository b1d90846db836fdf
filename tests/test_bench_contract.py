"""bench.py contract on the CPU: the reference arm (the oracle, --impl
reference) prints one JSON line with the GPU arm's metric string, unit and
config keys, a cpu_baseline and an e2e block (the driver divides the two arms'
values, so they must measure the same thing)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                        "--warmup", "3"], capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    src = open(os.path.join(ROOT, "bench.py")).read()
    assert d["impl"] == "reference"
    assert src.count('"metric": METRIC') == 2     # the same metric string in both arms
    assert d["metric"] == "selected-variant SpMV GB/s vs HBM peak; % of exhaustive-best variant"
    assert d["unit"] == "GB/s" and d["higher_is_better"] is True and d["value"] > 0
    assert d["warmup"] >= 3 and d["steps"] == 1 and d["data"] == "synthetic"
    assert d["config"]["workload"].startswith("3d27pt_stencil_512^3_fp32")
    assert d["config"]["sample_rows"] == 8 * 512 * 512 and d["config"]["sample_nnz"] == 8 * 27 * 510 ** 2 + 8 * 18 * 4 * 510 + 8 * 12 * 4
    # DIA compulsory bytes of configs[4] per row (§8(d)): in-range slots 3,619,156,990
    assert abs(d["config"]["bytes_per_row_credited"] - (3619156990 * 4 + 27 * 4 + 8 * 512 ** 3) / 512 ** 3) < 1e-9
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] == (os.cpu_count() or 1) and cb["value"] == d["value"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]


def test_stencil_rowptr_closed_form_matches_generator():
    """bench.py partitions configs[4] from a closed-form rowptr: it must equal
    the generator's rowptr (checked at n = 12, 17) and its total must be the
    (3n-2)^3 closed form (n = 512)."""
    import numpy as np
    sys.path.insert(0, ROOT)
    import bench
    import synth
    for n in (12, 17):
        assert np.array_equal(bench.stencil_rowptr_host(n), np.asarray(synth.stencil("3d27", n).rowptr, np.int64))
    rp = bench.stencil_rowptr_host(64)
    assert rp[-1] == (3 * 64 - 2) ** 3


def test_multi_gpu_request_relaunches_and_fails_cleanly_without_gpus():
    """`bench.py --gpus 2` without torchrun relaunches itself under
    torch.distributed.run (two ranks); on a box without 2 GPUs rank 0 prints a
    JSON error line naming n_gpus = 2 and the run exits non-zero."""
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1", "--warmup",
                        "3", "--quick", "--no-cpu"], capture_output=True, text=True, timeout=600, cwd=ROOT, env=env)
    assert r.returncode != 0
    lines = [json.loads(l) for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1 and lines[0]["n_gpus"] == 2 and "error" in lines[0], (r.stdout, r.stderr[-2000:])
