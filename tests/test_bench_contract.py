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
    assert src.count(f'"metric": "{d["metric"]}"') == 2     # the same string in both arms
    assert d["metric"] == "selected-variant SpMV GB/s vs HBM peak; % of exhaustive-best variant"
    assert d["unit"] == "GB/s" and d["higher_is_better"] is True and d["value"] > 0
    assert d["warmup"] >= 3 and d["steps"] == 1 and d["data"] == "synthetic"
    assert d["config"]["workload"].startswith("3d27pt_stencil_128^3_fp32")
    assert d["config"]["rows_per_gpu"] == 128 ** 3 and d["config"]["nnz_per_gpu"] == (3 * 128 - 2) ** 3
    assert d["config"]["bytes_per_step"] == 242087012     # DIA compulsory bytes of configs[1] (§8(d))
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] == d["value"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
