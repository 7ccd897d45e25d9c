"""bench.py host logic on CPU: the workload table is complete and the reference
arm (the CPU oracle) prints the contract's JSON line."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_workload_table():
    sys.path.insert(0, ROOT)
    import bench
    kinds = {"nodewise", "shadow", "saint", "pinsage", "pass_full", "layerwise", "walk"}
    for name, wl in bench.WORKLOADS.items():
        assert wl["kind"] in kinds, name
        assert "graph" in wl and "desc" in wl, name
        if wl["kind"] != "walk":
            assert wl["batch"] > 0, name
    assert set(bench.KERNEL_OF) >= kinds


def test_reference_arm_line():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                          "--workload", "graphsage_tiny", "--steps", "1", "--warmup", "0"],
                         capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads(out.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["value"] > 0
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] >= 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0
