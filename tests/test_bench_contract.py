"""The driver's bench contract, checked on CPU: the reference arm (the CPU
oracle, --impl reference) prints one JSON line with the contract's keys, and
our arm fails loudly without a GPU (no CPU fallback prints a number)."""
import json
import os
import subprocess
import sys

import pytest

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


def test_reference_arm_prints_the_contract_line():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--steps", "2",
                        "--warmup", "3"], cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.strip().startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "scaling", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["steps"] == 2 and d["warmup"] == 3
    assert d["value"] > 0 and d["cpu_baseline"]["kind"] == "oracle"
    assert d["cpu_baseline"]["value"] == d["value"] and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert "workload" in d["config"]


@pytest.mark.skipif(_gpu(), reason="checks the no-GPU behaviour")
def test_our_arm_fails_loudly_without_a_gpu():
    r = subprocess.run([sys.executable, "bench.py", "--steps", "1", "--warmup", "3"], cwd=ROOT,
                       capture_output=True, text=True, timeout=600)
    assert r.returncode != 0
    assert not [ln for ln in r.stdout.splitlines() if ln.strip().startswith("{")]


def _fake_reads_res(times, name="c1"):
    import bench_reads
    cfg = bench_reads.read_config(name, 8)
    cfg["policy"] = "sequential"
    st = dict(fill_bytes=16 << 20, major=4096, minor=0, evictions=4032, waits=10,
              downgrades=0, nofree=10)
    return dict(cfg=cfg, times=times, stats=[st] * len(times), err=0, link=55.0, raw_t=3e-4,
                raw_equal=True, reads=(16 << 20) // 16, clocks={}, parity=None,
                other_policies={})


def test_reads_summary_takes_the_slowest_rank():
    """The C1 / C3 objects of the default line: value = the whole job's fill
    bytes over the slowest rank's mean step (the contract's max over ranks)."""
    import argparse
    import bench_reads
    sys.path.insert(0, ROOT)
    args = argparse.Namespace(steps=2, warmup=3, workload="c1")
    fast, slow = _fake_reads_res([1e-3, 1e-3]), _fake_reads_res([2e-3, 2e-3])
    out = bench_reads.reads_summary(args, [fast, slow], 2, "m")
    assert out["ms_per_step"] == 2.0
    assert out["value"] == round(2 * (16 << 20) / 2e-3 / 1e9, 3)
    assert out["step_times"]["n"] == 4 and out["step_times"]["mean_ms"] == 1.5
    assert out["roofline"]["bound"] == "host_link" and 0 < out["roofline"]["frac"]
    assert "parity_vs_oracle" not in out  # rank 0 ran no oracle here
