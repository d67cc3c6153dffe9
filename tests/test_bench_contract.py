"""bench.py's reference arm (the oracle on the host cores, tier framing ④) runs on the CPU
box and prints one JSON line with the contract's keys; the GPU arm's line is checked on the
B200 (-m gpu)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                        "--steps", "2", "--warmup", "3", "--n", "48", "--cpu-seconds", "1"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    for key in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
                "higher_is_better", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert key in d, key
    assert d["impl"] == "reference" and d["unit"] == "GB/s" and d["value"] > 0
    assert d["e2e"]["value"] == d["value"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    sys.path.insert(0, ROOT)
    import bench
    assert d["config"]["workload"] == bench.workload_name(48)
    assert d["metric"] == bench.METRIC


@pytest.mark.gpu
def test_gpu_arm_json_line():
    """The driver's contract on the B200 (-m gpu): one JSON line with every key, the kernel
    roofline against the measured peak, e2e with host<->device bytes, clocks, and one
    proteus launch per sweep in the timed region."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--steps", "50",
                        "--warmup", "3", "--job-sweeps", "50", "--cpu-seconds", "1",
                        "--e2e-processes", "0"],
                       capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    for key in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
                "higher_is_better", "scaling", "vs_baseline", "dtype", "data", "config",
                "roofline", "cpu_baseline", "e2e", "gpu_launches", "clocks"):
        assert key in d, key
    assert d["n_gpus"] == 1 and d["steps"] == 50 and d["gpu_launches"] == 50
    rl = d["roofline"]
    assert rl["bound"] == "hbm" and rl["unit"] == "GB/s" and 0.3 < rl["frac"] < 1.2
    assert abs(rl["achieved"] / rl["peak"] - rl["frac"]) < 1e-3
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0
    assert d["e2e"]["d2h_bytes_per_step"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["clocks"]["samples"] >= 1
    assert d["speedup_vs_aot"]["cold_compiles"] == 1
    # CFG 1/3/4/5 beside the CFG 2 line (VERDICT r01 "Next" 5): every workload measured,
    # its oracle spot check passing, and the stencil attribution present
    su = d["suite"]
    assert "error" not in su, su
    for w in ("adam_run", "xs", "micro"):
        par = su[w]["cpu_baseline"]["parity"]
        assert all(v.get("ok", v.get("bit_exact")) for v in par.values()), (w, par)
    assert su["micro"]["kernel_speedup"] > 1.0 and su["xs"]["step_speedup"] > 1.0
    assert su["cache"]["compile_ms_p50"] > 0 and su["cache"]["hit_overhead_us"] < 5
    att = su["stencil_attribution"]
    assert att["jit_all_us"] < att["aot_us"]



@pytest.mark.gpu
def test_gpu_adam_workload_line():
    """bench.py --workload adam (CFG 1 over parameter shards): one JSON line, the SFU
    roofline (the folded adam_run is XU-pipe bound), one adam_run launch per bench step."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--workload", "adam",
                        "--steps", "50", "--warmup", "3"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["unit"] == "param-steps/s" and d["value"] > 1e11 and d["gpu_launches"] == 50
    assert d["roofline"]["bound"] == "sfu" and 0.2 < d["roofline"]["frac"] < 1.05
    assert d["e2e"]["value"] > 0 and d["jit"]["compiles"] == 1
