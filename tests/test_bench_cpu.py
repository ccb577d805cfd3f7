"""bench.py on CPU: the flop accounting behind every GFLOPS number and the
roofline denominators, and the reference arm's JSON contract.

The LAWN-41 counts (reading Q1) are checked against a brute-force
count of multiply-adds from each routine's definition at a tiny order (so a
wrong exponent or a dropped triangle factor fails), and the reference arm
(`--impl reference`, the fp64 oracle on host cores) must print one JSON line
with the driver's keys."""
import importlib.util
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def bench():
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def brute_force_flops(n):
    """2 flops per multiply-add, counted from the loop nests (side=L, lower,
    uplo triangle of C incl. the diagonal); TRMM/TRSM: the triangle's k <= i
    multiply-adds per column (n(n+1)/2 each) -- LAWN-41 counts n^2 per column
    for both (the diagonal scaling is counted as one multiply)."""
    gemm = 2 * n * n * n
    syrk = sum(2 * n for i in range(n) for j in range(n) if j <= i)       # C(i,j), i >= j: k terms
    syr2k = sum(4 * n for i in range(n) for j in range(n) if j <= i)
    trmm = n * sum(2 * (i + 1) - 1 for i in range(n))                    # (i+1) mults, i adds per row
    return {"sgemm": gemm, "ssymm": gemm, "ssyrk": syrk, "ssyr2k": syr2k, "strmm": trmm, "strsm": trmm}


@pytest.mark.parametrize("n", [1, 2, 7, 16])
def test_lawn41_counts(bench, n):
    fl = bench.flops(n)
    bf = brute_force_flops(n)
    for r in ("sgemm", "ssymm", "strmm", "strsm"):
        assert fl[r] == bf[r], r
    # SYRK: k n(n+1) multiply-adds-and-adds; SYR2K: 2 k n^2 + n (LAWN-41)
    assert fl["ssyrk"] == bf["ssyrk"] == n * n * (n + 1)
    assert fl["ssyr2k"] == 2 * n ** 3 + n and abs(bf["ssyr2k"] - fl["ssyr2k"]) <= 2 * n * n


def test_column_sampling_scales_linearly(bench):
    full, half = bench.flops(64), bench.flops(64, cols=32)
    for r in full:
        assert half[r] == pytest.approx(full[r] / 2)


def test_peak_denominators(bench):
    peaks = {"bf16_tflops": 1600.0, "bf16_tflops_sustained": 1400.0}
    tf32_3x = bench.fp32_3xtf32_peak(peaks, sustained=True)
    assert tf32_3x == pytest.approx(1400.0 * (1.1 / 2.25) / 3.0)
    assert bench.fp32_3xtf32_peak(peaks, sustained=False) == pytest.approx(1600.0 * (1.1 / 2.25) / 3.0)


def test_reference_arm_json_contract():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--steps", "1", "--warmup", "0",
                        "--cpu-seconds", "1"], cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for key in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
                "higher_is_better", "scaling", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert key in d, key
    assert d["impl"] == "reference" and d["value"] > 0 and d["higher_is_better"] is True
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["config"]["n"] == 8192


def test_spawn_command(bench):
    cmd = bench.spawn_command(8, ["bench.py", "--gpus", "8", "--steps", "5"], port=29555)
    assert cmd[1:4] == ["-m", "torch.distributed.run", "--nnodes=1"]
    assert "--nproc-per-node=8" in cmd
    i = cmd.index("--master-addr")
    assert cmd[i + 1] == "127.0.0.1" and cmd[cmd.index("--master-port") + 1] == "29555"
    assert cmd[-4:] == ["--gpus", "8", "--steps", "5"] and cmd[-5].endswith("bench.py")


def test_gpus_flag_spawns_ranks_reference_arm():
    """`bench.py --gpus 2` started WITHOUT torchrun re-launches itself with
    one process per GPU (torch.distributed.run, 127.0.0.1); for the reference
    arm rank 0 alone runs the oracle and prints the one JSON line."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--gpus", "2", "--steps", "1",
                        "--warmup", "0", "--cpu-seconds", "1"], cwd=ROOT, capture_output=True, text=True,
                       timeout=600, env=env)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["n_gpus"] == 2
