"""bench.py contract: one JSON line with the keys the driver reads (metric, value, unit, n_gpus, steps, warmup,
ms_per_step, higher_is_better, scaling, dtype, config.workload, roofline, cpu_baseline, e2e, gpu_launches, clocks)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
        "vs_baseline", "dtype", "data", "config"}


def _run(args, env=None, timeout=900):
    r = subprocess.run([sys.executable] + args, cwd=ROOT, capture_output=True, text=True, timeout=timeout,
                       env={**os.environ, **(env or {})})
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def test_reference_arm_cpu():
    d = _run(["bench.py", "--impl", "reference", "--config", "C1", "--steps", "3", "--warmup", "3"])
    assert KEYS <= set(d) and d["impl"] == "reference"
    assert d["unit"] == "s/iteration" and d["higher_is_better"] is False and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["e2e"]["h2d_bytes_per_step"] == 0
    assert d["config"]["workload"] == "C1"


def test_reference_arm_two_ranks_cpu():
    """Under torchrun (N > 1) rank 0 alone times the oracle on the whole job our arm times at that N (weak: N x the
    configuration) on all host cores (torchrun exports OMP_NUM_THREADS=1); the other ranks exit 0 without work."""
    d = _run(["-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr", "127.0.0.1",
              "--master-port", "29545", "bench.py", "--impl", "reference", "--gpus", "2", "--config", "C1",
              "--steps", "3", "--warmup", "3"])
    assert d["impl"] == "reference" and d["n_gpus"] == 2 and d["scaling"] == "weak"
    assert d["config"]["total_rows"] == 40_000 and d["config"]["n_obs_per_gpu"] == 20_000
    assert d["cpu_baseline"]["cores"] == d["cpu_baseline"]["host_cores"] >= 1


@pytest.mark.gpu
def test_bench_line_gpu(cuda_device):
    d = _run(["bench.py", "--config", "C1", "--steps", "5", "--warmup", "3", "--cpu-iters", "2"])
    assert KEYS <= set(d)
    assert d["n_gpus"] == 1 and d["steps"] == 5 and d["dtype"] == "f64"
    rf = d["roofline"]
    assert rf["bound"] == "hbm" and 0 < rf["frac"] < 1.5 and rf["peak"] > 1000
    assert d["gpu_launches"] == 5 * 4 and d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert "sm_mhz" in d["clocks"]


@pytest.mark.gpu
def test_bench_two_ranks_gloo_callback(cuda_device):
    """The multi-rank flow of bench.py (weak-scaling shapes, max over ranks, e2e, one line from rank 0) through the
    library's host-callback communicator, both ranks on cuda:0 (NCCL cannot put two ranks on one GPU)."""
    d = _run(["-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr", "127.0.0.1",
              "--master-port", "29541", "bench.py", "--gpus", "2", "--config", "C1", "--steps", "4", "--warmup",
              "3", "--comm", "gloo-callback", "--same-device"])
    assert d["n_gpus"] == 2 and d["scaling"] == "weak"
    assert d["config"]["n_obs_per_gpu"] == 20_000 and d["config"]["total_rows"] == 40_000
    assert d["config"]["parallelism"].startswith("dp2")
    assert d["gpu_launches"] == 4 * 9


@pytest.mark.gpu
def test_bench_repro_line(cuda_device):
    d = _run(["bench.py", "--config", "C1", "--steps", "4", "--warmup", "3", "--repro", "--cpu-iters", "1"])
    assert d["gpu_launches"] == 4 * 7 and "reproducible" in d["config"]["variant"]
    assert d["roofline"]["kernel"] == "repro iteration" and "repro" in d["cpu_baseline"]["sample"]


@pytest.mark.gpu
def test_bench_strong_scaling_two_ranks(cuda_device):
    """--scaling strong (C4 over 1/2/4/8 GPUs): the configuration itself is split over the ranks by the
    O-SHARD star ranges, at the reduced C4 shape C4s (n_att 3,000,000: the 24 MB shared slice of AR2), two ranks on
    cuda:0 through the host-callback communicator."""
    d = _run(["-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr", "127.0.0.1",
              "--master-port", "29543", "bench.py", "--gpus", "2", "--config", "C4s", "--scaling", "strong",
              "--steps", "4", "--warmup", "3", "--comm", "gloo-callback", "--same-device", "--no-e2e"])
    assert d["n_gpus"] == 2 and d["scaling"] == "strong" and d["config"]["scaling"] == "strong"
    assert d["config"]["total_rows"] == 7_800_000 and d["config"]["n_obs_per_gpu"] == 3_900_000
    assert d["gpu_launches"] == 4 * 9 and d["value"] > 0
