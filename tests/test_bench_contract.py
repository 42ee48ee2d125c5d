"""bench.py's JSON-line contract (the driver parses it).

CPU: the reference arm (`--impl reference`, the oracle on the host cores) on BASELINE.json configs[0]
prints one line with the contract keys, alone and under torchrun at 2 ranks (rank 0 only prints).
GPU: the CUDA arm on configs[0] prints roofline, cpu_baseline, e2e, clocks, gpu_launches and a clean
sampled parity.
"""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BASE_KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
             "scaling", "vs_baseline", "dtype", "data", "config", "e2e"}


def _lines(out):
    return [json.loads(l) for l in out.splitlines() if l.startswith("{")]


def _run(args, timeout=300):
    env = dict(os.environ, MASTER_ADDR="127.0.0.1")
    r = subprocess.run(args, cwd=ROOT, env=env, capture_output=True, text=True, timeout=timeout)
    assert r.returncode == 0, r.stderr[-2000:]
    return _lines(r.stdout)


def test_reference_arm_line():
    (d,) = _run([sys.executable, "bench.py", "--impl", "reference", "--config", "1", "--steps", "2",
                 "--warmup", "3"])
    assert BASE_KEYS <= d.keys()
    assert d["impl"] == "reference" and d["unit"] == "steps/s" and d["value"] > 0
    assert d["steps"] == 2 and d["warmup"] == 3 and d["higher_is_better"] is True
    assert "configs[0]" in d["config"]["workload"]
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] == d["value"] and cb["sample"]
    assert d["e2e"] == {"value": d["value"], "unit": "steps/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}


def test_reference_arm_torchrun_rank0_only():
    lines = _run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                  "--master-addr", "127.0.0.1", "--master-port", "29531", "bench.py", "--impl", "reference",
                  "--gpus", "2", "--config", "1", "--steps", "1", "--warmup", "3"])
    assert len(lines) == 1
    assert lines[0]["impl"] == "reference" and lines[0]["n_gpus"] == 2


@pytest.mark.gpu
def test_cuda_arm_line():
    (d,) = _run([sys.executable, "bench.py", "--config", "1", "--steps", "3", "--warmup", "3",
                 "--cpu-seconds", "1"])
    assert BASE_KEYS <= d.keys() and "impl" not in d
    assert d["value"] > 0 and d["n_gpus"] == 1 and d["scaling"] == "weak"
    rf = d["roofline"]
    assert rf["bound"] in ("hbm", "tensor", "alu") and rf["peak"] > 0 and rf["achieved"] > 0
    assert abs(rf["frac"] - rf["achieved"] / rf["peak"]) < 1e-9
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] > 0
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert d["gpu_launches"] > 0
    assert "sm_mhz" in d["clocks"] and "reasons" in d["clocks"]
    assert d["parity_sample"]["mismatched_walks"] == 0


def test_gpus_n_without_torchrun_launches_ranks():
    """`bench.py --gpus 2` outside torchrun re-launches itself with one process per GPU (the driver's
    launch line): one JSON line from rank 0 with n_gpus == 2, not a silent single-GPU run."""
    lines = _run([sys.executable, "bench.py", "--impl", "reference", "--gpus", "2", "--config", "1", "--steps", "1",
                  "--warmup", "3"])
    assert len(lines) == 1 and lines[0]["n_gpus"] == 2


def test_world_size_must_match_gpus():
    env = dict(os.environ, MASTER_ADDR="127.0.0.1")
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", "29533", "bench.py", "--impl", "reference",
                        "--gpus", "3", "--config", "1", "--steps", "1", "--warmup", "3"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=300)
    assert r.returncode != 0 and "WORLD_SIZE" in r.stderr
