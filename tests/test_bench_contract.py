"""bench.py contract checks that run without a GPU: the reference arm
(the CPU oracle) prints one JSON line with the required keys, also under a
2-process torchrun where rank 1 exits 0 without work."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(cmd, env=None):
    e = dict(os.environ)
    e.update(env or {})
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=600, env=e)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    return lines


def _check(line, workload="tiny"):
    d = json.loads(line)
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "scaling", "vs_baseline", "dtype", "data", "config",
              "cpu_baseline", "e2e", "impl"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0
    assert d["config"]["workload"] == workload
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0
    return d


def test_reference_arm_single_process():
    lines = _run([sys.executable, "bench.py", "--impl", "reference", "--config", "tiny",
                  "--steps", "2", "--warmup", "1", "--cpu-seconds", "0.3"])
    assert len(lines) == 1
    _check(lines[0])


def test_reference_arm_torchrun_two_ranks():
    lines = _run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
                  "--nproc-per-node", "2", "--master-addr", "127.0.0.1", "--master-port",
                  "29533", "bench.py", "--gpus", "2", "--impl", "reference", "--config", "tiny",
                  "--steps", "2", "--warmup", "1", "--cpu-seconds", "0.3"])
    assert len(lines) == 1          # rank 0 alone prints
    assert _check(lines[0])["n_gpus"] == 2


def test_reference_arm_rsbench():
    """--config rs-*: the reference arm times the RSBench oracle."""
    lines = _run([sys.executable, "bench.py", "--impl", "reference", "--config", "rs-tiny",
                  "--steps", "2", "--warmup", "1", "--cpu-seconds", "0.3"])
    assert len(lines) == 1
    d = _check(lines[0], "rs-tiny")
    assert d["metric"] == "RS lookups/sec"


def test_reference_arm_self_launch_two_ranks():
    """`bench.py --gpus 2` outside torchrun starts the two ranks itself
    (torch.distributed.run on 127.0.0.1) and relays rank 0's single line."""
    e = {k: v for k, v in os.environ.items()
         if k not in ("RANK", "WORLD_SIZE", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT")}
    r = subprocess.run([sys.executable, "bench.py", "--gpus", "2", "--impl", "reference",
                        "--config", "tiny", "--steps", "2", "--warmup", "1", "--cpu-seconds", "0.3"],
                       cwd=ROOT, capture_output=True, text=True, timeout=600, env=e)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    assert _check(lines[0])["n_gpus"] == 2
