"""bench.py's host-side contract, on the CPU (no GPU needed):

* `--impl reference` (the oracle timed on the host cores) prints ONE JSON line
  with the contract's keys (at least 3 warm-up steps whatever --warmup says), `impl: reference`,
  a `cpu_baseline` describing the run and an `e2e` block with zero transfer bytes — checked on
  the tiny C1 workload;
* `--gpus N` on a node with fewer than N CUDA devices refuses with one JSON error line and exit
  code 2 (never a silent 1-GPU number for an N-GPU request).
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(*args, timeout=600):
    env = dict(os.environ)
    env.pop("WORLD_SIZE", None)
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], cwd=ROOT, env=env,
                          capture_output=True, text=True, timeout=timeout)


def _json_lines(out):
    return [json.loads(line) for line in out.splitlines() if line.startswith("{")]


def test_reference_arm_prints_one_contract_line():
    r = _run("--impl", "reference", "--config", "C1", "--steps", "2", "--warmup", "1")
    assert r.returncode == 0, r.stderr[-2000:]
    lines = _json_lines(r.stdout)
    assert len(lines) == 1
    d = lines[0]
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["higher_is_better"] is False and d["unit"] == "ms"
    assert d["steps"] == 2 and d["warmup"] == 3 and d["value"] > 0     # W >= 3 is enforced
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert d["config"]["n"] == 1024 and d["config"]["cycles"] >= 1


def test_more_gpus_than_the_node_has_is_refused():
    import torch
    want = max(2, torch.cuda.device_count() + 1)          # N > 1: the multi-rank launcher
    r = _run("--gpus", str(want), timeout=300)
    assert r.returncode == 2
    lines = _json_lines(r.stdout)
    assert len(lines) == 1 and "error" in lines[0] and lines[0]["n_gpus"] == want
