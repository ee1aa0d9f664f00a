"""bench.py end to end on the GPU: the single-GPU line and the N>1 path the
driver's scaling run takes (torchrun, one process per rank).  With one device
the ranks share cuda:0 (SF_BENCH_SHARED_GPU=1: gloo process group, the p2p
transport over CUDA IPC on the same device), which exercises the same slab
decomposition, halo exchange, agglomeration and max-over-ranks timing."""
import json
import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _json_lines(out):
    return [json.loads(l) for l in out.splitlines() if l.startswith("{")]


def _run(cmd, env=None, timeout=900):
    e = dict(os.environ)
    e.update(env or {})
    r = subprocess.run(cmd, cwd=ROOT, env=e, capture_output=True, text=True, timeout=timeout)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    return r.stdout


def _torchrun(n, args, env=None):
    return _run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
                 f"--nproc-per-node={n}", "--master-addr=127.0.0.1",
                 f"--master-port={_free_port()}", "bench.py", "--gpus", str(n), *args],
                env={"SF_BENCH_SHARED_GPU": "1", **(env or {})})


def _check_line(d, n):
    assert d["n_gpus"] == n and d["unit"] == "DOF/s" and d["value"] > 0
    assert d["higher_is_better"] is True and d["scaling"] == "weak"
    assert d["gpu_launches"] > 0 and d["dtype"] == "f64"
    assert d["config"]["final_relres"] < 1e-10
    assert d["ms_per_step"] > 0


def test_bench_single_gpu_line():
    out = _run([sys.executable, "bench.py", "--steps", "2", "--warmup", "3", "--side", "128",
                "--no-cpu-baseline"])
    lines = _json_lines(out)
    assert len(lines) == 1
    d = lines[0]
    _check_line(d, 1)
    assert d["roofline"]["bound"] == "hbm" and 0 < d["roofline"]["frac"] <= 1.2
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] == 8 * 128**3


@pytest.mark.parametrize("n,quick", [(2, False), (4, True)])
def test_bench_torchrun_ranks(n, quick):
    out = _torchrun(n, ["--steps", "2", "--warmup", "3", "--side", "64", "--no-cpu-baseline",
                        *(["--quick"] if quick else [])])
    lines = _json_lines(out)
    assert len(lines) == 1, out          # rank 0 alone prints
    d = lines[0]
    _check_line(d, n)
    assert d["config"]["transport"] == "p2p"
    assert d["config"]["global"][2] * d["config"]["global"][1] * d["config"]["global"][0] == n * 64**3
    if not quick:   # side measurements ran over the ranks (C4 strong-scaling F-cycle, e2e)
        assert d["fcycle_strong"]["dof_s"] > 0 and d["e2e"]["value"] > 0


def test_bench_reference_arm_torchrun():
    out = _torchrun(2, ["--impl", "reference", "--steps", "1", "--warmup", "3", "--side", "64"])
    lines = _json_lines(out)
    assert len(lines) == 1, out
    d = lines[0]
    assert d["impl"] == "reference" and d["value"] > 0 and d["n_gpus"] == 2
    assert d["cpu_baseline"]["kind"] == "oracle"
    assert d["e2e"]["h2d_bytes_per_step"] == 0
