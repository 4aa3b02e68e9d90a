"""bench.py's multi-rank harness, host side (no GPU): `--gpus N` self-launch
under torchrun, the world-size check, and the reference arm's CPU leg.  The
end-to-end multi-rank run (2 gloo ranks on one GPU, checksums compared with a
single-GPU recomputation) is the -m gpu test at the bottom."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def test_self_launch_argv_is_torchrun_on_loopback():
    argv = bench.self_launch_argv(4, ["--gpus", "4", "--steps", "7"], 12345)
    assert argv[:3] == [sys.executable, "-m", "torch.distributed.run"]
    assert "--nproc-per-node=4" in argv and "--nnodes=1" in argv
    assert argv[argv.index("--master-addr") + 1] == "127.0.0.1"
    assert "--master-port=12345" in argv
    assert argv[-4:] == ["--gpus", "4", "--steps", "7"]
    assert argv[-5].endswith("bench.py")


class _A:
    def __init__(self, gpus, impl="ours"):
        self.gpus, self.impl = gpus, impl


def test_no_self_launch_when_single_or_under_torchrun(monkeypatch):
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    assert bench.maybe_self_launch(_A(None), []) is None
    assert bench.maybe_self_launch(_A(1), []) is None
    assert bench.maybe_self_launch(_A(4, "reference"), []) is None
    monkeypatch.setenv("WORLD_SIZE", "4")
    assert bench.maybe_self_launch(_A(4), []) is None


def test_self_launch_spawns_torchrun(monkeypatch):
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    seen = {}

    def fake_call(cmd):
        seen["cmd"] = cmd
        return 3
    monkeypatch.setattr(subprocess, "call", fake_call)
    assert bench.maybe_self_launch(_A(2), ["--gpus", "2"]) == 3
    assert "--nproc-per-node=2" in seen["cmd"]


def test_world_size_mismatch_is_an_error(monkeypatch):
    monkeypatch.setenv("WORLD_SIZE", "2")
    monkeypatch.setenv("RANK", "0")
    with pytest.raises(SystemExit) as e:
        bench.main(["--gpus", "4", "--no-extras"])
    assert "WORLD_SIZE=2" in str(e.value)


def test_reference_arm_reports_requested_gpus(capsys, monkeypatch):
    for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK"):
        monkeypatch.delenv(k, raising=False)
    bench.main(["--impl", "reference", "--gpus", "2", "--workload", "ps1", "--steps", "3", "--warmup", "3"])
    line = json.loads(capsys.readouterr().out.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["n_gpus"] == 2
    assert line["cpu_baseline"]["kind"] == "oracle" and line["e2e"]["h2d_bytes_per_step"] == 0


@pytest.mark.gpu
@pytest.mark.parametrize("workload", ["tr1", "ps1"])
def test_two_gloo_ranks_on_one_gpu_end_to_end(workload):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--dist-backend", "gloo",
                          "--workload", workload, "--steps", "5", "--warmup", "3", "--no-extras", "--no-e2e"],
                         capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    line = json.loads(lines[0])
    assert line["n_gpus"] == 2 and line["config"]["p_total"] == 2 * line["config"]["p_per_gpu"]
    assert line["checksums_match"] is True and len(line["checksums"]["per_rank"]) == 2
    assert line["cpu_baseline"]["gpu_matches_oracle_on_sample"] is True
