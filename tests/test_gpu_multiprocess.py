"""The one-process-per-GPU path (-m gpu): ranks as separate processes that share
buffers through CUDA IPC and synchronise with device barriers, every strategy,
against the oracle.  Both ranks run on cuda:0 here (the GPU box has one B200): the
same peer loads/stores/atomics that cross NVLink on a multi-GPU node stay inside one
device."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("world", [2])
def test_multiprocess_strategies_match_oracle(world):
    env = dict(os.environ, APT_TEST_DEVICE="0")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", "--master-port", "29533", os.path.join(ROOT, "tests", "mp_step.py"),
           "f32,bf16", "GDP,NFP,SNP,DNP", "5,5;5,5,5"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, env=env, cwd=ROOT)
    out = r.stdout + r.stderr
    line = [l for l in out.splitlines() if l.startswith("RESULT")]
    assert r.returncode == 0 and line and line[0] == "RESULT OK", out[-4000:]


@pytest.mark.parametrize("world", [2])
def test_multiprocess_gat_layer_matches_oracle(world):
    env = dict(os.environ, APT_TEST_DEVICE="0")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", "--master-port", "29534", os.path.join(ROOT, "tests", "mp_gat.py"),
           "GDP,NFP,SNP,DNP"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=env, cwd=ROOT)
    out = r.stdout + r.stderr
    line = [l for l in out.splitlines() if l.startswith("RESULT")]
    assert r.returncode == 0 and line and line[0] == "RESULT OK", out[-4000:]


@pytest.mark.parametrize("world", [2])
def test_multiprocess_link_trials_measure_peer_ops(world):
    env = dict(os.environ, APT_TEST_DEVICE="0")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", "--master-port", "29535", os.path.join(ROOT, "tests", "mp_links.py")]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=env, cwd=ROOT)
    out = r.stdout + r.stderr
    line = [l for l in out.splitlines() if l.startswith("RESULT")]
    assert r.returncode == 0 and line and line[0] == "RESULT OK", out[-4000:]
