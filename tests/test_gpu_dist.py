"""Cross-GPU paths on real kernels against the oracle: tests/dist_worker.py under torchrun with 2 and 3 ranks sharing
the visible GPU(s) over gloo (NCCL needs one GPU per rank; the driver's multi-GPU bench uses it)."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("world,port", [(2, 29611), (3, 29612)])
def test_dist_check_gloo(world, port):
    env = dict(os.environ, CDD_DIST_BACKEND="gloo", OMP_NUM_THREADS="1")
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
                        f"--nproc-per-node={world}", "--master-addr", "127.0.0.1",
                        "--master-port", str(port), os.path.join(ROOT, "tests", "dist_worker.py")],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    assert "dist_check ok" in r.stdout
