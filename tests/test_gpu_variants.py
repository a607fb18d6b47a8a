"""The non-default implementations behind the measurement knobs, each read once per
process: the parity tests of the kernels they replace, re-run in a child process with the knob set.
Keeps every variant the profiles compare bit-exact with the oracle."""
import os
import subprocess
import sys

import pytest

from tests.gpu_util import need_gpu

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


@pytest.mark.skipif(os.environ.get("ACCMG_VARIANT_CHILD") == "1", reason="already a variant run")
@pytest.mark.parametrize("env,files", [
    ({"ACCMG_FUSED_PUSH": "0"}, ["tests/test_gpu_compaction.py", "tests/test_gpu_jacobi.py"]),
    ({"ACCMG_COMPACT_IMPL": "1"}, ["tests/test_gpu_compaction.py", "tests/test_gpu_jacobi.py"]),
    ({"ACCMG_JACOBI_IMPL": "1"}, ["tests/test_gpu_jacobi.py"]),
    ({"ACCMG_J3D_VARIANT": "0"}, ["tests/test_gpu_jacobi3d.py"]),
    ({"ACCMG_J3D_VARIANT": "5"}, ["tests/test_gpu_jacobi3d.py"]),
    ({"ACCMG_KMEANS_TC_QW": "64"}, ["tests/test_gpu_kmeans_tc.py"]),
], ids=["no-fused-push", "compact-impl1", "jacobi-impl1", "j3d-v0", "j3d-v5", "kmeans-qw64"])
def test_variant_parity(env, files):
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider", *files,
                        "-k", "not fp32_pipe_path"], cwd=ROOT,
                       env=dict(os.environ, ACCMG_VARIANT_CHILD="1", **env), capture_output=True, text=True,
                       timeout=1200)
    assert r.returncode == 0, r.stdout[-3000:]
