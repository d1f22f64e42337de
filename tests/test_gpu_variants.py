"""The parity suite on the GA_NSPAN=0 build: the paper's routing, every size
above the bins on TBuddy (DESIGN.md "Spans" is the departure the
default build makes).  The variant is built by __graft_entry__.build() next to
libga.so (paper_conf_ppopp_geladog19_b200/_build.py VARIANTS) and loaded by a
child pytest through GA_LIB, so this process keeps the default library."""
import os
import subprocess
import sys

import pytest
import torch

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.timeout(1800, method="thread")
def test_parity_suite_on_nspan0_build():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ppopp_geladog19_b200 import _build
    lib = _build.build_variants()["nspan0"]                  # (re)built if missing or older than the sources
    assert os.path.exists(lib)
    env = dict(os.environ, GA_LIB=lib, GA_EXPECT_NSPAN="0")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-p", "no:cacheprovider",
                        "tests/test_gpu_parity.py", "tests/test_gpu_edge.py"],
                       cwd=ROOT, env=env, capture_output=True, text=True)
    tail = (r.stdout + r.stderr)[-4000:]
    assert r.returncode == 0, tail
    assert " passed" in tail and "failed" not in tail, tail
