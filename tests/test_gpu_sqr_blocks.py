"""The block-squaring experiment (FLB_SQR_BLOCKS=1 build) stays bit-exact: run the
parity suite's encrypt/decrypt cases against a library built with it, when that build exists."""

import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
VARIANT = os.path.join(ROOT, "build_variants", "sq.so")

pytestmark = pytest.mark.gpu


def _variant_current():
    """The variant exists and is newer than every source it is built from (else it is stale)."""
    if not os.path.exists(VARIANT):
        return False
    sys.path.insert(0, os.path.join(ROOT, "paper_conf_icde_zeng0fcpcwg23_b200"))
    import build  # noqa: E402
    t = os.path.getmtime(VARIANT)
    return all(os.path.getmtime(d) <= t for d in build.deps())


@pytest.mark.skipif(not _variant_current(), reason="FLB_SQR_BLOCKS=1 variant not built or stale "
                    "(FLB_LIB_PATH=build_variants/sq.so FLB_NVCC_EXTRA=-DFLB_SQR_BLOCKS=1 python "
                    "paper_conf_icde_zeng0fcpcwg23_b200/build.py --force)")
def test_block_squaring_variant_parity():
    env = dict(os.environ, FLB_LIB_PATH=VARIANT)
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "tests/test_gpu_parity.py",
                        "-k", "encrypt or decrypt or scalar"], cwd=ROOT, env=env, capture_output=True, text=True,
                       timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
