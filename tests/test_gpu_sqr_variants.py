"""The squaring experiments stay bit-exact (both measured slower on B200 and off by
default): run the parity suite's encrypt / decrypt / scalar-mul cases against a library built with
each of them, when that build exists and is current.
    FLB_SQR_BLOCKS=1: lane-local block squaring + reduce-only REDC   -> build_variants/sq.so
    FLB_SQR_SPLIT=1:  a^2 = L(L + 2HB) + H^2 R split squaring        -> build_variants/sqsplit.so
Build one with  FLB_LIB_PATH=build_variants/<name>.so FLB_NVCC_EXTRA=-D<FLAG>=1 python tools/build_variant.py"""

import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
VARIANTS = {"FLB_SQR_BLOCKS": "sq.so", "FLB_SQR_SPLIT": "sqsplit.so"}

pytestmark = pytest.mark.gpu


def _variant_current(path):
    """The variant exists and is newer than every source it is built from (else it is stale)."""
    if not os.path.exists(path):
        return False
    sys.path.insert(0, os.path.join(ROOT, "paper_conf_icde_zeng0fcpcwg23_b200"))
    import build  # noqa: E402
    t = os.path.getmtime(path)
    return all(os.path.getmtime(d) <= t for d in build.deps())


@pytest.mark.parametrize("flag", sorted(VARIANTS))
def test_squaring_variant_parity(flag):
    path = os.path.join(ROOT, "build_variants", VARIANTS[flag])
    if not _variant_current(path):
        pytest.skip(f"{flag}=1 variant not built or stale ({path})")
    env = dict(os.environ, FLB_LIB_PATH=path)
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "tests/test_gpu_parity.py",
                        "-k", "encrypt or decrypt or scalar"], cwd=ROOT, env=env, capture_output=True, text=True,
                       timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
