"""Build a variant of the CUDA library without importing the package (which would load the default
library): FLB_LIB_PATH=<out.so> FLB_NVCC_EXTRA="-D..." python tools/build_variant.py [-v]"""
import importlib.util
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
spec = importlib.util.spec_from_file_location("_flb_build", os.path.join(ROOT, "paper_conf_icde_zeng0fcpcwg23_b200", "build.py"))
mod = importlib.util.module_from_spec(spec)
spec.loader.exec_module(mod)
print(mod.build(force=True, verbose="-v" in sys.argv))
