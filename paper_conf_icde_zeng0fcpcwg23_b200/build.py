"""Builds the CUDA library in-tree: paper_conf_icde_zeng0fcpcwg23_b200/_flb.so (sm_100a).

    python -m paper_conf_icde_zeng0fcpcwg23_b200.build [--force] [-v]

The kernels of each (X, T) frame split are instantiated in their own object (csrc/flb_inst.cu
compiled once per split, the split lists come from csrc/flb_core.cuh), so nvcc runs in parallel
over the splits; the objects are then linked into one shared library.
"""

from __future__ import annotations

import glob
import os
import re
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
OUT = os.environ.get("FLB_LIB_PATH") or os.path.join(HERE, "_flb.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC",
    "-I", os.path.join(ROOT, "include"),
]
OBJ = os.path.join(HERE, "build", "obj" if "FLB_LIB_PATH" not in os.environ else "obj_" + os.path.basename(OUT))


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def splits():
    """(X, T, enc, dec) for every frame split named by FLB_ENC_COMBOS / FLB_DEC_COMBOS."""
    core = open(os.path.join(CSRC, "flb_core.cuh")).read()
    def combos(name):
        line = re.search(r"#define " + name + r"\(M\)(.*)", core).group(1)
        return [(int(a), int(b)) for a, b in re.findall(r"M\((\d+),\s*(\d+)\)", line)]
    enc, dec = combos("FLB_ENC_COMBOS"), combos("FLB_DEC_COMBOS")
    return [(x, t, int((x, t) in enc), int((x, t) in dec)) for x, t in sorted(set(enc) | set(dec))]


def jobs(extra):
    """(object path, nvcc argument list) per translation unit."""
    out = []
    for src in sources():
        name = os.path.splitext(os.path.basename(src))[0]
        if name == "flb_inst":
            for x, t, e, d in splits():
                obj = os.path.join(OBJ, f"flb_inst_{x}x{t}.o")
                defs = [f"-DFLB_INST_X={x}", f"-DFLB_INST_T={t}", f"-DFLB_INST_ENC={e}", f"-DFLB_INST_DEC={d}"]
                out.append((obj, defs + ["-c", src]))
            for s in (32, 64, 96, 128):
                out.append((os.path.join(OBJ, f"flb_inst_tc{s}.o"), [f"-DFLB_INST_TC={s}", "-DFLB_INST_ENC=0",
                                                                      "-DFLB_INST_DEC=0", "-c", src]))
        else:
            out.append((os.path.join(OBJ, name + ".o"), ["-c", src]))
    return out


def deps():
    return sources() + sorted(glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.hpp"))
                              + glob.glob(os.path.join(ROOT, "include", "*.h")))


def up_to_date() -> bool:
    if not os.path.exists(OUT):
        return False
    t = os.path.getmtime(OUT)
    return all(os.path.getmtime(d) <= t for d in deps())


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and up_to_date():
        return OUT
    extra = os.environ.get("FLB_NVCC_EXTRA", "").split() + (["-Xptxas", "-v"] if verbose else [])
    os.makedirs(OBJ, exist_ok=True)
    todo = jobs(extra)

    def compile_one(job):
        obj, args = job
        return subprocess.run([NVCC] + FLAGS + extra + args + ["-o", obj], capture_output=True, text=True)

    with ThreadPoolExecutor(max_workers=max(1, os.cpu_count() or 1)) as ex:
        results = list(ex.map(compile_one, todo))
    for (obj, _), r in zip(todo, results):
        sys.stderr.write(r.stdout + r.stderr)
        if r.returncode != 0:
            raise subprocess.CalledProcessError(r.returncode, f"nvcc -> {obj}")
    link = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-cudart", "shared",
            "-Xcompiler", "-fPIC"] + [o for o, _ in todo] + ["-o", OUT + ".tmp"]
    subprocess.run(link, check=True)
    os.replace(OUT + ".tmp", OUT)
    return OUT


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
