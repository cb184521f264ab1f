"""Per-phase cycles of the tensor-core Montgomery kernel (thread 0 of each CTA, summed), from a
FLB_TC_PROF=1 build:  FLB_LIB_PATH=build_variants/tcprof.so python tools/tc_phases.py [count]"""
import ctypes
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402

count = int(sys.argv[1]) if len(sys.argv) > 1 else 18944
mode = sys.argv[2] if len(sys.argv) > 2 else "keyholder"  # or "public" (k_tc_exp<128> at 2048 bits)
pub, priv = flb.keygen(2048, 0xF1B0 + 2048)
m = torch.randint(0, 2**31 - 1, (count, 64), dtype=torch.int32).cuda()
fn = flb.LIB.flb_debug_tc_prof128 if mode == "public" else flb.LIB.flb_debug_tc_prof
fn.argtypes = [ctypes.POINTER(ctypes.c_uint64), ctypes.c_int]
buf = (ctypes.c_uint64 * 16)()
enc = (lambda: flb.encrypt(pub, m, seed=1)) if mode == "public" else (lambda: flb.encrypt_crt(priv, m, seed=1))
enc()
torch.cuda.synchronize()
fn(buf, 1)
enc()
torch.cuda.synchronize()
fn(buf, 0)
names = ["P (product + sA/t_hi writes + barrier)", "M1 issue + wait", "N1 (q normalise + resolve + sA)",
         "M2 wait", "F (finish + borrow + writes)"]
out = {}
for S, o in (((128, 0),) if mode == "public" else ((32, 0), (64, 8))):
    calls = buf[o + 5]
    tot = sum(buf[o + i] for i in range(5))
    out["S=%d" % S] = {"calls": calls, "cycles_per_call": tot / max(calls, 1),
                       "phases": {n: round(buf[o + i] / max(calls, 1)) for i, n in enumerate(names)}}
print(json.dumps(out, indent=1))
