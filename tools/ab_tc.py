"""A/B timing of the tensor-core kernels for the library named by FLB_LIB_PATH (default: the
in-tree build): key-holder encryption at the C2 batch (k_tc_exp_dag) and decryption at 16,645 and
133,160 (k_tc_exp), median of 5 after a warm-up, plus a bit-exactness check against the CUDA-core
CIOS kernels (FLB_TC=0) on 4,096 elements.  One JSON line.
    FLB_LIB_PATH=build_variants/x.so python tools/ab_tc.py [bits] [count]"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402

bits = int(sys.argv[1]) if len(sys.argv) > 1 else 2048
count = int(sys.argv[2]) if len(sys.argv) > 2 else 133160
pub, priv = flb.keygen(bits, 0xF1B0 + bits)
g = torch.Generator().manual_seed(7)
m = torch.randint(-2**31, 2**31 - 1, (count, bits // 32), generator=g, dtype=torch.int32)
m[:, -1] = 0
m = m.cuda()


def timed(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        fn()
        e.record()
        torch.cuda.synchronize()
        ts.append(s.elapsed_time(e) / 1e3)
    return statistics.median(ts)


out = {"lib": os.path.basename(flb.library_path), "bits": bits, "count": count}
os.environ["FLB_TC"] = "1"
t = timed(lambda: flb.encrypt_crt(priv, m, seed=3))
out["enc_kh_ms"] = round(t * 1e3, 2)
out["enc_kh_per_s"] = round(count / t)
c = flb.encrypt_crt(priv, m, seed=3)
c2 = c[:16645].contiguous()
out["dec_16645_ms"] = round(timed(lambda: flb.decrypt(priv, c2)) * 1e3, 2)
out["dec_all_per_s"] = round(count / timed(lambda: flb.decrypt(priv, c), reps=3))
ok = torch.equal(flb.decrypt(priv, c), m)
small = m[:4096].contiguous()
ctc = flb.encrypt_crt(priv, small, seed=9)
os.environ["FLB_TC"] = "0"
ccios = flb.encrypt_crt(priv, small, seed=9)
dcios = flb.decrypt(priv, ctc)
os.environ["FLB_TC"] = "1"
out["bit_exact"] = bool(ok and torch.equal(ctc, ccios) and torch.equal(dcios, small))
print(json.dumps(out), flush=True)
