"""Kernel timing sweep (CUDA events) for tuning: encrypt/decrypt/add/reduce at a key size."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402

bits = int(os.environ.get("BITS", "2048"))
M = int(os.environ.get("M", "133160"))
reps = int(os.environ.get("REPS", "2"))
pub, priv = flb.keygen(bits, 0xF1B0 + bits)
p, q, n = priv.export()
m = torch.from_numpy(synthetic.ints_to_limbs(synthetic.uniform_below(n, 64, 1), pub.pt_words).view("int32")).cuda()
m = m.repeat((M + 63) // 64, 1)[:M].contiguous()


def timed(fn):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    best = 1e30
    for _ in range(reps):
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best


c = flb.encrypt(pub, m, seed=1)
res = {"limbs": os.environ.get("FLB_LIMBS", "16"), "bits": bits, "M": M}
t = timed(lambda: flb.encrypt(pub, m, seed=1, out=c))
mm, lp = flb.op_cost(pub, "encrypt")
res["enc_ms"] = t
res["enc_per_s"] = M / t * 1e3
res["enc_TLPs"] = lp * M / t / 1e9
c2 = torch.empty_like(c)
t = timed(lambda: flb.encrypt_crt(priv, m, seed=1, out=c2))
mm, lp = flb.op_cost(priv, "encrypt_crt")
res["enc_crt_ms"] = t
res["enc_crt_per_s"] = M / t * 1e3
res["enc_crt_TLPs"] = lp * M / t / 1e9
res["enc_crt_equal"] = bool(torch.equal(c, c2))
Md = min(M, int(os.environ.get("MD", str(M))))
d = flb.decrypt(priv, c[:Md])
t = timed(lambda: flb.decrypt(priv, c[:Md], out=d))
mm, lp = flb.op_cost(priv, "decrypt")
res["dec_ms"] = t
res["dec_per_s"] = Md / t * 1e3
res["dec_TLPs"] = lp * Md / t / 1e9
ok = torch.equal(d, m[:Md])
res["roundtrip_ok"] = bool(ok)
o = torch.empty_like(c)
t = timed(lambda: flb.add(pub, c, c, out=o))
res["add_per_s"] = M / t * 1e3
res["add_TLPs"] = 2 * (2 * pub.ct_words ** 2 + pub.ct_words) * M / t / 1e9
print(json.dumps(res))
