"""A/B timing of the modexp-heavy kernels for the library named by FLB_LIB_PATH (default: the
in-tree build): key-holder encrypt, public encrypt, decrypt at the given key size, one JSON line.
    FLB_LIB_PATH=build_variants/x.so python tools/ab_bench.py [bits] [count]"""
import json
import os
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


def timed(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(reps):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        fn()
        e.record()
        torch.cuda.synchronize()
        best = min(best, s.elapsed_time(e) / 1e3)
    return best


out = {"lib": flb.library_path, "bits": bits, "count": count}
os.environ["FLB_TC"] = "0"
c = flb.encrypt_crt(priv, m, seed=3)
t = timed(lambda: flb.encrypt_crt(priv, m, seed=3))
out["encrypt_keyholder_per_s"] = count / t
os.environ["FLB_TC"] = "1"
ctc = flb.encrypt_crt(priv, m, seed=3)
torch.cuda.synchronize()
bad = (ctc != c).any(dim=1).nonzero().flatten().tolist()
out["tc_mismatches"] = len(bad)
out["tc_first_bad"] = bad[:3]
t = timed(lambda: flb.encrypt_crt(priv, m, seed=3))
out["encrypt_keyholder_tc_per_s"] = count / t
os.environ["FLB_TC"] = "0"
t = timed(lambda: flb.encrypt(pub, m, seed=3), reps=1)
out["encrypt_public_per_s"] = count / t
for tc in ("0", "1"):
    os.environ["FLB_TC"] = tc
    sfx = "_tc" if tc == "1" else ""
    t = timed(lambda: flb.decrypt(priv, c))
    out["decrypt%s_per_s" % sfx] = count / t
    c2 = c[:16645]
    t = timed(lambda: flb.decrypt(priv, c2))
    out["decrypt%s_16645_per_s" % sfx] = c2.shape[0] / t
    d = flb.decrypt(priv, c)
    out["roundtrip%s_ok" % sfx] = bool(torch.equal(d, m))
os.environ["FLB_TC"] = "0"
out["crt_equals_public"] = bool(torch.equal(c, flb.encrypt(pub, m, seed=3)))
print(json.dumps(out))
