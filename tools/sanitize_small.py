"""Small runs of every kernel for compute-sanitizer (memcheck / racecheck / synccheck / initcheck).

    python tools/sanitize_small.py          # 37-element batches of every op (toy16 / 1024 / 2048 / 4096)
    python tools/sanitize_small.py dag      # + a 20,000-element key-holder encryption at 2048 bits: 157
                                            #   stage-1 and 157 stage-2 tiles per prime on 296 CTAs, so
                                            #   stage-2 tiles wait on flags set by other CTAs
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402
from tests.helpers import golden_keys  # noqa: E402

K = golden_keys()
dag = len(sys.argv) > 1 and sys.argv[1] == "dag"
for name in ("toy16", "1024", "2048", "4096"):
    p, q = K[name]
    pub, priv = flb.key_from_primes(p, q)
    n = p * q
    M = 37
    m = torch.from_numpy(synthetic.ints_to_limbs(synthetic.uniform_below(n, M, 1), pub.pt_words).view(np.int32)).cuda()
    c = flb.encrypt(pub, m, seed=1)
    c2 = flb.encrypt_crt(priv, m, seed=1)
    d = flb.decrypt(priv, c)
    a = flb.add(pub, c, c2)
    e = torch.randint(0, 2 ** 31, (M, 2), dtype=torch.int32).cuda()
    s = flb.scalar_mul(pub, c, e)
    offs = torch.tensor([0, 5, 5, 30, 37], dtype=torch.int64).cuda()
    r = flb.reduce_segments(pub, c, offs)
    mm = flb.debug_mont_mul(pub, c, c2)
    if name != "toy16":
        cd = flb.Codec(1.0, 29, 3, 7)
        x = torch.from_numpy(synthetic.c2_gradient(0, n=100)).cuda()
        pt = flb.pack(pub, cd, x)
        u = flb.unpack(pub, cd, pt, 100, summands=1)
        us = flb.unpack_sums(pub, cd, pt, 100)
    torch.cuda.synchronize()
    assert torch.equal(d, m) and torch.equal(c, c2)
# Table I fundamentals (csrc/flb_mp.cu)
a = torch.randint(-2**31, 2**31 - 1, (37, 33), dtype=torch.int32).cuda()
b = torch.randint(-2**31, 2**31 - 1, (37, 33), dtype=torch.int32).cuda()
flb.mp_add(a, b)
flb.mp_sub(a, b)
flb.mp_mul(a, b)
flb.mp_divmod(a, b)
b[:, 0] |= 1
flb.mp_mod_inv(a, b)
torch.cuda.synchronize()
if dag:
    p, q = K["2048"]
    pub, priv = flb.key_from_primes(p, q)
    M = 20000
    m = torch.from_numpy(synthetic.ints_to_limbs(synthetic.uniform_below(p * q, 64, 2), pub.pt_words)
                         .view(np.int32)).cuda().repeat(M // 64 + 1, 1)[:M].contiguous()
    c2 = flb.encrypt_crt(priv, m, seed=5)
    torch.cuda.synchronize()
    assert torch.equal(flb.decrypt(priv, c2), m)
print("sanitize run ok")
