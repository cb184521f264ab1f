"""One launch each of the non-modexp kernels at bench-like sizes, for ncu: hom-add (k_add, 2048-bit,
1,048,576 pairs), the C2 segmented product (k_plan_* + k_reduce, 16,645 x 8), the C3 multi-
exponentiation (k_bucket / k_scan_u64 / k_reduce / k_horner, 1,048,576 x 8 features), pack and unpack
(1,048,576 values).  Not a benchmark."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402
from paper_conf_icde_zeng0fcpcwg23_b200 import dist as fdist  # noqa: E402

pub, priv = flb.keygen(2048, 0xF1B0 + 2048)
M = 1 << 20
m = torch.randint(0, 2**31 - 1, (M, 64), dtype=torch.int32).cuda()
c = flb.encrypt_crt(priv, m, seed=1)
c2 = flb.encrypt_crt(priv, m, seed=2)
flb.add(pub, c, c2)                                    # k_add
cd = flb.Codec(1.0, 29, 3, 63)
x = torch.from_numpy(synthetic.c2_gradient(0)).cuda()
pt = flb.pack(pub, cd, x)                              # k_pack
rows = pt.shape[0]
ct8 = c[: 8 * rows].contiguous()
offs, idx = fdist.client_segments(8, rows, device="cuda")
agg = flb.reduce_segments(pub, ct8, offs, idx=idx, max_segment_len=8)  # k_plan_*, k_reduce
dec = flb.decrypt(priv, agg)
flb.unpack(pub, cd, dec, 1 << 20, summands=8)          # k_unpack
N, F = 1 << 20, 8
e = torch.from_numpy(synthetic.uniform_words(N * F, 1, 9).view(np.int32)).cuda()
iF = torch.arange(N, dtype=torch.int64, device="cuda").repeat(F)
offF = torch.arange(F + 1, dtype=torch.int64, device="cuda") * N
flb.multiexp_segments(pub, c, e, offF, idx=iF)         # k_bucket, k_scan_u64, k_reduce, k_horner
torch.cuda.synchronize()
print("ok")
