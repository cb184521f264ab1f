"""One k_crt_pre + k_encrypt_crt2 launch pair (key-holder encryption, 2048-bit), for ncu A/B of
kernel variants (FLB_LIB_PATH selects the library).  COUNT (default 37,888 = 2 rounds) elements."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402

count = int(os.environ.get("COUNT", "37888"))
pub, priv = flb.keygen(2048, 0xF1B0 + 2048)
g = torch.Generator().manual_seed(7)
m = torch.randint(-2**31, 2**31 - 1, (count, 64), generator=g, dtype=torch.int32)
m[:, -1] = 0
ct = flb.encrypt_crt(priv, m.cuda(), seed=1)
torch.cuda.synchronize()
print("ok", ct.shape)
