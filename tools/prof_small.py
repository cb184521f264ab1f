"""One wave of k_encrypt_crt (2048-bit) for a quick ncu look (M = 18,944)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402

M = int(os.environ.get("M", "18944"))
pub, priv = flb.keygen(2048, 0xF1B0 + 2048)
p, q, n = priv.export()
m = torch.from_numpy(synthetic.ints_to_limbs(synthetic.uniform_below(n, 64, 1), 64).view("int32")).cuda()
m = m.repeat((M + 63) // 64, 1)[:M].contiguous()
ct = flb.encrypt_crt(priv, m, seed=1)
torch.cuda.synchronize()
print("ok")
