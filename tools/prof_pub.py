"""One public-key encryption launch at 2048 bits (k_tc_exp<128>, the n^2 frame on the tensor cores) for
ncu.  Not a benchmark."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402

count = int(sys.argv[1]) if len(sys.argv) > 1 else 18944
pub, priv = flb.keygen(2048, 0xF1B0 + 2048)
m = torch.randint(0, 2**31 - 1, (count, 64), dtype=torch.int32).cuda()
c = flb.encrypt(pub, m, seed=1)
torch.cuda.synchronize()
print("ok", c.shape)
