"""One launch of k_encrypt_crt at the bench size (133,160 key-holder encryptions), for ncu."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402

pub, priv = flb.keygen(2048, 0xF1B0 + 2048)
cd = flb.Codec(1.0, 29, 3, 63)
pt = torch.cat([flb.pack(pub, cd, torch.from_numpy(synthetic.c2_gradient(c)).cuda()) for c in range(8)])
ct = flb.encrypt_crt(priv, pt, seed=1)
torch.cuda.synchronize()
print("ok", ct.shape)
