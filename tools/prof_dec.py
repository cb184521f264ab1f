"""The C2 decryption alone at bench size (for ncu): encrypt 16,645 ciphertexts (k_tc_exp_dag), then
decrypt them (k_tc_exp<64> + k_dec_finish).  Not a benchmark (no timing)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402

count = int(sys.argv[1]) if len(sys.argv) > 1 else 16645
pub, priv = flb.keygen(2048, 0xF1B0 + 2048)
g = torch.Generator().manual_seed(5)
m = torch.randint(-2**31, 2**31 - 1, (count, 64), generator=g, dtype=torch.int32)
m[:, -1] = 0
c = flb.encrypt_crt(priv, m.cuda(), seed=1)
d = flb.decrypt(priv, c)
torch.cuda.synchronize()
assert torch.equal(d.cpu(), m)
print("ok", count)
