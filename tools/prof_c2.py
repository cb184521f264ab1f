"""One launch of each C2 kernel at bench size (for ncu): pack, encrypt 133,160, reduce 16,645x8,
decrypt 16,645, unpack.  Not a benchmark (no timing)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402
from paper_conf_icde_zeng0fcpcwg23_b200 import dist as fdist  # noqa: E402

clients = int(os.environ.get("CLIENTS", "8"))
pub, priv = flb.keygen(2048, 0xF1B0 + 2048)
cd = flb.Codec(1.0, 29, 3, 63)
rows = cd.num_plaintexts(1 << 20)
pt = torch.cat([flb.pack(pub, cd, torch.from_numpy(synthetic.c2_gradient(c)).cuda()) for c in range(clients)])
ct = flb.encrypt(pub, pt, seed=1)
ct2 = flb.encrypt_crt(priv, pt, seed=1)
offs, idx = fdist.client_segments(clients, rows, device="cuda")
agg = flb.reduce_segments(pub, ct, offs, idx=idx, max_segment_len=clients)
dec = flb.decrypt(priv, agg)
out = flb.unpack(pub, cd, dec, 1 << 20, summands=clients)
torch.cuda.synchronize()
print("ok", out.shape)
