"""Which words of the tensor-core product phase differ from the exact product (debugging aid):
python tools/tc_product_debug.py [words] [square]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402

words = int(sys.argv[1]) if len(sys.argv) > 1 else 64
square = (sys.argv[2] != "0") if len(sys.argv) > 2 else True
vals = synthetic.uniform_below(1 << (32 * words), 128, 1)
a = torch.from_numpy(synthetic.ints_to_limbs(vals, words).view(np.int32)).cuda()
t = flb.debug_tc_product(a, a, square=square).cpu().numpy().view(np.uint32)
want = synthetic.ints_to_limbs([v * v for v in vals], 2 * words)
bad = np.nonzero((t != want).any(axis=1))[0]
print("elements wrong:", len(bad), "of 128")
for e in bad[:3]:
    diff = np.nonzero(t[e] != want[e])[0]
    print("elem", e, "wrong words:", diff.tolist())
