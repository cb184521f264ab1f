"""Writes tests/golden/keys.json: Paillier primes for the parity tests.

Calls ONLY oracle/ (oracle.paillier.keygen).  Seeds follow SURVEY.md §8(d): 0xF1B0 + k.
Run:  python tests/golden/make_keys.py
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
from oracle import paillier  # noqa: E402

keys = {}
for k in (1024, 2048, 3072, 4096):
    p, q = paillier.keygen(k, 0xF1B0 + k)
    keys[str(k)] = {"seed": 0xF1B0 + k, "p": hex(p), "q": hex(q)}
keys["toy16"] = {"seed": None, "p": hex(251), "q": hex(241), "note": "SURVEY §4 toy key, n = 60,491"}
keys["toy9"] = {"seed": None, "p": hex(19), "q": hex(17), "note": "SURVEY §4 toy key, n = 323"}
out = os.path.join(os.path.dirname(os.path.abspath(__file__)), "keys.json")
with open(out, "w") as f:
    json.dump(keys, f, indent=1)
print("wrote", out)
