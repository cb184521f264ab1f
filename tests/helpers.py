"""Shared test helpers: golden keys and limb-tensor marshalling (no method arithmetic)."""

import json
import os

import numpy as np

import synthetic

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def golden_keys():
    with open(os.path.join(GOLDEN, "keys.json")) as f:
        d = json.load(f)
    return {k: (int(v["p"], 16), int(v["q"], 16)) for k, v in d.items()}


def to_dev(values, words):
    import torch
    arr = synthetic.ints_to_limbs(values, words)
    return torch.from_numpy(arr.view(np.int32)).cuda()


def from_dev(t):
    return synthetic.limbs_to_ints(t.cpu().numpy())
