"""Montgomery multiplication by its definition (ORACLE — test infrastructure).

PAPER L98–L114 (Algorithm 1) and L146–L197 (Algorithm 2, parallel CIOS): the output is
A*B*R^-1 mod N with R a power of two above N.  The oracle is that definition written out —
no word loop, no CIOS — so it checks the CUDA thread-group CIOS (the debug entry
``flb_debug_mont_mul``) without sharing its structure.  Reading c7: R = 2^(32 s) for an
s-limb modulus frame (not Alg. 2's garbled 2^(w x)); reading c8: outputs are canonical in [0, N).
"""

from __future__ import annotations


def mont_mul(a: int, b: int, n_mod: int, limbs: int) -> int:
    """a * b * R^-1 mod N with R = 2^(32*limbs)."""
    r = 1 << (32 * limbs)
    if n_mod % 2 == 0 or n_mod >= r:
        raise ValueError("Montgomery needs an odd modulus below R")
    return a * b * pow(r, -1, n_mod) % n_mod
