"""CPU ORACLE for the FLBooster batched-Paillier hot path — TEST INFRASTRUCTURE ONLY.

This package is the plain, slow, obviously-correct definition of every result the CUDA
library computes.  It exists to check the CUDA path, never to stand in for it:

* only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
  ``--impl reference`` legs may import it;
* it shares no code with ``paper_conf_icde_zeng0fcpcwg23_b200`` (the product) and imports
  nothing from it; the only module both sides use is ``synthetic`` (seeded input
  generators with none of the method's arithmetic);
* every function is written from the paper, ``/root/reference/PAPER.md`` — cited as
  ``PAPER L<line> (<section / equation / algorithm>)`` — or, where the paper is silent or
  garbled, from the reading recorded in DESIGN.md §3 (``reading c<k>``, numbered as in
  SURVEY.md §8(c)).

Arithmetic is Python's arbitrary-precision ``int`` (big integers) and IEEE-754 binary64
``float`` (the codec); library primitives used as single steps: ``pow`` (modular
exponentiation), ``math.gcd``/``math.lcm``, ``pow(x, -1, n)`` (modular inverse), ``round``
(round-half-even).  No Montgomery form, no CRT, no windowing, no (1+mn) shortcut: those are
the method's reformulations and live only on the CUDA side.

Parity status per function (DESIGN.md §3 lists the pins):

* paillier.encrypt / decrypt / add / scalar_mul / reduce_segments — pinned (toy-key brute
  force, Paillier invariants, closed forms; tests/test_oracle_paillier.py).
* paillier.keygen — pinned (independent Fermat/trial-division primality checks, bit lengths).
* philox.philox4x32_10 — pinned (Random123 known-answer vectors, tests/golden/philox_kat.txt).
* philox.draw_r — "parity unpinned" by the paper: the derivation of r from Philox is a
  convention of this build (reading c4); it is pinned only to its own stated range/bit
  properties and to the KAT-pinned generator.
* codec.* — pinned by Eq. 7 at alpha=1/2, Eq. 9 slot order on hand-worked fixtures,
  Eq. 11/12 closed forms and the dequantisation error bound; slot order, capacity,
  rounding mode and NaN/clamp handling are conventions (readings c11–c17), so those
  choices are "parity unpinned" by the paper itself.
* montgomery.mont_mul — pinned (definition a*b*R^-1 mod N checked by multiplying back).
"""

from . import paillier, philox, codec, montgomery, modarith  # noqa: F401
