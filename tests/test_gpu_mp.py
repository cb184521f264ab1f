"""Table I fundamentals on the device (csrc/flb_mp.cu) against
oracle/modarith.py: add/sub with carry/borrow, full product, division with remainder, mod, and the
modular inverse for odd and even moduli — bit-exact on random operands of every frame (1 to 256
limbs, widths that are and are not multiples of 4) plus the edge cases (0, 1, all-ones, a < b,
b = 0, x >= n, non-invertible x, n in {0, 1})."""

import math
import random

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
from oracle import modarith  # noqa: E402
from tests.helpers import from_dev, to_dev  # noqa: E402

pytestmark = pytest.mark.gpu
WORDS = [1, 3, 8, 32, 33, 64, 100, 128, 200, 256]


def _operands(words, count, seed):
    rng = random.Random(seed)
    R = 1 << (32 * words)
    a = [rng.randrange(R) for _ in range(count)]
    # b of every magnitude (so quotients of every length appear)
    b = [rng.randrange(R) >> rng.randrange(0, 32 * words) for _ in range(count)]
    edge = [(0, 0), (0, 1), (1, 0), (R - 1, R - 1), (R - 1, 1), (1, R - 1), (R - 1, 0), (5, 7), (7, 5),
            (R - 1, R - 2), (R >> 1, (R >> 1) + 1)]
    for i, (x, y) in enumerate(edge):
        a[i], b[i] = x, y
    return a, b


def _vec(t):
    return t.cpu().numpy().view(np.uint32).tolist()


@pytest.mark.parametrize("words", WORDS)
def test_add_sub_mul(words):
    a, b = _operands(words, 300, 100 + words)
    ta, tb = to_dev(a, words), to_dev(b, words)
    cy = torch.empty(300, dtype=torch.int32, device="cuda")
    bo = torch.empty(300, dtype=torch.int32, device="cuda")
    s = from_dev(flb.mp_add(ta, tb, carry=cy))
    d = from_dev(flb.mp_sub(ta, tb, borrow=bo))
    m = from_dev(flb.mp_mul(ta, tb))
    cyl, bol = _vec(cy), _vec(bo)
    for i in range(300):
        assert (s[i], cyl[i]) == modarith.mp_add(a[i], b[i], words), i
        assert (d[i], bol[i]) == modarith.mp_sub(a[i], b[i], words), i
        assert m[i] == modarith.mp_mul(a[i], b[i]), i


@pytest.mark.parametrize("words", WORDS)
def test_divmod_and_mod(words):
    a, b = _operands(words, 200, 200 + words)
    ta, tb = to_dev(a, words), to_dev(b, words)
    q, r = flb.mp_divmod(ta, tb)
    q, r = from_dev(q), from_dev(r)
    r2 = from_dev(flb.mp_mod(ta, tb))
    for i in range(200):
        assert (q[i], r[i]) == modarith.mp_divmod(a[i], b[i], words), i
        assert r2[i] == r[i]


@pytest.mark.parametrize("words", [1, 3, 32, 64, 100, 128, 256])
def test_mod_inv_odd_and_even_moduli(words):
    rng = random.Random(300 + words)
    R = 1 << (32 * words)
    xs, ns = [], []
    for i in range(96):
        n = rng.randrange(2, R)
        if i % 3 == 0:
            n |= 1          # odd modulus
        elif i % 3 == 1:
            n &= ~1         # even modulus
            n = max(n, 2)
        x = rng.randrange(R)
        if i % 5 == 0:
            x = x % n       # reduced input
        if i % 7 == 0:
            g = rng.randrange(2, 1 << min(30, 32 * words - 2)) if words > 1 else 6
            x, n = (x // g) * g % R, max(2, (n // g) * g)   # shared factor: not invertible
        xs.append(x)
        ns.append(n)
    # edge cases: n = 0, 1, 2; x = 0, 1; x = n - 1; x = n; an RSA-style even modulus
    edge = [(3, 0), (3, 1), (1, 2), (0, 2), (0, 7), (1, 7), (6, 7), (7, 7), (R - 1, R - 2), (R - 2, R - 1),
            (17, 780)]
    for i, (x, n) in enumerate(edge):
        xs[i], ns[i] = x % R, n % R
    ok = torch.empty(96, dtype=torch.int32, device="cuda")
    inv = from_dev(flb.mp_mod_inv(to_dev(xs, words), to_dev(ns, words), ok=ok))
    okl = _vec(ok)
    for i in range(96):
        want = modarith.mod_inv(xs[i], ns[i])
        assert inv[i] == want, (i, xs[i], ns[i])
        assert okl[i] == (1 if ns[i] >= 2 and math.gcd(xs[i], ns[i]) == 1 else 0), i


def test_rsa_private_exponent_on_device():
    """mod_inv as Table I uses it for key generation: d = e^-1 mod lcm(p-1, q-1)."""
    n, e, d, p = modarith.rsa_keygen(1024, 11)
    q = n // p
    lam = math.lcm(p - 1, q - 1)
    got = from_dev(flb.mp_mod_inv(to_dev([e], 32), to_dev([lam], 32)))[0]
    assert got == d
