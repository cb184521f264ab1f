"""Pin for oracle/philox.py: Random123 known-answer vectors (tests/golden/philox_kat.txt)."""

import os

from oracle import philox

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "philox_kat.txt")


def _kat():
    rows = []
    with open(GOLDEN) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            w = [int(x, 16) for x in line.split()]
            rows.append((tuple(w[0:4]), tuple(w[4:6]), tuple(w[6:10])))
    return rows


def test_philox_kat():
    rows = _kat()
    assert len(rows) == 3
    for ctr, key, out in rows:
        assert philox.philox4x32_10(ctr, key) == out


def test_philox_words_layout():
    # word 4j+t is output t of block j with counter (index lo, index hi, j, 0)
    w = philox.philox_words(0x1122334455667788, 5, 9)
    b0 = philox.philox4x32_10((5, 0, 0, 0), (0x55667788, 0x11223344))
    b1 = philox.philox4x32_10((5, 0, 1, 0), (0x55667788, 0x11223344))
    b2 = philox.philox4x32_10((5, 0, 2, 0), (0x55667788, 0x11223344))
    assert w == list(b0) + list(b1) + [b2[0]]
