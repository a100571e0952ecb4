"""Pins of the oracle's PforDelta codec (oracle/pfd.cpp; the paper's comparison
scheme, §2.1.1, Fig. 3) — the NEXT-3 comparator."""
import numpy as np

import oracle
from conftest import read_golden
from helpers import bits_lsb_first


def _slots(words, m, b):
    s = bits_lsb_first(words[1:], m * b)
    return [int(s[i * b:(i + 1) * b][::-1], 2) if b else 0 for i in range(m)]


def test_fig3_worked_example():
    g = read_golden("pfd_fig3.txt")
    x = [int(v) for v in g["docids"][0]]
    b = int(g["b"][0][0])
    w, bo, ne = oracle.pfd_encode(x, b=b)
    m = len(x) - 1
    assert np.array_equal(np.diff(x), [int(v) for v in g["gaps"][0]])
    assert bo == b and ne == 3
    assert w[0] & 1023 == int(g["first_exception"][0][0])
    assert (w[0] >> 10) & 1023 == 3 and (w[0] >> 20) & 63 == b
    assert _slots(w, m, b) == [int(v) for v in g["slots"][0]]
    nsw = (m * b + 31) // 32
    assert list(w[1 + nsw:]) == [int(v) for v in g["exception_tail"][0]]
    assert np.array_equal(oracle.pfd_decode(w, x[0], len(x)), x)


def test_ninety_percent_rule():
    """b = bits of the largest of the ceil(0.9 m) smallest gaps."""
    def block(gaps):
        return np.cumsum([7] + list(gaps)).astype(np.uint32)
    # 10 gaps: 9 regular ones of value 1, one 1000 -> b = 1, one exception
    w, b, ne = oracle.pfd_encode(block([1] * 9 + [1000]))
    assert (b, ne) == (1, 1)
    # 20 gaps: 18 of value 3 (2 bits) and 2 huge at positions 9 and 19 -> b = 2;
    # 19 - 9 = 10 > 2^2, so 13 and 17 are forced exceptions: 4 in all
    w, b, ne = oracle.pfd_encode(block([3] * 9 + [1 << 20] + [3] * 9 + [1 << 21]))
    assert (b, ne) == (2, 4)
    # Fig. 3's gaps under the rule: ceil(7.2) = 8 regular -> b = bits(68) = 7, none
    w, b, ne = oracle.pfd_encode([100, 121, 163, 172, 185, 214, 282, 300, 347])
    assert (b, ne) == (7, 0)
    assert w[0] & 1023 == 8   # "no exception": first position = m


def test_forced_exceptions_keep_links_in_b_bits():
    """b = 1: exceptions at gap positions 0 and 5 are 5 apart > 2^1, so positions
    2 and 4 become (forced) exceptions; every link fits in one bit."""
    x = np.cumsum([10, 5, 1, 1, 1, 1, 7]).astype(np.uint32)   # gaps 5,1,1,1,1,7
    w, b, ne = oracle.pfd_encode(x, b=1)
    assert (b, ne) == (1, 4)
    m = len(x) - 1
    sl = _slots(w, m, 1)
    pos = [0]
    for _ in range(ne - 1):
        pos.append(pos[-1] + sl[pos[-1]] + 1)
    assert pos == [0, 2, 4, 5]
    assert np.array_equal(oracle.pfd_decode(w, int(x[0]), len(x)), x)


def test_size_closed_form_and_roundtrip_random():
    rng = np.random.default_rng(5)
    for trial in range(400):
        n = int(rng.integers(1, 513))
        N = int(rng.choice([n + 5, 10 * n, 1000 * n, 2 ** 31]))
        x = np.sort(rng.choice(N, size=n, replace=False)).astype(np.uint32)
        bsel = None if trial % 3 else int(rng.integers(1, 20))
        w, b, ne = oracle.pfd_encode(x, b=bsel)
        m = n - 1
        assert len(w) == 1 + (m * b + 31) // 32 + ne
        g = np.diff(x.astype(np.int64))
        if bsel is None and m:
            # at most 10% exceptions unless forced ones were needed
            assert (g >= (1 << b)).sum() <= m - (9 * m + 9) // 10
            assert (1 << (b - 1)) <= np.sort(g)[(9 * m + 9) // 10 - 1] < (1 << b)
        assert np.array_equal(oracle.pfd_decode(w, int(x[0]), n), x)


def test_brute_force_every_b_tiny():
    rng = np.random.default_rng(9)
    for _ in range(60):
        n = int(rng.integers(2, 40))
        x = np.sort(rng.choice(5000, size=n, replace=False)).astype(np.uint32)
        for b in range(1, 14):
            w, bo, ne = oracle.pfd_encode(x, b=b)
            g = np.diff(x.astype(np.int64))
            assert ne >= int((g >= (1 << b)).sum())
            assert np.array_equal(oracle.pfd_decode(w, int(x[0]), n), x)
