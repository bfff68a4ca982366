"""Pins for the oracle's Hamming position code (§4.2).

Independent of the oracle: the reflected-Gray order is built here by the reflect-and-prefix
construction, minimality is checked by brute force over all orders, and the worked values
come from tests/golden/hamming_worked_values.txt (the paper's printed numbers).
"""
import itertools
import os

import pytest

import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden", "hamming_worked_values.txt")


def _golden():
    rows = []
    for line in open(GOLD):
        if line.startswith("#") or not line.strip():
            continue
        rows.append([x.strip() for x in line.split("|")])
    return rows


def _hd(a: str, b: str) -> int:
    return sum(x != y for x, y in zip(a, b))


def _cumulative(seq):
    return sum(_hd(seq[i], seq[i + 1]) for i in range(len(seq) - 1))


def _reflected(k):
    """Reflect-and-prefix construction of the k-digit reflected order."""
    seq = ["0", "1"]
    for _ in range(k - 1):
        seq = ["0" + s for s in seq] + ["1" + s for s in reversed(seq)]
    return seq


def test_worked_values_from_paper():
    for kind, inp, exp, _cite in _golden():
        if kind == "cumulative":
            assert _cumulative(inp.split(",")) == int(exp)
        elif kind == "hamming":
            a, b = inp.split(",")
            assert _hd(a, b) == int(exp)
        elif kind == "order":
            k = int(inp)
            order = sorted((format(b, "0%db" % k) for b in range(2 ** k)),
                           key=lambda s: oracle.hamming_code(int(s, 2)))
            assert order == exp.split(",")
        elif kind == "code":
            assert oracle.hamming_code(int(inp, 2)) == int(exp)
        elif kind == "negcode":
            # a 2:8 segment vector with three nonzeros whose code is -25: the string at rank
            # 25 of the 8-digit order must have exactly three ones, and its code is -25.
            seq = _reflected(8)
            s = seq[25]
            assert s.count("1") == 3
            assert oracle.position_code(int(s, 2), 2) == int(exp)


@pytest.mark.parametrize("k", range(1, 11))
def test_rank_matches_reflect_and_prefix_order(k):
    seq = _reflected(k)
    for rank, s in enumerate(seq):
        assert oracle.hamming_code(int(s, 2)) == rank


@pytest.mark.parametrize("k", [2, 3])
def test_order_is_a_minimal_cumulative_hamming_order(k):
    """Brute force over every order starting at 0...0: the minimum cumulative distance is
    2^k - 1 and the oracle's order attains it (L387-393)."""
    strs = [format(b, "0%db" % k) for b in range(2 ** k)]
    best = min(_cumulative([strs[0]] + list(p)) for p in itertools.permutations(strs[1:]))
    assert best == 2 ** k - 1
    ours = sorted(strs, key=lambda s: oracle.hamming_code(int(s, 2)))
    assert _cumulative(ours) == best


def test_negation_only_for_violating_strings():
    for M in (4, 8, 16):
        for b in range(0, 2 ** M, max(1, 2 ** M // 4096)):
            c = oracle.position_code(b, 2)
            h = oracle.hamming_code(b)
            assert abs(c) == h
            assert (c < 0) == (bin(b).count("1") > 2 and h != 0)


def test_code_zero_only_for_empty():
    assert oracle.hamming_code(0) == 0
    for b in range(1, 1 << 12):
        assert oracle.hamming_code(b) != 0
