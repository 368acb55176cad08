"""Pins for the SOAP-text oracle parser (reading R19; §8(f) NEXT #2): a hand-written golden
fixture, and the round trip through the C text writer in synth/ (an independent program)."""
from __future__ import annotations

import os

import numpy as np
import pytest

import synth
from oracle.soap import parse_soap

GOLD = os.path.join(os.path.dirname(__file__), "golden", "soap_tiny.txt")


def _golden():
    text, reads = [], []
    for line in open(GOLD):
        line = line.rstrip("\n")
        if line.startswith("TEXT"):
            text.append(line[5:].replace("<TAB>", "\t"))
        elif line.startswith("READ"):
            f = line.split()
            reads.append((int(f[1]), int(f[2]), int(f[3]), int(f[4]),
                          [int(x) for x in f[5].split(",")], [int(x) for x in f[6].split(",")]))
    return ("\n".join(text) + "\n").encode(), reads


def test_golden_fixture():
    text, want = _golden()
    r = parse_soap(text, "chr7", 33, 1000)
    assert len(r["pos"]) == len(want)
    for i, (pos, ln, st, h, b, q) in enumerate(want):
        o0, o1 = int(r["off"][i]), int(r["off"][i + 1])
        assert (int(r["pos"][i]), int(r["len"][i]), int(r["strand"][i]), int(r["hits"][i])) == \
            (pos, ln, st, h)
        assert list(r["bases"][o0:o1]) == b and list(r["quals"][o0:o1]) == q
    # unterminated last line parses the same; chr None keeps the chr8 line too
    assert len(parse_soap(text.rstrip(b"\n"), "chr7", 33, 1000)["pos"]) == 3
    assert len(parse_soap(text, None, 33, 1000)["pos"]) == 4


@pytest.mark.parametrize("q_offset", [33, 64])
def test_round_trip_through_c_writer(q_offset):
    w = synth.generate("C1", n_sites=3_000, depth=6.0, seed=12)
    text = synth.soap_text(w, "chrZ", q_offset)
    r = parse_soap(text, "chrZ", q_offset, int(w["origin"]))
    for k in ("pos", "len", "strand", "hits", "bases", "quals"):
        assert np.array_equal(r[k], np.asarray(w[k])[:len(r[k])] if k in ("bases", "quals")
                              else np.asarray(w[k])), k
    assert np.array_equal(r["off"], np.asarray(w["off"]) - w["off"][0])


@pytest.mark.parametrize("bad", ["r\tAC\tII\t1\ta\t3\t+\tc\t5",        # len != |seq|
                                 "r\tAC\tII\t1\ta\t2\t*\tc\t5",        # strand
                                 "r\tAX\tII\t1\ta\t2\t+\tc\t5",        # base
                                 "r\tAC\t I\t1\ta\t2\t+\tc\t5",        # quality < offset
                                 "r\tAC\tII\t0\ta\t2\t+\tc\t5",        # hits 0
                                 "r\tAC\tII\t1\ta\t2\t+\tc\t5x",       # location
                                 "r\tAC\tII\t1\ta\t2\t+\tc"])          # 8 fields
def test_malformed_lines_raise(bad):
    good = "r\tAC\tII\t1\ta\t2\t+\tc\t5\n"
    with pytest.raises(ValueError, match="line 1"):
        parse_soap((good + bad + "\n").encode(), "c")
