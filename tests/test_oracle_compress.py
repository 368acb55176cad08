"""Pins for the oracle's output compression (§V-B; byte format = reading
R17, oracle/compress.c).  What fixes it independently of the encoder: a block whose every word
was derived by hand from the format (tests/golden/compress_tiny.txt), exact round trip on
adversarial tables (decode is a separate code path), and structural identities that follow
from the definitions of RLE and DICT."""
from __future__ import annotations

import os

import numpy as np
import pytest

import oracle
from tests._records import records

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "compress_tiny.txt")


def _tiny():
    r = np.zeros(3, oracle.RECORD_DTYPE)
    r["pos"] = [100, 101, 102]
    r["ref"] = [0, 4, 2]
    r["genotype"] = [0, 255, 5]
    r["quality"] = [20, 0, 20]
    r["base1"] = [0, 4, 2]
    r["base2"] = [4, 4, 1]
    r["avgq1"] = [30, 0, 30]
    r["avgq2"] = [0, 0, 25]
    r["known"] = [0, 0, 1]
    r["cnt_uni1"] = [5, 0, 3]
    r["cnt_all1"] = [5, 0, 4]
    r["cnt_uni2"] = [0, 0, 2]
    r["cnt_all2"] = [0, 0, 2]
    r["depth"] = [5, 0, 6]
    r["rank_p"] = [1, 1, 0.5]
    r["copy_num"] = [1, 0, 1]
    r["post1"] = [1, 1, 0.75]
    return r


def _golden_words():
    out = []
    for line in open(GOLDEN):
        line = line.split("#")[0].strip()
        if line:
            out.append(int(line, 16))
    return np.array(out, np.uint32)


def test_golden_tiny_block():
    w = oracle.compress(_tiny(), 4)
    g = _golden_words()
    assert len(w) == len(g) and np.array_equal(w, g), (w.tolist(), g.tolist())
    assert oracle.decompress(g, 3).tobytes() == _tiny().tobytes()


@pytest.mark.parametrize("kind,n,B", [("call", 100_000, 65536), ("call", 4097, 1024),
                                      ("runs", 70_001, 8192), ("random", 20_000, 8192),
                                      ("random", 33, 16), ("const", 5000, 4096),
                                      ("call", 1, 65536), ("call", 17, 16)])
def test_round_trip(kind, n, B):
    r = records(n, seed=n % 97, kind=kind)
    w = oracle.compress(r, B)
    d = oracle.decompress(w, n)
    assert d.tobytes() == r.tobytes()
    # blocks: one per B records, each announcing its own size
    i, nb = 0, 0
    while i < len(w):
        assert w[i] == 0x31435347 and w[i + 5] == B
        assert w[i + 1] == min(B, n - nb * B)
        i += int(w[i + 4])
        nb += 1
    assert i == len(w) and nb == (n + B - 1) // B


def test_empty_stream():
    assert len(oracle.compress(records(0), 1024)) == 0
    assert len(oracle.decompress(np.zeros(0, np.uint32), 10)) == 0


def test_constant_columns_are_one_run():
    """RLE of a constant column is one run of length n; DICT of one value needs 0 bits."""
    n = 3000
    r = records(n, kind="const")
    w = oracle.compress(r, 4096)
    # the six RLE sections are the last 6 x 5 words: [R=1, D=1, v, D=1, n]
    tail = w[-30:].reshape(6, 5)
    assert (tail[:, 0] == 1).all() and (tail[:, 1] == 1).all()
    assert (tail[:, 3] == 1).all() and (tail[:, 4] == n).all()


def test_raw_dictionary_above_4096_distinct():
    """More than 4096 distinct run values: RAW mode, values verbatim (still round-trips)."""
    n = 10_000
    r = records(n, seed=5, kind="random")
    w = oracle.compress(r, 16384)
    assert (w == 0xFFFFFFFF).any()
    assert oracle.decompress(w, n).tobytes() == r.tobytes()


def test_malformed_stream_rejected():
    g = _golden_words()
    for cut in (1, 10, 40, 81):
        with pytest.raises(ValueError):
            oracle.decompress(g[:cut], 3)
    bad = g.copy()
    bad[0] ^= 1
    with pytest.raises(ValueError):
        oracle.decompress(bad, 3)


def test_ratio_on_call_like_table():
    """The call-like table compresses well below the 40-byte record (paper: 14-16x vs text)."""
    n = 200_000
    r = records(n, seed=3)
    w = oracle.compress(r, 65536)
    assert r.nbytes / (4 * len(w)) > 5
