"""Pins for the packed read format (reading R21, oracle/pack.py; SURVEY.md §8(f) NEXT #2 "compressed
temp input"): a hand-encoded two-read example byte by byte, and the round trip
unpack(pack(w)) == w on inputs that reach every branch (N bases, >= 128 hits, 1-bp and 256-bp
reads, quality runs, block boundaries)."""
from __future__ import annotations

import struct

import numpy as np
import pytest

import synth
from oracle import pack as opk
from tests._util import workload


def _tiny():
    return workload("ACGTACGTACGTACGT", [
        dict(pos=7, strand=0, hits=1, bases="ACGTN", quals=[30, 30, 30, 20, 2]),
        dict(pos=9, strand=1, hits=200, bases="GG", quals=[40, 40])])


def test_hand_encoded_example():
    buf = opk.pack(_tiny(), block_reads=1024)
    # header: 2 reads, 7 bases, runs (30x3)(20x1)(2x1)(40x2), one N, one hits exception, 1 block
    assert buf[:4] == b"GSR1"
    v = struct.unpack_from("<IQQQQQII6Q", buf, 4)
    assert v[:8] == (1, 2, 7, 4, 1, 1, 1, 1024)
    # sections: blocks @128 (40 B), meta @176 (4 arrays of 16 B), bases @240, runs @256,
    # nexc @272, hexc @288; total 304
    assert list(v[8:]) == [128, 176, 240, 256, 272, 288] and len(buf) == 304
    assert struct.unpack_from("<5Q", buf, 128) == (7, 0, 0, 0, 0)
    assert struct.unpack_from("<2I", buf, 176) == (0, 2)           # pos - pos0
    assert buf[192:194] == bytes([4, 1])                          # len - 1
    assert buf[208:210] == bytes([0, 0x80 | 127])                 # strand << 7 | min(hits-1,127)
    assert buf[224:226] == bytes([2, 0])                          # runs - 1
    # codes A C G T N G G = 0 1 3 2 (0) 3 3, four per byte from the low bits
    assert buf[240:242] == bytes([0 | 1 << 2 | 3 << 4 | 2 << 6, 0 | 3 << 2 | 3 << 4])
    assert struct.unpack_from("<4H", buf, 256) == (30 << 8 | 2, 20 << 8, 2 << 8, 40 << 8 | 1)
    assert struct.unpack_from("<I", buf, 272) == (4,)             # the N: base 4 of the block
    assert struct.unpack_from("<2I", buf, 288) == (1, 200)        # read 1 of the block: 200 hits


def _check_roundtrip(w, block_reads):
    u = opk.unpack(opk.pack(w, block_reads))
    n = len(w["pos"])
    assert np.array_equal(u["pos"], np.asarray(w["pos"], np.uint64))
    assert np.array_equal(u["len"], np.asarray(w["len"], np.uint16))
    assert np.array_equal(u["strand"], np.asarray(w["strand"], np.uint8))
    assert np.array_equal(u["hits"], np.asarray(w["hits"], np.uint16))
    off = np.asarray(w["off"], np.int64)
    for k in ("bases", "quals"):
        src = np.concatenate([np.asarray(w[k])[off[r]:off[r] + int(w["len"][r])] for r in range(n)]) \
            if n else np.zeros(0, np.uint8)
        assert np.array_equal(u[k], src), k


@pytest.mark.parametrize("block_reads", [1, 7, 1024])
def test_roundtrip_edge_reads(block_reads):
    rng = np.random.default_rng(3)
    reads = []
    for k in range(60):
        L = int(rng.choice([1, 2, 5, 100, 256]))
        q = np.repeat(rng.integers(0, 64, L), 1)[:L]
        q[: L // 2] = q[0]                       # a long run
        b = rng.integers(0, 5, L)
        reads.append(dict(pos=int(rng.integers(0, 400)), strand=int(rng.integers(2)),
                          hits=int(rng.choice([1, 2, 127, 128, 129, 65535])), bases=list(b),
                          quals=list(q)))
    _check_roundtrip(workload("A" * 700, reads), block_reads)


def test_roundtrip_synthetic_and_size():
    w = synth.generate("C1", n_sites=20_000, depth=10.0, seed=9)
    buf = opk.pack(w, 256)
    _check_roundtrip(w, 256)
    raw = 2 * len(w["bases"]) + 21 * len(w["pos"])
    assert len(buf) < raw / 3.5                  # ~4.7x smaller at the synthetic quality runs


def test_rejects_out_of_range():
    w = _tiny()
    bad = dict(w, quals=np.array(w["quals"]).copy())
    bad["quals"][0] = 64
    with pytest.raises(ValueError):
        opk.pack(bad)
    bad = dict(w, pos=np.array([0, 2 ** 33], np.uint64))
    with pytest.raises(ValueError):
        opk.pack(bad)


def test_hand_encoded_reference_relative_example():
    """Version 2: the same two reads against reference ACGTACGTACGTACGT.  Read 0 at 7: reference
    TACGT, read ACGTN -> every base differs (codes 0 1 3 2 4); read 1 at 9: reference CG, read
    GG -> base 0 differs (code 3).  Exceptions: block-relative base index << 3 | code."""
    w = _tiny()
    buf = opk.pack(w, 1024, ref=w["ref"], origin=0)
    v = struct.unpack_from("<IQQQQQII6Q", buf, 4)
    assert v[:8] == (2, 2, 7, 4, 6, 1, 1, 1024)
    s_blk, s_meta, s_bases, s_runs, s_nexc, s_hexc = v[8:]
    assert s_bases == s_runs == 240                    # no base plane
    assert struct.unpack_from("<6I", buf, s_nexc) == (0 << 3 | 0, 1 << 3 | 1, 2 << 3 | 3,
                                                      3 << 3 | 2, 4 << 3 | 4, 5 << 3 | 3)
    assert struct.unpack_from("<2I", buf, s_hexc) == (1, 200)
    u = opk.unpack(buf, ref=w["ref"])
    assert list(u["bases"]) == [0, 1, 3, 2, 4, 3, 3]
    with pytest.raises(ValueError):
        opk.unpack(buf)                                # needs the reference


@pytest.mark.parametrize("block_reads", [7, 1024])
def test_reference_relative_roundtrip(block_reads):
    w = synth.generate("C1", n_sites=20_000, depth=10.0, seed=9)
    ref = np.asarray(w["ref"]).copy()
    ref[5000:5100] = 4                                 # an N block under some reads
    ref[7000] |= 8                                     # a known-SNP flag (ignored by the code)
    buf1 = opk.pack(w, block_reads)
    buf2 = opk.pack(w, block_reads, ref=ref, origin=int(w["origin"]))
    assert len(buf2) < 0.75 * len(buf1)
    u = opk.unpack(buf2, ref=ref, origin=int(w["origin"]))
    for k in ("bases", "quals", "pos", "strand", "hits"):
        assert np.array_equal(u[k], opk.unpack(buf1)[k]), k
    assert np.array_equal(u["bases"], np.asarray(w["bases"]))
