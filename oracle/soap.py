"""Oracle for SOAP alignment text -> reads (reading R19; input file 1,
P:L206-212, in SOAPsnp's format).  TEST INFRASTRUCTURE ONLY: plain Python string
handling, one line at a time, for small inputs.  Shares nothing with the CUDA parser.

Each '\\n'-terminated line (the last may be unterminated; empty lines are skipped) is split on
tabs into at least 9 fields: id, seq, qual, n_hits, a/b, len, strand, chr, location.  Lines of
another chromosome (when chr_name is given) are skipped; every other line must be well formed
(else ValueError naming the 0-based line): len == |seq| == |qual| in 1..256, seq over ACGTN in
either case -> 0 1 2 3 4, qualities ord(c) - q_offset in 0..63, n_hits >= 1 (saturating at
65535), strand '+' (0) or '-' (1), location >= 1 -> pos = location - 1 + loc_base.  Numbers are
plain decimal digit strings of 1..19 digits.
"""
from __future__ import annotations

import numpy as np

_CODE = {"A": 0, "C": 1, "T": 2, "G": 3, "N": 4}


def _num(s: str, line: int) -> int:
    if not (1 <= len(s) <= 19) or not all("0" <= c <= "9" for c in s):
        raise ValueError(f"line {line}: bad number {s!r}")
    return int(s)


def parse_soap(text: bytes, chr_name: str | None = None, q_offset: int = 33, loc_base: int = 0):
    lines = text.split(b"\n")
    if lines and lines[-1] == b"":
        lines.pop()                      # the terminator of the last line
    pos, ln, strand, hits, bases, quals = [], [], [], [], [], []
    for i, raw in enumerate(lines):
        if not raw:
            continue
        f = raw.decode("latin-1").split("\t")
        if len(f) < 9:
            raise ValueError(f"line {i}: {len(f)} fields")
        if chr_name and f[7] != chr_name:
            continue
        seq, qual = f[1], f[2]
        n = _num(f[5], i)
        if not (1 <= n <= 256) or len(seq) != n or len(qual) != n:
            raise ValueError(f"line {i}: length")
        if f[6] not in ("+", "-"):
            raise ValueError(f"line {i}: strand")
        h = _num(f[3], i)
        loc = _num(f[8], i)
        if h < 1 or loc < 1:
            raise ValueError(f"line {i}: hits/location")
        b = [_CODE.get(c.upper(), -1) for c in seq]
        q = [ord(c) - q_offset for c in qual]
        if min(b) < 0 or min(q) < 0 or max(q) > 63:
            raise ValueError(f"line {i}: base/quality character")
        pos.append(loc - 1 + loc_base)
        ln.append(n)
        strand.append(1 if f[6] == "-" else 0)
        hits.append(min(h, 65535))
        bases.extend(b)
        quals.extend(q)
    off = np.zeros(len(ln) + 1, np.uint64)
    off[1:] = np.cumsum(np.asarray(ln, np.uint64)) if ln else []
    return dict(pos=np.asarray(pos, np.uint64), len=np.asarray(ln, np.uint16), off=off,
                bases=np.asarray(bases, np.uint8), quals=np.asarray(quals, np.uint8),
                strand=np.asarray(strand, np.uint8), hits=np.asarray(hits, np.uint16))
