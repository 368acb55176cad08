"""CPU ORACLE of the packed read format (reading R21) — TEST INFRASTRUCTURE ONLY.

SURVEY.md §8(f) NEXT #2's second half: GSNP's first pass writes "a compressed copy of the input"
(about a third of its size) that the second pass reads back (§V-A; Fig. 10b
P:L1076-1085).  On B200 the same idea shrinks what crosses PCIe: the reads travel packed and are
unpacked in HBM.  The paper gives no byte format, so R21 defines one from what the
paper says the data look like — four-letter bases (2 bits, N as an exception list) and qualities
that come in runs of equal value (the observation §V-B's RLE rests on).

This module is the plain definition: an encoder and a decoder written as straightforward Python
loops over reads (numpy only for the bit packing), sharing nothing with libgsnp's encoder or the
GPU decoder.  Layout (all little-endian; every section starts 16-byte aligned):

  header, 128 bytes:
    0 magic b"GSR1"  4 version u32 (1; 2 below)  8 n_reads u64  16 n_bases u64  24 n_runs u64
    32 n_nexc u64  40 n_hexc u64  48 n_blocks u32  52 block_reads u32
    56 section offsets u64[6]: blocks, meta, bases, runs, nexc, hexc   104..127 zero
  blocks  n_blocks x 5 u64: pos0 (first read's position), and the numbers of bases, runs,
          N exceptions and hits exceptions before the block
  meta    pos_rel u32[n_reads] (pos - block pos0), len_m1 u8[n_reads], sh u8[n_reads]
          (strand << 7 | min(hits - 1, 127)), nrun_m1 u8[n_reads] (each array 16-byte aligned)
  bases   2 bits per base, all reads' bases concatenated: base k at bits 2(k % 4) of byte k / 4;
          A=0 C=1 T=2 G=3, N stored as 0 and listed in nexc
  runs    u16 per run: q << 8 | (run length - 1); maximal runs of equal quality inside each read,
          in base order (a run never crosses a read)
  nexc    u32 per N base: its base index minus the block's first base index
  hexc    u32 pairs (read index minus the block's first read index, hits) for hits >= 128

Reads are blocks of block_reads consecutive reads; within a block pos - pos0 must fit in 32 bits.
Unpacking yields off = [0, len0, len0+len1, ...] (bases contiguous).

Version 2 (reference-relative bases): aligned reads mostly repeat the reference under them, so
with the reference at hand (it is resident on the device anyway) a base is predicted as the
reference code at its site (N where the reference is N) and only the bases that differ are
stored: the bases section is empty and the nexc section lists u32 (base index minus the block's
first base index) << 3 | code for every mismatching base (codes 0..4).  Everything else is as in
version 1.  A version-2 stream decodes only against the same reference.
"""
from __future__ import annotations

import struct

import numpy as np

MAGIC = b"GSR1"
HDR = 128


def _a16(x: int) -> int:
    return (x + 15) & ~15


def pack(w: dict, block_reads: int = 1024, ref=None, origin: int = 0) -> bytes:
    """Encode the read arrays of w (pos, len, off, bases, quals, strand, hits) in format R21;
    with ref (codes, known-SNP bit 3 allowed) and origin, version 2 (reference-relative)."""
    v2 = ref is not None
    if v2:
        ref = np.asarray(ref, np.uint8)
    pos = np.asarray(w["pos"], np.uint64)
    ln = np.asarray(w["len"], np.int64)
    off = np.asarray(w["off"], np.int64)
    bases_in = np.asarray(w["bases"], np.uint8)
    quals_in = np.asarray(w["quals"], np.uint8)
    strand = np.asarray(w["strand"], np.uint8)
    hits = np.asarray(w["hits"], np.int64)
    n = len(pos)
    nblk = (n + block_reads - 1) // block_reads
    blocks = np.zeros((nblk, 5), np.uint64)
    pos_rel = np.zeros(n, np.uint32)
    len_m1 = np.zeros(n, np.uint8)
    sh = np.zeros(n, np.uint8)
    nrun_m1 = np.zeros(n, np.uint8)
    codes, runs, nexc, hexc = [], [], [], []
    n_bases = 0
    for b in range(nblk):
        r0 = b * block_reads
        blocks[b] = (int(pos[r0]), n_bases, len(runs), len(nexc), len(hexc) // 2)
        base0 = n_bases
        for r in range(r0, min(n, r0 + block_reads)):
            L = int(ln[r])
            if not 1 <= L <= 256:
                raise ValueError(f"read {r}: length {L}")
            d = int(pos[r]) - int(pos[r0])
            if not 0 <= d < 2 ** 32:
                raise ValueError(f"read {r}: position out of its block's 32-bit range")
            if int(strand[r]) > 1 or int(hits[r]) < 1:
                raise ValueError(f"read {r}: strand/hits")
            pos_rel[r] = d
            len_m1[r] = L - 1
            h = int(hits[r]) - 1
            sh[r] = int(strand[r]) << 7 | min(h, 127)
            if h >= 127:
                hexc += [r - r0, int(hits[r])]
            bb = bases_in[int(off[r]):int(off[r]) + L]
            qq = quals_in[int(off[r]):int(off[r]) + L]
            if v2:
                s0 = int(pos[r]) - origin
                if s0 < 0 or s0 + L > len(ref):
                    raise ValueError(f"read {r}: outside the reference")
            for i in range(L):
                c = int(bb[i])
                if c > 4 or int(qq[i]) > 63:
                    raise ValueError(f"read {r}: base/quality out of range")
                if v2:
                    rc = int(ref[s0 + i]) & 7
                    pred = rc if rc < 4 else 4
                    if c != pred:
                        nexc.append((n_bases + i - base0) << 3 | c)
                    continue
                if c == 4:
                    nexc.append(n_bases + i - base0)
                    c = 0
                codes.append(c)
            k = 0
            nr = 0
            while k < L:                     # maximal runs of equal quality
                q = int(qq[k])
                e = k + 1
                while e < L and int(qq[e]) == q:
                    e += 1
                runs.append(q << 8 | (e - k - 1))
                nr += 1
                k = e
            nrun_m1[r] = nr - 1
            n_bases += L
    if v2:
        packed_bases = np.zeros(0, np.uint8)
    else:
        cd = np.zeros(_a16((n_bases + 3) // 4) * 4, np.uint8)
        cd[:n_bases] = codes
        packed_bases = (cd[0::4] | cd[1::4] << 2 | cd[2::4] << 4 | cd[3::4] << 6).astype(np.uint8)
        packed_bases = packed_bases[:(n_bases + 3) // 4]
    secs = [blocks.tobytes(), None, packed_bases.tobytes(), np.asarray(runs, np.uint16).tobytes(),
            np.asarray(nexc, np.uint32).tobytes(), np.asarray(hexc, np.uint32).tobytes()]
    meta = b""
    for arr in (pos_rel, len_m1, sh, nrun_m1):
        bts = arr.tobytes()
        meta += bts + b"\0" * (_a16(len(bts)) - len(bts))
    secs[1] = meta
    offs, cur = [], HDR
    for sct in secs:
        offs.append(cur)
        cur = _a16(cur + len(sct))
    hdr = MAGIC + struct.pack("<IQQQQQII6Q", 2 if v2 else 1, n, n_bases, len(runs), len(nexc), len(hexc) // 2,
                              nblk, block_reads, *offs)
    hdr += b"\0" * (HDR - len(hdr))
    out = bytearray(cur)
    out[:HDR] = hdr
    for o, sct in zip(offs, secs):
        out[o:o + len(sct)] = sct
    return bytes(out)


def header(buf: bytes) -> dict:
    if bytes(buf[:4]) != MAGIC:
        raise ValueError("not a GSR1 stream")
    v = struct.unpack_from("<IQQQQQII6Q", buf, 4)
    keys = ("version", "n_reads", "n_bases", "n_runs", "n_nexc", "n_hexc", "n_blocks",
            "block_reads")
    d = dict(zip(keys, v[:8]))
    d["sections"] = list(v[8:14])
    return d


def unpack(buf: bytes, ref=None, origin: int = 0) -> dict:
    """Decode a GSR1 stream back to read arrays (off rebuilt contiguous from 0); a version-2
    stream needs the reference it was packed against."""
    h = header(buf)
    v2 = h["version"] == 2
    if v2 and ref is None:
        raise ValueError("version-2 stream: the reference is needed")
    n, nb, B = h["n_reads"], h["n_bases"], h["block_reads"]
    s_blk, s_meta, s_bases, s_runs, s_nexc, s_hexc = h["sections"]
    blocks = np.frombuffer(buf, np.uint64, h["n_blocks"] * 5, s_blk).reshape(-1, 5)
    o = s_meta
    pos_rel = np.frombuffer(buf, np.uint32, n, o)
    o = _a16(o + 4 * n)
    len_m1 = np.frombuffer(buf, np.uint8, n, o)
    o = _a16(o + n)
    sh = np.frombuffer(buf, np.uint8, n, o)
    o = _a16(o + n)
    nrun_m1 = np.frombuffer(buf, np.uint8, n, o)
    pb = np.frombuffer(buf, np.uint8, 0 if v2 else (nb + 3) // 4, s_bases)
    runs = np.frombuffer(buf, np.uint16, h["n_runs"], s_runs)
    nexc = np.frombuffer(buf, np.uint32, h["n_nexc"], s_nexc)
    hexc = np.frombuffer(buf, np.uint32, 2 * h["n_hexc"], s_hexc).reshape(-1, 2)
    pos = np.zeros(n, np.uint64)
    ln = len_m1.astype(np.uint16) + 1
    off = np.zeros(n + 1, np.uint64)
    off[1:] = np.cumsum(ln.astype(np.uint64))
    strand = (sh >> 7).astype(np.uint8)
    hits = ((sh & 127).astype(np.uint16) + 1)
    bases = np.zeros(nb, np.uint8)
    if v2:                                   # the reference under every base
        ref = np.asarray(ref, np.uint8)
        for b in range(h["n_blocks"]):
            for r in range(b * B, min(n, (b + 1) * B)):
                s0 = int(blocks[b][0]) + int(pos_rel[r]) - origin
                rc = ref[s0:s0 + int(ln[r])] & 7
                bases[int(off[r]):int(off[r + 1])] = np.where(rc < 4, rc, 4)
    else:
        for k in range(4):
            bases[k::4] = (pb >> (2 * k)) & 3
    quals = np.zeros(nb, np.uint8)
    ri = 0
    for b in range(h["n_blocks"]):
        r0 = b * B
        pos0, base0, run0, ne0, he0 = (int(x) for x in blocks[b])
        assert run0 == ri
        r1 = min(n, r0 + B)
        for r in range(r0, r1):
            pos[r] = pos0 + int(pos_rel[r])
            k = int(off[r])
            for _ in range(int(nrun_m1[r]) + 1):
                v = int(runs[ri])
                ri += 1
                quals[k:k + (v & 255) + 1] = v >> 8
                k += (v & 255) + 1
            assert k == int(off[r + 1])
        ne1 = int(blocks[b + 1][3]) if b + 1 < h["n_blocks"] else h["n_nexc"]
        for e in nexc[ne0:ne1]:
            if v2:
                bases[base0 + (int(e) >> 3)] = int(e) & 7
            else:
                bases[base0 + int(e)] = 4
        he1 = int(blocks[b + 1][4]) if b + 1 < h["n_blocks"] else h["n_hexc"]
        for rr, hv in hexc[he0:he1]:
            hits[r0 + int(rr)] = hv
    return dict(pos=pos, len=ln, off=off, bases=bases, quals=quals, strand=strand, hits=hits)
