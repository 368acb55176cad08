"""The library's packed-read encoder (gsnp_pack_reads, host code — no GPU needed) is byte-identical
to the oracle's plain encoder of reading R21 (oracle/pack.py) and reports sizes / range errors as
the ABI states."""
from __future__ import annotations

import numpy as np
import pytest

import synth
from oracle import pack as opk
from paper_conf_icpp_luzlwfl11_b200 import gsnp
from tests.test_oracle_pack import _tiny
from tests._util import workload


def _edge():
    rng = np.random.default_rng(5)
    reads = []
    for _ in range(300):
        L = int(rng.choice([1, 2, 3, 4, 5, 99, 100, 256]))
        reads.append(dict(pos=int(rng.integers(0, 900)), strand=int(rng.integers(2)),
                          hits=int(rng.choice([1, 3, 127, 128, 300, 65535])),
                          bases=list(rng.integers(0, 5, L)),
                          quals=list(np.repeat(rng.integers(0, 64, L // 3 + 1), 3)[:L])))
    return workload("A" * 1200, reads)


@pytest.mark.parametrize("block_reads", [1, 3, 64, 1024, 4096])
def test_library_encoder_equals_oracle(block_reads):
    for w in (_tiny(), _edge(), synth.generate("C1", n_sites=30_000, depth=12.0, seed=21)):
        a = gsnp.pack_reads(w, block_reads)
        b = np.frombuffer(opk.pack(w, block_reads), np.uint8)
        assert a.tobytes() == b.tobytes()
        assert gsnp.packed_sizes(a) == (len(w["pos"]), int(np.asarray(w["len"], np.int64).sum()))


def test_encoder_errors():
    w = _tiny()
    bad = dict(w, bases=np.array(w["bases"]).copy())
    bad["bases"][1] = 5
    with pytest.raises(gsnp.GsnpError) as e:
        gsnp.pack_reads(bad)
    assert e.value.status == -2
    with pytest.raises(gsnp.GsnpError) as e:
        gsnp.pack_reads(w, 5000)
    assert e.value.status == -1
    with pytest.raises(gsnp.GsnpError):
        gsnp.packed_sizes(np.zeros(200, np.uint8))


@pytest.mark.parametrize("block_reads", [3, 1024])
def test_library_reference_relative_encoder_equals_oracle(block_reads):
    w = synth.generate("C1", n_sites=30_000, depth=12.0, seed=21)
    ref = np.asarray(w["ref"]).copy()
    ref[100:300] = 4
    a = gsnp.pack_reads(w, block_reads, ref=ref, origin=int(w["origin"]))
    b = np.frombuffer(opk.pack(w, block_reads, ref=ref, origin=int(w["origin"])), np.uint8)
    assert a.tobytes() == b.tobytes()
    bad = dict(w, pos=np.asarray(w["pos"]).copy())
    bad["pos"][-1] = len(ref) - 5                      # past the reference end
    with pytest.raises(gsnp.GsnpError) as e:
        gsnp.pack_reads(bad, block_reads, ref=ref, origin=int(w["origin"]))
    assert e.value.status == -2
