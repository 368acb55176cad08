"""GPU dense ablation (gsnp_call_dense): SOAPsnp's Alg. 1
over per-site dense base_occ arrays on the device must give the oracle's records (the paper's
dense == sparse claim) — and byte-identical records to the sparse gsnp_call."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import synth
from paper_conf_icpp_luzlwfl11_b200 import gsnp
from tests._parity import compare
from tests._util import workload

pytestmark = pytest.mark.gpu

OP = oracle.Params()


def _run(w, w0, w1, chunk):
    C = oracle.calib_counts(OP, w)
    p = oracle.p_matrix(OP, C)
    rec_o, dbg = oracle.call_window(OP, w, p, w0, w1, debug=True)
    with gsnp.Context.from_workload(w) as ctx:
        ctx.calibrate(w)
        rec_d = ctx.call_dense(w, w0, w1, chunk_sites=chunk)
        rec_s = ctx.call(w, w0, w1)
    rep = compare(w, rec_d, rec_o, dbg["L10"])
    assert rec_d.tobytes() == rec_s.tobytes()
    return rep


def test_dense_c1_matches_oracle_and_sparse():
    w = synth.generate("C1")
    _run(w, 0, len(w["ref"]), 1024)


@pytest.mark.parametrize("chunk", [32, 96, 4096])
def test_dense_ragged_chunks(chunk):
    """Chunk edges inside the window (reads straddle them) and a ragged last chunk."""
    w = synth.generate("C1", n_sites=3_000, depth=15.0, seed=5)
    _run(w, 37, 2_911, chunk)


@pytest.mark.parametrize("depth,dup", [(40.0, 0.1), (100.0, 0.1)])
def test_dense_deep_with_duplicates(depth, dup):
    w = synth.generate("C1", n_sites=2_000, depth=depth, dup_rate=dup, seed=int(depth) + 1)
    _run(w, 0, 2_000, 512)


def test_dense_saturated_cell_is_capacity_then_recovers():
    """256 identical unique bases at one site overflow the paper's 1-byte cell."""
    ref = "ACGT" * 100
    reads = [dict(pos=100, strand=0, hits=1, bases=ref[100:200], quals=30) for _ in range(256)]
    w = workload(ref, reads)
    with gsnp.Context.from_workload(w) as ctx:
        ctx.calibrate(w)
        with pytest.raises(gsnp.GsnpError) as e:
            ctx.call_dense(w, 0, 400, chunk_sites=128)
        assert e.value.status == -7
        # 255 copies fit; the context is clean again after the failure
        w2 = workload(ref, reads[:255])
        ctx.calibrate(w2)
        assert ctx.call_dense(w2, 0, 400, chunk_sites=128).tobytes() == ctx.call(w2, 0, 400).tobytes()


def test_dense_device_io_and_bad_chunk():
    import torch
    w = synth.generate("C1", n_sites=2_000, depth=10.0, seed=9)
    dev = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda()
           for k in ("pos", "len", "off", "bases", "quals", "strand", "hits")}
    with gsnp.Context.from_workload(w) as ctx:
        ctx.calibrate(w)
        out = torch.zeros(40 * 2_000, dtype=torch.uint8, device="cuda")
        ctx.call_dense(dev, 0, 2_000, out, chunk_sites=256)
        torch.cuda.synchronize()
        assert out.cpu().numpy().tobytes() == ctx.call(w, 0, 2_000).tobytes()
        for bad in (0, 31, 33):
            with pytest.raises(gsnp.GsnpError):
                ctx.call_dense(w, 0, 2_000, chunk_sites=bad)


def test_dense_out_of_range_quality_is_status():
    w = synth.generate("C1", n_sites=2_000, depth=10.0, seed=10)
    with gsnp.Context.from_workload(w) as ctx:
        ctx.calibrate(w)
        bad = dict(w, quals=w["quals"].copy())
        bad["quals"][7] = 50                                   # > q_max (40)
        with pytest.raises(gsnp.GsnpError) as e:
            ctx.call_dense(bad, 0, 2_000, chunk_sites=512)
        assert e.value.status == -2
        assert ctx.call_dense(w, 0, 2_000, chunk_sites=512).tobytes() == ctx.call(w, 0, 2_000).tobytes()
