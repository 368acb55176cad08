"""GPU SOAP-text parsing (gsnp_parse_soap, reading R19) vs the oracle
parser (oracle/soap.py) — element by element, bit-exact — and end to end into gsnp_call."""
from __future__ import annotations

import numpy as np
import pytest

import synth
from oracle.soap import parse_soap
from paper_conf_icpp_luzlwfl11_b200 import gsnp
from tests.test_oracle_soap import _golden

pytestmark = pytest.mark.gpu
KEYS = ("pos", "len", "off", "bases", "quals", "strand", "hits")


def _np(r):
    return {k: (v.cpu().numpy() if hasattr(v, "cpu") else np.asarray(v)) for k, v in r.items()}


def _same(a, b):
    for k in KEYS:
        assert np.array_equal(np.asarray(a[k]), np.asarray(b[k])), k


@pytest.fixture(scope="module")
def ctx():
    w = synth.generate("C1", n_sites=2_000)
    with gsnp.Context.from_workload(w) as c:
        yield c


@pytest.mark.parametrize("device", [True, False])
def test_golden(ctx, device):
    text, _ = _golden()
    _same(_np(ctx.parse_soap(text, "chr7", 33, 1000, device=device)), parse_soap(text, "chr7", 33, 1000))
    _same(_np(ctx.parse_soap(text, None, 33, 1000)), parse_soap(text, None, 33, 1000))
    t2 = text.rstrip(b"\n") + b"\n\n\n" + text.rstrip(b"\n")            # empty lines, no final \n
    _same(_np(ctx.parse_soap(t2, "chr7", 33, 5)), parse_soap(t2, "chr7", 33, 5))


def test_chromosome_filter_multi_tile_and_unaligned_device_text(ctx):
    import torch
    a = synth.generate("C1", n_sites=400_000, depth=15.0, seed=21)
    b = synth.generate("C1", n_sites=100_000, depth=15.0, seed=22)
    ta, tb = synth.soap_text(a, "chrA", 33), synth.soap_text(b, "chrB", 33)
    # interleave blocks of lines of the two chromosomes
    la, lb = ta.split(b"\n"), tb.split(b"\n")
    mixed = b"\n".join(la[:5000] + lb[:3000] + la[5000:] + lb[3000:])
    for name in ("chrA", "chrB"):
        want = parse_soap(mixed, name, 33, 7)
        _same(_np(ctx.parse_soap(mixed, name, 33, 7)), want)
        dev = torch.zeros(len(mixed) + 3, dtype=torch.uint8, device="cuda")
        dev[3:] = torch.frombuffer(bytearray(mixed), dtype=torch.uint8).cuda()
        _same(_np(ctx.parse_soap(dev[3:], name, 33, 7)), want)
    assert len(parse_soap(mixed, "chrA", 33, 7)["pos"]) == len(a["pos"])


@pytest.mark.parametrize("bad", ["r\tAC\tII\t1\ta\t3\t+\tc\t5", "r\tAC\tII\t1\ta\t2\t*\tc\t5",
                                 "r\tAX\tII\t1\ta\t2\t+\tc\t5", "r\tAC\t I\t1\ta\t2\t+\tc\t5",
                                 "r\tAC\tII\t0\ta\t2\t+\tc\t5", "r\tAC\tII\t1\ta\t2\t+\tc\t5x",
                                 "r\tAC\tII\t1\ta\t2\t+\tc"])
def test_malformed_is_range_error(ctx, bad):
    good = "r\tAC\tII\t1\ta\t2\t+\tc\t5\n"
    with pytest.raises(gsnp.GsnpError) as e:
        ctx.parse_soap((good + bad + "\n" + good).encode(), "c")
    assert e.value.status == -2 and "line 1" in str(e.value)
    # a line of another chromosome is skipped, not checked (as in the oracle)
    if bad.count("\t") >= 8:
        r = ctx.parse_soap((good + bad.replace("\tc\t", "\td\t") + "\n").encode(), "c")
        assert len(r["pos"]) == 1


def test_parse_then_call_equals_direct_arrays():
    w = synth.generate("C1", n_sites=20_000, depth=12.0, seed=23)
    text = synth.soap_text(w, "chr21", 64)
    with gsnp.Context.from_workload(w) as c:
        reads = c.parse_soap(text, "chr21", 64, int(w["origin"]))
        _same(_np(reads), parse_soap(text, "chr21", 64, int(w["origin"])))
        c.calibrate(reads)
        rec_p = c.call(reads, 0, 20_000)
        c.calibrate(w)
        rec_d = c.call(w, 0, 20_000)
    assert rec_p.tobytes() == rec_d.tobytes()


def test_capacity_query_and_empty(ctx):
    text, _ = _golden()
    out = {k: np.zeros(1, d) for k, d in (("pos", np.uint64), ("len", np.uint16), ("off", np.uint64),
                                          ("bases", np.uint8), ("quals", np.uint8),
                                          ("strand", np.uint8), ("hits", np.uint16))}
    with pytest.raises(gsnp.GsnpError) as e:
        ctx.parse_soap(text, "chr7", 33, 0, out=out)
    assert e.value.status == -7
    r = _np(ctx.parse_soap(b"", None))
    assert len(r["pos"]) == 0 and list(r["off"]) == [0]
