"""Windowed calling (windows of >= 256 K sites) through gsnp_call_async: the
windows together give exactly the one-window records, with no host round trip per window; device
errors are deferred to gsnp_wait; the kernel variant (32/64/128 key slots) is picked per window
on the device and every variant gives the same records."""
from __future__ import annotations

import numpy as np
import pytest

import synth
from paper_conf_icpp_luzlwfl11_b200 import gsnp

pytestmark = pytest.mark.gpu

KEYS = ("pos", "len", "off", "bases", "quals", "strand", "hits")


def _dev(w):
    import torch
    return {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda() for k in KEYS}


def _window_reads(w, dev, a, b):
    ra, rb = synth.read_range(w, a, b)
    return gsnp.make_reads(dict(dev, pos=dev["pos"][ra:rb], len=dev["len"][ra:rb],
                                off=dev["off"][ra:rb + 1], strand=dev["strand"][ra:rb],
                                hits=dev["hits"][ra:rb]))


@pytest.mark.parametrize("cfg,win", [("C2", 1 << 18), ("C5", 100_003)])
def test_async_windows_equal_one_call(cfg, win):
    import torch
    w = synth.generate(cfg, n_sites=3_000_000) if cfg == "C2" else synth.generate(cfg, n_sites=1_000_000)
    lo, hi = w["region"]
    dev = _dev(w)
    with gsnp.Context.from_workload(w, stream=torch.cuda.current_stream()) as ctx:
        ctx.calibrate(dev)
        one = torch.empty(40 * (hi - lo), dtype=torch.uint8, device="cuda")
        ctx.call(dev, lo, hi, one)
        many = torch.zeros_like(one)
        for a in range(lo, hi, win):
            b = min(hi, a + win)
            ctx.call_async(_window_reads(w, dev, a, b), a, b, many[40 * (a - lo):40 * (b - lo)])
        ctx.wait()
        assert torch.equal(one, many)


def test_variants_give_identical_records():
    """C3-like 30X input (mean depth estimate 27.6) called as one window (the 32-slot kernel, its
    33-64-key sites through k_list_sites) and as windows small enough that the overlapping reads'
    estimate picks the 64-slot kernel (500 sites: (500 + 99) / 500 x 27.6 = 33) or the 128-slot
    kernel (64 sites: 70) — at this depth every site stays on a thread path in all three, where
    keys are summed in canonical order, so the records are byte-identical."""
    import torch
    w = synth.generate("C3", n_sites=2_000_000)
    lo, hi = w["region"]
    dev = _dev(w)
    with gsnp.Context.from_workload(w, stream=torch.cuda.current_stream()) as ctx:
        ctx.calibrate(dev)
        one = torch.empty(40 * (hi - lo), dtype=torch.uint8, device="cuda")
        ctx.call(dev, lo, hi, one)
        r_all = gsnp.make_reads(dev)
        for win in (64, 500, 5_000, 300_000):
            many = torch.zeros_like(one)
            for a in range(lo, hi, win):            # all reads passed: small windows look deep
                b = min(hi, a + win)
                ctx.call_async(r_all, a, b, many[40 * (a - lo):40 * (b - lo)])
            ctx.wait()
            assert torch.equal(one, many), win


def test_async_errors_are_deferred():
    import torch
    w = synth.generate("C1", n_sites=50_000, depth=10.0, seed=13)
    dev = _dev(w)
    bad = dict(dev, pos=dev["pos"].flip(0).contiguous())
    out = torch.zeros(40 * 50_000, dtype=torch.uint8, device="cuda")
    with gsnp.Context.from_workload(w) as ctx:
        ctx.calibrate(dev)
        ctx.call_async(gsnp.make_reads(dev), 0, 10_000, out[:400_000])
        ctx.call_async(gsnp.make_reads(bad), 10_000, 20_000, out[400_000:800_000])   # unsorted
        with pytest.raises(gsnp.GsnpError) as e:
            ctx.wait()
        assert e.value.status == -3
        ctx.wait()                                   # cleared
        with pytest.raises(gsnp.GsnpError) as e:      # host-side argument errors are immediate
            ctx.call_async(gsnp.make_reads(w), 0, 100, out)
        assert e.value.status == -1
        ctx.call_async(gsnp.make_reads(dev), 0, 50_000, out)
        ctx.wait()
        ref = ctx.call(w, 0, 50_000)
    assert out.cpu().numpy().view(gsnp.RECORD_DTYPE).tobytes() == ref.tobytes()
