"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle on the same seeded inputs."""
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


def _ctx(w, **kw):
    return gsnp.Context.from_workload(w, **kw)


def _oracle_all(w, P=OP, w0=None, w1=None, counts=None):
    C = oracle.calib_counts(P, w) if counts is None else counts
    p = oracle.p_matrix(P, C)
    w0 = int(w["origin"]) if w0 is None else w0
    w1 = int(w["origin"]) + len(w["ref"]) if w1 is None else w1
    rec, dbg = oracle.call_window(P, w, p, w0, w1, debug=True)
    return C, p, rec, dbg


def _check_window(ctx, w, w0, w1, C_or, p_or, P=OP):
    rec_o, dbg_o = oracle.call_window(P, w, p_or, w0, w1, debug=True)
    dg = ctx.debug_window(w, w0, w1)
    assert np.array_equal(dg["off"], dbg_o["off"])
    assert np.array_equal(dg["keys_sorted"], dbg_o["keys"])
    # builder output: same multiset per site
    off = dg["off"].astype(np.int64)
    built = dg["keys_built"].copy()
    for s in range(len(off) - 1):
        built[off[s]:off[s + 1]].sort()
    assert np.array_equal(built, dbg_o["keys"])
    assert np.array_equal(dg["counters"], dbg_o["counters"])
    rep = compare(w, dg["records"], rec_o, dbg_o["L10"], dbg_o["post10"], dg["L10"], dg["post10"])
    # production path (no debug buffers) gives the same records
    rec_g = ctx.call(w, w0, w1)
    assert rec_g.tobytes() == dg["records"].tobytes()
    return rep


@pytest.fixture(scope="module")
def c1():
    w = synth.generate("C1")
    C, p, rec, dbg = _oracle_all(w)
    return w, C, p, rec, dbg


def test_c1_calibration_tables_bit_exact(c1):
    w, C, p, _, _ = c1
    with _ctx(w) as ctx:
        counts = ctx.calibrate_count(w)
        assert np.array_equal(counts.reshape(64, 256, 4, 4), C)
        ctx.calibrate_finalize(counts)
        t = ctx.get_tables()
        assert np.array_equal(t["counts"], C)
        L = OP.max_read_len
        assert np.array_equal(t["p"][:, :L], p[:, :L])
        # T rows are Alg. 2's value for every (q_adj, coord, base, genotype), q_adj in [1, q_max]
        # (adjust never leaves that range); the other rows are never indexed
        import math
        log10 = np.vectorize(math.log10)            # glibc log10, as Alg. 2 on the host
        Q = OP.q_max + 1
        for n in range(10):
            want = log10(0.5 * p[1:Q, :L, oracle.GA1[n], :] + 0.5 * p[1:Q, :L, oracle.GA2[n], :])
            assert np.array_equal(t["T"][1:Q, :, :, n], want)
        assert not t["T"][Q:].any() and not t["T"][0].any()
        # adjust table == the oracle's adjust in every cell
        adj = t["adj"]
        for qq in range(64):
            for pcr in range(1, adj.shape[1] + 3):
                for g in range(0, adj.shape[2] + 3):
                    got = adj[qq, min(pcr, adj.shape[1]) - 1, min(g, adj.shape[2] - 1)]
                    assert got == oracle.adjust(OP, qq, pcr, g), (qq, pcr, g)


def test_c1_window_parity(c1):
    w, C, p, _, _ = c1
    with _ctx(w) as ctx:
        ctx.calibrate(w)
        rep = _check_window(ctx, w, 0, len(w["ref"]), C, p)
        assert rep["sites"] == 10_000
        # sub-windows with ragged edges
        for a, b in ((0, 1), (1, 129), (4_000, 4_517), (9_950, 10_000), (123, 123)):
            if a < b:
                _check_window(ctx, w, a, b, C, p)


@pytest.mark.parametrize("depth,dup", [(3.0, 0.0), (40.0, 0.1), (100.0, 0.1)])
def test_depth_classes_parity(depth, dup):
    """Exercises every segment-length class (8/16/32/64/128/256) and the deep CTA path."""
    w = synth.generate("C1", n_sites=6_000, depth=depth, dup_rate=dup, seed=int(depth))
    C, p, _, _ = _oracle_all(w, w0=0, w1=1)
    with _ctx(w) as ctx:
        ctx.calibrate(w)
        _check_window(ctx, w, 0, 6_000, C, p)


def _pile_workload(n_reads, seed=0, hits_frac=0.0):
    """All reads start within a few bases: a deep site (exercises the CTA deep path)."""
    rng = np.random.default_rng(seed)
    ref = rng.integers(0, 4, 600).astype(np.uint8)
    reads = []
    for k in range(n_reads):
        p = 200 + int(rng.integers(0, 5))
        b = ref[p:p + 100].copy()
        err = rng.random(100) < 0.05
        b[err] = (b[err] + rng.integers(1, 4, err.sum())) % 4
        reads.append(dict(pos=p, strand=int(rng.integers(2)),
                          hits=1 if rng.random() >= hits_frac else 2,
                          bases=b, quals=list(rng.integers(2, 41, 100))))
    return workload(ref, reads)


@pytest.mark.parametrize("n", [255, 257, 300, 700, 2000])
def test_deep_pile_parity(n):
    w = _pile_workload(n, seed=n)
    C, p, _, _ = _oracle_all(w, w0=0, w1=1)
    with _ctx(w) as ctx:
        ctx.calibrate(w)
        _check_window(ctx, w, 150, 450, C, p)


def test_edge_cases_parity():
    rng = np.random.default_rng(1)
    ref = "".join("ACTG"[i] for i in rng.integers(0, 4, 500))
    ref = ref[:100] + "N" * 20 + ref[120:]
    reads = [
        dict(pos=0, strand=0, bases="A" * 50, quals=0),                     # q = 0, short read
        dict(pos=5, strand=1, bases="NNNN" + "C" * 96, quals=2),            # N bases
        dict(pos=5, strand=1, bases="NNNN" + "C" * 96, quals=2),            # PCR duplicate
        dict(pos=40, strand=0, hits=3, bases="G" * 100, quals=30),          # multi-hit only
        dict(pos=90, strand=0, bases="T" * 100, quals=40),                  # over the N block
        dict(pos=395, strand=1, bases="A" * 105, quals=35),                 # len 105 > 100
    ]
    reads[-1]["bases"] = "A" * 100
    reads.append(dict(pos=400, strand=0, bases="ACGT" * 25, quals=list(rng.integers(0, 41, 100))))
    kp = [1e-6] * 10
    kp[3] = 0.5
    w = workload(ref, reads, known=[(95, kp), (450, kp)])
    C, p, _, _ = _oracle_all(w, w0=0, w1=1)
    with _ctx(w) as ctx:
        ctx.calibrate(w)
        _check_window(ctx, w, 0, 500, C, p)
        _check_window(ctx, w, 99, 121, C, p)


def test_empty_reads_and_depth_zero():
    ref = np.array([0, 1, 2, 3, 4] * 40, np.uint8)
    w = workload(ref, [])
    C, p, rec, dbg = _oracle_all(w)
    with _ctx(w) as ctx:
        ctx.calibrate(w)
        rec_g = ctx.call(w, 0, 200)
        compare(w, rec_g, rec, dbg["L10"], dbg["post10"])
        assert (rec_g["genotype"][4::5] == 255).all()


def test_coefficient_variants_parity():
    w = synth.generate("C1", n_sites=3_000, depth=25.0, dup_rate=0.1, seed=9)
    for kw in (dict(global_dep=1.0, pcr_dep=1.0), dict(global_dep=0.95, pcr_dep=0.7),
               dict(global_dep=0.8, pcr_dep=1.0)):
        P = oracle.Params(**kw)
        C, p, _, _ = _oracle_all(w, P, w0=0, w1=1)
        with _ctx(w, **kw) as ctx:
            ctx.calibrate(w)
            _check_window(ctx, w, 0, 3_000, C, p, P)


def test_device_inputs_and_outputs_match_host(c1):
    import torch
    w, C, p, rec_o, _ = c1
    dev = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda()
           for k in ("pos", "len", "off", "bases", "quals", "strand", "hits")}
    with _ctx(w) as ctx:
        counts = torch.zeros(64 * 256 * 16, dtype=torch.uint64, device="cuda")
        ctx.calibrate_count(dev, counts)
        assert np.array_equal(counts.cpu().numpy().reshape(64, 256, 4, 4), C)
        ctx.calibrate_finalize(counts)
        out = torch.zeros(40 * 10_000, dtype=torch.uint8, device="cuda")
        ctx.call(dev, 0, 10_000, out)
        rec_d = out.cpu().numpy().view(gsnp.RECORD_DTYPE)
        rec_h = ctx.call(w, 0, 10_000)
        assert rec_d.tobytes() == rec_h.tobytes()


def test_errors_are_statuses():
    w = synth.generate("C1", n_sites=2_000)
    with _ctx(w) as ctx:
        with pytest.raises(gsnp.GsnpError) as e:
            ctx.call(w, 0, 10)
        assert e.value.status == -4                       # before calibration
        ctx.calibrate(w)
        bad = dict(w)
        bad["pos"] = w["pos"][::-1].copy()
        with pytest.raises(gsnp.GsnpError) as e:
            ctx.call(bad, 0, 2_000)
        assert e.value.status == -3
        bad = dict(w)
        bad["quals"] = w["quals"].copy()
        bad["quals"][5] = 50
        with pytest.raises(gsnp.GsnpError) as e:
            ctx.call(bad, 0, 2_000)
        assert e.value.status == -2
        with pytest.raises(gsnp.GsnpError) as e:
            ctx.call(w, 0, 100, out=np.zeros(10, gsnp.RECORD_DTYPE))
        assert e.value.status == -7
        with pytest.raises(gsnp.GsnpError) as e:
            ctx.call(w, 1_990, 2_010)
        assert e.value.status == -2
        rec = ctx.call(w, 0, 2_000)                        # still usable after errors
        assert len(rec) == 2_000


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_variable_length_reads_parity(seed):
    """Reads of unequal length: '-' strand reads ending at the same coordinate share a cycle
    from different starts; same-start reads of unequal length do not."""
    rng = np.random.default_rng(100 + seed)
    S = 600
    ref = rng.integers(0, 4, S).astype(np.uint8)
    reads = []
    for _ in range(260):
        ln = int(rng.integers(30, 101))
        p = int(rng.integers(0, S - ln))
        st = int(rng.integers(2))
        b = ref[p:p + ln].copy()
        err = rng.random(ln) < 0.05
        b[err] = (b[err] + rng.integers(1, 4, err.sum())) % 4
        q = list(rng.integers(2, 41, ln))
        reads.append(dict(pos=p, strand=st, hits=1 if rng.random() > 0.05 else 2, bases=b, quals=q))
        if rng.random() < 0.3:                 # partner ending at the same coordinate on '-'
            ln2 = int(rng.integers(30, 101))
            p2 = p + ln - ln2
            if 0 <= p2 <= S - ln2:
                reads.append(dict(pos=p2, strand=1, bases=ref[p2:p2 + ln2],
                                  quals=list(rng.integers(2, 41, ln2))))
        if rng.random() < 0.2:                 # same start, other length / strand
            ln3 = int(rng.integers(30, 101))
            if p + ln3 <= S:
                reads.append(dict(pos=p, strand=int(rng.integers(2)), bases=ref[p:p + ln3],
                                  quals=list(rng.integers(2, 41, ln3))))
    w = workload(ref, reads)
    C, p, _, _ = _oracle_all(w, w0=0, w1=1)
    with _ctx(w) as ctx:
        ctx.calibrate(w)
        _check_window(ctx, w, 0, S, C, p)


@pytest.mark.parametrize("read_len", [150, 250])
def test_long_reads_full_quality_range_parity(read_len):
    """max_read_len 256 and q_max 63: 150/250-bp reads with qualities up to 63 (256-cycle tables;
    at 250 bp the calibration's shared histogram stops short of the last cycles, which go to
    global atomics)."""
    w = synth.generate("C1", n_sites=4_000, depth=25.0, read_len=read_len, q_hi=63, seed=77)
    P = oracle.Params(max_read_len=256, q_max=63)
    C, p, _, _ = _oracle_all(w, P, w0=0, w1=1)
    with _ctx(w, max_read_len=256, q_max=63) as ctx:
        counts = ctx.calibrate_count(w)
        assert np.array_equal(counts.reshape(64, 256, 4, 4), C)
        ctx.calibrate_finalize(counts)
        _check_window(ctx, w, 0, 4_000, C, p, P)


def test_unaligned_device_reads_calibrate_and_call(c1):
    """Device byte arrays at an odd address: the calibration's TMA stages must fall back to
    global loads (bulk copies need 16-byte alignment) and give the same counts and records."""
    import torch
    w, C, p, rec, _ = c1
    dev = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda()
           for k in ("pos", "len", "off", "strand", "hits")}
    for k in ("bases", "quals"):
        buf = torch.zeros(len(w[k]) + 3, dtype=torch.uint8, device="cuda")
        buf[3:] = torch.from_numpy(np.ascontiguousarray(w[k])).cuda()
        dev[k] = buf[3:]
    with _ctx(w) as ctx:
        counts = ctx.calibrate_count(dev)
        assert np.array_equal(counts.reshape(64, 256, 4, 4), C)
        ctx.calibrate_finalize(counts)
        got = ctx.call(dev, int(w["origin"]), int(w["origin"]) + len(w["ref"]))
    compare(w, got, rec, c1[4]["L10"])


@pytest.mark.parametrize("case", ["26x_dups", "40x_32slot", "pile"])
def test_listed_sites_thread_path_parity(case, monkeypatch):
    """k_list_sites (the 32-slot kernel's sites with 33-64 unique keys, one thread per site,
    chunked thread path) on small inputs: GSNP_LIST_MIN=0 sends every list through it (by default
    lists under 16 K sites take the warp path).  At 40X with the 32-slot kernel forced
    (GSNP_MID_AT) and in a 700-read pile, sites beyond 64 keys go on to the warp and CTA paths
    through the second list."""
    monkeypatch.setenv("GSNP_LIST_MIN", "0")
    if case == "26x_dups":
        w, win = synth.generate("C1", n_sites=6_000, depth=26.0, dup_rate=0.1, seed=26), (0, 6_000)
    elif case == "40x_32slot":
        monkeypatch.setenv("GSNP_MID_AT", "1000")
        w, win = synth.generate("C1", n_sites=6_000, depth=40.0, dup_rate=0.1, seed=40), (0, 6_000)
    else:
        w, win = _pile_workload(700, seed=7), (150, 450)
    C, p, _, _ = _oracle_all(w, w0=0, w1=1)
    with _ctx(w) as ctx:
        ctx.calibrate(w)
        _check_window(ctx, w, win[0], win[1], C, p)
