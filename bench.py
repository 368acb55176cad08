#!/usr/bin/env python
"""bench.py — GSNP hot path on B200: genome sites/s (device-timed) + roofline of the top kernel.

One step = the whole hot path over one shard of synthetic input:
calibration count (GPU histogram) -> [N>1: NCCL all-reduce of the 2 MiB counts] -> finalize
(host p matrix + score table, upload) -> gsnp_call over every site of the shard.  Inputs are
resident in HBM before timing.  N=1 workload: BASELINE.json configs[1] (C2, chr21-like 48 Mb,
20X).  Multi-GPU: weak scaling, each rank a contiguous C2-sized shard of a larger genome.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl reference]

--impl reference times the CPU oracle (the reference arm of this tier) on a bounded sample.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "genome sites/sec at 1/2/4/8 B200 (device-timed) + % of HBM roofline"
UNIT = "sites/s"


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.rows = []
        self.stop = threading.Event()
        self.th = threading.Thread(target=self._run, daemon=True)

    def _run(self):
        while not self.stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                                      "--format=csv,noheader,nounits"], capture_output=True,
                                     text=True, timeout=5).stdout.strip()
                if out:
                    self.rows.append([x.strip() for x in out.split(",")])
            except Exception:
                pass
            self.stop.wait(0.1)

    def __enter__(self):
        self.th.start()
        return self

    def __exit__(self, *a):
        self.stop.set()
        self.th.join(timeout=10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4)
                          if len(r) > 2 + i and r[2 + i].lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons,
                "samples": len(self.rows)}


def _l2_gather_peak(live: bool = True):
    """Measured ceiling of random 80-byte row gathers from an L2-resident 2 MB table."""
    exe = os.path.join(ROOT, "tools", "l2_gather_peak")
    if live and os.path.exists(exe):
        try:
            out = subprocess.run([exe], capture_output=True, text=True, timeout=60).stdout
            return float(json.loads(out.strip().splitlines()[-1])["l2_gather_gbs"]), "measured live"
        except Exception:
            pass
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "l2_gather_peak.json")))
        return float(d["l2_gather_gbs"]), "measured (profiles/l2_gather_peak.json)"
    except Exception:
        return 6650.0, "fallback (HBM copy peak)"


def _dist():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


STRONG = ("C3", "C4")          # BASELINE configs quoted as one genome sharded over the GPUs


def shard_plan(cfg_name: str, ws: int):
    """Contiguous shards of the config's genome, one per rank.  C3/C4 (strong scaling, BASELINE
    configs[2..3]): the whole genome split by expected aligned bases — shard.plan_by_bases over a
    thin sample of read starts drawn with the generator's placement density (no full generation).
    Other configs (weak scaling): rank r holds a config-sized piece of a ws-times longer genome."""
    import synth
    from paper_conf_icpp_luzlwfl11_b200 import shard
    base = synth.CONFIGS[cfg_name]
    if cfg_name in STRONG:
        starts = synth.sample_read_starts(base, 2_000_000, seed=base.seed)
        ln = np.full(len(starts), base.read_len, np.int64)
        return base, shard.plan_by_bases(starts, ln, base.n_sites, base.origin, ws)
    n = base.n_sites
    if ws == 1:
        return base, [(base.origin, base.origin + n)]
    genome = base.scaled(n_sites=n * ws, n_lead_frac=base.n_lead_frac / ws,
                         n_blocks=base.n_blocks * ws)
    return genome, [(r * n, (r + 1) * n) for r in range(ws)]


def make_shard(cfg_name: str, rank: int, ws: int):
    """This rank's shard: the reads covering its sites (read-length halo included) and the
    reference under them, generated region by region (shard.py)."""
    import synth
    genome, plan = shard_plan(cfg_name, ws)
    lo, hi = plan[rank]
    if lo == genome.origin and hi == genome.origin + genome.n_sites:
        return synth.generate(genome)
    return synth.generate(genome.scaled(region_lo=lo - genome.origin, region_hi=hi - genome.origin))


def count_keys(w, w0: int, w1: int, chunk: int = 1 << 20) -> int:
    """Unique non-N aligned bases at sites [w0, w1) (one score-table row each), counted read chunk
    by read chunk (bounded memory at C3/C4 sizes)."""
    pos = np.asarray(w["pos"], np.int64)
    ln = np.asarray(w["len"], np.int64)
    off = np.asarray(w["off"], np.int64)
    keys = 0
    for a in range(0, len(pos), chunk):
        b = min(len(pos), a + chunk)
        uni = np.repeat(np.asarray(w["hits"][a:b]) == 1, ln[a:b])
        ok = uni & (np.asarray(w["bases"][off[a]:off[b]]) < 4)
        if pos[a] < w0 or pos[b - 1] + ln[a:b].max() > w1:          # reads crossing the edges
            site = np.repeat(pos[a:b], ln[a:b]) + (np.arange(off[a], off[b]) -
                                                  np.repeat(off[a:b], ln[a:b]))
            ok &= (site >= w0) & (site < w1)
        keys += int(np.count_nonzero(ok))
    return keys


def input_bytes(w) -> int:
    return sum(int(np.asarray(w[k]).nbytes) for k in ("pos", "len", "off", "bases", "quals",
                                                      "strand", "hits"))


def _oracle_step(w, lo, hi, procs=None):
    """One oracle step over sites [lo, hi) of w: calibration counts over the reads that touch the
    sites, p matrix, and every record — P independent single-threaded oracle processes over
    windows (SURVEY.md §8(d) timing protocol, tests/_mp.py).  Returns (records, stats)."""
    import oracle
    import synth
    from tests._mp import calib_parallel, call_parallel
    P = oracle.Params()
    t0 = time.perf_counter()
    ra, rb = synth.read_range(w, lo, hi)
    sub = w if (ra == 0 and rb == len(w["pos"])) else synth.slice_reads(w, ra, rb)
    C, cst = calib_parallel(P, sub, procs)
    tp = time.perf_counter()
    p = oracle.p_matrix(P, C)
    tp = time.perf_counter() - tp
    rec, _, _, st = call_parallel(P, sub, p, lo, hi, procs=procs)
    wall = time.perf_counter() - t0
    return rec, {"wall_s": wall, "cpu_s": cst["cpu_s"] + tp + st["cpu_s"], "procs": st["procs"],
                 "sites": hi - lo, "reads": rb - ra}


def cpu_baseline_full(w, rec_gpu=None):
    """cpu_baseline: the oracle as it stands over the WHOLE shard (calibration + every site) on all
    host cores.  Also compares its records with the GPU's (full-config parity counters)."""
    lo, hi = w["region"]
    rec, st = _oracle_step(w, lo, hi)
    out = {"value": st["sites"] / st["wall_s"], "unit": UNIT, "cores": st["procs"], "kind": "oracle",
           "sample": f"the whole shard: calibration over all {st['reads']} reads + all {st['sites']} "
                     f"sites, {st['procs']} single-threaded oracle processes over windows",
           "wall_s": round(st["wall_s"], 2), "core_seconds": round(st["cpu_s"], 1),
           "per_core_value": st["sites"] / st["cpu_s"]}
    if rec_gpu is not None and len(rec_gpu) == len(rec):
        out["parity"] = {f: int(np.count_nonzero(rec_gpu[f] != rec[f]))
                         for f in ("genotype", "quality", "base1", "base2", "depth", "cnt_uni1")}
        out["parity"]["note"] = ("mismatching records per field, GPU vs oracle over the whole shard "
                                 "(tests/test_gpu_fullsize.py applies the near-tie / near-integer rules)")
    return out


def run_reference(args):
    """--impl reference: the oracle (this tier's reference arm) on the host cores, each step a
    bounded contiguous sample (1/8) of the shard, timed step by step (measured ms_per_step)."""
    ws, rank, _ = _dist()
    if rank != 0:
        return 0
    w = make_shard(args.config, 0, 1)
    lo, hi = w["region"]
    S = hi - lo
    n = max(1, S // args.ref_frac)
    s0 = lo + (S - n) // 2                       # mid-shard (C2 starts with its leading N block)
    for _ in range(args.warmup):
        _oracle_step(w, s0, s0 + max(1, n // 16))
    times, st = [], None
    for _ in range(args.steps):
        _, st = _oracle_step(w, s0, s0 + n)
        times.append(st["wall_s"])
    ms = 1e3 * float(np.mean(times))
    v = n / (ms / 1e3)
    desc = (f"oracle calibrate+call over sites [{s0},{s0 + n}) (1/{args.ref_frac} of the {S}-site "
            f"shard, {st['reads']} reads) per step, {st['procs']} single-threaded processes")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": args.config, "sample": desc},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": st["procs"], "kind": "oracle",
                             "sample": desc},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def run_gpu(args):
    import torch
    from paper_conf_icpp_luzlwfl11_b200 import gsnp
    ws, rank, local = _dist()
    if ws != args.gpus:
        args.gpus = ws
    # debug knobs to exercise the multi-rank flow on a one-GPU box (not for timing):
    # GSNP_BENCH_BACKEND=gloo (collectives staged through host memory), GSNP_BENCH_SAME_GPU=1
    backend = os.environ.get("GSNP_BENCH_BACKEND", "nccl")
    if os.environ.get("GSNP_BENCH_SAME_GPU"):
        local = 0
    torch.cuda.set_device(local)
    dist = None
    if ws > 1:
        import torch.distributed as dist
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)

    def all_reduce_(t, op=None):
        kw = {} if op is None else {"op": op}
        if backend == "nccl":
            dist.all_reduce(t, **kw)
        else:
            c = t.cpu()
            dist.all_reduce(c, **kw)
            t.copy_(c)
    from paper_conf_icpp_luzlwfl11_b200 import shard
    w = make_shard(args.config, rank, ws)
    w0, w1 = w["region"]                      # this rank's sites; w["ref"] also covers the halo
    S = w1 - w0
    stream = torch.cuda.current_stream()
    keys = ("pos", "len", "off", "bases", "quals", "strand", "hits")
    host = {k: torch.from_numpy(np.ascontiguousarray(w[k])) for k in keys}
    dev = {k: v.cuda() for k, v in host.items()}
    torch.cuda.synchronize()
    ctx = gsnp.Context.from_workload(w, device=local, stream=stream,
                                     flags=gsnp.GSNP_RANK_SUM | gsnp.GSNP_TIMING)
    counts = torch.zeros(64 * 256 * 16, dtype=torch.uint64, device="cuda")
    out = torch.empty(40 * S, dtype=torch.uint8, device="cuda")
    rd = gsnp.make_reads(dev)
    # calibration counts a read only on the rank that owns its start (no double counting)
    ora, orb = shard.owned_reads(w["pos"], w0, w1)

    def owned(d):
        return dict(d, pos=d["pos"][ora:orb], len=d["len"][ora:orb], off=d["off"][ora:orb + 1],
                    strand=d["strand"][ora:orb], hits=d["hits"][ora:orb])

    def step():
        ctx.calibrate_count(owned(dev), counts)
        if dist is not None:
            all_reduce_(counts.view(torch.int64))
        ctx.calibrate_finalize(counts)
        ctx.call_reads(rd, w0, w1, out)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    ctx.stage_times(reset=True)
    l0 = ctx.launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if dist is not None:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            step()
        ev1.record(stream)
        torch.cuda.synchronize()
    if dist is not None:
        dist.barrier()
    ms_total = ev0.elapsed_time(ev1)
    launches = ctx.launch_count() - l0
    st = ctx.stage_times(reset=True)
    t = torch.tensor([ms_total], dtype=torch.float64, device="cuda")
    if dist is not None:
        all_reduce_(t, dist.ReduceOp.MAX)
    ms_max = float(t.item())
    ms_step = ms_max / args.steps
    # per-rank shard sizes (all-gathered; the max-over-ranks time above covers every rank)
    mine = [S, int(len(w["pos"])), int(w["off"][-1] - w["off"][0]), float(ms_total / args.steps)]
    if dist is not None:
        allv = [None] * ws
        dist.all_gather_object(allv, mine)
    else:
        allv = [mine]
    total_sites = sum(int(v[0]) for v in allv)
    value = total_sites / (ms_step / 1e3)
    strong = args.config in STRONG

    # ---- e2e: the same step through the public API with pinned host inputs and outputs, the
    # host->device copy of the reads and the device->host copy of the result inside the timed
    # region.  Transfers overlap compute: reads go up in chunks on a copy stream while the
    # calibration counts each chunk that has arrived; the result of each window chunk comes down
    # while the next chunk is being called.  Two results: the 40-byte records (gsnp_call), and the
    # paper's output form, the RLE-DICT-compressed records (gsnp_call_compressed, §V-B) — the
    # headline e2e.
    # e2e pipeline: the reads go up in KR chunks (the calibration counts each chunk as it lands);
    # the window is called in K chunks of geometrically shrinking size (geometric, 2:1 per step), so each chunk's
    # result download hides under the next chunk's compute and the exposed tail is the smallest
    KR = int(os.environ.get("GSNP_E2E_READ_CHUNKS", "8"))
    K = int(os.environ.get("GSNP_E2E_CHUNKS", "4"))   # packed input, B 32768: 2/3/4 chunks 30.6/30.3/29.9 ms
    CZ_B = int(os.environ.get("GSNP_E2E_CZ_B", "32768"))     # 65536 / 16384: +0.7% / +1.6% e2e time
    pinned = {k: v.pin_memory() for k, v in host.items()}
    out_h = torch.empty(40 * S, dtype=torch.uint8).pin_memory()
    dev2 = {k: torch.empty_like(v, device="cuda") for k, v in host.items()}
    h2d = sum(v.numel() * v.element_size() for v in pinned.values())
    nr_all = int(len(w["pos"]))
    rcut = [nr_all * i // KR for i in range(KR + 1)]
    ocut = [int(w["off"][r]) for r in rcut]
    wt = [2.0 ** (K - 1 - j) for j in range(K)]
    wcut = [w0 + int(S * sum(wt[:j]) / sum(wt)) for j in range(K + 1)]
    wcut[-1] = w1
    copy_stream = torch.cuda.Stream()
    part = torch.zeros_like(counts)
    zcap = 11 * max(b - a for a, b in zip(wcut, wcut[1:])) + 4096   # words per chunk (> 10/record)
    zdev = torch.empty(K * zcap, dtype=torch.int32, device="cuda")
    zh = torch.empty(K * zcap, dtype=torch.int32).pin_memory()
    znw = [0] * K
    gofs = [0] * ws                           # global word offset of each rank's compressed output

    bd = {}                                   # breakdown events of the last e2e step

    def _ev(name, st):
        e = torch.cuda.Event(enable_timing=True)
        e.record(st)
        bd[name] = e

    # packed reads (R21, §8(f) NEXT #2's compressed input): the host holds the shard's reads in the
    # packed form — written once by gsnp_pack_reads, like GSNP's first-pass temp file
    # — and every e2e step ships them through the C ABI's host-buffer path
    # (gsnp_unpack_reads: chunked H2D on the library's copy stream, decoded in HBM as chunks land)
    t_pack = time.perf_counter()
    packed = torch.from_numpy(gsnp.pack_reads(w, 1024, ref=w["ref"], origin=int(w["origin"]))).pin_memory()
    t_pack = time.perf_counter() - t_pack
    h2d_packed = packed.numel()

    def e2e_step(compressed, packed_in=False):
        evs = []
        _ev("start", stream)
        if packed_in:
            ctx.unpack_reads(packed, out=dev2)             # H2D of the packed stream + decode
            _ev("h2d_done", stream)
            counts.zero_()
            ctx.calibrate_count(owned(dev2), counts)
            if dist is not None:
                all_reduce_(counts.view(torch.int64))
            _ev("count_done", stream)
            ctx.calibrate_finalize(counts)
            _ev("finalize_done", stream)
            return e2e_calls(compressed)
        copy_stream.wait_stream(stream)
        with torch.cuda.stream(copy_stream):
            for i in range(KR):
                a, b, oa, ob = rcut[i], rcut[i + 1], ocut[i], ocut[i + 1]
                for k in ("pos", "len", "strand", "hits"):
                    dev2[k][a:b].copy_(pinned[k][a:b], non_blocking=True)
                dev2["off"][a:b + 1].copy_(pinned["off"][a:b + 1], non_blocking=True)
                dev2["bases"][oa:ob].copy_(pinned["bases"][oa:ob], non_blocking=True)
                dev2["quals"][oa:ob].copy_(pinned["quals"][oa:ob], non_blocking=True)
                e = torch.cuda.Event()
                e.record(copy_stream)
                evs.append(e)
        _ev("h2d_done", copy_stream)
        counts.zero_()
        for i in range(KR):                   # count chunk i (owned reads only) once it landed
            stream.wait_event(evs[i])
            a, b = max(rcut[i], ora), min(rcut[i + 1], orb)
            if a < b:
                sub = dict(dev2, pos=dev2["pos"][a:b], len=dev2["len"][a:b],
                           off=dev2["off"][a:b + 1], strand=dev2["strand"][a:b],
                           hits=dev2["hits"][a:b])
                ctx.calibrate_count(sub, part)
                counts.view(torch.int64).add_(part.view(torch.int64))
        if dist is not None:
            all_reduce_(counts.view(torch.int64))
        _ev("count_done", stream)
        ctx.calibrate_finalize(counts)
        _ev("finalize_done", stream)
        return e2e_calls(compressed)

    def e2e_calls(compressed):
        rd2 = gsnp.make_reads(dev2)
        for j in range(K):                    # call window chunk j, then ship its result
            lo, hi = wcut[j], wcut[j + 1]
            _ev(f"call{j}_start", stream)
            if compressed:
                znw[j] = ctx.call_compressed(rd2, lo, hi, zdev[j * zcap:(j + 1) * zcap], CZ_B)
                src, dst = zdev[j * zcap:j * zcap + znw[j]], zh[j * zcap:j * zcap + znw[j]]
            else:
                src = out[40 * (lo - w0):40 * (hi - w0)]
                ctx.call_reads(rd2, lo, hi, src)
                dst = out_h[40 * (lo - w0):40 * (hi - w0)]
            _ev(f"call{j}_end", stream)
            e = torch.cuda.Event()
            e.record(stream)
            copy_stream.wait_event(e)
            with torch.cuda.stream(copy_stream):
                dst.copy_(src, non_blocking=True)
        if compressed and dist is not None:   # §8(e) collective 2: where each rank's stream goes
            gofs[:] = shard.gather_output_offsets(
                dist, sum(znw), "cuda" if backend == "nccl" else "cpu")[0]
        _ev("calls_done", stream)
        stream.wait_stream(copy_stream)
        _ev("end", stream)

    def breakdown():
        names = ["start", "h2d_done", "count_done", "finalize_done", "calls_done", "end"]
        out = {f"{a}->{b}": round(bd[a].elapsed_time(bd[b]), 3) for a, b in zip(names, names[1:])}
        out["call_spans"] = [round(bd[f"call{j}_start"].elapsed_time(bd[f"call{j}_end"]), 3)
                             for j in range(K)]
        return out

    def time_e2e(compressed, packed_in=False):
        for _ in range(max(1, args.warmup // 2)):
            e2e_step(compressed, packed_in)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        n_e2e = max(2, min(args.steps, 5))
        ctx.stage_times(reset=True)
        e0.record(stream)
        for _ in range(n_e2e):
            e2e_step(compressed, packed_in)
        e1.record(stream)
        torch.cuda.synchronize()
        te = torch.tensor([e0.elapsed_time(e1) / n_e2e], dtype=torch.float64, device="cuda")
        if dist is not None:
            all_reduce_(te, dist.ReduceOp.MAX)
        return float(te.item())

    def dev_stages(n):
        return {k: round(v[0] / n, 3) for k, v in ctx.stage_times(reset=True).items() if v[1]}
    te_rec = time_e2e(False)
    bd_rec = breakdown()
    bd_rec["device_stage_ms"] = dev_stages(max(2, min(args.steps, 5)))
    ok_rec = bool(torch.equal(out_h, out.cpu()))
    def check_cz():      # the shipped streams == the device compressor on the device step's records
        ok = True
        for j in range(K):
            lo, hi = wcut[j], wcut[j + 1]
            ref, nw = ctx.compress(out[40 * (lo - w0):40 * (hi - w0)], CZ_B,
                                   torch.empty(zcap, dtype=torch.int32, device="cuda"))
            ok &= nw == znw[j] and bool(torch.equal(ref.cpu(), zh[j * zcap:j * zcap + nw]))
        return ok
    te_cz = time_e2e(True)
    bd_cz = breakdown()
    bd_cz["device_stage_ms"] = dev_stages(max(2, min(args.steps, 5)))
    ok_cz = check_cz()
    d2h_cz = 4 * sum(znw)
    te_pk = time_e2e(True, packed_in=True)
    bd_pk = breakdown()
    bd_pk["device_stage_ms"] = dev_stages(max(2, min(args.steps, 5)))
    ok_pk = check_cz() and all(bool(torch.equal(dev2[k], dev[k])) for k in ("pos", "bases", "quals"))
    e2e = {"value": total_sites / (te_pk / 1e3), "unit": UNIT, "h2d_bytes_per_step": h2d_packed,
           "d2h_bytes_per_step": 4 * sum(znw), "ms_per_step": te_pk, "check": ok_pk,
           "input": "packed reads R21 v2 (bases relative to the reference) in pinned host memory "
                    "(%.2f B/base; packed once by gsnp_pack_reads in %.2f s on the host, outside the "
                    "step) -> gsnp_unpack_reads (C ABI, host buffer: chunked H2D + k_unpack against the "
                    "context's device reference)" % (h2d_packed / max(1, len(w["bases"])), t_pack),
           "result": "RLE-DICT-compressed records (gsnp_call_compressed, §V-B) in %d window chunks "
                     "(geometric, 2:1 per step), each chunk's download overlapped with the next call" % K,
           "breakdown_ms": bd_pk,
           "raw_input": {"value": total_sites / (te_cz / 1e3), "ms_per_step": te_cz,
                         "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h_cz, "check": ok_cz,
                         "input": "unpacked read arrays, %d chunks, counted as they land" % KR,
                         "breakdown_ms": bd_cz},
           "records": {"value": total_sites / (te_rec / 1e3), "ms_per_step": te_rec,
                       "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": out_h.numel(),
                       "check": ok_rec, "result": "40-byte records (gsnp_call), unpacked input",
                       "breakdown_ms": bd_rec}}
    if ws > 1:
        e2e["rank_offsets_words"] = gofs      # all-gathered per-rank compressed sizes (§8(e))

    # ---- §8(f) NEXT #1, outside the step: RLE-DICT compression (§V-B) of this shard's records,
    # device to device, blocks of 65536 records.  CUDA events on the library's stream.
    nw = gsnp.ctypes.c_uint64(0)                       # size query (status CAPACITY expected)
    gsnp.lib().gsnp_compress(ctx.h, gsnp._ptr(out), S, CZ_B, None, 0, gsnp.ctypes.byref(nw))
    cz_words = int(nw.value)
    cz_out = torch.empty(cz_words, dtype=torch.int32, device="cuda")
    ctx.compress(out, CZ_B, cz_out)
    ctx.stage_times(reset=True)
    c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n_cz = 5
    c0.record(stream)
    for _ in range(n_cz):
        ctx.compress(out, CZ_B, cz_out)
    c1.record(stream)
    torch.cuda.synchronize()
    cz_ms = c0.elapsed_time(c1) / n_cz
    cz_kernel_ms = ctx.stage_times(reset=True)["compress"][0] / n_cz
    compress = {"block_sites": CZ_B, "ms": cz_ms, "kernel_ms": cz_kernel_ms,
                "records_per_s": S / (cz_ms / 1e3), "in_bytes": 40 * S, "out_bytes": 4 * cz_words,
                "ratio": 40 * S / (4 * cz_words),
                "note": "device records -> device stream, whole shard; not part of the step "
                        "(SURVEY §8(f) #1)"}

    # ---- windowed calling, outside the step: the paper calls a chromosome in windows of >= 256 K
    # sites (Fig. 11).  The same shard in 2^18-site windows through
    # gsnp_call_async (device reads, each window's read range with its halo; no host round trip
    # per window) after one calibration; CUDA events on the library's stream.
    windowed = None
    if ws == 1 and args.config not in STRONG:
        import synth
        windowed = []
        for WIN in (1 << 18, 1 << 22):
          wins = [(a, min(w1, a + WIN)) for a in range(w0, w1, WIN)]
          wrd = []
          for a, b in wins:
            ra, rb = synth.read_range(w, a, b)
            wrd.append(gsnp.make_reads(dict(dev, pos=dev["pos"][ra:rb], len=dev["len"][ra:rb],
                                            off=dev["off"][ra:rb + 1], strand=dev["strand"][ra:rb],
                                            hits=dev["hits"][ra:rb])))

          def win_step():
            ctx.calibrate_count(owned(dev), counts)
            ctx.calibrate_finalize(counts)
            for (a, b), r in zip(wins, wrd):
                ctx.call_async(r, a, b, out[40 * (a - w0):40 * (b - w0)])
            ctx.wait()
          win_step()
          torch.cuda.synchronize()
          ctx.stage_times(reset=True)
          v0, v1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
          n_w = 3
          v0.record(stream)
          for _ in range(n_w):
              win_step()
          v1.record(stream)
          torch.cuda.synchronize()
          wms = v0.elapsed_time(v1) / n_w
          windowed.append({"window_sites": WIN, "windows": len(wins), "ms_per_step": wms,
                           "value": S / (wms / 1e3), "vs_one_window": ms_step / wms,
                           "note": "calibration + every window through gsnp_call_async, one gsnp_wait"})

    # ---- §8(f) NEXT #3, outside the step: the dense ablation (Fig. 5) — SOAPsnp's
    # Alg. 1 over per-site dense base_occ arrays (gsnp_call_dense) vs the sparse path, same
    # sub-window of this shard, same records.  CUDA events on the library's stream.
    dense = None
    side = ws == 1 and args.config not in STRONG      # side legs (outside the step): N=1, C1/C2/C5
    if not args.no_dense and side:
        dlo = w0 + min(S // 4, 8_000_000)
        dhi = min(w1, dlo + (1 << 22))
        nd = dhi - dlo
        dout = torch.empty(40 * nd, dtype=torch.uint8, device="cuda")
        sout = torch.empty(40 * nd, dtype=torch.uint8, device="cuda")
        DCH = 16384

        def t_dense():
            ctx.call_dense(rd, dlo, dhi, dout, chunk_sites=DCH)

        def t_sparse():
            ctx.call_reads(rd, dlo, dhi, sout)
        res = {}
        for name, fn in (("dense", t_dense), ("sparse", t_sparse)):
            fn()
            torch.cuda.synchronize()
            ctx.stage_times(reset=True)
            d0, d1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            d0.record(stream)
            for _ in range(3):
                fn()
            d1.record(stream)
            torch.cuda.synchronize()
            res[name] = (d0.elapsed_time(d1) / 3, ctx.stage_times(reset=True))
        dst = res["dense"][1]
        dense = {"sites": nd, "window": [dlo, dhi], "chunk_sites": DCH,
                 "dense_ms": res["dense"][0], "sparse_ms": res["sparse"][0],
                 "dense_over_sparse": res["dense"][0] / res["sparse"][0],
                 "dense_stage_ms": {k: round(dst[k][0] / 3, 3) for k in
                                    ("dense_count", "dense_lik", "dense_recycle")},
                 "same_records": bool(torch.equal(dout, sout)),
                 "note": "paper: GPU dense 14-17x slower than GSNP on an M2050 (P:L915-917)"}
        del dout, sout

    # ---- §8(f) NEXT #2, outside the step: input packing on the GPU — this shard's reads as SOAP
    # alignment text (resident in HBM), parsed into the gsnp_reads arrays (gsnp_parse_soap).
    parse = None
    if not args.no_parse and side:
        import synth
        text = synth.soap_text(w, "chr21", 33)
        tdev = torch.frombuffer(bytearray(text), dtype=torch.uint8).cuda()
        del text
        pout = {k: torch.empty_like(v) for k, v in dev.items()}
        pout["off"] = torch.empty_like(dev["off"])
        lb = int(w["origin"])
        ctx.parse_soap(tdev, "chr21", 33, lb, out=pout)
        torch.cuda.synchronize()
        ctx.stage_times(reset=True)
        p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        n_p = 5
        p0.record(stream)
        for _ in range(n_p):
            got = ctx.parse_soap(tdev, "chr21", 33, lb, out=pout)
        p1.record(stream)
        torch.cuda.synchronize()
        p_ms = p0.elapsed_time(p1) / n_p
        p_kms = ctx.stage_times(reset=True)["parse"][0] / n_p
        sv = {torch.uint16: torch.int16, torch.uint64: torch.int64}

        def _sg(t):
            return t.view(sv.get(t.dtype, t.dtype))
        off0 = _sg(dev["off"])[0]
        ok = all(torch.equal(_sg(got[k]), _sg(dev[k]) - off0 if k == "off" else _sg(dev[k]))
                 for k in got)
        nbt = int(tdev.numel())
        parse = {"text_bytes": nbt, "reads": int(len(w["pos"])), "ms": p_ms, "kernel_ms": p_kms,
                 "text_GB_per_s": nbt / (p_ms / 1e3) / 1e9, "reads_per_s": len(w["pos"]) / (p_ms / 1e3),
                 "check": bool(ok),
                 "note": "SOAP text in HBM -> gsnp_reads arrays; not part of the step (SURVEY §8(f) #2)"}
        del tdev, pout, got

    if rank != 0:
        if dist is not None:
            dist.destroy_process_group()
        return 0
    # ---- roofline.  The metric is SURVEY.md §8(d)'s: METHOD bytes — what the
    # method must move through HBM: 18.2 B per aligned base (2 B read input, 0.16 B read metadata,
    # 4 B key write, 8 B sort read+write, 4 B key read) + 53 B per site (1 B reference, 12 B
    # offsets and counters, 40 B record) — per launch of the dominant kernel, k_call_tile (a3-a8
    # fused: it moves only the compulsory part of these bytes; keys stay on chip), over its average
    # launch time (CUDA events on the library's stream), against MEASURED_PEAKS.json's HBM copy
    # bandwidth.  Beside it: the whole step (+ the calibration's second read of the input,
    # 2.16 B/base), k_calib_count's own stream, and the L2 view of the score-table gather (80 B per
    # unique base vs the live gather ceiling of tools/l2_gather_peak).
    peak, peak_kind = _peaks()
    # per call: gsnp_call launches the three k_call_tile instantiations (32/64/128 slots; the two
    # the window's depth does not pick return at once) — their events sum to the call's kernel time
    # — and the kernels that finish the sites k_call_tile lists (k_list_sites, k_warp_sites,
    # k_big_sites): the method bytes cover every site, so their time is counted with it
    call_ms, call_n = st["call_tile"]
    call_ms += st.get("warp_sites", (0.0, 0))[0] + st.get("big_sites", (0.0, 0))[0]
    call_avg_ms = call_ms / args.steps
    cal_ms, cal_n = st["calib_count"]
    cal_avg_ms = cal_ms / args.steps
    nreads = int(len(w["pos"]))
    nbases = int(w["off"][-1] - w["off"][0])
    keys = count_keys(w, w0, w1)
    method_call = 18.2 * nbases + 53.0 * S
    call_gbs = method_call / (call_avg_ms / 1e3) / 1e9
    own_reads = orb - ora
    own_bases = int(w["off"][orb] - w["off"][ora]) if own_reads else 0
    method_cal = 2.16 * own_bases                       # bases + quals + read metadata
    cal_gbs = method_cal / (cal_avg_ms / 1e3) / 1e9 if cal_n else 0.0
    step_gbs = (method_call + method_cal) / (ms_step / 1e3) / 1e9
    compulsory = 2 * nbases + 21 * nreads + 1 * S + 40 * S    # fused kernel's HBM floor
    t_bytes = 80 * keys                              # score-table rows gathered per launch
    l2_achieved = t_bytes / (call_avg_ms / 1e3) / 1e9
    l2_peak, l2_kind = _l2_gather_peak(live=not args.no_cpu)
    stage_share = {k: round(v[0] / max(ms_total, 1e-9), 4) for k, v in st.items()}
    traffic = None
    tr_path = os.path.join(ROOT, "profiles", "call_tile_dram_bytes.json")
    if os.path.exists(tr_path):
        try:
            tr = json.load(open(tr_path))
            if tr.get("workload") == args.config:
                traffic = tr.get("bytes_per_launch")
        except Exception:
            traffic = None
    roofline = {
        "bound": "hbm", "achieved": call_gbs, "peak": peak, "unit": "GB/s", "frac": call_gbs / peak,
        "traffic": traffic, "peak_kind": f"MEASURED_PEAKS.json hbm_gbs ({peak_kind})",
        "kernel": "k_call_tile (+ k_list_sites, k_warp_sites, k_big_sites for the sites it lists)",
        "launch_ms": call_avg_ms, "alg_bytes_per_launch": method_call,
        "alg_bytes": "SURVEY §8(d) method bytes: 18.2 B per aligned base + 53 B per site",
        "units_per_launch": {"bases": nbases, "sites": S, "unique_keys": keys},
        "step_view": {"achieved": step_gbs, "frac": step_gbs / peak,
                      "alg_bytes_per_step": method_call + method_cal,
                      "alg_bytes": "k_call_tile's method bytes + the calibration read (2.16 B/base)"},
        "calib_view": {"kernel": "k_calib_count", "launch_ms": cal_avg_ms, "achieved": cal_gbs,
                       "frac": cal_gbs / peak, "alg_bytes_per_launch": method_cal},
        "compulsory_view": {"alg_bytes_per_launch": compulsory,
                            "achieved": compulsory / (call_avg_ms / 1e3) / 1e9,
                            "note": "inputs 2 B/base + 21 B/read + ref 1 B/site + record 40 B/site"},
        "l2_view": {"achieved": l2_achieved, "peak": l2_peak, "frac": l2_achieved / l2_peak,
                    "peak_kind": l2_kind, "alg_bytes_per_launch": t_bytes,
                    "alg_bytes": "80 B score-table row per unique base, gathered from L2"}}
    cpu = None
    if not args.no_cpu and ws == 1:            # the oracle baseline: rank 0 at N=1 only
        rec_gpu = out.cpu().numpy().view(gsnp.RECORD_DTYPE)
        cpu = cpu_baseline_full(w, rec_gpu)
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": ws, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
        "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic",
        "config": {"workload": args.config, "sites_per_gpu": S, "reads_per_gpu": nreads,
                   "total_sites": total_sites,
                   "per_rank": [{"sites": int(v[0]), "reads": int(v[1]), "bases": int(v[2]),
                                 "ms_per_step": round(v[3], 3)} for v in allv],
                   "bases_per_gpu": nbases, "depth": synth_depth(args.config),
                   "read_len": 100, "l2": "inputs (%.2f GB/GPU) > L2 126 MB; no flush" %
                   (input_bytes(w) / 1e9),
                   "parallelism": f"shard{ws}" + (" (plan_by_bases)" if strong else ""),
                   "stage_ms_per_step": {k: round(v[0] / args.steps, 4) for k, v in st.items()},
                   "stage_share": stage_share},
        "roofline": roofline,
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": launches,
        "clocks": clk.summary(),
        "compress": compress,
        "windowed": windowed,
        "dense_ablation": dense,
        "parse": parse,
    }
    print(json.dumps(line), flush=True)
    ctx.close()
    if dist is not None:
        dist.destroy_process_group()
    return 0


def synth_depth(name):
    import synth
    return synth.CONFIGS[name].depth


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C2")
    ap.add_argument("--impl", default="gsnp", choices=["gsnp", "reference"])
    ap.add_argument("--no-cpu", action="store_true",
                    help="skip the cpu_baseline leg and the live L2-gather microbenchmark")
    ap.add_argument("--ref-frac", type=int, default=8,
                    help="--impl reference: each step is this fraction (1/k) of the shard")
    ap.add_argument("--no-dense", action="store_true", help="skip the dense-ablation leg")
    ap.add_argument("--no-parse", action="store_true", help="skip the SOAP-text parsing leg")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    return run_gpu(args)


if __name__ == "__main__":
    sys.exit(main())
