"""Host logic of the multi-GPU bench modes (CPU): the N-block layout synth reports without
generating the genome is the one it generates, and bench.shard_plan's strong-scaling plans for
C3/C4 (shard.plan_by_bases over a thin sample of read starts) tile the genome and balance the
expected aligned bases."""
from __future__ import annotations

import numpy as np
import pytest

import bench
import synth


@pytest.mark.parametrize("cfg", ["C2", "C3", "C4"])
def test_n_intervals_match_generation(cfg):
    base = synth.CONFIGS[cfg].scaled(n_sites=3_000_000, depth=0.5)
    w = synth.generate(base)
    m = np.zeros(base.n_sites, bool)
    for a, b in synth.n_intervals(base):
        m[a:b] = True
    assert np.array_equal(m, w["ref"] == 4)


@pytest.mark.parametrize("cfg,world", [("C3", 2), ("C3", 8), ("C4", 8)])
def test_strong_plans_tile_and_balance(cfg, world):
    genome, plan = bench.shard_plan(cfg, world)
    base = synth.CONFIGS[cfg]
    assert plan[0][0] == base.origin and plan[-1][1] == base.origin + base.n_sites
    assert all(a < b for a, b in plan) and all(plan[i][1] == plan[i + 1][0] for i in range(world - 1))
    # expected aligned bases per shard ~ non-N sites per shard (reads start uniformly on them)
    iv = synth.n_intervals(base)
    def non_n(a, b):
        cover = sum(max(0, min(b, int(y)) - max(a, int(x))) for x, y in iv)
        return (b - a) - cover
    load = np.array([non_n(a, b) for a, b in plan], np.float64)
    assert load.max() <= 1.01 * load.mean()


def test_weak_plans_are_config_sized():
    genome, plan = bench.shard_plan("C2", 4)
    n = synth.CONFIGS["C2"].n_sites
    assert plan == [(r * n, (r + 1) * n) for r in range(4)]
    assert genome.n_sites == 4 * n
