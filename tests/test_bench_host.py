"""CPU checks of bench.py's host-side helpers (no GPU): the e2e placement
helper never fails the bench and never widens the CPU set, and the N > 1
slabs partition a field into block-aligned, contiguous, covering pieces."""
from __future__ import annotations

import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_bind_to_gpu_numa_is_safe_without_a_gpu():
    before = os.sched_getaffinity(0)
    prev, why = bench.bind_to_gpu_numa(0)
    try:
        assert isinstance(why, str) and why
        now = os.sched_getaffinity(0)
        if prev is None:
            assert now == before and why.startswith("not bound")
        else:
            assert prev == before and now < before
    finally:
        os.sched_setaffinity(0, before)


def test_slabs_partition_block_aligned():
    for n in (0, 1, 31, 32, 1000, 280_953_867):
        for world in (1, 2, 3, 8):
            pieces = [bench.slab(n, r, world) for r in range(world)]
            assert pieces[0][0] == 0 and pieces[-1][1] == n
            for (a0, a1), (b0, b1) in zip(pieces, pieces[1:]):
                assert a1 == b0 and a0 <= a1
            for a, _ in pieces[1:]:
                assert a % 32 == 0 or a == n
