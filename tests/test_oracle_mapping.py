"""Pins for the mapping oracles (a1 plan geometry, a2 group partition, a5
simd worksharing owner, a12 shard partition) against values the paper prints
(tests/golden/*.json, each with its citation) and invariants of the
definitions."""
import json
import os

import numpy as np
import pytest

import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")
SIMDLENS = (1, 2, 4, 8, 16, 32)


def load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def test_paper_group_count_range_T128():
    g = load("paper_mapping.json")
    T = g["threads_per_team"]
    counts, sizes = [], []
    for S in SIMDLENS:
        if S < 2:  # "if the group size is less than two ... run on all threads" (2-level)
            continue
        G = oracle.plan_geometry(T, S)[0]
        counts.append(G)
        sizes.append(S)
    assert min(counts) == g["num_groups_min"] and max(counts) == g["num_groups_max"]
    assert min(sizes) == g["threads_per_group_min"] and max(sizes) == g["threads_per_group_max"]


def test_paper_fig2_one_group_per_warp():
    f = load("paper_mapping.json")["fig2"]
    m = oracle.group_map(f["threads_per_team"], 32)
    assert len(set(m[:, 0])) == f["groups"]
    for w in range(f["groups"]):
        lanes = m[w * 32:(w + 1) * 32]
        assert lanes[:, 3].sum() == f["mains_per_warp"]
        assert (lanes[:, 3] == 0).sum() == f["workers_per_warp"]


def test_paper_sharing_default_split():
    g = load("paper_sharing.json")
    for S in SIMDLENS:
        G, slot, _ = oracle.plan_geometry(256, S, g["sharing_bytes"], 0)
        assert G * slot == g["sharing_bytes"]            # divided evenly
    # a 24-byte SpMV payload does not fit a 16-byte slot (S=2, T=256): global fallback
    assert oracle.plan_geometry(256, 2, 2048, 24) == (128, 16, 1)
    assert oracle.plan_geometry(256, 4, 2048, 24) == (64, 32, 0)
    assert oracle.plan_geometry(256, 4, g["sharing_bytes_original"], 24) == (64, 16, 1)


@pytest.mark.parametrize("T", [32, 128, 256, 1024])
@pytest.mark.parametrize("S", SIMDLENS)
def test_group_map_invariants(T, S):
    m = oracle.group_map(T, S)
    grp, gid, size, lead, mask = (m[:, i] for i in range(5))
    assert np.all(size == S)
    # equal-size groups of adjacent threads, never spanning a warp
    for g in np.unique(grp):
        members = np.nonzero(grp == g)[0]
        assert members.size == S
        assert np.all(np.diff(members) == 1)
        assert len(set(members // 32)) == 1
        assert sorted(gid[members]) == list(range(S))
        assert lead[members].sum() == 1 and gid[members][lead[members] == 1][0] == 0
        masks = mask[members].view(np.uint32)
        assert len(set(masks.tolist())) == 1
        expected = 0
        for t in members:
            expected |= 1 << (t % 32)
        assert int(masks[0]) == expected
        assert bin(int(masks[0])).count("1") == S
    assert len(np.unique(grp)) == T // S


@pytest.mark.parametrize("S", SIMDLENS)
def test_simd_owner_cyclic(S):
    for trip in (0, 1, S - 1, S, S + 1, 3 * S + 1, 100):
        if trip < 0:
            continue
        own = oracle.simd_owner(trip, S)
        assert own.size == trip
        assert np.all(own >= 0) and np.all(own < S)
        # Fig 8: lane id runs iterations id, id+S, ...: exactly ceil((trip-id)/S) of them
        for lane in range(S):
            assert (own == lane).sum() == max(0, -(-(trip - lane) // S))
        assert np.array_equal(own, np.arange(trip) % S)


@pytest.mark.parametrize("bad", [(256, 0), (256, 3), (256, 64), (48, 4), (16, 4), (2048, 4)])
def test_plan_rejects_invalid(bad):
    assert oracle.plan_geometry(*bad) is None


@pytest.mark.parametrize("n,P", [(0, 1), (1, 4), (7, 8), (1024, 3), (10_000_001, 8)])
def test_shard_partition_covers(n, P):
    seen = 0
    for r in range(P):
        chunk, b, cnt = oracle.shard_rows(n, P, r)
        assert chunk == -(-n // P)
        assert b == min(r * chunk, n) and cnt >= 0
        assert b == seen or cnt == 0
        seen += cnt
    assert seen == n


def test_sharing_slots_are_8_byte_aligned_even_split():
    # DESIGN.md R8: sharing/G rounded down to the 8-byte payload alignment
    assert oracle.plan_geometry(256, 8, 1000, 24) == (32, 24, 0)      # 1000/32 = 31.25 -> 24
    assert oracle.plan_geometry(1024, 2, 2048, 24) == (512, 0, 1)     # 4 B -> 0: fallback
    for T in (64, 256, 1024):
        for S in (2, 4, 8, 16, 32):
            G, slot, _ = oracle.plan_geometry(T, S, 2048, 0)
            assert slot % 8 == 0 and G * slot <= 2048 and G * (slot + 8) > 2048 - 8 * G
