"""Pins for the oracle's §3 selection rules (cc_edges case 1 / case 2 and the
subgraph packing), CPU only.

Each fixture in tests/golden/sec3_*.txt is a small graph whose expected
inserted edges (in insertion order, with weights) and tiles (centre, members,
t) were derived by hand, line by line, §3 (P@30023-32416) and
readings R21-R28; the derivation is in each file.  The
fixtures are built so that reversing any single decision changes the
expected output (DESIGN.md §3 "§3 mutation run", tools/mutate_sec3.py):

  S1 sec3_case1_order   case-1 centre order (need asc, id asc), pair tie-break, subgraph order
  S2 sec3_case1_pairs   pair order by common neighbours (P@31015), stop at high, d-desc tie-break
  S3 sec3_case2_sibling case-2 sibling / partner = fewest internal edges (P@31268), t = 4
  S4 sec3_case2_order   case 1 before case 2, case-2 centre order (CC desc), id tie-break
  S5 sec3_skip          the case-1 skip rule, one-directional sibling edges (P@31860)
  S6 sec3_case2_passes  case-2 round-robin passes, internal degrees recomputed per pass

The same expectations are checked against the production C++ transform
(libgraffix, host-only graph) so that a misreading shared by both sides would
still be caught by the hand-derived values.
"""
import numpy as np
import pytest

from golden_io import load_sec3
from oracle import transform as T
from oracle.graph import from_raw

FIXTURES = ["sec3_case1_order.txt", "sec3_case1_pairs.txt", "sec3_case2_sibling.txt",
            "sec3_case2_order.txt", "sec3_skip.txt", "sec3_case2_passes.txt"]


def _oracle(name):
    raw, meta, added, tiles = load_sec3(name)
    g = from_raw(raw)
    th = T.ppm(float(meta["cc_threshold"]))
    got_added, L = T.cc_edges(T.identity(g), th, int(meta["budget"]))
    got_tiles = T.subgraphs(L, g.n, th, int(meta.get("smax", 64)), 0)
    return g, meta, added, tiles, got_added, got_tiles


@pytest.mark.parametrize("name", FIXTURES)
def test_sec3_added_edges_in_order(name):
    _, _, added, _, got, _ = _oracle(name)
    assert [tuple(int(x) for x in e) for e in got] == added


@pytest.mark.parametrize("name", FIXTURES)
def test_sec3_tiles(name):
    _, _, _, tiles, _, got = _oracle(name)
    assert [(int(c), [int(x) for x in mem], int(t)) for c, mem, t in got] == tiles


@pytest.mark.parametrize("name", FIXTURES)
def test_sec3_full_transform_matches_fixture(name):
    """Through T.transform (apply_smem): the inserted edges land in the
    logical graph with their weights and kind, the tile list is the same."""
    raw, meta, added, tiles = load_sec3(name)
    g = from_raw(raw)
    kn = T.Knobs(smem=True, cc_threshold=float(meta["cc_threshold"]), added_edge_budget=int(meta["budget"]))
    tg = T.transform(g, kn)
    L = tg.logical()
    adds = sorted((int(s), int(d), int(w)) for s, d, w, a in zip(L.src, L.dst, L.w, L.added) if a)
    assert adds == sorted(added)
    assert [(int(c), list(m), int(t)) for c, m, t in tg.tiles] == tiles


@pytest.fixture(scope="module")
def gx():
    from paper_conf_icpp_0001n20_b200 import build
    build.build()
    import paper_conf_icpp_0001n20_b200 as m
    return m


@pytest.mark.parametrize("name", FIXTURES)
def test_sec3_library_matches_fixture(gx, name):
    """The production transform (C++, host-only graph, no device) reproduces
    the hand-derived edges and tiles."""
    raw, meta, added, tiles = load_sec3(name)
    G = gx.Graph.host_only(raw.row_ptr, raw.col, raw.w)
    info = G.transform(gx.Knobs(smem=True, cc_threshold=float(meta["cc_threshold"]),
                                added_edge_budget=int(meta["budget"])))
    ex = G.export()
    rp, col, w, ad, s2o = ex["row_ptr"], ex["col"], ex["w"], ex["edge_added"], ex["slot_to_orig"]
    got = []
    for s in range(ex["n_slots"]):
        for e in range(rp[s], rp[s + 1]):
            if ad[e]:
                got.append((int(s2o[s]), int(s2o[col[e]]), int(w[e])))
    assert sorted(got) == sorted(added)
    assert info["edges_added_smem"] == len(added)
    tp, tm = ex["tile_ptr"], ex["tile_members"]
    lt = [(int(ex["tile_centre"][i]), sorted(int(s2o[x]) for x in tm[tp[i]:tp[i + 1]]), int(ex["tile_iters"][i]))
          for i in range(len(ex["tile_centre"]))]
    assert lt == tiles


def test_sec3_every_selection_mutant_is_killed():
    """tools/mutate_sec3.py: each of 21 single-decision mutants of cc_edges /
    subgraphs (reversed orders, dropped rules, > vs >=, dropped weight term,
    single case-2 pass, ...) fails at least one hand-derived fixture."""
    import subprocess
    import sys
    import os
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, os.path.join(root, "tools", "mutate_sec3.py")], capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "SURVIVED" not in r.stdout and "NOT APPLIED" not in r.stdout
