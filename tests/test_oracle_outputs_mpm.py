"""Pins of the oracle's k-core outputs and of its MPM
iteration (f3) -- checked against what the paper and the mathematics fix,
never against the oracle itself:

* the Fig. 1 / Fig. 2 worked example (
  tests/golden/fig1_fig2_reconstruction.json);
* closed forms: MPM on the path P_n needs floor((n-1)/2) changing iterations
  (the value 1 travels one hop inward from each end per iteration), on a
  star exactly 1, on K_n and C_n none; K_n's k-cores;
* independent algorithms: the k-core by deletion (no core numbers) must equal
  {v : BZ core >= k}; the MPM fixpoint must equal the BZ core on every
  labelled graph with <= 6 vertices and on random graphs;
* a theorem: MPM iterates never increase and never drop below the core;
* brute force: the induced subgraph's arc set, by pairs.
"""
import itertools
import json
import os

import numpy as np
import pytest

import kcgen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _fig1():
    g = json.load(open(os.path.join(GOLD, "fig1_fig2_reconstruction.json")))
    idx = {s: i for i, s in enumerate(g["labels"])}
    rp, ci = kcgen.csr_from_edges(len(idx), [(idx[a], idx[b]) for a, b in g["edges"]])
    return g, idx, rp, ci


def _all_graphs_union(nv):
    """Disjoint union of every labelled graph on nv vertices."""
    pairs = list(itertools.combinations(range(nv), 2))
    edges = []
    for gi in range(1 << len(pairs)):
        for q, (a, b) in enumerate(pairs):
            if (gi >> q) & 1:
                edges.append((gi * nv + a, gi * nv + b))
    return kcgen.csr_from_edges((1 << len(pairs)) * nv, edges)


# ------------------------------------------------------------------ MPM
def test_mpm_fig2_first_iterate():
    g, idx, rp, ci = _fig1()
    a0, it0 = oracle.mpm(rp, ci, max_iters=0)
    assert it0 == 0
    assert [a0[idx[s]] for s in g["labels"]] == [g["expected_degree"][s] for s in g["labels"]]
    a1, it1 = oracle.mpm(rp, ci, max_iters=1)
    assert it1 == 1
    assert a1[idx[g["fig2_vertex"]]] == g["fig2_hindex"]  # v drops 6 -> 3
    assert [a1[idx[s]] for s in g["labels"]] == [g["mpm_first_iterate"][s] for s in g["labels"]]
    a, it = oracle.mpm(rp, ci)
    assert it == g["mpm_iterations"]
    assert [a[idx[s]] for s in g["labels"]] == [g["expected_core"][s] for s in g["labels"]]


@pytest.mark.parametrize("n", [2, 3, 4, 5, 10, 11, 64, 101])
def test_mpm_path_iteration_count(n):
    rp, ci = kcgen.csr_from_edges(n, [(i, i + 1) for i in range(n - 1)])
    a, it = oracle.mpm(rp, ci)
    assert np.all(a == 1)
    assert it == (n - 1) // 2
    # after t iterations exactly the vertices within distance t of an end hold 1
    for t in range(0, (n - 1) // 2 + 1):
        at, _ = oracle.mpm(rp, ci, max_iters=t)
        dist = np.minimum(np.arange(n), n - 1 - np.arange(n))
        want = np.where(dist <= t, 1, 2)
        assert np.array_equal(at, want), t


def test_mpm_closed_forms():
    for n in (3, 6, 20):
        rp, ci = kcgen.csr_from_edges(n, list(itertools.combinations(range(n), 2)))
        a, it = oracle.mpm(rp, ci)
        assert it == 0 and np.all(a == n - 1)
        rp, ci = kcgen.csr_from_edges(n, [(i, (i + 1) % n) for i in range(n)])
        a, it = oracle.mpm(rp, ci)
        assert it == 0 and np.all(a == 2)
    L = 50
    rp, ci = kcgen.csr_from_edges(L + 1, [(0, i) for i in range(1, L + 1)])
    a, it = oracle.mpm(rp, ci)
    assert it == 1 and np.all(a == 1)
    rp, ci = kcgen.csr_from_edges(7, [])
    a, it = oracle.mpm(rp, ci)
    assert it == 0 and np.all(a == 0)


@pytest.mark.parametrize("nv", [4, 5, 6])
def test_mpm_fixpoint_equals_core_exhaustive(nv):
    rp, ci = _all_graphs_union(nv)
    a, _ = oracle.mpm(rp, ci)
    assert np.array_equal(a, oracle.bz_core(rp, ci))


def test_mpm_iterates_monotone_and_bounded_by_core():
    for spec in [kcgen.rmat(9, 8, seed=3), kcgen.er(400, 6, seed=4), kcgen.chunglu(500, 2.1, 3000, seed=5)]:
        rp, ci = kcgen.generate_host(spec)
        core = oracle.bz_core(rp, ci)
        a_fin, its = oracle.mpm(rp, ci)
        assert np.array_equal(a_fin, core)
        prev, _ = oracle.mpm(rp, ci, max_iters=0)
        for t in range(1, its + 1):
            at, _ = oracle.mpm(rp, ci, max_iters=t)
            assert np.all(at <= prev) and np.all(at >= core), t
            prev = at
        assert np.array_equal(prev, core)


# ------------------------------------------------------------ k-cores
def test_kcore_members_fig1():
    g, idx, rp, ci = _fig1()
    for k, members in g["kcore_members"].items():
        mask = oracle.kcore_members(rp, ci, int(k))
        assert sorted(np.nonzero(mask)[0].tolist()) == sorted(idx[s] for s in members), k


def test_kcore_members_closed_forms():
    n = 9
    rp, ci = kcgen.csr_from_edges(n, list(itertools.combinations(range(n), 2)))
    for k in range(0, n + 2):
        assert oracle.kcore_members(rp, ci, k).sum() == (n if k <= n - 1 else 0)
    # star: 1-core is everything, 2-core empty
    rp, ci = kcgen.csr_from_edges(11, [(0, i) for i in range(1, 11)])
    assert oracle.kcore_members(rp, ci, 1).sum() == 11
    assert oracle.kcore_members(rp, ci, 2).sum() == 0


def test_kcore_members_equals_core_threshold():
    """Two independent algorithms: deletion at fixed k vs BZ core numbers (nestedness)."""
    for spec in [kcgen.rmat(11, 16, seed=1), kcgen.chunglu(3000, 2.1, 30000, seed=2), kcgen.er(2000, 12, seed=3)]:
        rp, ci = kcgen.generate_host(spec)
        core = oracle.bz_core(rp, ci)
        for k in sorted(set([0, 1, 2, int(core.max()), int(core.max()) + 1, int(np.median(core))])):
            assert np.array_equal(oracle.kcore_members(rp, ci, k).astype(bool), core >= k), k


def test_induced_csr_bruteforce():
    rp, ci = kcgen.generate_host(kcgen.rmat(8, 8, seed=7))
    n = rp.size - 1
    rng = np.random.default_rng(0)
    keep = (rng.random(n) < 0.5).astype(np.uint8)
    srp, sci, vm = oracle.induced_csr(rp, ci, keep)
    assert oracle.validate_csr(srp, sci) == 0
    assert vm.tolist() == np.nonzero(keep)[0].tolist()
    got = {(int(vm[i]), int(vm[sci[x]])) for i in range(vm.size) for x in range(srp[i], srp[i + 1])}
    want = {(v, int(u)) for v in range(n) for u in ci[rp[v]:rp[v + 1]] if keep[v] and keep[u]}
    assert got == want
