"""Input generator (kcgen/) checks on the host: valid simple symmetric CSRs,
determinism, owner-range slicing, and the shape statistics the configs need."""
import numpy as np
import pytest

import kcgen
import oracle


@pytest.mark.parametrize("spec", [kcgen.rmat(10, 16, seed=1), kcgen.er(2000, 10, seed=2),
                                  kcgen.chunglu(3000, 2.1, 20000, seed=3),
                                  kcgen.rmat(13, 4, seed=7, a=0.45, b=0.15, c=0.15)])
def test_generated_csr_is_valid_and_deterministic(spec):
    rp, ci = kcgen.generate_host(spec)
    assert rp.shape[0] == spec.num_vertices + 1
    assert rp[0] == 0 and rp[-1] == ci.shape[0]
    assert oracle.validate_csr(rp, ci) == 0
    rp2, ci2 = kcgen.generate_host(spec)
    assert np.array_equal(rp, rp2) and np.array_equal(ci, ci2)
    rp3, ci3 = kcgen.generate_host(spec.with_seed(spec.seed + 100))
    assert not (rp3.shape == rp.shape and np.array_equal(rp3, rp) and np.array_equal(ci3, ci))


def test_edge_list_matches_csr():
    spec = kcgen.rmat(9, 8, seed=4)
    rp, ci = kcgen.generate_host(spec)
    n = spec.num_vertices
    edges = set()
    for i in range(spec.num_edges):
        u, v = kcgen.edge(spec, i)
        assert 0 <= u < n and 0 <= v < n
        if u != v:
            edges.add((u, v))
            edges.add((v, u))
    src = np.repeat(np.arange(n), np.diff(rp))
    assert set(zip(src.tolist(), ci.tolist())) == edges


def test_er_endpoints_are_uniform_draws():
    spec = kcgen.er(1000, 8, seed=3)
    us = np.array([kcgen.edge(spec, i) for i in range(spec.num_edges)])
    # uniform: each half of the id range gets ~half of the endpoints
    frac = (us < 500).mean()
    assert 0.47 < frac < 0.53


def test_owner_ranges_partition_the_graph():
    spec = kcgen.chunglu(2048, 2.1, 12000, seed=5)
    rp, ci = kcgen.generate_host(spec)
    n = spec.num_vertices
    for P in (2, 3, 8):
        bounds = [(r * n) // P for r in range(P + 1)]
        parts = [kcgen.generate_host(spec, bounds[r], bounds[r + 1]) for r in range(P)]
        cat_ci = np.concatenate([p[1] for p in parts])
        cat_deg = np.concatenate([np.diff(p[0]) for p in parts])
        assert np.array_equal(cat_ci, ci) and np.array_equal(cat_deg, np.diff(rp))


def test_permutation_is_bijection():
    # permute on a graph where every id appears (complete-ish ER) -> relabelled ids cover [0,n)
    spec = kcgen.rmat(8, 64, seed=3)
    us = {kcgen.edge(spec, i)[0] for i in range(spec.num_edges)}
    assert len(us) > 0.9 * 256
    assert max(us) < 256


def test_rmat_s16_shape():
    """C1 shape: n=65,536, ~0.9M undirected edges, many isolated
    vertices, heavy-tailed degrees, deep core hierarchy."""
    rp, ci = kcgen.generate_host(kcgen.CONFIGS["C1"])
    deg = np.diff(rp)
    m = ci.shape[0] // 2
    assert rp.shape[0] - 1 == 65536
    assert 850_000 < m < 960_000
    assert 0.2 < (deg == 0).mean() < 0.4
    assert deg.max() > 5000
    core = oracle.bz_core(rp, ci)
    assert 150 < core.max() < 300


def test_chunglu_cdf():
    spec = kcgen.chunglu(1000, 2.1, 100)
    cdf = kcgen.build_cdf(spec)
    assert cdf[-1] == 1.0 and np.all(np.diff(cdf) > 0)
    w = (np.arange(1, 1001, dtype=np.float64)) ** (-1 / 1.1)
    assert np.allclose(cdf, np.cumsum(w) / w.sum(), rtol=1e-12)
