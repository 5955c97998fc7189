"""T0 units on the GPU (SURVEY 8(c) test tiers): the Fig. 8 ballot compaction
primitive, the level-skip minimum (SURVEY Q10 / DESIGN reading R5), and the
north-star C symbol ``kcore_decompose`` called directly through ctypes on real
graphs (not through the binding's ``_ex`` path)."""
import ctypes
import json
import os

import numpy as np
import pytest

import kcgen
import oracle

torch = pytest.importorskip("torch")
import paper_conf_icde_ahmady0gcz23_b200 as kc  # noqa: E402

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden")
DEV = "cuda:0"


def _lib():
    lib = kc.library()
    lib.kcore_test_ballot_compact.argtypes = [ctypes.c_void_p] * 2 + [ctypes.c_int32] + [ctypes.c_void_p] * 4
    lib.kcore_decompose.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64,
                                    ctypes.c_void_p, ctypes.c_void_p]
    return lib


def test_fig8_ballot_compaction():
    """P:L368-370 (Fig. 8): p=[1,0,0,1,1,1,0,1] over a..h gives the exclusive
    prefix a=[0,1,1,1,2,3,4,4]; e advances by 5; a,d,e,f,h land in order."""
    g = json.load(open(os.path.join(GOLD, "fig8_ballot.json")))
    lib = _lib()
    names = g["vids"]
    vid = torch.arange(len(names), dtype=torch.int32, device=DEV)
    pred = torch.tensor(g["p"], dtype=torch.int32, device=DEV)
    prefix = torch.full((len(names),), -7, dtype=torch.int32, device=DEV)
    buf = torch.full((len(names),), -1, dtype=torch.int32, device=DEV)
    e0 = 3  # e_old: the cursor need not start at 0
    e = torch.tensor([e0], dtype=torch.int32, device=DEV)
    rc = lib.kcore_test_ballot_compact(vid.data_ptr(), pred.data_ptr(), len(names), prefix.data_ptr(),
                                       buf.data_ptr() - 4 * e0, e.data_ptr(), None)
    assert rc == 0
    assert prefix.cpu().tolist() == g["exclusive_prefix"]
    assert int(e.item()) - e0 == g["e_advance"]
    got = [names[i] for i in buf.cpu().tolist()[:g["e_advance"]]]
    assert got == g["appended_in_order"]


def test_ballot_compaction_many_warps():
    """Random predicates over 300 warps: per-warp prefixes are exclusive popcounts,
    every selected id is appended exactly once, and each warp's ids are contiguous
    and in lane order."""
    rng = np.random.default_rng(8)
    n = 300 * 32 + 17  # ragged last warp
    p = (rng.random(n) < 0.37).astype(np.int32)
    lib = _lib()
    vid = torch.arange(n, dtype=torch.int32, device=DEV)
    pred = torch.from_numpy(p).to(DEV)
    prefix = torch.empty(n, dtype=torch.int32, device=DEV)
    buf = torch.full((n,), -1, dtype=torch.int32, device=DEV)
    e = torch.zeros(1, dtype=torch.int32, device=DEV)
    assert lib.kcore_test_ballot_compact(vid.data_ptr(), pred.data_ptr(), n, prefix.data_ptr(), buf.data_ptr(),
                                         e.data_ptr(), None) == 0
    pre = prefix.cpu().numpy()
    for w in range(0, n, 32):
        pw = p[w:w + 32]
        assert np.array_equal(pre[w:w + 32], np.concatenate([[0], np.cumsum(pw)[:-1]]))
    tot = int(e.item())
    assert tot == int(p.sum())
    out = buf.cpu().numpy()[:tot]
    assert np.array_equal(np.sort(out), np.nonzero(p)[0])
    # each warp's block is contiguous and ascending (lane order)
    blocks = {}
    for pos, v in enumerate(out):
        blocks.setdefault(v // 32, []).append(pos)
    for w, pos in blocks.items():
        assert pos == list(range(pos[0], pos[0] + len(pos)))
        assert list(out[pos[0]:pos[0] + len(pos)]) == sorted(out[pos[0]:pos[0] + len(pos)])


def _hub_clique(t, leaves, attach):
    """K_t (core t-1) plus a hub with `leaves` pendant leaves and `attach` edges
    into the clique (attach < t-1).  At level 1 the scan-time minimum degree
    above k is min(t-1, ...) but peeling the leaves takes the hub from
    leaves+attach down to `attach`: the level skip must go to `attach`, which
    only the peel-reported minimum (old-1 > k) knows."""
    e = [(i, j) for i in range(t) for j in range(i + 1, t)]
    hub = t
    e += [(hub, i) for i in range(attach)]
    e += [(hub, t + 1 + x) for x in range(leaves)]
    n = t + 1 + leaves
    want = np.ones(n, dtype=np.int32)
    want[:t] = t - 1
    want[hub] = attach
    return kcgen.csr_from_edges(n, e), want


@pytest.mark.parametrize("t,leaves,attach", [(8, 20, 3), (12, 5000, 5), (40, 200_000, 2), (6, 3, 4)])
def test_level_skip_uses_peel_minimum(t, leaves, attach):
    (rp, ci), want = _hub_clique(t, leaves, attach)
    ref = oracle.bz_core(rp, ci)
    assert np.array_equal(ref, want)  # the construction is what the docstring says
    r = torch.from_numpy(rp).to(DEV)
    c = torch.from_numpy(ci).to(DEV)
    for kw in (dict(), dict(bloom=False), dict(algo=kc.ALGO_HOSTLOOP)):
        core, st = kc.kcore_decompose(r, c, stats=True, **kw)
        assert np.array_equal(core.cpu().numpy(), want), kw
        # level skipping visits exactly the distinct core values (no empty level counted)
        assert st.levels == len(np.unique(want)), (kw, st.levels)
        assert st.kmax == t - 1


def test_level_skip_gaps():
    """Disjoint cliques K_3, K_9, K_40, K_41 and a path: core values {1,2,8,39,40};
    every gap between them is one level-skip jump."""
    parts = [kcgen.csr_from_edges(s, [(i, j) for i in range(s) for j in range(i + 1, s)]) for s in (3, 9, 40, 41)]
    parts.append(kcgen.csr_from_edges(50, [(i, i + 1) for i in range(49)]))
    rp, ci = kcgen.disjoint_union(parts)
    want = oracle.bz_core(rp, ci)
    assert sorted(set(want.tolist())) == [1, 2, 8, 39, 40]
    core, st = kc.kcore_decompose(torch.from_numpy(rp).to(DEV), torch.from_numpy(ci).to(DEV), stats=True)
    assert np.array_equal(core.cpu().numpy(), want)
    assert st.levels == 5 and st.kmax == 40


@pytest.mark.parametrize("cfg", ["C1", "chunglu-small", "er-small"])
def test_north_star_symbol_direct(cfg):
    """kcore_decompose(rowptr, colidx, n, m, core_out, stream) -- the north-star
    signature itself, raw device pointers, on the caller's stream."""
    spec = {"C1": kcgen.CONFIGS["C1"], "chunglu-small": kcgen.chunglu(1 << 16, 2.1, 1 << 20),
            "er-small": kcgen.er(1 << 16, 24)}[cfg]
    rp, ci = kcgen.generate_host(spec)
    ref = oracle.bz_core(rp, ci)
    lib = _lib()
    r = torch.from_numpy(rp).to(DEV)
    c = torch.from_numpy(ci).to(DEV)
    n, m = rp.size - 1, ci.size
    s = torch.cuda.Stream()
    core = torch.full((n,), -5, dtype=torch.int32, device=DEV)
    torch.cuda.synchronize()
    rc = lib.kcore_decompose(r.data_ptr(), c.data_ptr(), n, m, core.data_ptr(), s.cuda_stream)
    assert rc == 0
    s.synchronize()
    assert np.array_equal(core.cpu().numpy(), ref)
    # inputs untouched (const)
    assert np.array_equal(r.cpu().numpy(), rp) and np.array_equal(c.cpu().numpy(), ci)
