"""GPU parity of the k-shell / k-core outputs and of the MPM
kernel (f3), through the C ABI, against the CPU oracle.  Integer results:
bit-exact.  MPM runs the bulk-synchronous iteration, so every
iterate a_t -- not only the fixpoint -- must equal the oracle's."""
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


def _dev(rp, ci):
    return (torch.from_numpy(np.asarray(rp, dtype=np.int64)).to(DEV),
            torch.from_numpy(np.asarray(ci, dtype=np.int32)).to(DEV))


def _graphs():
    g = json.load(open(os.path.join(GOLD, "fig1_fig2_reconstruction.json")))
    idx = {s: i for i, s in enumerate(g["labels"])}
    out = [kcgen.csr_from_edges(len(idx), [(idx[a], idx[b]) for a, b in g["edges"]])]
    out.append(kcgen.csr_from_edges(1000, [(i, i + 1) for i in range(999)]))  # path: 499 iterations
    L = 5000
    out.append(kcgen.csr_from_edges(L + 1, [(0, i) for i in range(1, L + 1)]))  # star: big vertex
    for spec in [kcgen.rmat(10, 16, seed=2), kcgen.er(3000, 10, seed=3), kcgen.chunglu(4000, 2.1, 40000, seed=4),
                 kcgen.rmat(13, 16, seed=5)]:
        out.append(kcgen.generate_host(spec))
    out.append(kcgen.csr_from_edges(9, []))
    return out


def test_kshell_mask_subgraph_vs_oracle():
    for rp, ci in _graphs() + [kcgen.generate_host(kcgen.CONFIGS["C1"])]:
        r, c = _dev(rp, ci)
        core = kc.kcore_decompose(r, c)
        ref = oracle.bz_core(rp, ci)
        assert np.array_equal(core.cpu().numpy(), ref)
        kmax = int(ref.max()) if ref.size else 0
        for k in sorted({0, 1, 2, kmax // 2, kmax, kmax + 1}):
            shell = kc.kcore_kshell(core, k).cpu().numpy()
            assert shell.tolist() == np.nonzero(ref == k)[0].tolist(), k
            mask, cnt = kc.kcore_kcore_mask(core, k)
            want = oracle.kcore_members(rp, ci, k)  # deletion definition, no core numbers
            assert np.array_equal(mask.cpu().numpy(), want) and cnt == int(want.sum()), k
            srp, sci, vm = kc.kcore_kcore_subgraph(r, c, core, k)
            orp, oci, ovm = oracle.induced_csr(rp, ci, want)
            assert np.array_equal(srp.cpu().numpy(), orp), k
            assert np.array_equal(sci.cpu().numpy(), oci), k
            assert np.array_equal(vm.cpu().numpy(), ovm), k


def test_mpm_every_iterate_matches_oracle():
    for rp, ci in _graphs():
        r, c = _dev(rp, ci)
        a_ref, it_ref = oracle.mpm(rp, ci)
        ts = sorted({0, 1, 2, 3, it_ref // 2, max(it_ref - 1, 0), it_ref, it_ref + 5})
        for t in ts:
            a_o, i_o = oracle.mpm(rp, ci, max_iters=t)
            a_g, i_g = kc.kcore_mpm(r, c, max_iters=t)
            assert i_g == i_o, (t, i_g, i_o)
            assert np.array_equal(a_g.cpu().numpy(), a_o), t
        a_g, i_g = kc.kcore_mpm(r, c)
        assert i_g == it_ref and np.array_equal(a_g.cpu().numpy(), a_ref)


def test_mpm_C1_full_and_repeatable():
    rp, ci = kcgen.generate_host(kcgen.CONFIGS["C1"])
    r, c = _dev(rp, ci)
    a_ref, it_ref = oracle.mpm(rp, ci)
    assert np.array_equal(a_ref, oracle.bz_core(rp, ci))
    for rep in range(5):
        a_g, i_g, st = kc.kcore_mpm(r, c, stats=True)
        assert i_g == it_ref and np.array_equal(a_g.cpu().numpy(), a_ref), rep
    assert st.levels == it_ref and st.arcs_walked >= ci.size


@pytest.mark.slow
@pytest.mark.parametrize("name", ["C2", "C3"])
def test_mpm_fixpoint_configs(name):
    """Full-size configs: the MPM fixpoint equals the BZ core."""
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    ref = oracle.bz_core(r.cpu().numpy(), c.cpu().numpy())
    a, it = kc.kcore_mpm(r, c)
    assert np.array_equal(a.cpu().numpy(), ref), (name, it)


@pytest.mark.slow
def test_outputs_full_size_C2():
    """Outputs at a BASELINE config's full size (C2: 4.2M vertices, 134M arcs)
    against the oracle's deletion-definition k-core and induced subgraph."""
    r, c = kcgen.generate_device(kcgen.CONFIGS["C2"])
    rp, ci = r.cpu().numpy(), c.cpu().numpy()
    core = kc.kcore_decompose(r, c)
    kmax = int(core.max())
    for k in (kmax // 2, kmax):
        want = oracle.kcore_members(rp, ci, k)
        mask, cnt = kc.kcore_kcore_mask(core, k)
        assert np.array_equal(mask.cpu().numpy(), want) and cnt == int(want.sum()), k
        shell = kc.kcore_kshell(core, k).cpu().numpy()
        assert np.array_equal(shell, np.nonzero((core == k).cpu().numpy())[0]), k
        srp, sci, vm = kc.kcore_kcore_subgraph(r, c, core, k)
        orp, oci, ovm = oracle.induced_csr(rp, ci, want)
        assert np.array_equal(srp.cpu().numpy(), orp) and np.array_equal(vm.cpu().numpy(), ovm), k
        assert np.array_equal(sci.cpu().numpy(), oci), k
