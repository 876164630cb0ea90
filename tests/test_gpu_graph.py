"""GPU: graph mode (the whole fault-free factorisation captured into one CUDA graph and replayed,
include/abft.h abft_graph_release) gives bit-identical results to direct launches, on the first
(capturing) call, on replays, after a key change, and with ABFT off; an injection list bypasses it."""
import numpy as np
import pytest

import oracle
import synthetic as syn

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def P():
    import torch
    import paper_conf_ipps_chenlc16_b200 as p
    assert torch.cuda.is_available()
    return p


def factor(P, n, nb, graph, monkeypatch, opt=None, inj=None):
    import torch
    monkeypatch.setenv("ABFT_GRAPH", "1" if graph else "0")
    A = torch.empty(n, n, dtype=torch.float64, device="cuda").T
    P.abft_gen_spd(n, A)
    st, rep = P.abft_potrf_ex(n, nb, A, opt=opt, inj=inj)
    torch.cuda.synchronize()
    return st, rep, P.to_numpy_colmajor(A)


@pytest.mark.parametrize("n,nb", [(1024, 128), (2048, 256), (1536, 512)])
def test_graph_equals_direct(P, n, nb, monkeypatch):
    st0, r0, L0 = factor(P, n, nb, False, monkeypatch)
    for rep in range(3):   # capture, then replays of the cached graph
        st1, r1, L1 = factor(P, n, nb, True, monkeypatch)
        assert st0 == st1 == 0
        assert np.array_equal(np.tril(L0), np.tril(L1))
        assert r0["n_checks"] == r1["n_checks"] and r1["n_events"] == 0
    ref = oracle.potrf(syn.spd_matrix(n), nb, abft=False)
    s = np.sqrt(np.diag(syn.spd_matrix(n)))[:, None]
    err = np.max(np.abs(np.tril(L1) - np.tril(ref.L)) / np.maximum(np.abs(np.tril(ref.L)), 1e-3 * s))
    assert err <= 1e-11
    P.abft_graph_release()


def test_graph_key_change_abft_off_and_injection_bypass(P, monkeypatch):
    st, r, La = factor(P, 1024, 256, True, monkeypatch)
    st2, r2, Lb = factor(P, 2048, 256, True, monkeypatch)          # new key: recapture
    assert st == st2 == 0
    off = P.options(abft_enabled=False)
    st3, r3, Lc = factor(P, 1024, 256, True, monkeypatch, opt=off)
    st4, r4, Ld = factor(P, 1024, 256, False, monkeypatch, opt=off)
    assert st3 == st4 == 0 and np.array_equal(np.tril(Lc), np.tril(Ld)) and r3["n_checks"] == 0
    inj = syn.inj_array([dict(k=0, hook="REST", row=700, col=100, bit=50)])
    st5, r5, _ = factor(P, 1024, 256, True, monkeypatch, inj=inj)  # injections: direct path
    assert st5 == 0 and r5["n_events"] == 1
    assert P.abft_graph_release() == 0
