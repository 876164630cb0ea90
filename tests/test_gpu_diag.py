"""GPU: the diagonal-block factorisation (POTRF + inverse) on its own (the
recursive DMMA path of potrf.cu through the abft_dev_chol_inv diagnostic entry) against the CPU
oracle's POTF2 (PAPER.md:155-168 restated, reading A2/A3) on the same block, plus the LAPACK info
of a non-SPD block. Tolerances: L floor-relative 1e-11 (reading A18), |L inv(L) - I| <= 64 nb eps."""
import numpy as np
import pytest

import oracle
import synthetic as syn

pytestmark = pytest.mark.gpu
EPS = 2.0 ** -52


@pytest.fixture(scope="module")
def P():
    import torch
    import paper_conf_ipps_chenlc16_b200 as p
    assert torch.cuda.is_available()
    return p


def run_block(P, A):
    import torch
    nb = A.shape[0]
    At = P.colmajor(A)
    Li = torch.full((nb, nb), np.nan, dtype=torch.float64, device="cuda").T
    st = P.abft_dev_chol_inv(nb, At, Li)
    torch.cuda.synchronize()
    return st, P.to_numpy_colmajor(At), P.to_numpy_colmajor(Li)


@pytest.fixture(params=["tasks", "tasks_chunked", "rec"])
def chol_path(request, monkeypatch):
    """The diagonal-block paths: the one-launch task graph (default where nb % 64 == 0,
    nb >= 128), the same graph split into short launches at its step boundaries
    (ABFT_CHOL_CHUNKS) and the recursive multi-launch path (ABFT_CHOL=recursive), all read by the
    library per call."""
    monkeypatch.delenv("ABFT_CHOL_CHUNKS", raising=False)
    if request.param.startswith("tasks"):
        monkeypatch.delenv("ABFT_CHOL", raising=False)
        if request.param == "tasks_chunked":
            monkeypatch.setenv("ABFT_CHOL_CHUNKS", "3")
    else:
        monkeypatch.setenv("ABFT_CHOL", "recursive")
    return request.param


@pytest.mark.parametrize("nb", [29, 64, 96, 128, 192, 512, 1024])
def test_chol_inv_matches_oracle(P, nb, chol_path):
    A = syn.spd_matrix(nb, seed=nb + 7)
    st, L, Li = run_block(P, A)
    assert st == 0
    ref = oracle.potrf(A, nb, abft=False)
    assert ref.status == 0
    s = np.sqrt(np.diag(A))[:, None]
    Lr = np.tril(ref.L)
    err = np.max(np.abs(np.tril(L) - Lr) / np.maximum(np.abs(Lr), 1e-3 * s))
    assert err <= 1e-11, err
    # strict upper of A untouched
    assert np.array_equal(np.triu(L, 1), np.triu(A, 1))
    # inverse: lower with zero upper, L inv(L) = I
    assert np.all(np.triu(Li, 1) == 0.0)
    resid = np.max(np.abs(np.tril(L) @ Li - np.eye(nb)))
    assert resid <= 64 * nb * EPS, resid


@pytest.mark.parametrize("bad", [0, 63, 64, 200, 511])
def test_chol_inv_not_spd_info(P, bad, chol_path):
    """A leading minor of order bad+1 that is not positive: LAPACK info = bad + 1."""
    import torch
    nb = 512
    A = syn.spd_matrix(nb, seed=11)
    A[bad, bad] = -1.0
    st, _, _ = run_block(P, A)
    assert st == 2
    ref = oracle.potrf(A, nb, abft=False)
    assert ref.status == 2
    At = P.colmajor(A)
    st2, rep = P.abft_potrf_ex(nb, nb, At, opt=P.options(abft_enabled=False))
    torch.cuda.synchronize()
    assert st2 == 2 and rep["info"] == ref.info == bad + 1
