"""NEXT-4: several right-hand sides of one system solved together
(spcg_solve_multi).

Each right-hand side is an independent run of Algorithm 1, so each is
checked against the oracle's PCG on its own b exactly as a single solve is (SURVEY
§8(c.4)): |k - k_oracle| <= 1 to eps, x element-wise within 1e-8 ||x_oracle||_inf
at forced k.  Also: a right-hand side that converges early is frozen (its k and x
are those of its own stopping test) while the others continue; nrhs = 3 (a padded
group) and nrhs = 6 (two groups); b = 0 stops at k = 0; layouts the multi-RHS kernel
does not cover are refused with SPCG_ERR_INVALID_ARG.
"""
import numpy as np
import pytest

import gen
import oracle
import paper_conf_sc_maacsh25_b200 as lib
from parity_util import check_x_elementwise

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _rhs_block(A, seeds):
    return np.stack([gen.rhs(A, seed=s)[0] for s in seeds])


@pytest.mark.parametrize("params,nrhs", [((150, 67, 4), 2), ((256, 192, 4), 4), ((150, 67, 4), 3),
                                         ((200, 130, 4), 6)])
def test_multi_rhs_matches_oracle_per_rhs(params, nrhs):
    A = gen.make("aniso_layered", *params)
    h = lib.SPCG(A, mode="alg2", K=0, sptrsv="wchain")
    L, U, _ = oracle.setup(A, mode="alg2", K=0)
    Bh = _rhs_block(A, range(99, 99 + nrhs))
    B = torch.from_numpy(Bh).cuda()
    X, infos = h.solve_multi(B, eps=1e-8, kmax=20000)
    refs = [oracle.pcg(A, L, U, Bh[j], 1e-8, 20000) for j in range(nrhs)]
    for j in range(nrhs):
        assert infos[j]["status"] == 0, (j, infos[j])
        assert abs(infos[j]["iterations"] - refs[j]["k"]) <= 1, (j, infos[j], refs[j]["k"])
    # forced k: every right-hand side runs exactly k iterations
    k = max(r["k"] for r in refs)
    Xf, inf_f = h.solve_multi(B, eps=0.0, kmax=k)
    Xf = Xf.cpu().numpy()
    for j in range(nrhs):
        assert inf_f[j]["iterations"] == k
        rf = oracle.pcg(A, L, U, Bh[j], 0.0, k)
        check_x_elementwise(Xf[j], rf["x"])
    h.close()


def test_multi_rhs_freezes_converged_and_zero_rhs():
    A = gen.make("aniso_layered", 150, 67, 4)
    h = lib.SPCG(A, mode="alg2", K=0, sptrsv="wchain")
    L, U, _ = oracle.setup(A, mode="alg2", K=0)
    b0 = gen.rhs(A, seed=99)[0]
    Bh = np.stack([b0, np.zeros(A.n), 1e-6 * b0])       # b = 0 stops at k = 0; a scaled b stops earlier
    X, infos = h.solve_multi(torch.from_numpy(Bh).cuda(), eps=1e-8, kmax=20000)
    X = X.cpu().numpy()
    assert infos[1]["iterations"] == 0 and np.all(X[1] == 0.0)
    for j in (0, 2):
        ro = oracle.pcg(A, L, U, Bh[j], 1e-8, 20000)
        assert abs(infos[j]["iterations"] - ro["k"]) <= 1
        assert np.abs(X[j] - ro["x"]).max() <= 1e-6 * np.abs(ro["x"]).max() + 1e-14
    assert infos[2]["iterations"] < infos[0]["iterations"]
    h.close()


def test_multi_rhs_refuses_other_layouts():
    A = gen.make("poisson3d", 13, 11, 9)
    h = lib.SPCG(A, mode="alg2", K=0, sptrsv="chunked")
    B = torch.from_numpy(_rhs_block(A, (99, 100))).cuda()
    with pytest.raises(lib.SpcgError) as e:
        h.solve_multi(B)
    assert e.value.status == lib.ERR_INVALID_ARG
    h.close()
