"""NEXT-3: the ratio-sweep / paper-Oracle study (tools/ratio_sweep.py).

CPU: the statistics are pinned against independent definitions — Spearman against
scipy.stats.spearmanr (tie-free data), the paper's "Oracle" (the best
fixed ratio by exhaustive search) against hand-built cases, the Fig. 7 match count.
GPU: the sweep on small matrices through the C ABI; every run's iteration count is
within +-1 of the oracle's PCG on the oracle's own setup, and the
chosen t of Algorithm 2 is the oracle's.
"""
import os
import sys

import numpy as np
import pytest

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
import ratio_sweep as rs  # noqa: E402


def _run(ms, k, levels, status=0, pct=0.0):
    return {"ms": ms, "k": k, "ms_per_iter": ms / k, "levels": levels, "status": status, "chosen_pct": pct}


def test_spearman_matches_scipy():
    stats = pytest.importorskip("scipy.stats")
    rng = np.random.default_rng(3)
    for _ in range(20):
        a = rng.standard_normal(17)
        b = a * rng.uniform(-1, 2) + rng.standard_normal(17)
        assert abs(rs.spearman(a, b) - stats.spearmanr(a, b).statistic) < 1e-12
    assert rs.spearman([1, 2, 3], [3, 2, 1]) == pytest.approx(-1.0)
    assert rs.spearman([1, 1, 1], [1, 2, 3]) is None or abs(rs.spearman([1, 1, 1], [1, 2, 3])) <= 1.0


def test_paper_oracle_picks_fastest_converged():
    res = {"t1": _run(10.0, 10, 50), "t5": _run(8.0, 12, 40), "t10": _run(5.0, 20, 30, status=1)}
    assert rs.paper_oracle(res) == "t5"                 # t10 did not converge
    res["t10"]["status"] = 0
    assert rs.paper_oracle(res) == "t10"
    tie = {"t1": _run(5.0, 10, 50), "t5": _run(5.0, 10, 40), "t10": _run(6.0, 10, 30)}
    assert rs.paper_oracle(tie) == "t1"                 # ties -> the smaller ratio
    assert rs.paper_oracle({"t1": _run(1.0, 1, 1, status=-4)}) is None


def test_summarize_counts_and_correlation():
    rows = []
    for lv_pcg, (l1, l5, l10), alg2 in [(100, (99, 90, 60), 10.0), (200, (199, 150, 120), 5.0),
                                        (50, (50, 49, 48), 1.0)]:
        res = {"pcg": _run(10.0, 10, lv_pcg), "alg2": _run(5.0, 10, l5, pct=alg2)}
        # per-iteration time proportional to the levels: speedup is monotone in the reduction
        for t, lv in zip(rs.FIXED, (l1, l5, l10)):
            res[t] = _run(10.0 * lv / lv_pcg, 10, lv)
        rows.append(rs.row_of("m", 0, 1, res))
    s = rs.summarize(rows)
    assert s["points"] == 9 and s["matrices"] == 3
    assert s["spearman_wavefront_reduction_vs_per_iter_speedup"] == pytest.approx(1.0)
    # the oracle is the fewest-levels ratio here (t10 everywhere): alg2 matches on row 0 only
    assert [r["oracle_pct"] for r in rows] == [10.0, 10.0, 10.0]
    assert s["alg2_matches_oracle"] == 1


@pytest.mark.gpu
def test_sweep_runs_match_oracle_iterations():
    pytest.importorskip("torch")
    import gen
    import oracle
    rows = rs.run_sweep(rs.SMALL, reps=1)
    for (fam, params, K), row in zip(rs.SMALL, rows):
        A = gen.make(fam, *params)
        b, _ = gen.rhs(A)
        for tag, kw in rs.RUNS:
            mode = kw["mode"]
            L, U, info = oracle.setup(A, mode=mode, K=K, fixed_pct=kw.get("fixed_pct", 0.0))
            ro = oracle.pcg(A, L, U, b, 1e-8, 20000)
            run = row["runs"][tag]
            assert run["status"] == 0
            assert abs(run["k"] - ro["k"]) <= 1, (fam, tag, run["k"], ro["k"])
            if mode == "alg2":
                assert run["chosen_pct"] == info["chosen_pct"]
    s = rs.summarize(rows)
    assert s["matrices"] == len(rs.SMALL)
