"""NEXT row f1 on the GPU: the paper-literal MadPipe-DP and Algorithm 1
 through the C ABI, bit-exact against the oracle."""
import math

import numpy as np
import pytest

import chaingen
import oracle
import paper_conf_ipps_beaumontes22_b200 as mp

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    c = mp.Context(0)
    yield c
    c.close()


def _cases(n, seed):
    rng = np.random.default_rng(seed)
    for _ in range(n):
        L = int(rng.integers(1, 10))
        P = int(rng.integers(1, 5))
        ch = chaingen.tiny(rng, L)
        M = int((3 * ch["W"].sum() + 3 * ch["a"].sum()) * rng.uniform(0.2, 0.9)) + 1
        beta = float(rng.choice([math.inf, rng.uniform(5.0, 60.0)]))
        yield ch, P, M, beta, int(rng.choice([2, 4, 11])), int(rng.choice([4, 16, 51])), int(rng.choice([5, 21, 101]))


def test_literal_tables(ctx):
    rng = np.random.default_rng(1)
    for ch, P, M, beta, n_m, n_v, n_t in _cases(25, 71):
        pre = oracle.prep(ch, P, beta)
        That = pre["lb"] + rng.uniform(0, 1) * (pre["ub"] - pre["lb"])
        A, ARG = ctx.literal_table(ch, P, M, beta, n_m, n_v, n_t, That)
        A_ref, ARG_ref = oracle.literal_table(ch, P, M, beta, n_m, n_v, n_t, That)
        assert np.array_equal(A, A_ref)
        assert np.array_equal(ARG, ARG_ref)


def test_algorithm1(ctx):
    for ch, P, M, beta, n_m, n_v, n_t in _cases(25, 72):
        got = ctx.solve_paper(ch, P, M, beta, n_m, n_v, n_t, K=10)
        ref = oracle.literal_solve(ch, P, M, beta, n_m, n_v, n_t, K=10)
        assert np.array_equal(got["T"], ref["T"]) and np.array_equal(got["That"], ref["That"])
        assert got["rc"] == ref["rc"]
        if ref["rc"] == 0:
            assert got["period"] == ref["period"] and got["best_iter"] == ref["best_iter"]
            assert got["stages"] == ref["stages"]


def test_algorithm1_paper_discretisation_resnet(ctx):
    """The paper's own setting: ResNet-50-shaped chain, 11 x 51 x 21 levels (t_P reduced
    from 101 to keep the oracle within seconds), K = 10."""
    ch = chaingen.resnet50()
    ch = {k: (v[:31] if k == "a" else v[:30]) if k != "name" else v for k, v in ch.items()}
    args = (4, 6 * 10**9, 12e9, 11, 51, 21)
    got = ctx.solve_paper(ch, *args, K=10)
    ref = oracle.literal_solve(ch, *args, K=10)
    assert np.array_equal(got["T"], ref["T"]) and got["stages"] == ref["stages"]
    assert got["period"] == ref["period"]
