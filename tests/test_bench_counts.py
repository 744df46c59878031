"""The roofline numerators bench.py reports are the algorithm's actual work.

bench.stage_rooflines restates the paper's §5.1 operation counts. Here they are
checked against an independent count: the multiply-adds the CPU oracle's own Algorithm-1
contractions perform (every np.einsum inside oracle.fmm_stages, counted from its operand shapes
and attributed to the Algorithm-1 stage the oracle logs next). One complex-data x real-operator
multiply-add is 2C = 4 real flops (C = 2).
"""
import math

import numpy as np
import pytest

import bench
import synth_inputs as SI
from oracle import fmmfft_oracle as O


def einsum_macs(subscripts, *ops):
    lhs = subscripts.split("->")[0].split(",")
    size = {}
    for term, a in zip(lhs, ops):
        for c, n in zip(term, a.shape):
            size[c] = n
    return math.prod(size.values())


@pytest.mark.parametrize("N,P,B,Q,M_L", [(1 << 12, 16, 2, 16, 16), (1 << 13, 8, 3, 8, 16), (1 << 12, 4, 2, 4, 32)])
def test_stage_flops_match_oracle_contractions(monkeypatch, N, P, B, Q, M_L):
    calls = []
    real = np.einsum

    def counting(subscripts, *ops, **kw):
        calls.append((subscripts, einsum_macs(subscripts, *ops)))
        return real(subscripts, *ops, **kw)

    per_stage = {}

    class Log(O.StageLog):
        def __call__(self, name, level=None):
            per_stage[name] = per_stage.get(name, 0) + sum(m for _, m in calls)
            calls.clear()
            super().__call__(name, level)

    monkeypatch.setattr(O.np, "einsum", counting)
    L = O.tree_levels(N, P, M_L)
    S = SI.complex_uniform(0, N).reshape(2 ** L, M_L, P)
    O.fmm_stages(S, N, P, B, Q, Log())
    C = 2
    fl = {k: 2 * C * v for k, v in per_stage.items()}
    # S2T's einsum runs over all P slots; p = 0 is the identity (reading R1), not FMM work
    fl["S2T"] = fl["S2T"] * (P - 1) / P
    r = bench.stage_rooflines(N, P, B, Q, M_L, 1, L, "c64", False, False, "k")
    assert r["s2m"][1] == fl["S2M"]
    assert r["s2t"][1] == pytest.approx(fl["S2T"])
    assert r["m2m"][1] == fl["M2M"]
    # M2L over levels B+1..L plus L2L (the fused "down" stage), and M2L-B (the "top" stage)
    m2l_levels = 2 * C * sum(3 * Q * Q * 2 ** lev * (P - 1) for lev in range(B + 1, L + 1))
    m2l_base = 2 * C * (2 ** B - 3) * 2 ** B * Q * Q * (P - 1)
    assert fl["M2L"] == m2l_levels + m2l_base
    assert r["top"][1] == m2l_base
    assert r["down"][1] == m2l_levels + fl["L2L"]
    fused = bench.stage_rooflines(N, P, B, Q, M_L, 1, L, "c64", True, False, "k")
    assert fused["top"][1] == fl["M2M"] + fl["M2L"] + fl["L2L"]
    # wide tree with the cluster top (levels B..top_L in k_tree_pc): the three stages partition the work
    for top_L in range(B + 1, L + 1):
        h = bench.stage_rooflines(N, P, B, Q, M_L, 1, L, "c64", False, False, "k", top_L=top_L)
        assert h["m2m"][1] + h["top"][1] + h["down"][1] == pytest.approx(fl["M2M"] + fl["M2L"] + fl["L2L"])
        f = bench.stage_rooflines(N, P, B, Q, M_L, 1, L, "c64", False, False, "k", top_L=top_L, s2m_m2m=True)
        assert f["s2m"][1] + f["m2m"][1] + f["top"][1] + f["down"][1] == pytest.approx(
            fl["S2M"] + fl["M2M"] + fl["M2L"] + fl["L2L"])
