"""NEXT-3, the analytic wasted-GPU-time model (§5, eqs. 1-8).

The oracle (oracle/model.py, the equations written out) is pinned by the
values the paper prints in Table 8, eq. 9 and eq. 10, and
by the calculus the paper states (dW/dc = 0 at c*, W convex).  The library's
jitc_waste_model is then checked against the oracle."""
import json
import math
import os

import pytest

from oracle import model as M

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "table8.json")))
F = 2 / (992 * 86400)   # 2 failures per day on 992 GPUs


def _close(got, printed, rel, digits):
    """Within rel of the printed value, or within one unit of its last printed
    digit: Table 8 truncates rather than rounds some entries (e.g. BERT-L-PT
    c* at N=4 is 0.347/hr, printed 0.34; GPT2-8B 0.179, printed 0.17, while its
    own N=1024 entry 2.85 = 16 x 0.178)."""
    return abs(got - printed) <= max(rel * abs(printed), 10 ** (-digits))


def _digits(x):
    s = repr(x)
    return len(s.split(".")[1]) if "." in s else 0


@pytest.mark.parametrize("model", list(GOLD["periodic"]))
def test_periodic_rows_of_table8(model):
    inp = GOLD["inputs"][model]
    for N, (c_hr, wf_pct) in GOLD["periodic"][model].items():
        N = int(N)
        # The paper prints 2-3 significant digits and does not state f beyond
        # "2 failures per day on 992 GPUs"; beyond truncation its N=8192 rows
        # drift up to ~3% from the closed form (most rows are within 1%).
        rel = 0.035
        cs = M.c_star(N, F, inp["o"]) * 3600
        wf = 100 * M.waste_fraction(M.w_star(N, F, inp["o"], inp["r"]))
        assert _close(cs, c_hr, rel, _digits(c_hr)), (model, N, cs, c_hr)
        assert _close(wf, wf_pct, rel, _digits(wf_pct)), (model, N, wf, wf_pct)


@pytest.mark.parametrize("model", list(GOLD["user_jit_wf_percent"]))
def test_user_jit_rows_of_table8(model):
    inp = GOLD["inputs"][model]
    for N, wf_pct in GOLD["user_jit_wf_percent"][model].items():
        N = int(N)
        w = M.w_user_jit(N, F, inp["o"], inp["r"], inp["m"], inp["o_jit"])
        got = 100 * M.waste_fraction(w)
        assert _close(got, wf_pct, 0.04 if N == 8192 else 0.02, _digits(wf_pct)), (model, N, got, wf_pct)


def test_eq9_and_eq10_bert_l_pt():
    """eq. 9: c* ~ sqrt(N)/6 per hour for o = 5 s; eq. 10: w* = 4.8e-4 sqrt(N)
    + 2.3e-7 N with the paper's f = 2e-3 per GPU per day, r = 9.9 s."""
    f_day = 2e-3 / 86400
    for N in (4, 64, 1024, 8192):
        # the paper writes "≈ sqrt(N)/6 hr": the exact factor is 0.173
        assert abs(M.c_star(N, f_day, 5.0) * 3600 - math.sqrt(N) / 6) / (math.sqrt(N) / 6) < 0.05
        a, b = GOLD["eq10_coefficients_BERT-L-PT"]
        w = M.w_star(N, f_day, 5.0, 9.9)
        assert abs(w - (a * math.sqrt(N) + b * N)) / w < 0.02


def test_c_star_minimises_eq1():
    """dW/dc = 0 at c* (eq. 2) and W is convex (d2W/dc2 > 0): W(c*) is below
    W at nearby frequencies, and W(c*) equals w* (eq. 4/5)."""
    for (N, o, r) in [(4, 5.0, 9.9), (1024, 18.8, 28.6), (8192, 1.4, 8.8)]:
        cs = M.c_star(N, F, o)
        w0 = M.waste_periodic(N, F, o, r, cs)
        assert abs(w0 - M.w_star(N, F, o, r)) <= 1e-12 * max(1, w0)
        for k in (0.5, 0.9, 1.1, 2.0):
            assert M.waste_periodic(N, F, o, r, k * cs) > w0


def test_transparent_jit_is_flat_in_N_for_small_m():
    """eq. 8: only N f m / 2 grows with N; with m < 1 s it stays below the
    periodic fraction at large N (the paper's conclusion)."""
    for m in (0.08, 0.3):
        w4, w8k = M.w_transparent_jit(4, F, m, 0.0069), M.w_transparent_jit(8192, F, m, 0.0069)
        assert w8k - w4 < 1e-4
        assert M.waste_fraction(w8k) < M.waste_fraction(M.w_star(8192, F, 5.0, 9.9))


def test_library_matches_oracle():
    from paper_conf_eurosys_guptakkvgkrs24_b200 import build, jitc as J
    build.build()
    cases = [(N, o, r, m, oj) for N in (1, 4, 1024, 8192) for (o, r, m, oj) in
             [(5.0, 9.9, 0.418, 0.0076), (18.8, 28.6, 2.953, 0.0), (0.3, 0.55, 1.0, 0.0)]]
    for N, o, r, m, oj in cases:
        got = J.waste_model(J.MODEL_PERIODIC_OPTIMAL, N, F, o, r)
        assert math.isclose(got["c_opt"], M.c_star(N, F, o), rel_tol=1e-12)
        assert math.isclose(got["w"], M.w_star(N, F, o, r), rel_tol=1e-12)
        assert math.isclose(got["w_f"], M.waste_fraction(M.w_star(N, F, o, r)), rel_tol=1e-12)
        c = 3 * M.c_star(N, F, o)
        assert math.isclose(J.waste_model(J.MODEL_PERIODIC, N, F, o, r, c=c)["w"],
                            M.waste_periodic(N, F, o, r, c), rel_tol=1e-12)
        assert math.isclose(J.waste_model(J.MODEL_USER_JIT, N, F, o, r, m, oj)["w"],
                            M.w_user_jit(N, F, o, r, m, oj), rel_tol=1e-12)
        assert math.isclose(J.waste_model(J.MODEL_TRANSPARENT_JIT, N, F, m=m, o_jit=oj)["w"],
                            M.w_transparent_jit(N, F, m, oj), rel_tol=1e-12)
    with pytest.raises(J.JitcError):
        J.waste_model(J.MODEL_PERIODIC, 4, F, 5.0, 9.9, c=0.0)
