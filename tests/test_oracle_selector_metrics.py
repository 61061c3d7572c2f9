"""Pins for oracle/selector.py and oracle/metrics.py (CPU only).

Tab I is compared against the printed table (tests/golden/table1_policy.txt);
the classifier with the Q9 thresholds must reproduce every Tab II label; and
Tab I + Tab II must reproduce the paper's statement of which pairs it co-ran
("Slate concurrently runs RG with all the other kernels ... For all
pairings for which Slate gains less than 10%, Slate runs the kernels
consecutively").
"""
import itertools
import os

import pytest

from oracle import metrics as M
from oracle import selector as S

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _rows(name):
    return [l.split() for l in open(os.path.join(GOLDEN, name)) if l.strip() and not l.startswith("#")]


def test_table1_literal_matches_print():
    rows = _rows("table1_policy.txt")
    header = rows[0][1:]
    for r in rows[1:]:
        for c, v in zip(header, r[1:]):
            assert S.TABLE1_LITERAL[(r[0], c)] == v


def test_table1_symmetric_reading():
    for a, b in itertools.product(S.CATEGORIES, repeat=2):
        assert S.TABLE1[(a, b)] == S.TABLE1[(b, a)]
    # the two cells the print has asymmetric (Q8) follow the H_C row
    assert S.TABLE1[("M_M", "H_C")] == "solo" and S.TABLE1[("H_M", "H_C")] == "corun"
    diff = [k for k in S.TABLE1 if S.TABLE1[k] != S.TABLE1_LITERAL[k]]
    assert sorted(diff) == [("H_M", "H_C"), ("M_M", "H_C")]


def _labels():
    rows = _rows("table2_profiles.txt")
    peak = [r for r in rows if r[0] == "peak"][0]
    pk_bw, pk_fl = float(peak[1]), float(peak[2])
    out = {}
    for r in rows:
        if r[0] == "peak":
            continue
        c, m, cat = S.classify(float(r[4]), float(r[3]), 0.0, pk_bw, pk_fl, 0.0)
        out[r[0]] = (c, m, cat, r[1][0], r[2][0])
    return out


def test_classifier_reproduces_table2():
    for name, (c, m, cat, c_paper, m_paper) in _labels().items():
        assert (c, m) == (c_paper, m_paper), name
    cats = {k: v[2] for k, v in _labels().items()}
    assert cats == {"BS": "M_M", "GS": "M_M", "MM": "M_M", "RG": "L_C", "TR": "H_M"}


@pytest.mark.parametrize("literal", [False, True])
def test_pairings_reproduce_section_VE(literal):
    cats = {k: v[2] for k, v in _labels().items()}
    corun = set()
    for a, b in itertools.combinations_with_replacement(sorted(cats), 2):
        if S.policy(cats[a], cats[b], literal) == "corun":
            corun.add(frozenset((a, b)))
    assert corun == {frozenset(p) for p in [("RG",), ("RG", "BS"), ("RG", "GS"), ("RG", "MM"), ("RG", "TR")]}
    assert len(list(itertools.combinations_with_replacement(cats, 2))) == 15


def test_select_algorithm():
    # next kernel first, then the rest of the queue, else solo
    assert S.select("H_C", ["H_M", "L_C"]) == 0
    assert S.select("H_C", ["M_M", "H_M"]) == 1
    assert S.select("H_C", ["M_M", "H_C"]) is None
    assert S.select("M_M", []) is None
    # a head bypassed too often blocks look-ahead (Q13)
    assert S.select("H_C", ["M_M", "H_M"], bypassed=[4, 0]) is None


def test_split_fluid_model():
    # A compute tenant scales linearly; B saturates memory at 1/4 of the SMs
    n = 148
    curve_a = {s: 148.0 / s for s in (18, 37, 74, 111, 148)}
    curve_b = {s: max(1.0, 37.0 / s) for s in (18, 37, 74, 111, 148)}
    s, t = S.choose_split(curve_a, curve_b, n)
    assert 30 <= s <= 44
    assert t < 2.0                          # solo sum is 2.0
    # no gain possible when both scale linearly: best makespan equals the solo sum
    lin = {k: 148.0 / k for k in (37, 74, 148)}
    _, t2 = S.choose_split(lin, lin, n)
    assert abs(t2 - 2.0) < 1e-9
    assert S.interp_time(curve_a, 148) == 1.0 and S.interp_time(curve_a, 200) == 1.0


def test_turnaround_split_reading_q41():
    """The ANTT objective against closed forms.  Linear curves T_i(s) = W_i n / s
    are work-conserving: every split has makespan W_A + W_B, so all are feasible,
    A's completion is W_A + W_B whatever s, and B's is W_B n / s while B runs
    first -- ANTT falls as B (the shorter job) gets more SMs: the objective gives
    it all but one step, the textbook shortest-job-first limit."""
    n = 148
    wa, wb = 3.0, 1.0
    lin_a = {k: wa * n / k for k in (37, 74, 148)}
    lin_b = {k: wb * n / k for k in (37, 74, 148)}
    s, t = S.choose_split(lin_a, lin_b, n, objective="antt")
    assert s == n - 2 and abs(t - (wa + wb)) < 1e-9
    ta, tb = S.corun_times(lin_a, lin_b, n, s)
    assert abs(ta - (wa + wb)) < 1e-9 and abs(tb - wb * n / (n - 2)) < 1e-9
    assert abs(S.corun_antt(lin_a, lin_b, n, s) - 0.5 * ((wa + wb) / wa + n / (n - 2))) < 1e-12
    # swapped roles: the shorter job is A, so B gets the least
    s2, _ = S.choose_split(lin_b, lin_a, n, objective="antt")
    assert s2 == 2
    # a memory job B saturating at 37 SMs beside a linear compute job A: every
    # s >= 37 finishes B at its solo time and A then loses time with every SM
    # more, so the turnaround objective stops at the knee rounded up to the
    # step (38); the makespan objective gives B fewer (30: B finishes later,
    # A earlier, the two ends closer together)
    curve_a = {k: n / k for k in (18, 37, 74, 111, 148)}
    curve_b = {k: max(1.0, 37.0 / k) for k in (18, 37, 74, 111, 148)}
    s_m, t_m = S.choose_split(curve_a, curve_b, n)
    s_a, t_a = S.choose_split(curve_a, curve_b, n, objective="antt", slack=0.5)
    assert s_m == 30 and abs(t_m - 1.25) < 1e-12
    assert s_a == 38 and S.corun_times(curve_a, curve_b, n, 38)[1] == 1.0
    assert S.corun_antt(curve_a, curve_b, n, 38) < S.corun_antt(curve_a, curve_b, n, 30)
    # the slack bounds the makespan given up for turnaround
    for slack in (0.0, 0.02, 0.1):
        _, tt = S.choose_split(curve_a, curve_b, n, objective="antt", slack=slack)
        assert tt <= t_m * (1 + slack) + 1e-12
    _, t0 = S.choose_split(curve_a, curve_b, n, objective="antt", slack=0.0)
    assert abs(t0 - t_m) < 1e-12


def test_saturation_cap_reading_q29():
    # throughput linear between (37, 1/2T) and (74, 1/T): rate(s) = s / (74 T) there,
    # so rate >= 0.9 / T first holds at s = ceil(0.9 * 74) = 67
    curve = {148: 1.0, 74: 1.0, 37: 2.0}
    assert S.saturation_sms(curve, 148, 0.9) == 67
    assert S.saturation_sms(curve, 148, 1.0) == 74
    # a linearly scaling kernel needs 90% of the chip for 90% of its rate
    lin = {k: 148.0 / k for k in (37, 74, 148)}
    assert S.saturation_sms(lin, 148, 0.9) == 134          # ceil(0.9 * 148)
    # bounds restrict the split; an empty window falls back to the nearest bound
    curve_a = {s: 148.0 / s for s in (18, 37, 74, 111, 148)}
    curve_b = {s: max(1.0, 74.0 / s) for s in (18, 37, 74, 111, 148)}
    s_free, _ = S.choose_split(curve_a, curve_b, 148)
    s_cap, t_cap = S.choose_split(curve_a, curve_b, 148, hi_b=40)
    assert s_free > 40 and s_cap == 40
    assert abs(t_cap - S.corun_makespan(curve_a, curve_b, 148, 40)) < 1e-12
    s_lo, _ = S.choose_split(curve_a, curve_b, 148, lo_b=100)
    assert s_lo >= 100 and s_lo % 2 == 0
    assert S.choose_split(curve_a, curve_b, 148, lo_b=147)[0] == 146
    assert S.choose_split(curve_a, curve_b, 148, hi_b=1)[0] == 2


def test_metrics_closed_forms():
    # P10: perfect overlap of equal jobs, no slowdown -> G = 2, STP = 2, ANTT = 1
    assert M.gain([1, 1], [1, 1]) == 2.0
    assert M.stp([1, 1], [1, 1]) == 2.0 and M.antt([1, 1], [1, 1]) == 1.0
    # fully serialised "co-run" -> G = 1, not complementary (P:L99 needs T' < T)
    assert M.gain([1, 1], [1, 2]) == 1.0 and not M.complementary([1, 1], [1, 2])
    # sequential schedule of equal jobs: turnarounds 1, 2 -> STP 1.5, ANTT 1.5
    ta = M.sequential_turnarounds([1, 1])
    assert ta == [1, 2] and M.stp([1, 1], ta) == 1.5 and M.antt([1, 1], ta) == 1.5
    assert M.utilisation(6.5e12, 1.0, 6.5e12) == 1.0
    # STP <= n for any schedule without super-linear speed-up
    assert M.stp([2, 3, 5], [2, 3, 5]) == 3.0


def test_fluid_corun_reading_q31():
    n = 148
    pts = (18, 37, 74, 111, 148)
    # both tenants scale linearly: no split beats running them back to back
    lin = {k: 148.0 / k for k in pts}
    ok, _, g = S.fluid_corun(lin, 1, lin, 1, n)
    assert not ok and abs(g - 1.0) < 1e-9
    # A scales linearly (1 ms on the chip), B saturates at 37 SMs (1 ms):
    # by hand at s = 38, B ends at 1 ms while A ran at 110/148 of its rate, A's
    # remaining 1 - 110/148 ends 38/148 ms later: makespan 1.2568 (the chooser
    # may only do better), against 2 ms back to back
    sat = {k: max(1.0, 37.0 / k) for k in pts}
    ok, s, g = S.fluid_corun(lin, 1, sat, 1, n)
    assert ok and g >= 2.0 / (1.0 + 38.0 / 148) - 1e-9 and 30 <= s <= 48
    # the same pair with B's job 100x shorter: nothing worth a co-run
    ok, _, g = S.fluid_corun(lin, 1, sat, 0.01, n)
    assert not ok and g < 1.05
    # work scales the jobs: 10 launches of A against 10 of B is the 1-vs-1 decision
    assert S.fluid_corun(lin, 10, sat, 10, n)[1:] == pytest.approx(S.fluid_corun(lin, 1, sat, 1, n)[1:])


# ------------------------------------------------------------------ k-way split (NEXT-4)
def test_k_way_makespan_closed_forms():
    n = 48
    lin = {s: 48.0 / s for s in (6, 12, 24, 48)}          # perfectly linear: T(s) = 48 / s, T(n) = 1
    # work conservation: with linear curves and SMs handed on, any split of k jobs
    # finishes at the sum of their full-chip times
    for shares in ([24, 24], [6, 42], [12, 12, 24], [6, 18, 12, 12]):
        assert abs(S.corun_makespan_k([lin] * len(shares), shares) - len(shares)) < 1e-9
    # two co-runners: the k-way model is the 2-way one (pinned separately)
    a = {148: 1.0, 74: 1.3, 37: 2.4}
    b = {148: 2.0, 74: 2.1, 37: 2.9}
    for s in (20, 74, 100):
        assert abs(S.corun_makespan_k([a, b], [148 - s, s]) - S.corun_makespan(a, b, 148, s)) < 1e-9
    s2, t2 = S.choose_split(a, b, 148)
    sk, tk = S.choose_split_k([a, b], 148)
    assert sk == [148 - s2, s2] and abs(tk - t2) < 1e-9


def test_k_way_saturating_jobs_overlap_fully():
    # three jobs that each reach full speed on a third of the chip run side by side
    n = 48
    sat = {16: 1.0, 48: 1.0}                              # T(s) = 1 for s >= 16 (and s/16 below)
    shares, t = S.choose_split_k([sat, sat, sat], n, step=4)
    assert shares == [16, 16, 16] and abs(t - 1.0) < 1e-9
    assert S.corun_makespan_k([sat] * 3, [8, 20, 20]) > 1.0 + 1e-9


def test_kway_admission_reading_q49():
    """Closed forms on linear and saturating curves.  Work-conserving (linear)
    compute jobs gain nothing from joining: whatever the shares, the chip does
    the same total work (gain exactly 1), and a linear job joining a pair that
    already gives its compute partner every SM past the memory job's knee gains
    nothing either.  A small-grid compute job that saturates at 30 SMs joins a
    (linear compute, memory) pair: the pair alone ends at 1.257 and C after it
    at 1.757; joined on shares (80, 38, 30), by hand: A progresses on 80 SMs
    until C ends (0.5), on 110 until B ends (1.0), then on all 148, so the
    makespan is 1 + (148 - 80*0.5 - 110*0.5)/148 = 1.358 -- the best shares do
    a little better, gain 1.3.  A second memory job never joins (Q37)."""
    n = 148
    lin = lambda w: {k: w * n / k for k in (18, 30, 37, 74, 110, 111, 148)}
    sat = lambda w, knee: {k: w * max(1.0, knee / k) for k in (18, 30, 37, 74, 111, 148)}
    ok, shares, g = S.kway_admit([lin(1.0), lin(1.0), lin(1.0)], [2, 2, 2], [74, 74], n, 2)
    assert not ok and abs(g - 1.0) < 1e-9 and sum(shares) == n
    ok, _, g = S.kway_admit([lin(1.0), sat(1.0, 37), lin(1.0)], [2, 4, 2], [110, 38], n, 2)
    assert not ok and g < 1.01
    assert abs(S.corun_makespan_k([lin(1.0), sat(1.0, 37), sat(0.5, 30)], [80, 38, 30]) - 1.358108) < 1e-5
    ok, shares, g = S.kway_admit([lin(1.0), sat(1.0, 37), sat(0.5, 30)], [2, 4, 2], [110, 38], n, 2)
    assert ok and g >= 1.29 and sum(shares) == n and all(x % 2 == 0 and x >= 2 for x in shares)
    ok, _, _ = S.kway_admit([lin(1.0), sat(1.0, 37), sat(1.0, 37)], [2, 4, 3], [110, 38], n, 2)
    assert not ok
