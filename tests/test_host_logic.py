"""CPU-only checks of the C-ABI library: it loads without a GPU, exports every
symbol include/slate.h declares, refuses to run without a GPU (no CPU
fallback), and its host-side selector logic agrees with the oracle."""
import itertools
import os
import random
import re

import pytest

from oracle import selector as OS

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def S():
    from paper_conf_ipps_allenf019_b200 import build
    build.build()
    from paper_conf_ipps_allenf019_b200 import slate
    return slate


def _declared():
    txt = open(os.path.join(ROOT, "include", "slate.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(slate_[a-z_0-9]+)\s*\(", txt)))


def test_exports_every_declared_symbol(S):
    import ctypes
    lib = ctypes.CDLL(S.LIB_PATH)
    names = _declared()
    assert len(names) >= 17
    for n in names:
        assert hasattr(lib, n), n
    assert sorted(S.EXPORTED) == names


def test_no_cpu_fallback(S):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(S.SlateError) as e:
        S.Session(None, 0)
    assert e.value.status == S.ECUDA
    assert S.status_string(S.ECUDA) == "SLATE_ECUDA"


def test_policy_matches_oracle(S):
    for a, b in itertools.product(OS.CATEGORIES, repeat=2):
        for lit in (False, True):
            assert S.policy(a, b, lit) == OS.policy(a, b, lit)


def test_classify_matches_oracle(S):
    fr = [0.0, 0.005, 0.0099, 0.01, 0.05, 0.0999, 0.1, 0.2, 0.2499, 0.25, 0.5, 0.8499, 0.85, 1.0, 1.2]
    for m, f, t in itertools.product(fr, fr, [0.0, 0.02, 0.5]):
        c, mm, cat = OS.classify(m, f, t, 1.0, 1.0, 1.0)
        assert S.classify(m, f, t) == (c, mm, cat)


def test_select_matches_oracle(S):
    rng = random.Random(5)
    for _ in range(2000):
        active = rng.choice(OS.CATEGORIES)
        q = [rng.choice(OS.CATEGORIES) for _ in range(rng.randrange(0, 6))]
        byp = [rng.randrange(0, 6) for _ in q]
        assert S.select(active, q) == OS.select(active, q)
        assert S.select(active, q, bypassed=byp) == OS.select(active, q, bypassed=byp)


def test_choose_split_matches_oracle(S):
    rng = random.Random(7)
    pts = [148, 111, 74, 49, 37, 18]
    for _ in range(200):
        knee_a, knee_b = rng.uniform(10, 148), rng.uniform(10, 148)
        ta, tb = rng.uniform(0.2, 5), rng.uniform(0.2, 5)
        ca = {s: ta * max(1.0, knee_a / s) for s in pts}
        cb = {s: tb * max(1.0, knee_b / s) for s in pts}
        s1, t1 = S.choose_split(ca, cb, 148)
        s2, t2 = OS.choose_split(ca, cb, 148)
        assert abs(t1 - t2) <= 1e-9 * t2
        assert s1 == s2 or abs(OS.corun_makespan(ca, cb, 148, s1) - t2) <= 1e-9 * t2


def test_choose_split_bounds_and_saturation_match_oracle(S):
    rng = random.Random(11)
    pts = [148, 111, 74, 49, 37, 18]
    for _ in range(200):
        knee_a, knee_b = rng.uniform(10, 148), rng.uniform(10, 148)
        ca = {s: rng.uniform(0.2, 5) * max(1.0, knee_a / s) for s in pts}
        cb = {s: rng.uniform(0.2, 5) * max(1.0, knee_b / s) for s in pts}
        for c in (ca, cb):
            frac = rng.choice([0.5, 0.8, 0.9, 1.0])
            assert S.saturation_sms(c, 148, frac) == OS.saturation_sms(c, 148, frac)
        lo = rng.choice([0, 0, rng.randrange(1, 148)])
        hi = rng.choice([0, 0, rng.randrange(1, 148)])
        s1, t1 = S.choose_split(ca, cb, 148, 2, lo, hi)
        s2, t2 = OS.choose_split(ca, cb, 148, 2, lo, hi)
        assert abs(t1 - t2) <= 1e-9 * t2
        assert s1 == s2 or abs(OS.corun_makespan(ca, cb, 148, s1) - t2) <= 1e-9 * t2


def test_turnaround_split_matches_oracle(S):
    """Reading Q41: slate_choose_split_obj(ANTT) == oracle choose_split(objective="antt")."""
    rng = random.Random(41)
    pts = [148, 111, 74, 49, 37, 18]
    for _ in range(300):
        knee_a, knee_b = rng.uniform(10, 148), rng.uniform(10, 148)
        ca = {s: rng.uniform(0.2, 5) * max(1.0, knee_a / s) for s in pts}
        cb = {s: rng.uniform(0.2, 5) * max(1.0, knee_b / s) for s in pts}
        slack = rng.choice([0.0, 0.02, 0.05, 0.2])
        lo = rng.choice([0, 0, rng.randrange(1, 148)])
        s1, t1, a1 = S.choose_split(ca, cb, 148, 2, lo, 0, objective="antt", slack=slack, with_antt=True)
        s2, t2 = OS.choose_split(ca, cb, 148, 2, lo, 0, objective="antt", slack=slack)
        a2 = OS.corun_antt(ca, cb, 148, s2)
        assert abs(a1 - a2) <= 1e-9 * a2 and abs(t1 - t2) <= 1e-9 * t2 or s1 == s2
        r1 = S.fluid_corun(ca, 7, cb, 13, 148, 2, lo, 0, objective="antt", slack=slack)
        r2 = OS.fluid_corun(ca, 7, cb, 13, 148, 2, lo, 0, objective="antt", slack=slack)
        assert abs(r1[2] - r2[2]) <= 1e-9 * r2[2]


def test_fluid_corun_matches_oracle(S):
    rng = random.Random(13)
    pts = [148, 111, 74, 49, 37, 18]
    for _ in range(200):
        knee_a, knee_b = rng.uniform(10, 148), rng.uniform(10, 148)
        ca = {s: rng.uniform(0.02, 0.5) * max(1.0, knee_a / s) for s in pts}
        cb = {s: rng.uniform(0.02, 0.5) * max(1.0, knee_b / s) for s in pts}
        wa, wb = rng.choice([1, 7, 64]), rng.choice([1, 13, 640])
        lo = rng.choice([0, 0, rng.randrange(1, 148)])
        hi = rng.choice([0, 0, rng.randrange(1, 148)])
        r1 = S.fluid_corun(ca, wa, cb, wb, 148, 2, lo, hi)
        r2 = OS.fluid_corun(ca, wa, cb, wb, 148, 2, lo, hi)
        assert abs(r1[2] - r2[2]) <= 1e-9 * r2[2]
        assert r1[0] == r2[0] or abs(r2[2] - 1.05) < 1e-9


def test_kind_geometry(S):
    assert S.kind_geometry(S.KIND_TRIAD) == (1, 1024)
    assert S.kind_geometry(S.KIND_SGEMM_NAIVE) == (16, 16)
    tm, tn = S.kind_geometry(S.KIND_GEMM_BF16)
    assert (tm, tn) == (256, 256)          # one CTA-pair tile per original block
    with pytest.raises(S.SlateError):
        S.kind_geometry(99)


def test_choose_iters_closed_forms(S):
    """NEXT-4 task size: budget / (T_solo * workers / B), capped by two tasks per
    worker and by the kind's cap, at least 1."""
    # Black-Scholes P = 1 on B200: 65.5 us, 4 x 148 workers, 8192 blocks -> 4.73 us per block -> 4
    assert S.choose_iters(0.0655, 4, 148, 8192, 10, 20.0) == 4
    # P = 32: 25 us per block, over the budget -> 1
    assert S.choose_iters(0.349, 4, 148, 8192, 10, 20.0) == 1
    # tiny blocks: the balance bound (two tasks per worker) or the cap decides
    assert S.choose_iters(0.001, 8, 148, 65536, 10, 20.0) == 10
    assert S.choose_iters(0.001, 8, 148, 4736, 10, 20.0) == 2
    # fewer blocks than workers: 1
    assert S.choose_iters(0.5, 8, 148, 100, 10, 20.0) == 1
    # a longer budget buys longer tasks, linearly
    assert S.choose_iters(0.0655, 4, 148, 8192, 10, 40.0) == 6


def test_k_way_split_matches_oracle(S):
    """slate_choose_split_k / slate_corun_makespan_k == oracle selector (random curves)."""
    rng = random.Random(170)
    for trial in range(6):
        k = 3 if trial % 2 else 2
        curves = []
        for _ in range(k):
            t148 = rng.uniform(0.5, 3.0)
            curves.append({148: t148, 74: t148 * rng.uniform(1.05, 2.0), 37: t148 * rng.uniform(2.1, 4.0)})
        n, step = 148, 4 if k == 3 else 2
        s_c, t_c = S.choose_split_k(curves, n, step)
        s_o, t_o = OS.choose_split_k(curves, n, step)
        assert s_c == s_o and abs(t_c - t_o) < 1e-9 * t_o
        shares = s_o
        assert abs(S.corun_makespan_k(curves, shares) - OS.corun_makespan_k(curves, shares)) < 1e-9 * t_o


def test_kway_admit_matches_oracle(S):
    """NEXT-4 (Q49): slate_kway_admit == oracle selector.kway_admit on random groups."""
    rng = random.Random(49)
    pts = [148, 111, 74, 49, 37, 18]
    for _ in range(60):
        curves, cats = [], []
        for _ in range(3):
            knee = rng.uniform(10, 148)
            curves.append({s: rng.uniform(0.2, 3) * max(1.0, knee / s) for s in pts})
            cats.append(rng.choice([2, 2, 3, 4]))
        a = rng.randrange(2, 147, 2)
        r1 = S.kway_admit(curves, cats, [a, 148 - a], 148, 2)
        r2 = OS.kway_admit(curves, cats, [a, 148 - a], 148, 2)
        assert r1[0] == r2[0]
        if r2[1] is not None:
            assert abs(r1[2] - r2[2]) <= 1e-9 * r2[2]
