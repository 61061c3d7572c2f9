"""Pins for oracle/decode.py and oracle/protocol.py (CPU only).

decode: brute force over every small grid, every task size and every task start
-- Listing 2's incremental walk must equal the closed form at
every block, and the closed form must equal numpy's unravel_index (a library
routine, independent of the oracle).
protocol: exhaustive interleavings of tiny configurations and seeded random
interleavings of large ones -- every block exactly once, exact counters, no
deadlock or livelock, across resize sequences.
"""
import itertools

import numpy as np
import pytest

from oracle import decode as D
from oracle import protocol as P
from oracle import tenants as T


def test_decode_matches_unravel_index():
    for grid in [(1, 1, 1), (7, 1, 1), (3, 5, 1), (4, 3, 2), (1, 6, 5), (7, 7, 7)]:
        gx, gy, gz = grid
        for g in range(gx * gy * gz):
            z, y, x = np.unravel_index(g, (gz, gy, gx))    # C order: x fastest
            assert D.decode(g, grid) == (x, y, z)
            assert D.linear((x, y, z), grid) == g


def test_listing2_walk_brute_force():
    # P1: every grid with Gx, Gy, Gz in [1, 7], every iters in [1, 12], every start
    rng = range(1, 8)
    for gx, gy, gz in itertools.product(rng, rng, rng):
        grid = (gx, gy, gz)
        total = gx * gy * gz
        for iters in range(1, 13):
            for g in range(total):
                walk = D.listing2_walk(g, iters, grid)
                assert walk == [D.decode(b, grid) for b in range(g, min(g + iters, total))]
            assert D.listing2_walk(total, iters, grid) == []      # Q3: fetch past the end runs nothing


def test_task_partition_is_exact():
    # tasks {0, iters, 2 iters, ...} partition the block range
    for total in [1, 9, 10, 11, 103, 1024]:
        for iters in [1, 3, 10, 16]:
            seen = []
            for g in range(0, total, iters):
                seen += [D.linear(xyz, (total, 1, 1)) for xyz in D.listing2_walk(g, iters, (total, 1, 1))]
            assert seen == list(range(total))
            ex = T.expected_counters(total, iters)
            assert ex["tasks_done"] == len(range(0, total, iters))
            assert ex["next_clamped"] >= total and ex["next_clamped"] - total < iters


@pytest.mark.parametrize("cfg", [
    P.Config(blocks=4, iters=2, ranks=2, occ=1, lo=0, hi=1, resizes=[(0, 0), (0, 1)]),
    P.Config(blocks=3, iters=1, ranks=2, occ=1, lo=1, hi=1, resizes=[(0, 1)]),
    P.Config(blocks=5, iters=2, ranks=2, occ=1, lo=0, hi=0, resizes=[(1, 1)]),
    P.Config(blocks=3, iters=3, ranks=2, occ=1, lo=0, hi=1, resizes=[(1, 1), (0, 0)]),
    P.Config(blocks=4, iters=1, ranks=1, occ=2, lo=0, hi=0, resizes=[]),
    P.Config(blocks=3, iters=1, ranks=2, occ=1, lo=0, hi=1, resizes=[(1, 1), (0, 1)], abort=True),
    P.Config(blocks=4, iters=2, ranks=2, occ=1, lo=0, hi=1, resizes=[(0, 0)], abort=True),
])
def test_protocol_exhaustive(cfg):
    n = P.explore(cfg)
    assert n > 10


@pytest.mark.parametrize("cfg", [
    P.Config(blocks=4, iters=2, ranks=2, occ=1, lo=0, hi=1, resizes=[(0, 0), (0, 1)], faa_retire=False),
    P.Config(blocks=3, iters=1, ranks=2, occ=1, lo=1, hi=1, resizes=[(0, 1)], faa_retire=False),
    P.Config(blocks=3, iters=1, ranks=2, occ=1, lo=0, hi=1, resizes=[(1, 1), (0, 1)], abort=True, faa_retire=False),
])
def test_protocol_exhaustive_single_step_retire(cfg):
    """The same invariants with "retire unless last" as one atomic step."""
    assert P.explore(cfg) > 10


def test_faa_retire_needs_the_undo():
    """Q22 with the runtime's fetch-and-add retire: a last live worker that
    took live to 0 and left anyway (no undo) strands the remaining tasks: the
    mutation must fail on some interleaving."""
    class NoUndo(P.Model):
        def apply(self, act):
            if act[0] == "step":
                c = self.ctas[act[1]]
                if c[0] == P.RETIRING:
                    self.exit(c, False)
                    return
            super().apply(act)

    cfg = P.Config(blocks=4, iters=1, ranks=2, occ=1, lo=0, hi=1, resizes=[(1, 1)], grid=1)
    with pytest.raises(P.ProtocolViolation):
        stack, seen = [NoUndo(cfg)], set()
        import copy
        while stack:
            x = stack.pop()
            k = x.key()
            if k in seen:
                continue
            seen.add(k)
            if x.done():
                x.check_final()
                continue
            acts = x.actions()
            if not acts:
                raise P.ProtocolViolation("deadlock")
            for a in acts:
                y = copy.deepcopy(x)
                y.apply(a)
                y.check_step()
                stack.append(y)


def test_protocol_random_seeds():
    cfgs = [
        P.Config(blocks=1000, iters=3, ranks=8, occ=2, lo=0, hi=7, resizes=[(0, 3), (5, 7), (0, 7)]),
        P.Config(blocks=997, iters=10, ranks=6, occ=3, lo=2, hi=3, resizes=[(0, 5), (4, 4), (1, 2)]),
        P.Config(blocks=50, iters=1, ranks=4, occ=1, lo=0, hi=3, resizes=[(3, 3)] * 3 + [(0, 0)]),
        P.Config(blocks=300, iters=1, ranks=6, occ=1, lo=0, hi=5, resizes=[(0, 2), (3, 5), (1, 1), (0, 5)], abort=True),
    ]
    for cfg in cfgs:
        for seed in range(40):
            m = P.simulate(cfg, seed)
            assert m.blocks_done == cfg.blocks


def test_protocol_detects_a_broken_rule():
    """The model must be able to fail: without the last-worker rule, a shrink onto
    ranks that hold no worker strands the remaining tasks."""
    class Broken(P.Model):
        def apply(self, act):
            if act[0] == "step":
                c = self.ctas[act[1]]
                if c[0] == P.CHECK and not self.in_range(c):
                    self.exit(c, True)
                    return
            super().apply(act)

    cfg = P.Config(blocks=4, iters=1, ranks=2, occ=1, lo=0, hi=1, resizes=[(1, 1)], grid=1)
    failed = False
    import random
    for seed in range(200):
        rng = random.Random(seed)
        m = Broken(cfg)
        try:
            steps = 0
            while not m.done() and steps < 10000:
                acts = m.actions()
                if not acts:
                    raise P.ProtocolViolation("deadlock")
                m.apply(acts[rng.randrange(len(acts))])
                steps += 1
            m.check_final()
        except P.ProtocolViolation:
            failed = True
            break
    assert failed


def test_protocol_abort_needs_the_combined_word():
    """Q28: if abandoning a task and retiring were two steps (a worker may retire
    while the last other worker exits on an empty return list), a returned task
    could be orphaned: the mutation must fail."""
    class Split(P.Model):
        def actions(self):
            acts = super().actions()
            for i, c in enumerate(self.ctas):   # abort allowed even as the last live worker
                if c[0] == P.EXEC and self.cfg.abort and not self.in_range(c) and self.live == 1:
                    acts.append(("abort", i))
            return acts

    cfg = P.Config(blocks=2, iters=1, ranks=2, occ=1, lo=0, hi=1, resizes=[(1, 1)], grid=1, abort=True,
                   faa_abort=False)
    m = Split(cfg)
    with pytest.raises(P.ProtocolViolation):
        # explore every interleaving of the broken model
        import copy
        stack, seen = [m], set()
        while stack:
            x = stack.pop()
            k = x.key()
            if k in seen:
                continue
            seen.add(k)
            if x.done():
                x.check_final()
                continue
            acts = x.actions()
            if not acts:
                raise P.ProtocolViolation("deadlock")
            for a in acts:
                y = copy.deepcopy(x)
                y.apply(a)
                stack.append(y)


@pytest.mark.parametrize("cfg", [
    P.Config(blocks=3, iters=1, ranks=2, occ=1, lo=0, hi=1, resizes=[(1, 1), (0, 1)], abort=True, faa_abort=False),
    P.Config(blocks=4, iters=2, ranks=2, occ=1, lo=0, hi=1, resizes=[(0, 0)], abort=True, faa_abort=False),
])
def test_protocol_exhaustive_single_step_abort(cfg):
    """Q28 with "abandon unless last" as one atomic step (the round-1 CAS loop)."""
    assert P.explore(cfg) > 10


@pytest.mark.parametrize("cfg", [
    P.Config(blocks=2, iters=1, ranks=2, occ=1, lo=0, hi=1, resizes=[(1, 1)], grid=1, abort=True),
    P.Config(blocks=2, iters=1, ranks=2, occ=1, lo=0, hi=1, resizes=[(0, 0), (1, 1)], abort=True),
])
def test_protocol_exhaustive_faa_abort(cfg):
    """Q50: abandon-and-retire by one fetch-and-add on {live, returned}, the last
    live worker taking its unit back (or, if a taker claimed it, publishing it
    and leaving): exactly-once, no orphaned return, termination, in every
    interleaving -- including a single-CTA grid, where the abandoning worker is
    always the last.  (The abort configurations of test_protocol_exhaustive and
    the random-seed runs use this model too: it is the default.)"""
    assert P.explore(cfg) > 10


def test_faa_abort_needs_the_take_back():
    """Mutation: a last live worker that abandons by fetch-and-add and simply
    leaves (no take-back) orphans its task -- the model must find it."""
    class NoTakeBack(P.Model):
        def apply(self, act):
            if act[0] == "step" and self.ctas[act[1]][0] == P.ABORT_LAST:
                c = self.ctas[act[1]]
                self.ret_pub.append(c[4])
                self.exit(c, False)
                return
            super().apply(act)

    cfg = P.Config(blocks=2, iters=1, ranks=2, occ=1, lo=0, hi=1, resizes=[(1, 1)], grid=1, abort=True)
    import copy
    stack, seen, failed = [NoTakeBack(cfg)], set(), False
    while stack and not failed:
        x = stack.pop()
        k = x.key()
        if k in seen:
            continue
        seen.add(k)
        try:
            if x.done():
                x.check_final()
                continue
            acts = x.actions()
            if not acts:
                raise P.ProtocolViolation("deadlock")
            for a in acts:
                y = copy.deepcopy(x)
                y.apply(a)
                y.check_step()
                stack.append(y)
        except P.ProtocolViolation:
            failed = True
    assert failed


def test_grid_completion_waits_for_topup_blocks():
    """Stream order with top-ups (leave_main): the launch's own grid
    completes only after every block ran, even when a top-up grid (a grow) took the
    last tasks -- and the CTA that waits cannot starve the top-up (liveness is part
    of the exhaustive exploration).  Without the rule the exploration finds a grid
    that completes with blocks still running on the top-up."""
    cfgs = [P.Config(blocks=4, iters=2, ranks=2, occ=1, lo=0, hi=1, resizes=[(0, 0), (0, 1)]),
            P.Config(blocks=3, iters=1, ranks=2, occ=1, lo=0, hi=0, resizes=[(0, 1)])]
    for cfg in cfgs:
        assert P.explore(cfg) > 0
    bad = P.Config(blocks=4, iters=2, ranks=2, occ=1, lo=0, hi=1, resizes=[(0, 0), (0, 1)], leave_main=False)
    with pytest.raises(P.ProtocolViolation, match="grid completed"):
        P.explore(bad)
