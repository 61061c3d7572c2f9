"""Discrete-event model of the slate task queue and resize protocol  (test infrastructure only).

This is the *scheduling* half of the oracle: it computes no tenant output, it
checks the invariant that makes Slate's transformation semantics-preserving --
every original block runs exactly once, whatever the placement of worker CTAs
and whatever sequence of resize events arrives.

Paper steps modelled, in the paper's order:
  Lst1   a CTA reads its SM id and checks it against the inclusive
                      bound [sm_low, sm_high] (reading Q5); out of range -> return.
  Lst2   a worker atomically pulls SLATE_ITERS consecutive blocks from
                      slateIdx, clamps the last task (reading Q3 -- a fetch
                      at or past slateMax exits before running anything), runs the
                      blocks in order, and leaves the loop on a retreat signal or
                      when the queue is exhausted -- checked only between tasks.
  §III-C / Lst3       a resize changes the SM range; progress is carried in
  (P:L123-127,          slateIdx.  The paper terminates and
   P:L237-263)          relaunches the workers; the north star forbids the relaunch,
                      so here (reading Q6) shrink = workers outside the new range
                      retire at their next task boundary, grow = CTAs waiting in
                      standby join, or a top-up launch bound to the newly granted
                      ranks adds workers that share the same slateIdx.
  exit conditions     (1) wrong SM, (2) queue exhausted, (3) retreated / joined late
  

Two liveness rules of the B200 design are modelled so the
model can show they are sufficient:
  * an out-of-range CTA waits in standby while the tenant has fewer live
    workers than its target occ*|range| (so a launch cannot burn its whole grid
    on foreign SMs), and leaves when the target is met or the queue is drained;
    after a timeout with zero live workers it runs anyway;
  * the last live worker of a tenant never retires while tasks remain (the
    runtime decrements live and puts the unit back if it was the last:
    ``Config.faa_retire``; the transient zero is explored too).

``simulate`` runs one seeded random interleaving; ``explore`` enumerates every
interleaving of a tiny configuration (depth-first, memoised on state).  Both
raise ``ProtocolViolation`` on any broken invariant or deadlock.
"""
import random
from dataclasses import dataclass, field


class ProtocolViolation(AssertionError):
    pass


PENDING, PROLOGUE, STANDBY, FETCH, EXEC, CHECK, EXITED, RETIRING, WAITDONE, CLAIMED, ABORT_OK, ABORT_LAST = range(12)


@dataclass
class Config:
    blocks: int               # B = slateMax, the number of original blocks
    iters: int                # SLATE_ITERS, blocks per task
    ranks: int                # number of SMs N
    occ: int                  # max resident worker CTAs per SM
    lo: int                   # initial inclusive SM range [lo, hi]
    hi: int
    resizes: list = field(default_factory=list)   # [(lo, hi), ...] applied in order at random times
    grid: int = 0             # CTAs per launch; default occ * ranks (one full wave)
    abort: bool = False       # long-task tenants: a retiring worker may abandon its task
    leave_main: bool = True   # the CTA whose exit completes the launch's own grid waits until every block ran
                              # (a top-up grid may still hold blocks, and the queue's next
                              # launch starts when this grid completes).  False: it just exits
    faa_retire: bool = True   # retire as the runtime does it (Q22): live -= 1 in one atomic
                              # step, and if that took live from 1 to 0, live += 1 in a later step
                              # and stay; other CTAs may act in between.  False: one atomic
                              # "retire unless last" step
                              # mid-way and return it (Q28)
    faa_abort: bool = True    # abandon-and-retire as the runtime does it (Q50): one
                              # fetch-and-add on {live, returned} (live -1, returned +1); the
                              # task is published to the ring in a later step.  If live went
                              # 1 -> 0 the worker, in a later step, takes the unit back and
                              # resumes its task unless the returned count is 0 (a taker claimed
                              # it: then it publishes and leaves).  Takers claim a count and wait
                              # for a publication.  False: one atomic "abandon unless last" step


def _in(rank, lo, hi):
    return lo <= rank <= hi


class Model:
    """Mutable protocol state; ``actions()`` lists the enabled atomic steps."""

    def __init__(self, cfg):
        self.cfg = cfg
        self.next = 0                      # slateIdx
        self.epoch = 0
        self.lo, self.hi = cfg.lo, cfg.hi  # the resize word {epoch, lo, hi}
        self.live = 0                      # live worker CTAs of the tenant
        self.ret_count = 0                 # returned units committed and not yet claimed (Q28)
        self.ret_pub = []                  # published returned task starts, FIFO (the ring)
        self.cov = [0] * cfg.blocks        # executions per original block
        self.blocks_done = 0
        self.tasks_done = 0
        self.task_starts = []
        self.resize_i = 0
        grid = cfg.grid or cfg.occ * cfg.ranks
        # per CTA: [state, rank, launch_lo, launch_hi, g, n, seen_epoch, was_worker, main]
        # (main: a CTA of the launch's own grid; top-up CTAs are not)
        self.ctas = [[PENDING, -1, 0, cfg.ranks - 1, 0, 0, -1, False, True] for _ in range(grid)]
        self.main_exited = 0               # main CTAs that have left (joined or not)
        self.grid = grid
        self.resident = [0] * cfg.ranks    # resident CTAs per SM (placement capacity)

    # ------------------------------------------------------------ helpers
    def target(self):
        return self.cfg.occ * (self.hi - self.lo + 1)

    def in_range(self, c):
        return _in(c[1], self.lo, self.hi) and _in(c[1], c[2], c[3])

    def exit(self, c, worker):
        if worker:
            self.live -= 1
        if c[8]:                           # a CTA of the launch's own grid leaves (worker or not)
            self.main_exited += 1
            if self.main_exited == self.grid and self.cfg.leave_main and self.blocks_done < self.cfg.blocks:
                c[0] = WAITDONE            # the one completing the grid waits for every block (leave_main)
                return
        c[0] = EXITED
        self.resident[c[1]] -= 1

    def key(self):
        return (self.next, self.epoch, self.lo, self.hi, self.live, self.main_exited, self.ret_count, tuple(self.ret_pub),
                tuple(self.cov),
                self.blocks_done,
                self.tasks_done, tuple(sorted(self.task_starts)), self.resize_i,
                tuple(tuple(c) for c in self.ctas), tuple(self.resident))

    # ------------------------------------------------------------ actions
    def actions(self):
        acts = []
        for i, c in enumerate(self.ctas):
            st = c[0]
            if st == PENDING:
                for r in range(self.cfg.ranks):
                    if self.resident[r] < self.cfg.occ:
                        acts.append(("place", i, r))
            elif st in (PROLOGUE, FETCH, EXEC, CHECK, RETIRING, ABORT_OK, ABORT_LAST):
                acts.append(("step", i))
                # Q28: a worker outside the range may abandon its running task and
                # retire -- one fetch-and-add (faa_abort), or one atomic step that
                # refuses the last live worker
                if st == EXEC and self.cfg.abort and not self.in_range(c) and (self.cfg.faa_abort or self.live > 1):
                    acts.append(("abort", i))
            elif st == CLAIMED:
                if self.ret_pub:                   # the claimed unit has been published
                    acts.append(("step", i))
            elif st == STANDBY:
                acts.append(("step", i))
                if self.live == 0 and (self.next < self.cfg.blocks or self.ret_count or self.ret_pub):
                    acts.append(("timeout", i))
            elif st == WAITDONE and self.blocks_done == self.cfg.blocks:
                acts.append(("step", i))
        if self.resize_i < len(self.cfg.resizes):
            acts.append(("resize",))
        return acts

    def apply(self, act):
        cfg = self.cfg
        if act[0] == "resize":
            lo, hi = cfg.resizes[self.resize_i]
            self.resize_i += 1
            old = (self.lo, self.hi)
            self.epoch += 1
            self.lo, self.hi = lo, hi
            # grow: ranks not in the old range get a top-up launch bound to the new range
            # (the runtime's rule); CTAs it places on old ranks leave
            if lo < old[0] or hi > old[1]:
                for _ in range(cfg.occ * cfg.ranks):
                    self.ctas.append([PENDING, -1, lo, hi, 0, 0, -1, False, False])
            return
        if act[0] == "place":
            _, i, r = act
            c = self.ctas[i]
            c[0], c[1] = PROLOGUE, r
            self.resident[r] += 1
            return
        i = act[1]
        c = self.ctas[i]
        st = c[0]
        if act[0] == "abort":
            if cfg.faa_abort:                  # fetch-and-add: live -1, returned +1; publish later
                was_last = self.live == 1
                self.live -= 1
                self.ret_count += 1
                c[0] = ABORT_LAST if was_last else ABORT_OK
                return
            self.ret_count += 1                # one atomic step: return the task, retire
            self.ret_pub.append(c[4])
            self.exit(c, True)
            return
        if act[0] == "timeout":            # standby with no live worker: run anyway (liveness)
            self.live += 1
            c[0], c[7] = FETCH, True
            return
        if st == WAITDONE:                 # every block ran: the last main CTA leaves, the grid completes
            c[0] = EXITED
            self.resident[c[1]] -= 1
            return
        if st == ABORT_OK:                 # publish the abandoned task, leave (live already -1)
            self.ret_pub.append(c[4])
            self.exit(c, False)
            return
        if st == ABORT_LAST:               # it was the last live worker: take the unit back ...
            if self.ret_count >= 1:
                self.ret_count -= 1
                self.live += 1
                c[0] = EXEC                # ... and resume its task (none of it ran)
            else:                          # a taker claimed it: publish for the taker, leave
                self.ret_pub.append(c[4])
                self.exit(c, False)
            return
        if st == CLAIMED:                  # the ring slot of the claim is published
            g = self.ret_pub.pop(0)
            c[0], c[4], c[5] = EXEC, g, min(cfg.iters, cfg.blocks - g)
            return
        if st in (PROLOGUE, STANDBY):
            # Lst1: leader reads the SM id and the bound; here also the queue state
            if self.next >= cfg.blocks and not self.ret_count:
                self.exit(c, False)        # exit (2): nothing left to do
            elif self.in_range(c):
                self.live += 1
                c[0], c[6], c[7] = FETCH, self.epoch, True
            elif self.live >= self.target():
                self.exit(c, False)        # exit (1): wrong SM and the tenant is fully staffed
            else:
                c[0] = STANDBY             # wait: the tenant is under-staffed
        elif st == FETCH:
            if self.ret_count:             # Q28: returned tasks first -- claim a unit, then wait for its slot
                self.ret_count -= 1
                c[0] = CLAIMED
                return
            # Lst2 (2): globIdx = atomicAdd(&slateIdx, SLATE_ITERS)
            g = self.next
            self.next += cfg.iters
            if g >= cfg.blocks:            # Q3: never run a task that starts past the end
                self.exit(c, True)         # exit (2): the returned list was empty in the same atomic step
            else:
                c[0], c[4], c[5] = EXEC, g, min(cfg.iters, cfg.blocks - g)
                self.task_starts.append(g)
        elif st == EXEC:
            # Lst2 (3)-(5): run the task's blocks in order
            for b in range(c[4], c[4] + c[5]):
                self.cov[b] += 1
            self.blocks_done += c[5]
            self.tasks_done += 1
            c[0] = CHECK
        elif st == CHECK:
            # Lst2 (1) loop condition: retreat is examined only between tasks
            c[6] = self.epoch
            if self.in_range(c):
                c[0] = FETCH
            elif cfg.faa_retire:
                was_last = self.live == 1
                self.live -= 1             # fetch-and-add: live -= 1
                c[0], c[5] = RETIRING, int(was_last)
            elif self.live == 1 and (self.next < cfg.blocks or self.ret_count):
                c[0] = FETCH               # stay (the last live worker never retires)
            else:
                self.exit(c, True)         # exit (3): retreated
        elif st == RETIRING:
            if c[5]:                       # it was the last live worker: put the unit back, stay
                self.live += 1
                c[0] = FETCH
            else:
                self.exit(c, False)        # exit (3): retreated (its unit of live is already gone)

    # ------------------------------------------------------------ invariants
    def done(self):
        return all(c[0] in (EXITED,) for c in self.ctas) and self.resize_i == len(self.cfg.resizes)

    def check_final(self):
        cfg = self.cfg
        tasks = -(-cfg.blocks // cfg.iters)
        if self.cov != [1] * cfg.blocks:
            raise ProtocolViolation("coverage not exactly-once: %r" % self.cov)
        if self.blocks_done != cfg.blocks or self.tasks_done != tasks:
            raise ProtocolViolation("counters %d/%d" % (self.blocks_done, self.tasks_done))
        if sorted(self.task_starts) != list(range(0, cfg.blocks, cfg.iters)):
            raise ProtocolViolation("task starts %r" % self.task_starts)
        if min(self.next, tasks * cfg.iters) != tasks * cfg.iters:
            raise ProtocolViolation("next_clamped")
        if self.live != 0:
            raise ProtocolViolation("live workers at the end")
        if self.ret_count or self.ret_pub:
            raise ProtocolViolation("returned tasks never executed")

    def check_step(self):
        if any(v > 1 for v in self.cov):
            raise ProtocolViolation("block executed twice")
        # stream order: the launch's own grid completes (its next launch may start)
        # only when every block has run, whatever top-up grids still hold
        if self.blocks_done < self.cfg.blocks and all(c[0] == EXITED for c in self.ctas if c[8]):
            raise ProtocolViolation("the launch's grid completed with %d blocks still to run"
                                    % (self.cfg.blocks - self.blocks_done))


def simulate(cfg, seed, max_steps=10_000_000):
    """One random interleaving; returns the final model (invariants checked)."""
    rng = random.Random(seed)
    m = Model(cfg)
    steps = 0
    while not m.done():
        acts = m.actions()
        if not acts:
            raise ProtocolViolation("deadlock: tasks left %d" % (cfg.blocks - m.blocks_done))
        m.apply(acts[rng.randrange(len(acts))])
        m.check_step()
        steps += 1
        if steps > max_steps:
            raise ProtocolViolation("no termination")
    m.check_final()
    return m


def explore(cfg, limit=2_000_000):
    """Every interleaving of a tiny configuration.

    Builds the full reachable state graph, checks the invariants in every state
    and at every terminal state, and checks liveness: from every reachable state
    some terminal state is reachable (no deadlock, no livelock).  Returns the
    number of distinct states.
    """
    import copy
    succ = {}
    terminal = set()
    stack = [Model(cfg)]
    while stack:
        m = stack.pop()
        k = m.key()
        if k in succ:
            continue
        if len(succ) > limit:
            raise ProtocolViolation("state space larger than limit")
        if m.done():
            m.check_final()
            succ[k] = []
            terminal.add(k)
            continue
        acts = m.actions()
        if not acts:
            raise ProtocolViolation("deadlock in state %r" % (k,))
        nxt = []
        for a in acts:
            m2 = copy.deepcopy(m)
            m2.apply(a)
            m2.check_step()
            nxt.append(m2.key())
            stack.append(m2)
        succ[k] = nxt
    # liveness: backward reachability from the terminal states
    pred = {k: [] for k in succ}
    for k, ns in succ.items():
        for n in ns:
            pred[n].append(k)
    good = set(terminal)
    work = list(terminal)
    while work:
        k = work.pop()
        for p in pred[k]:
            if p not in good:
                good.add(p)
                work.append(p)
    if len(good) != len(succ):
        raise ProtocolViolation("%d states cannot reach completion" % (len(succ) - len(good)))
    return len(succ)
