"""CPU oracle for the Slate slate-kernel hot path.

TEST INFRASTRUCTURE ONLY. Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py`` (its ``cpu_baseline`` leg and ``--impl reference``) may import
anything under ``oracle/``.  The product path (``paper_conf_ipps_allenf019_b200``
and its CUDA library) never imports, links or executes this package, and this
package imports nothing from the product path: the two share no code.  The only
shared module is ``paper_conf_ipps_allenf019_b200/inputs.py``, the seeded input
generator, which holds none of the method's arithmetic -- and the oracle does
not even import that: every oracle function takes its inputs as arguments.

Citations ``P:L<n> §<sec>`` are lines of the paper text and its
section; ``Lst<n>``/``Tab <n>`` are its listings/tables; readings ``Q<n>`` are
listed in DESIGN.md §Readings (taken from SURVEY.md §8(c)).

Modules
  decode    -- K(B,T) -> K*(B*,T) block-index decode (§III-A, Lst2(4)).
  tenants   -- per-tenant block bodies in fp64, run block by block in linear
               order (the plain definition: "must preserve the semantics",
               P:L79 "K and K* are isomorphic").
  protocol  -- seeded discrete-event model of the task queue + resize protocol
               (Lst2 P:L199-231, §III-C, exit conditions P:L243-245).
  selector  -- workload classification + Tab I policy + selection algorithm
               (§III-B).
  metrics   -- the paper's throughput criterion and STP/ANTT.

Parity status (every function is pinned by a ``-m "not gpu"`` test unless
listed here): resize latency is measured only -- "parity unpinned" (the paper
reports no resize latency).
"""
