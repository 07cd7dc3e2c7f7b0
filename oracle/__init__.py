"""CPU oracle for the MSCCL-IR interpreter — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import anything from this package. The product path
(``paper_conf_asplos_cowanmmsx23_b200``) never imports it and shares no code with it:
this package has its own IR parser, its own chunk-geometry rule implementation, its
own reduction arithmetic and its own abstract machine.

Citations are ``P:L<n>`` = line n of the paper text (MSCCLang, ASPLOS '23), section
named alongside.

Modules
-------
irparse   : reads the MSCCL-IR text (tree of Fig. 4).
geometry  : chunk -> element span rule (reading R1 / SURVEY Q1-Q3).
numerics  : one correctly rounded binary op per reduce, in the buffer dtype.
mpi_ref   : brute-force collective definitions (P:L785-813 AllReduce, P:L2460-2461
            AllToAll), fp64 / exact integers.
sim       : executes an IR over per-rank host buffers with bounded FIFOs and
            cross-thread-block semaphores.
symbolic  : multiset and ordered-tree chunk labels; collective postconditions
            (P:L761-821).
validate  : structural rules V1-V9 of DESIGN.md, incl. abstract-machine deadlock check,
            and V10 (races=True): no happens-before race (``races``).
races     : happens-before race detection between instructions (program order, deps,
            k-th send -> k-th receive) and the
            independent check of the loader's direct-placement marking (reading R15).

Parity status: every function is pinned by ``tests/test_oracle_*.py`` (see DESIGN.md
"Oracle pins"). The reduction order the paper's own All-Pairs program used is not
printed in the paper: ``parity unpinned`` for that *paper* program; our two-shot /
one-shot programs fix the ascending-rank order (reading R7) and that order is
pinned by an independent fold.
"""
