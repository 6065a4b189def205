"""ORACLE — test infrastructure only.

Plain, slow, obviously-correct CPU reference for the variable-size batched GEMM method of
Li et al., "A Coordinated Tiling and Batching Framework for Efficient GEMM on GPUs"
(PPoPP'19; /root/reference/PAPER.md, cited as P<line>).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` leg may import anything under ``oracle/``.  The product package
``paper_conf_ppopp_li0yjl19_b200`` never imports it, and this package never imports the
product.  The only shared module is ``vbinputs`` (seeded input draws, no GEMM arithmetic).

Contents
* ``gemm``      — fp64 triple-loop GEMM in plain C (``gemm_ref.c``), P31/P133.
* ``plan_ref``  — tiling engine (§4, P245–255, Eq. 1), tile enumeration (P133–135, P157),
                  threshold / binary batching (§5, P259–270, Eq. 5), five-array encoding
                  (§6, P282–284, Fig. 6/7) and the LPT GEMM->rank sharder (BASELINE.json).
* ``forest_ref`` — the on-line batching-policy selector (random forest, §5, P272–274),
                  evaluated on trees that are a B200 platform constant (reading C-25).
* ``conv_ref``  — stride-1 zero-padded 2-D convolution in fp64 (NHWC x HWIO), the definition
                  behind the implicit-GEMM convolution path (NEXT-3, P45, P338–352).
* ``checks``    — normwise error, coverage map and plan invariants.

Parity status: every function is pinned (see DESIGN.md §3 and tests/test_oracle_*.py) except
the threshold-batching fill rule, whose source passage (P261) is garbled: it is pinned only
by consistency with P352 and derived values ("parity partially unpinned", C-9).
"""
