"""ORACLE -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct CPU implementations of what the CRSD hot path
computes, written from PAPER.md (Sun et al., ICPP 2011) and the readings listed
in DESIGN.md. Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``
(its ``cpu_baseline`` leg and ``--impl reference``) may import anything here.
The product (``paper_conf_icpp_sunzwzyr11_b200``, ``libcrsd.so``) never does,
and the two share no code; only ``gen/`` (seeded inputs, no method arithmetic)
serves both.

Modules and their pins (tests/test_oracle_pins.py, tests/test_oracle_cg_pins.py,
all ``-m "not gpu"``)
  coo.coo_spmv     -- y = alpha*A*x + beta*y by definition (C, long double):
                      dense brute force, scipy.sparse, stencil closed forms
  coo.rows_spmv    -- the same definition on sampled rows (full-size parity):
                      dense brute force on shuffled samples (first/last/empty
                      rows, beta != 0), bitwise vs coo_spmv, closed forms
  coo.parity_error -- the pass criterion max_r |y - y_ref| / scale_r: hand cases
                      (scale-0 rows exact, NaN fails, max not mean)
  coo.coo_spmv_native -- the definition accumulated in the matrix dtype, 1..N
                      OpenMP threads (the timed CPU baseline, not a checker):
                      summation bound vs coo_spmv, thread-count invariance,
                      closed forms
  crsd_ref         -- CRSD construction step by step in the paper's order,
                      paper-layout arrays (Fig. 4) and the B200 layout: Fig. 2
                      -> Fig. 4 / Table III golden, grouping example, DIA
                      special case, hand-worked presence cases
  crsd_ref.paper_ell_rows -- the paper's ELL scatter-row pass (P:L395-411,
                      P:L703-719), paper evaluation order: Fig. 2 by hand,
                      the definition
  decode           -- independent CRSD decoder + invariants I1-I8: round trip
                      of the paper-order construction, corrupted layouts rejected
  closed_forms     -- analytic A*x for 5/7/27-point stencils: the interior
                      values of SURVEY.md §8(c) (0, 0, -4/-6/-54), boundary A*1
  cg_ref           -- textbook conjugate gradient (Hestenes-Stiefel / Saad
                      Alg. 6.18) on the definition SpMV: finite termination vs
                      closed-form and LAPACK solutions, first step, orthogonality

Every function listed has at least one pin that does not re-derive it from
itself; none is "parity unpinned".
"""
