"""ORACLE -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct CPU implementations of what the CRSD hot path
computes, written from PAPER.md (Sun et al., ICPP 2011) and the readings listed
in DESIGN.md. Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``
(its ``cpu_baseline`` leg and ``--impl reference``) may import anything here.
The product (``paper_conf_icpp_sunzwzyr11_b200``, ``libcrsd.so``) never does,
and the two share no code; only ``gen/`` (seeded inputs, no method arithmetic)
serves both.

Modules
  coo          -- y = alpha*A*x + beta*y by definition (C, long double)   [pinned]
  crsd_ref     -- CRSD construction step by step in the paper's order,
                  paper-layout arrays (Fig. 4) and the B200 layout      [pinned]
  decode       -- independent CRSD decoder + structural invariants I1-I8 [pinned]
  closed_forms -- analytic A*x for 5/7/27-point stencils                [pinned]
  cg_ref       -- textbook conjugate gradient (Hestenes-Stiefel / Saad
                  Alg. 6.18) on the definition SpMV                    [pinned]
  crsd_ref.paper_ell_rows -- the paper's ELL scatter-row pass
                  (P:L395-411), paper evaluation order       [pinned]

Every function is pinned by ``tests/test_oracle_pins.py`` and
``tests/test_oracle_cg_pins.py`` (``-m "not gpu"``);
none is "parity unpinned".
"""
