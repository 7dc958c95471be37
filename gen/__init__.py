"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This package holds NO arithmetic of the CRSD method (no offset grouping, no
segmenting, no SpMV). It only draws matrices in COO form with the shapes of
the paper's workloads (FDM/FVM stencils, broken diagonals, scatter points,
banded matrices) and the vectors they are multiplied with. The recipes are
stated in DESIGN.md ("Input recipe") and follow SURVEY.md §8(d).
"""
from .matrices import (  # noqa: F401
    COO,
    stencil,
    stencil_5pt,
    stencil_7pt,
    stencil_27pt,
    inject_scatter,
    config1,
    config2,
    config3,
    config4,
    config5,
    band,
    random_diagonal,
    vectors,
    nonzero_uniform,
    spd_stencil_scatter,
)
