"""Seeded synthetic input generators shared by the CUDA path and the oracle.

This package is the ONLY code both sides use.  It holds none of the method's
arithmetic: it draws table contents (energies, cross-section values,
concentrations, SU(3) links, multipole data) and returns plain numpy arrays.
Everything the paper's hot path computes -- lookup sampling, the unionized
energy grid and its index grid, the binary search, interpolation,
accumulation, argmax/hash, the SU(3) products, the fork/join runtime -- is
implemented twice, independently: in ``oracle/`` (plain C) and in
``paper_conf_cgo_hubercgtddcd22_b200/csrc`` (CUDA for sm_100a).

Recipes follow DESIGN.md "Input recipe" (the paper names the proxy apps and
their command lines only, PAPER.md:926-944 / 955-956 / 978-979 / 1020; table
structure is the apps' public structure, marked [ext] in SURVEY.md).
"""
from . import xs, su3, rs  # noqa: F401
