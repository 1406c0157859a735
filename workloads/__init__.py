"""Seeded input generators and literal workload tables.

This is the ONLY module shared by the oracle (``oracle/``) and the product
(``paper_conf_asplos_0001cgrnls0trm26_b200``) — through the tests and bench.py.
It holds no layout arithmetic: layouts appear here as literal tables of which
logical bit each hardware bit carries, and random layouts are
built by construction (random assignments / triangular constructions), never by
composing, inverting or classifying anything.
"""
from .configs import CONFIGS, spec_to_bases, bit_coords  # noqa: F401
from . import gen  # noqa: F401
