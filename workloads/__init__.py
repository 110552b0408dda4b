"""Seeded synthetic workload generators (integers and bf16-exact values only).

The one module shared by the oracle (`oracle/`) and the harness (`bench.py`,
`tests/`). It holds none of the method's arithmetic; see SURVEY.md §8(c) C1.
"""
from . import configs, prng, inputs, weights  # noqa: F401
