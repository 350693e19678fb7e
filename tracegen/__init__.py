"""tracegen — seeded synthetic inputs shared by the product path and the oracle.

This module holds input formats and workload generators only; it contains none of the race-check
arithmetic (no lowering, no vector clocks, no shadow logic), so both sides can consume its output
without sharing method code (see DESIGN.md §"Oracle independence").
"""
from .program import *  # noqa: F401,F403
from . import configs, fuzz  # noqa: F401
