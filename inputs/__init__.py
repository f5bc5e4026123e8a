"""Seeded synthetic inputs shared by the oracle tests, the CUDA tests and bench.py.

Holds no KTILER arithmetic (see synth.py).  ``synth`` is numpy (CPU); ``gpu`` is the
device twin used to fill multi-GB inputs in HBM.
"""
from . import synth  # noqa: F401
