"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and
bench.py.

This package holds INPUT GENERATION ONLY (task rule ③): the counter-based
node-tensor generator (``synth.h`` in C, ``gen.synth_node`` in numpy) and the
graph-set recipes of SURVEY.md §8(d) (``workloads``).  It contains none of the
method's arithmetic — no contraction, no scheduling, no reduction — and imports
neither ``oracle`` nor the CUDA package.
"""
from .gen import NodeSpec, GraphSpec, Workload, synth_node, node_scale  # noqa: F401
from . import workloads  # noqa: F401
