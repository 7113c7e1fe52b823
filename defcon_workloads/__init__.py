"""Seeded synthetic workloads for the DEFCON hot path (shared by tests and bench).

This package holds NO arithmetic of the method: it only draws seeded random
inputs with the shapes and value distributions of the paper's workloads
(``inputs``) and lists the BASELINE.json configurations plus the FLOP/byte
model used for roofline reporting (``configs``).  Both the CPU oracle
(``oracle/``) and the CUDA product path consume the same arrays it returns.
"""
