"""Seeded synthetic-input module shared by the oracle (oracle/) and the CUDA path.

Holds no method arithmetic: the C header ``capgpu_gen.h`` (counter-based
generator) and ``configs.py`` (the five BASELINE.json workloads as plain data).
"""
