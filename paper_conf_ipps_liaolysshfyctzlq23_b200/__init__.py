"""Mimose on B200: budget-respecting, input-aware checkpointed training step.

The product is the C-ABI library ``libmimose.so`` built from ``csrc/`` (host
C++ runtime + sm_100a CUDA kernels).  :mod:`.binding` is a thin ctypes layer
over it; :mod:`.workload` holds the seeded synthetic input generators (shared
with the test oracle, no method arithmetic).
"""
