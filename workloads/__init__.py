"""Seeded synthetic-workload descriptions shared by the oracle side and the CUDA
side (tests, bench).  Holds shapes, names, seeds and value-distribution
parameters only -- none of the method's arithmetic (no packing, no hashing, no
selection) and not the generator formula itself: each side implements the
counter-based generator on its own (oracle/jitc_oracle.c, the K4 kernel)."""
from .configs import *  # noqa: F401,F403
