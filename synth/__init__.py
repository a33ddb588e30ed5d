"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

Holds no scheduler arithmetic (see profiles.py docstring).
"""
from .profiles import Profile, make_profile, requeue, table_iii_combo1, TABLE_II  # noqa: F401
from .configs import Query, CONFIGS, config, PER_CLIENT, PER_GPU  # noqa: F401
