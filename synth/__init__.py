"""Seeded synthetic ICFG inputs (shared by the oracle and the CUDA path).

Holds input construction only — never any of the method's arithmetic.
"""
from .icfg import *  # noqa: F401,F403
from .icfg import Icfg, IcfgBuilder  # noqa: F401
from .tiny_random import random_tiny  # noqa: F401
from .generator import PRESETS, GenConfig, corpus_app, corpus_config, generate, preset  # noqa: F401
