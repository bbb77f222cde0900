"""bcgen — seeded synthetic trace generators (input fixtures only).

Serves both the oracle tests and the CUDA path; holds none of the method's
arithmetic.  See format.py for the record layout.
"""
from .format import *  # noqa: F401,F403
from .builder import TraceBuilder, gaddr  # noqa: F401
from .fuzz import random_trace  # noqa: F401
from .configs import make_config, CONFIGS  # noqa: F401
