"""MemXCT CPU oracle (fp64, single-threaded C) -- TEST INFRASTRUCTURE ONLY.

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` / ``--impl reference``
legs may import this package.  The product package never imports it, and it never imports the
product package.  See memxct_oracle.c for the passages each function follows.
"""
from .oracle import *  # noqa: F401,F403
