"""CPU oracle for the EGEMM-TC hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
``paper_conf_ppopp_fengwcz0d21_b200`` never imports it and shares no code with it.
"""
from .oracle import *  # noqa: F401,F403
