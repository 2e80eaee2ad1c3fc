"""CPU oracle for the SLAM-Share tracking hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
(``paper_conf_conext_dhakalrwcr22_b200``) never imports it and shares no code with it.
"""
from .oracle import *  # noqa: F401,F403
