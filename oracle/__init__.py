"""CPU oracle -- TEST INFRASTRUCTURE ONLY.

Plain cycle-accurate 2-state E-AIG simulator (oracle.cpp) plus an independent
Python twin (twin.py).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py`` (cpu_baseline leg and ``--impl reference``) may import this
package.  The product path (``paper_conf_dac_guozwlr25_b200``) never does.
"""
from .oracle import Oracle, build_oracle, oracle_digest  # noqa: F401
