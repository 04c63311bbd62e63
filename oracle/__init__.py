"""CPU oracle for the Paraprox Stencil & Partition approximation.

TEST INFRASTRUCTURE ONLY: only ``tests/``, ``__graft_entry__.smoke()`` and the
``cpu_baseline`` / ``--impl reference`` legs of ``bench.py`` may import this
package.  It shares no code with the CUDA product path
(``paper_conf_asplos_samadijlm14_b200``) and never imports it.
"""
from .oracle import *  # noqa: F401,F403
