"""fsmgen -- seeded synthetic DFAs and input streams for the spec-k FSM workloads.

This module is the ONLY code shared by the oracle side (``oracle/``) and the product side
(``paper_conf_ppopp_xiaja20_b200``).  It holds workload definitions and random-number
generators, and none of the spec-k method's arithmetic (no look-back, no local processing, no
merge, no re-execution).
"""
from . import dfas, streams  # noqa: F401
from .dfas import DFA  # noqa: F401
from .streams import MASTER_SEED  # noqa: F401
