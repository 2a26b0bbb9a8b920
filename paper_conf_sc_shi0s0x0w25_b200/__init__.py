"""B200-native hot path of Moment (Shi et al., SC '25): multi-hop CSR neighbour sampling and the
topology-aware feature gather, behind the C ABI of include/moment.h (libmoment.so).

The Python layer is argument marshalling only (`moment.py`); see DESIGN.md.
"""
from . import moment  # noqa: F401
from .moment import *  # noqa: F401,F403
from . import boxes  # noqa: F401,E402
from . import layout  # noqa: F401,E402
