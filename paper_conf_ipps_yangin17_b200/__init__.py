"""B200-native (sm_100a) hot path of Yang, Ito & Nakano's rearrangement
photomosaic (IPDPS-W 2017): the all-pairs tile error matrix E (Eq. 1) and the
colour-class parallel 2-swap local search (Algorithm 2), behind the C-ABI
library ``libpm.so`` (include/pm.h).  The Python layer only marshals
arguments; every step of the path runs in the CUDA kernels.

``synth`` (seeded inputs) imports nothing else; the C-ABI binding is loaded
lazily by ``paper_conf_ipps_yangin17_b200.pm`` and fails loudly if the
library is missing.
"""
__all__ = ["synth", "pm"]
