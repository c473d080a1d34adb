"""B200-native per-length encoder runtimes for Arlo's polymorphing (ICPP '24).

The compute path lives in ``libarlo.so`` (hand-written sm_100a CUDA behind the
C ABI of ``include/arlo.h``); ``arlo`` is the thin ctypes binding.  Importing
this package does not load the library; ``from paper_conf_icpp_tanlyl024_b200
import arlo`` does, and fails loudly if it is missing.
"""
__all__ = ["arlo", "workload"]
