"""B200-native MG-Join hot path (Paul, Lu, He, Lau, SIGMOD '21).

The join itself runs in ``libmgj.so`` (hand-written sm_100a CUDA behind the
C ABI declared in ``include/mgj.h``); ``mgj`` is the thin ctypes binding.
"""
