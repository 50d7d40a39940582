"""B200-native OP-PIC particle loop (Lantra, Wright, Mudalige, ICPP '24).

libopp.so (csrc/, C ABI in include/opp.h) holds the hand-written sm_100a
kernels; ``opp`` is the thin ctypes binding with the ABI's names and ``app``
a Mini-FEM-PIC-style application on top of it.  Importing ``opp`` fails loudly
if the library has not been built -- there is no CPU fallback.
"""
__all__ = ["opp", "app"]
