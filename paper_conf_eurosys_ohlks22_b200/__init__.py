"""B200-native data-parallel hot path of out-of-order backprop (Oh et al., EuroSys'22).

The product is libooo.so (C ABI in include/ooo.h: hand-written sm_100a
kernels + the stream/event/NCCL scheduler).  This package holds its build
script, the thin ctypes binding (``stack``), the workload shapes
(``configs``) and the seeded input generators (``synth``).  Importing the
package does not load the library; ``stack.OooStack`` does, and raises if it
has not been built.
"""
__all__ = ["configs", "synth", "stack", "build"]
