"""B200-native batched sum-check prover (BatchZK hot path, ASPLOS'25).

The compute path lives in the C-ABI library ``libbzk.so`` (include/bzk.h,
csrc/); :mod:`.bzk` is the thin ctypes binding.  Importing this package does not
load the library; the first call into :mod:`.bzk` does, and raises if it is
missing -- there is no CPU fallback.
"""
__all__ = ["bzk", "inputs"]
