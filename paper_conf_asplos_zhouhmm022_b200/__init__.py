"""B200-native ValueExpert value-trace analysis (ASPLOS '22, Zhou et al.).

The hot path lives in libve.so (hand-written CUDA for sm_100a behind the C ABI
of include/ve.h); `ve` is the thin ctypes binding with the same names.
"""
