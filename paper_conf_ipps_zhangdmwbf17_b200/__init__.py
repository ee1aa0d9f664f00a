"""B200-native (sm_100a, fp64) HPGMG-FV hot path of Snowflake (Zhang et al., IPDPSW 2017).

libsf.so (csrc/, C ABI in include/sf.h) holds every kernel; ``sf`` is its thin
ctypes binding; ``inputs`` holds the seeded synthetic problem generators.
"""
__all__ = ["sf", "inputs", "build"]
