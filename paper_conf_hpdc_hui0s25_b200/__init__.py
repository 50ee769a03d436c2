"""B200-native batched pipeline-construction search of FluidFaaS (HPDC '25).

``ffs``       -- binding of the C ABI (include/ffs.h) implemented by libffs.so (sm_100a).
``workload``  -- seeded synthetic inputs (profile tables, cluster state, requests).
"""
__all__ = ["workload", "ffs"]
