"""B200-native FP64 Landau Jacobian (Adams, Brennan, Knepley, Wang, IPDPS 2022).

The compute path is liblandau.so (CUDA, sm_100a) behind the C ABI in include/landau.h;
``paper_conf_ipps_adamsbkw22_b200.landau`` is its thin ctypes binding.  Nothing here falls back to
the CPU: if the shared library is missing, the binding raises.
"""
