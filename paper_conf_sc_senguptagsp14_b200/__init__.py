"""B200-native Strings (SC14) multi-tenant GPU scheduler hot path.

The product is the C-ABI library ``lib/libstrings_sched.so`` (declared in
``include/strings_sched.h``); ``strings`` is its ctypes binding and
``runner`` drives whole workloads through it.
"""
