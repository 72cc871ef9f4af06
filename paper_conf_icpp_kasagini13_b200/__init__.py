"""B200-native offline permutation (Kasagi, Nakano, Ito, ICPP 2013).

    from paper_conf_icpp_kasagini13_b200 import Plan
    plan = Plan(p)              # offline: König colourings -> packed schedules (C++)
    plan.apply(a, b)            # hot path: sm_100a kernels, b[p[i]] = a[i]

The product is libperm.so (C ABI, include/perm.h); this package only binds it.
The binding is loaded on first use (so `python -m ....build` can run before the
library exists); using any name below without a built libperm.so raises.
"""
_EXPORTS = ("Plan", "PermError", "scatter_baseline", "gather_baseline", "copy_kernel",
            "last_error", "version", "LIB_PATH", "nccl_unique_id")

__all__ = list(_EXPORTS)


def __getattr__(name):
    if name in _EXPORTS:
        from . import _lib
        return getattr(_lib, name)
    raise AttributeError(name)
