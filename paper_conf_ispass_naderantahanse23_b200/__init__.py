"""B200-native Sieve stratification (ISPASS'23) -- Python binding of libsieve.so.

See include/sieve.h for the C-ABI and DESIGN.md for the design.  The binding only marshals
arguments; every step of the path runs in the library's sm_100a kernels.
"""
from .sieve import (ADOPT, EXPORTED, LIB_PATH, MEM_DEVICE, MEM_HOST, PHASES, STRATUM_DTYPE, Ctx,
                    Group, Params, SieveError, Strata, Trace, cycle_cov, default_params, get_unique_id,
                    kernel_launches, limbs_to_u128, load_csv, load_trace, min_strata, predict, predict_multi, stratify,
                    stratify_sweep, tier_census, torch_caching_allocator, trace_columns, u128_to_limbs,
                    version)
from . import distributed  # noqa: F401

__all__ = ["Ctx", "Group", "Params", "SieveError", "Strata", "Trace", "default_params",
           "get_unique_id", "load_csv", "load_trace", "min_strata", "trace_columns", "predict", "stratify", "version", "STRATUM_DTYPE",
           "LIB_PATH", "EXPORTED", "MEM_HOST", "MEM_DEVICE", "ADOPT", "u128_to_limbs",
           "limbs_to_u128", "torch_caching_allocator", "distributed"]
