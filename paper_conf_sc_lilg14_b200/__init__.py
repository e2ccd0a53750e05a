"""paper_conf_sc_lilg14_b200 — B200-native concrete race checking (the data-parallel hot path of SESA, SC'14).

The product is ``libsesa.so`` (C ABI, include/sesa.h) built from ``csrc/`` for sm_100a; ``sesa`` is its thin
ctypes binding.  See DESIGN.md.
"""
from .sesa import (ACCESS_DTYPE, FLOW_DTYPE, RACE_DTYPE, SesaError, Trace, load, nccl_unique_id,  # noqa: F401
                   to_device)

__all__ = ["Trace", "SesaError", "load", "nccl_unique_id", "to_device", "ACCESS_DTYPE", "RACE_DTYPE",
           "FLOW_DTYPE"]
