"""numpy views of the ABI structs (layout only; mirrors include/sesa.h sizes 32 / 40 / 104 bytes)."""
import numpy as np

REC_DTYPE = np.dtype(
    [("addr", "<u8"), ("value_hash", "<u8"), ("block", "<u4"), ("thread", "<u4"), ("interval", "<u4"),
     ("size", "<u2"), ("space", "u1"), ("rw", "u1")], align=True)
RACE_DTYPE = np.dtype(
    [("addr", "<u8"), ("first", "<u8"), ("second", "<u8"), ("block", "<u4"), ("interval", "<u4"),
     ("space", "u1"), ("kind", "u1"), ("reserved", "u1", (2,)), ("epoch", "<u4")], align=True)
FLOW_DTYPE = np.dtype(
    [("base", "<u8"), ("bstride", "<i8"), ("tstride", "<i8"), ("istride", "<i8"), ("value_seed", "<u8"),
     ("block_lo", "<u4"), ("block_hi", "<u4"), ("nthreads", "<u4"), ("interval", "<u4"),
     ("pmask", "<u4"), ("pval", "<u4"), ("pmod", "<u4"), ("prem", "<u4"), ("plo", "<u4"), ("phi", "<u4"),
     ("fkind", "<u4"), ("fc", "<u4"), ("fm", "<u4"), ("count", "<u4"),
     ("size", "<u2"), ("space", "u1"), ("rw", "u1"), ("flags", "<u4")], align=True)
assert REC_DTYPE.itemsize == 32 and RACE_DTYPE.itemsize == 40 and FLOW_DTYPE.itemsize == 104
