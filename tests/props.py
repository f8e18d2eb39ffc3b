"""Closed-form properties of the reuse histogram that hold at any size
(used where the LRU-stack oracle cannot finish; pinned against the oracle in
test_oracle_pins.py::test_kernel_scope_properties_match_oracle)."""
import numpy as np


def kernel_scope_properties(t, lb):
    """(mass, inf, streaming) of the kernel-scope reuse histogram from the
    definitions (P:L248, P:L252, P:L237 streaming) -- no LRU stack needed."""
    mem = (t.meta & 3) < 2
    line = (t.addr[mem] // lb).astype(np.uint64)
    st = (t.meta[mem] & 3) == 1
    n = len(line)
    order = np.lexsort((np.arange(n), line))            # by line, then trace position
    ls, ss = line[order], st[order]
    new_line = np.r_[True, ls[1:] != ls[:-1]]
    # epoch = stores to the line at or before the position (running count per line)
    cs = np.cumsum(ss)
    base = np.maximum.accumulate(np.where(new_line, cs - ss, 0))
    epoch = cs - base
    # renamed key = (line, epoch); keys are contiguous runs in this order
    new_key = new_line | (epoch != np.r_[-1, epoch[:-1]])
    kid = np.cumsum(new_key) - 1
    counts = np.bincount(kid)
    inf = int(new_key.sum())                           # first use of every renamed element
    streaming = int((counts == 1).sum())
    return n, inf, streaming
