"""Slab decomposition helpers for lora_stencil_run_dist (host logic only; no compute).

The global padded grid (N0 + 2R, ...) is split along the slowest axis: rank q owns interior
rows/planes [start_q, start_q + n_q) and holds the padded local array
global[start_q : start_q + n_q + 2R] (its halo rows are the neighbours' edge rows or the physical
boundary).  The per-step exchange itself is native (csrc/dist.cpp, NCCL); its plan is exposed by
lora_stencil_dist_exchange_plan so it can be checked on CPU.
"""
from __future__ import annotations


def slab_bounds(N0: int, nranks: int, rank: int, align: int = 1):
    """(start, count) of rank's interior rows: near-even split in units of `align` rows
    (the last rank takes the remainder rows that do not fill a unit)."""
    if not (0 <= rank < nranks) or N0 < nranks:
        raise ValueError("need 0 <= rank < nranks <= N0")
    units, tail = divmod(N0, align)
    base, rem = divmod(units, nranks)
    start = (rank * base + min(rank, rem)) * align
    count = (base + (1 if rank < rem else 0)) * align
    if rank == nranks - 1:
        count += tail
    return start, count


def local_slice(global_padded, start: int, count: int, radius: int):
    """The padded local array of a slab (a view for numpy / torch)."""
    return global_padded[start:start + count + 2 * radius]


def local_shape(global_shape, nranks: int, rank: int, align: int = 1):
    s, c = slab_bounds(global_shape[0], nranks, rank, align)
    return (c,) + tuple(global_shape[1:]), s
