"""Schedule oracle for the fine-grained SM scheduling of COMET (Fig. 8).
TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The paper's model (Fig. 8): a GEMM is cut into 128x128x128 "tiles"
(= one output tile x one 128-channel K-block).  A tile whose activation block is INT8 costs
more than an INT4 tile (on the paper's A100 the INT4 tensor core is 2x faster, P:L166:
cost 2 : 1).  Every SM runs its assigned tiles in order.

  * naive (Fig. 8b): tiles are dealt round-robin, one per SM per *iteration*, with a
    barrier after every iteration -> makespan = sum over iterations of the slowest tile.
  * barrier minimisation (Fig. 8c): same dealing, a single barrier before the
    write-back -> makespan = max over SMs of the SM's summed cost.
  * tile remapping (Fig. 8d): any whole-tile assignment -> max over SMs of summed cost.
  * tile decomposition (Fig. 8e): a tile's K-range may be split between SMs
    (stream-K [42]) -> max over SMs of summed (fractional) cost.

Parity: pinned by the Fig. 8 worked example (tests/golden/fig8_schedule.json).
"""
from __future__ import annotations

from fractions import Fraction


def unit_cost(tags, kb: int, cost_int4, cost_int8):
    """Cost of one (output tile, K-block) unit: depends only on the block's precision tag."""
    return cost_int8 if tags[kb] else cost_int4


def makespan_naive_barrier(n_units: int, n_sm: int, cost_of_unit) -> Fraction:
    """Round-robin, one unit per SM per iteration, barrier after each iteration (Fig. 8b)."""
    total = Fraction(0)
    for start in range(0, n_units, n_sm):
        total += max(Fraction(cost_of_unit(u)) for u in range(start, min(start + n_sm, n_units)))
    return total


def makespan_round_robin(n_units: int, n_sm: int, cost_of_unit) -> Fraction:
    """Round-robin dealing with a single barrier before write-back (Fig. 8c)."""
    loads = [Fraction(0)] * n_sm
    for u in range(n_units):
        loads[u % n_sm] += Fraction(cost_of_unit(u))
    return max(loads)


def makespan(per_sm_segments, tags, cost_int4, cost_int8) -> Fraction:
    """per_sm_segments: for each SM a list of (tile, kb_begin, kb_end) half-open K-block ranges.
    Makespan = max over SMs of the summed unit costs (Fig. 8d/8e)."""
    loads = []
    for segs in per_sm_segments:
        load = Fraction(0)
        for (_tile, kb0, kb1) in segs:
            for kb in range(kb0, kb1):
                load += Fraction(unit_cost(tags, kb, cost_int4, cost_int8))
        loads.append(load)
    return max(loads) if loads else Fraction(0)


def check_cover(per_sm_segments, n_tiles: int, nb: int) -> None:
    """Every (tile, K-block) unit is covered exactly once (invariant I11)."""
    seen = {}
    for sm, segs in enumerate(per_sm_segments):
        for (tile, kb0, kb1) in segs:
            if not (0 <= tile < n_tiles and 0 <= kb0 < kb1 <= nb):
                raise AssertionError(f"bad segment {(tile, kb0, kb1)} on SM {sm}")
            for kb in range(kb0, kb1):
                if (tile, kb) in seen:
                    raise AssertionError(f"unit {(tile, kb)} covered twice")
                seen[(tile, kb)] = sm
    missing = n_tiles * nb - len(seen)
    if missing:
        raise AssertionError(f"{missing} units not covered")


def lower_bound(n_tiles: int, tags, n_sm: int, cost_int4, cost_int8) -> Fraction:
    """Perfect-balance bound: total cost / #SMs (what decomposition reaches, Fig. 8e)."""
    total = sum(Fraction(unit_cost(tags, kb, cost_int4, cost_int8)) for kb in range(len(tags)))
    return total * n_tiles / n_sm
