"""Seeded synthetic INPUT generators shared by the oracle side and the CUDA side.

This package holds none of XPlacer's arithmetic (no shadow records, no
diagnosis): it only produces event traces -- allocations, host and device
accesses, transfers, epoch boundaries and diagnose points -- in the shapes of
the paper's workloads.  Both `oracle/` and the CUDA path
consume the same traces; neither imports the other.
"""
