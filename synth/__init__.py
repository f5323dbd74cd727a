"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the method (no stencil, no sin/cos
iteration, no ghost logic). It only produces input grids, following the input
recipe in DESIGN.md §3 (SURVEY.md §8(c) "Input generator"):

    splitmix64(z): z += 0x9E3779B97F4A7C15; z = (z ^ z>>30) * 0xBF58476D1CE4E5B9;
                   z = (z ^ z>>27) * 0x94D049BB133111EB; return z ^ z>>31
    u0[gidx] = (splitmix64(gidx + seed*0x9E3779B97F4A7C15) >> 11) * 2^-53
    gidx = (z*ny + y)*nx + x over the GLOBAL grid

Values are U[0,1) doubles, position-addressable, so any sub-block (a tile, a
z-slab of one rank, a cone-oracle neighbourhood) can be regenerated on its own.
A second, independent C implementation of the same counter-based generator
lives in synth/splitmix.c (multi-threaded, for grids of tens of GB).
"""
from .splitmix import (GOLDEN_GAMMA, splitmix64, uniform_at, uniform_grid,
                       uniform_block, constant_grid, linear_grid, sine_grid,
                       sine_grid_dirichlet, fill_uniform_native)

__all__ = ["GOLDEN_GAMMA", "splitmix64", "uniform_at", "uniform_grid",
           "uniform_block", "constant_grid", "linear_grid", "sine_grid",
           "sine_grid_dirichlet", "fill_uniform_native"]
