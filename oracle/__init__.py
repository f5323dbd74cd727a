"""oracle/ — TEST INFRASTRUCTURE ONLY (not part of the product path).

Plain, slow, obviously-correct CPU implementations of what the tiled GPU path
computes, written from PAPER.md (Bastem et al., ICPP 2017). Only `tests/`,
`__graft_entry__.smoke()` and `bench.py` (its `cpu_baseline` leg and
`--impl reference`) may import this package. It never imports the product
package `paper_conf_icpp_bastemuzas17_b200`, and the product never imports it.

Contents (each function cites the passage it follows):
  heat_c / heat_np        untiled fp64 Jacobi heat step (reading R1)
  sincos_c / sincos_py    compute-intensive kernel listing
  ghost_map               brute-force ghost-source map of one tile
  tiled_heat              heat on tiles with ghost shells built from ghost_map
  cone_block              exact sub-block of a huge run (dependency cone)
  ResidencyOracle         the cache-list state machine of P:L88-L90
Pins (tests/test_oracle.py, -m "not gpu"): closed forms (constant, linear,
sine eigenmodes, delta Green's function), invariants (shift, reflections,
transpose, conservation, max principle), tiled == untiled, brute force.
"""
from .oracle import (BC_PERIODIC, BC_DIRICHLET, heat_c, heat_np, sincos_c,
                     sincos_py, ghost_map, tiled_heat, cone_block,
                     ResidencyOracle, lib_path, build)

__all__ = ["BC_PERIODIC", "BC_DIRICHLET", "heat_c", "heat_np", "sincos_c",
           "sincos_py", "ghost_map", "tiled_heat", "cone_block",
           "ResidencyOracle", "lib_path", "build"]
