"""iBFS hot path on B200: joint bitwise traversal of i concurrent BFS instances.

Product API (all compute in libibfs.so, hand-written sm_100a CUDA; no CPU fallback):
  Graph.from_csr / Graph.from_edges  -> ibfs_load_csr / ibfs_load_edges
  Graph.plan                          -> ibfs_plan_groups  (outdegree-based GroupBy)
  Graph.run                           -> ibfs_run_ex       (depth rows + statistics)
  dist.run_sharded                    -> groups sharded over torch.distributed ranks
See include/ibfs.h and DESIGN.md.
"""
from ._build import build  # noqa: F401
from ._lib import IbfsError, load  # noqa: F401
from .graph import Graph, RunStats, use_torch_allocator  # noqa: F401

__all__ = ["Graph", "RunStats", "IbfsError", "build", "load", "use_torch_allocator"]
