"""paper_conf_dac_0159layhrr24_b200 — B200-native DGR differentiable DAG-forest solver.

The product is ``libdgr.so`` (C ABI in ``include/dgr.h``, sm_100a kernels in ``csrc/``).
``dgr.py`` is the thin Python binding: argument marshalling only, every step of the
solver iteration runs in the CUDA kernels.  There is no CPU fallback: without the
extension or a GPU the binding raises.
"""
from .dgr import (BuiltForest, DgrError, Loss, Solver, Weights, build_forest, lib_path, load_library,  # noqa: F401
                  nccl_unique_id, partition, plan_info, torch_allreduce)

__all__ = ["Solver", "Weights", "Loss", "DgrError", "partition", "nccl_unique_id", "load_library", "lib_path", "plan_info",
           "build_forest", "BuiltForest", "torch_allreduce"]
