"""B200-native PDL-mapped blocked matmul (Sandrieser, Benkner, Pllana, IPDPS 2011).

``pdl``     -- ctypes binding of libpdl.so (pdl_load / task_matmul / pdl_run / pdl_query).
``runtime`` -- one-process-per-GPU driver: BLOCK plan from libpdl, operand-panel
               exchange over torch.distributed (NCCL on NVLink), local task via libpdl.
"""
from . import pdl  # noqa: F401  (fails loudly if libpdl.so is missing)

__all__ = ["pdl"]
