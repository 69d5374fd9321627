"""B200-native SMIless co-optimisation hot path (exhaustive SLA-constrained min-cost plan search).

The product is the C-ABI library libsmiless.so (include/smiless.h): CUDA kernels for
sm_100a, one NVRTC-specialised evaluator per DAG.  `smiless` is its thin ctypes binding,
`dist` the multi-GPU driver (torch.distributed + NCCL for the final exchange only).
"""
from .smiless import (Planner, PlanResult, SmilessError, load_library, planner_for,  # noqa: F401
                      FLAG_NO_PRUNE, FLAG_ARRIVALS_ON_DEVICE, FLAG_FORCE_INT64, OK, INFEASIBLE)
