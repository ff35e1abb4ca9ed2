"""mpx — model-driven multi-path GPU→GPU transfers on B200 (Sojoodi et al., SC-W '25).

The product is libmpx.so (include/mp.h): a host C++ model evaluator / Algorithm 1
selector and hand-written sm_100a transfer kernels.  ``mp`` is the thin ctypes
binding; ``dist`` bootstraps multi-rank contexts over torch.distributed.
"""
from .mp import (Context, MPError, lib, MP_PATH_DIRECT, MP_PATH_GPU, MP_PATH_HOST,  # noqa: F401
                 MP_MODEL_PAPER, MP_MODEL_B200)
