"""B200-native EGG-SynC synchronization update (Jorgensen & Assent, EDBT 2023).

The product is ``libeggsync.so`` (hand-written CUDA for sm_100a behind the C ABI
in include/eggsync.h).  This package holds its thin ctypes binding
(:mod:`.eggsync`), the multi-GPU driver (:mod:`.distributed`) and the seeded
input generator (:mod:`.datagen`).  Importing the package does not load the
library; the first call does, and fails loudly if it is missing.
"""
from .eggsync import (EggSyncError, Context, cluster, step, sync_step, sync_lambda, lib, last_error,  # noqa: F401
                      OK, NOT_CONVERGED, EINVAL, EDOMAIN, ENOMEM, ECUDA, ENCCL, MAX_D)

__all__ = ["EggSyncError", "Context", "cluster", "step", "sync_step", "sync_lambda", "lib", "last_error"]
