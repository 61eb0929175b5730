"""Gallatin on B200: device-side malloc/free over a concurrent vEB tree (sm_100a).

Python face of ``libgallatin.so`` (C-ABI in ``include/gallatin.h``; device
header ``include/gallatin/device.cuh``).  PAPER.md = "Gallatin: A
General-Purpose GPU Memory Manager" (McCoy & Pandey, PPoPP'24).  Importing the
package loads the CUDA library; there is no CPU fallback.
"""
from ._native import (  # noqa: F401
    GallatinError, Graph, Veb, declared_functions, gallatin_destroy, gallatin_drain, gallatin_free,
    gallatin_free_host, gallatin_init, gallatin_is_initialized, gallatin_malloc, gallatin_malloc_host,
    gallatin_probe, gallatin_replay, gallatin_reset, gallatin_snapshot, gallatin_stamp, gallatin_stats,
    gallatin_usable, gallatin_verify, gallatin_version, lib, oracle_params,
)

lib()  # fail loudly at import when the CUDA library is missing
