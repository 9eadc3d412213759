"""B200-native Stokes-FO (Blatter-Pattyn) residual + forward-AD Jacobian cell
evaluator: the hot path Antepara et al. (SC-W '24) profile in MALI/Albany,
rebuilt as hand-written sm_100a CUDA behind a C ABI (include/stokesfo.h).

    stokesfo  -- ctypes binding of libstokesfo.so (same names as the C ABI)
    synth     -- seeded synthetic footprints and fields (inputs only)
    halo      -- torch.distributed plumbing for the multi-GPU halo sum
    build     -- in-tree nvcc build for sm_100a
"""
from .stokesfo import (StokesFO, StokesFOError, mesh_extrude, mesh_halo_list, mesh_localize,  # noqa: F401
                       mesh_lateral_faces, mesh_partition_columns)
