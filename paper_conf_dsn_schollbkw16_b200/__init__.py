"""B200-native ABFT-SpMV with implicit error localization (Schoell et al.,
DSN 2016).  The compute path is libabft.so (include/abft.h, sm_100a CUDA);
this package is its thin binding plus the seeded input generators."""
from .abft import (AUTOCORRECT, CHECK, DEBUG_CHECKSUMS, NOCHECK, AbftError, CsrDevice, Dist,
                   DistHandle, Handle, Inject, burst_table, dist_unique_id, encode, halo_plan, lib,
                   lib_path)

__all__ = ["encode", "Handle", "CsrDevice", "Inject", "AbftError", "lib", "lib_path",
           "burst_table", "CHECK", "NOCHECK", "AUTOCORRECT", "DEBUG_CHECKSUMS", "Dist",
           "DistHandle", "dist_unique_id", "halo_plan"]
