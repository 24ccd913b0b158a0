"""paper_conf_icdcs_dengr24_b200 — B200-native hot path of MEGA (Deng & Rao, ICDCS'24):
multi-head GAT attention over a traversal-reorganised exact graph layout.

The product is libmega.so (include/mega.h); this package is its thin binding.
"""
from .mega import (MEGA_BF16, MEGA_BWD_PHASE_DST, MEGA_BWD_PHASE_SRC, MEGA_F32, MEGA_FLAG_ELER_IN_CTX,  # noqa: F401
                   SLOPE, Layout, MegaError, lib, mega_abi_version, mega_gat_bwd, mega_gat_fwd,
                   mega_gat_workspace_bytes, mega_layout_bind_device, mega_layout_device_bytes, mega_layout_load,
                   mega_layout_save, mega_layout_stats_get, mega_layout_view_get, mega_preprocess, mega_project_bwd,
                   mega_project_fwd)
