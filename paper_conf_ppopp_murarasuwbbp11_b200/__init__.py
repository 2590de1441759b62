"""B200-native compact sparse grids (Murarasu et al., PPoPP'11): compression
(hierarchization) and the decompression hot path (batched evaluation) as
hand-written sm_100a CUDA kernels behind the C ABI ``include/sg.h``.

Importing this package loads ``libsg.so`` (built in-tree by
``python -m paper_conf_ppopp_murarasuwbbp11_b200.build``); there is no CPU
fallback.
"""
from ._sg import (SG_EVAL_PRESORTED, SG_F32, SG_F64, SgError, sg_build_info, sg_create, sg_destroy,  # noqa: F401
                  sg_evaluate, sg_evaluate_host, sg_evaluate_workspace_bytes, sg_get_layout, sg_gp2idx,
                  sg_gp2idx_device, sg_grid_coords_device, sg_hierarchize, sg_idx2gp, sg_idx2gp_device,
                  sg_kernel_launch_count, sg_profile_enable, sg_profile_read, sg_sfc_order, sg_evaluate_ordered, sg_evaluate_plane,
                  sg_plane_workspace_bytes, sg_part_bounds, sg_evaluate_part)
from .grid import BoundaryGrid, Grid  # noqa: F401
from .multi import evaluate_distributed, evaluate_sharded_grid, partition  # noqa: F401
