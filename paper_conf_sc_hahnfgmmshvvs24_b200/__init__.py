"""B200-native MDNorm + BinMD single-crystal TOF cross-section hot path (Hahn et al., SC'24 W).

The product is the C-ABI library libmdnorm.so (include/mdnorm.h); this package is its thin
Python binding (same function names) plus the multi-GPU shard plan / reduce (dist.py).
"""
from .mdnorm import (  # noqa: F401
    Grid, MdnError, MDN_ACC_F32, MDN_ACC_F64, MDN_PRIV_AUTO, MDN_PRIV_OFF, MDN_PRIV_ON,
    mdnorm_set_privatization, mdnorm_accumulation_paths,
    mdnorm_create_grid, mdnorm_destroy, mdnorm_set_instrument, mdnorm_set_flux,
    mdnorm_accumulate, mdnorm_accumulate_runs, binmd_accumulate, mdnorm_histograms,
    mdnorm_cross_section, mdnorm_reset, mdnorm_stats, mdn_last_error, mdn_version,
    mdnorm_set_pixel_krange, mdnorm_set_flux_tables, binmd_accumulate_err, mdnorm_error_histogram, mdnorm_cross_section_err,
    mdnorm_accumulate_matrices, binmd_accumulate_matrices, mdnorm_debug_trajectories,
    binmd_debug_bins, mdnorm_debug_compose, packed_histograms, mdn_divide,
    mdnorm_debug_set_max_slab, mdnorm_debug_last_launch, mdnorm_debug_flux_guess, binmd_box_bounds, binmd_accumulate_boxes,
)
from .dist import plan_shards, reduce_packed, reduce_scatter_packed, RankPlan  # noqa: F401
