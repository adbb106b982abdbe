"""gpuscout-b200: B200-native batched bottleneck attribution (GPUscout, SC-W 2023).

The product is the C-ABI library libgpuscout_b200.so (include/gpuscout_b200.h, sources in csrc/);
this package is its thin Python binding (binding.py), the text report (report.py) and the
multi-GPU orchestration (dist.py).
"""
from .binding import (GS_JOIN_CONSUMER, GS_JOIN_LINE, GS_JOIN_PC, GS_HIST_AUTO, GS_HIST_GLOBAL, GS_HIST_PRIVATE, GS_HIST_WINDOW, GS_HIST_PARTITION, RANKED_DTYPE, RULES,
                      SITE_DTYPE, Context, GsError, gs_attribute_counts, gs_attribute_samples, gs_detect, gs_load_sass,
                      gs_pack_samples, gs_rank_sites, gs_rank_sites_slice, gs_register_pressure, load_library)

__all__ = ["Context", "GsError", "load_library", "gs_load_sass", "gs_detect", "gs_pack_samples",
           "gs_attribute_samples", "gs_attribute_counts", "gs_rank_sites", "gs_rank_sites_slice", "gs_register_pressure", "SITE_DTYPE", "RANKED_DTYPE", "RULES", "GS_HIST_AUTO",
           "GS_HIST_GLOBAL", "GS_HIST_PRIVATE", "GS_HIST_WINDOW", "GS_HIST_PARTITION", "GS_JOIN_PC", "GS_JOIN_LINE", "GS_JOIN_CONSUMER"]
