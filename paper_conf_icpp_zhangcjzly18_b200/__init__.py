"""B200-native FFS-VA prepositive filter cascade (SDD + SNM + T-YOLO) — Python face of libffsva.so.

See include/ffsva.h for the C-ABI and DESIGN.md for the design. ``ffsva`` is the ctypes binding.
"""
from .ffsva import (  # noqa: F401
    Context, PreparedBatch, Stream, StreamDesc, Tyolo, Scheduler, FfsvaError, RESULT_DTYPE, STAT_NAMES, EXPORTS, lib,
    ffsva_open_stream, ffsva_set_reference, ffsva_snm_load, ffsva_filter_batch, ffsva_sdd_batch,
    ffsva_batch_prepare, ffsva_batch_launch, ffsva_batch_fetch, ffsva_batch_device_outputs, ffsva_batch_destroy,
    ffsva_get_reference, ffsva_stream_info, ffsva_stats_copy, ffsva_close, ffsva_kernel_launches, ffsva_version,
)
