"""B200-native MultiCL device-mapper search (Aji et al., IEEE CLUSTER 2015).

The product is ``libmcl.so`` (C ABI in ``include/mcl.h``); this package is its thin
binding plus the seeded workload generators. See DESIGN.md.
"""
from .mcl import (  # noqa: F401
    EXPORTED,
    MCL_E_CUDA,
    MCL_E_INVAL,
    MCL_E_NCCL,
    MCL_E_NOMEM,
    MCL_E_RANGE,
    MCL_OK,
    Mapper,
    MclError,
    load_library,
    mcl_comm_destroy,
    mcl_comm_init,
    mcl_comm_unique_id,
    mcl_device_sms,
    mcl_last_error_string,
    mcl_last_launch_info,
    mcl_map_queues,
    mcl_mapper_create,
    mcl_mapper_destroy,
    mcl_probe_int_rate,
    mcl_status_string,
    mcl_version,
)
