"""B200-native (sm_100a) Image-Domain Gridding hot path: plan / grid / degrid behind a C ABI.

Veenboer, Petschow, Romein, "Image-Domain Gridding on Graphics Processors", IPDPS 2017.
The product is libidg_b200.so (include/idg.h); this package is its ctypes binding plus the
multi-GPU sharding glue (torch.distributed, NCCL).  No CPU fallback exists.
"""
from .idg import (IDGError, METADATA_DTYPE, Plan, adder_workspace, degrid, degrid_bands, degrid_host,
                  degrid_host_splitter, grid, grid_bands, grid_host, grid_host_adder, ipc_close, ipc_handle, ipc_open,
                  kernel_variants, last_variant, launch_count, lib, profiling_enable, profiling_read, profiling_reset,
                  rho_benchmark, workspace)

__all__ = ["IDGError", "METADATA_DTYPE", "Plan", "adder_workspace", "degrid", "degrid_bands", "degrid_host",
           "degrid_host_splitter", "grid", "grid_bands", "grid_host", "grid_host_adder", "ipc_close", "ipc_handle",
           "ipc_open", "kernel_variants", "last_variant", "launch_count", "lib", "profiling_enable", "profiling_read",
           "profiling_reset", "rho_benchmark", "workspace"]
