"""B200-native DASP SpMV hot path (Lu & Liu, SC'23): y = alpha*A*x + beta*y.

The product is ``libdasp.so`` (C-ABI in ``include/dasp.h``; sm_100a kernels in ``csrc/``).
``dasp`` is its argument-marshalling binding; ``multigpu`` is the row-slab NCCL mode.
"""
from .dasp import (DASP_VARIANT_CUDACORE, DASP_VARIANT_DEFAULT, DASP_VARIANT_MMA, DaspError, Plan,  # noqa: F401
                   dasp_partition_rows, dasp_plan_copy_array, dasp_plan_create, dasp_plan_create_device, dasp_plan_destroy,
                   dasp_plan_get_info, dasp_plan_read_timing, dasp_plan_set_timing, dasp_remap_columns,
                   dasp_spmv, dasp_spmv_host, dasp_spmv_scatter, dasp_version)
