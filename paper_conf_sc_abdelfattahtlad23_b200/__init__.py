"""B200-native batched band LU with partial pivoting (dgbtrf) and banded
solve (dgbtrs / dgbsv), after Abdelfattah et al., SC-W 2023.

The product is libbandlu.so (C ABI, include/bandlu.h; sm_100a CUDA kernels in
csrc/).  ``binding`` marshals torch CUDA tensors into it; ``inputs`` is the
seeded synthetic workload generator.  Nothing here imports oracle/.
"""
from .binding import (AUTO, COLS, GENERIC, ROWS, TC, THIN, THREAD, TPM, WINDOW, BandLUError, dgbsv_batched, dgbsv_strided_batched,  # noqa: F401
                      dgbsv_strided_batched_host, dgbtrf_batched, dgbtrf_strided_batched, dgbtrfs_strided_batched, dgbtrs_batched,
                      dgbtrs_strided_batched, load, ptr_array, rows_available, tc_available, thread_available, tpm_available, thin_available, cols_available, jit_band, jit_check, trf_variant, trs_rows_available,
                      trs_variant, trfs_plan, TRFS_TWO_LAUNCH, TRFS_FUSED, TRFS_THIN)

__all__ = ["dgbtrf_strided_batched", "dgbtrfs_strided_batched", "dgbtrs_strided_batched", "dgbsv_strided_batched", "dgbtrf_batched",
           "dgbtrs_batched", "dgbsv_batched", "dgbsv_strided_batched_host", "ptr_array", "load",
           "trf_variant", "trs_variant", "trfs_plan", "TRFS_TWO_LAUNCH", "TRFS_FUSED", "tc_available", "rows_available", "thread_available", "THREAD", "TPM", "THIN", "thin_available", "COLS", "cols_available", "TRFS_THIN", "tpm_available", "jit_band", "jit_check", "trs_rows_available", "AUTO", "ROWS", "GENERIC", "WINDOW", "TC", "BandLUError"]
