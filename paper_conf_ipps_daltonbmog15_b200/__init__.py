"""B200-native merge-path sparse operations (Dalton et al., IPDPS 2015).

The product path is libmsp.so (hand-written sm_100a CUDA behind the C ABI
of include/msp.h); this package is its thin Python binding.  Importing it
loads the library and fails loudly if it has not been built.
"""
from ._lib import EXPORTS, MspError, lib  # noqa: F401
from .ops import (CsrTensor, SpAddPlan, SpGemmPlan, SpGemmRadixPlan, csr_check, gather_values, rebase_offsets, row_split,  # noqa: F401
                  set_operation, spadd, spadd_fused, spgemm, spmv, spmv_nnz_split, spmv_workspace_bytes, workspace)

from . import dist  # noqa: F401,E402

lib()
