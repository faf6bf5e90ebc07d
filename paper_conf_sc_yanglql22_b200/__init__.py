"""B200-native WholeGraph mini-batch preparation (Yang et al., SC'22).

The hot path -- multi-hop neighbour sampling, append-unique and global gather
over a multi-GPU distributed shared memory -- runs in hand-written sm_100a CUDA
kernels behind the C ABI declared in include/wg.h (libwg.so).  This package is
the thin Python binding (argument marshalling) plus the batch pipeline.
"""

from ._lib import (LIB_PATH, WG_DSM_COL32, WG_DSM_CSR_REPLICATED, WG_DSM_HASHED, WG_DSM_PAD64,  # noqa: F401
                   WG_DSM_WHOLE_ROWS, WG_DSM_WIDE_HASH, WG_UNIQUE_COMPACT, WG_UNIQUE_DIRECT, WG_UNIQUE_WIDE, WgError,
                   lib)
from .dsm import DSM, ThreadAllgather, TorchDistAllgather, local_num_edges, shard_csr  # noqa: F401
from .pipeline import (MiniBatchLoader, MiniBatchPipeline, PreparedBatch, capacities, pack_inputs,  # noqa: F401
                       required_keys)
