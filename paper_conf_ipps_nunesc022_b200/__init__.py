"""B200-native (sm_100a) CSMV batched commit pipeline.

CSMV (Nunes, Castro, Romano, IPDPS 2022) is a client-server multi-versioned
STM for GPUs.  The hot path -- client transactions over K-version rings,
warp pre-validation, batched submission to a persistent shared-memory server,
client write-back and ordered GTS publication -- is one fused persistent
CUDA kernel behind the C ABI in include/csmv.h (libcsmv.so).  Python here is
argument marshalling (csmv.py), the paper's workload presets (workloads.py)
and the partitioned multi-GPU runner (partition.py).
"""
from .csmv import Store, Workload, CsmvError, lib, zipf_table  # noqa: F401
from . import workloads  # noqa: F401
