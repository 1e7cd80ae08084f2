"""B200-native (sm_100a) DGI pre-training hot path of Mars (ICPP'21).

The product is ``libmars.so`` (CUDA kernels + C ABI, ``include/mars.h``); this
package holds it and a thin ctypes binding (``mars.py``) with the ABI's names.
It never imports ``oracle/`` and has no CPU fallback.
"""
from .mars import (DGI, Graph, MarsError, MARS_BF16, MARS_FP32, PHASES, config_default,  # noqa: F401
                   corruption_samples,
                   debug_gemm, featurize, placer_create, Placer, ppo_create, Ppo, dgi_create, dp_connect, dp_export, dgi_export_activations, dgi_step, encode, free,
                   graph_export_csr, graph_load, graph_load_shard, graph_shard_info, lib,
                   nccl_get_unique_id, num_params, shard_attach, shard_connect,
                   shard_connect_local, shard_export, shard_partition, version, LIB_PATH, SIGNATURES)
