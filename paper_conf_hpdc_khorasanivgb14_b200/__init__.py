"""B200-native CuSha shard-processing path (Khorasani et al., HPDC'14).

The product is ``libcusha.so`` (C ABI in ``include/cusha.h``; CUDA sources in
``csrc/``); ``cusha`` is its thin Python binding.  Build with
``python -m paper_conf_hpdc_khorasanivgb14_b200.build``.
"""
from . import cusha  # noqa: F401

__all__ = ["cusha"]
