"""B200-native hot path of Vista's Staged CNN feature transfer (Nakandala & Kumar, SIGMOD 2020).

The product is the C-ABI library libvista.so (include/vista.h): sm_100a tcgen05/TMA
implicit-GEMM conv + FC, tap, join/concat and LR kernels behind vista_plan /
vista_transfer / vista_train.  This package only holds that library's sources
(csrc/) and a thin ctypes binding (vista.py).
"""
from .vista import (ALEXNET, RESNET50, TAP_NAMES, VGG16, Vista, VistaError, lib, vista_avgpool, vista_conv2d,
                    vista_ingest, vista_join, vista_lrn, vista_maxpool, vista_nccl_unique_id, vista_shard_range, vista_tap,
                    torch_dist_allreduce)

__all__ = ["ALEXNET", "VGG16", "RESNET50", "TAP_NAMES", "Vista", "VistaError", "lib", "vista_conv2d", "vista_tap",
           "vista_maxpool", "vista_lrn", "vista_avgpool", "vista_ingest", "vista_shard_range",
           "vista_nccl_unique_id", "vista_join", "torch_dist_allreduce"]
