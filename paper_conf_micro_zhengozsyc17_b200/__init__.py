"""vp — a B200-native VersaPipe pipeline runtime (Zheng et al., MICRO-50 2017).

The product is ``csrc/`` (CUDA for sm_100a behind the C ABI in ``include/vp.h``,
built into ``libvp.so``) and the thin ctypes binding ``vp.py``.  Importing this
package is cheap; ``from paper_conf_micro_zhengozsyc17_b200 import vp`` loads the
native library and raises if it is missing (there is no CPU fallback).
"""
import os

# Coarse / fine / hybrid models run one persistent kernel per stage group, each in its
# own stream; they must map to distinct hardware queues to co-run (SURVEY §5 "Config").
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
