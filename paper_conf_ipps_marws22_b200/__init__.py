"""B200-native hot path of Adaptive SGD (Ma, Rusu, Wu, Sim, IPDPSW'22).

libasgd.so (csrc/, C ABI in include/asgd.h) holds every step of the path:
sm_100a CUDA kernels for the local SGD step and the merge, host C++ for the
scheduler and Alg. 1 / Alg. 2.  This package is the thin Python binding
(api.py) and the driver (train.py).  There is no CPU fallback: without the
built library (python -m paper_conf_ipps_marws22_b200.build) imports of the
binding raise.
"""
from . import api, train  # noqa: F401
from ._lib import AsgdError, LIB_PATH  # noqa: F401

__all__ = ["api", "train", "AsgdError", "LIB_PATH"]
