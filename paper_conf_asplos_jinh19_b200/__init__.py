"""B200-native Split-CNN split window operators (Jin & Hong, ASPLOS'19).

The product is ``libsplitcnn.so`` (C ABI in ``include/splitcnn.h``, CUDA kernels for
sm_100a in ``csrc/``).  ``splitcnn`` is the thin ctypes binding (same names as the C
calls), ``plan.SplitPlan`` caches plan geometry, ``net.SplitNet`` runs a split VGG/ResNet
conv stack through the library.  Importing ``splitcnn`` fails loudly if the library is not
built: there is no CPU fallback.
"""
__all__ = ["splitcnn", "plan", "net"]
