"""B200-native cuMF_SGD hot path (Xie, Tan, Fong, Liang, HPDC'17).

The compute path is libmf_b200.so (C ABI, include/mf.h); ``mf.py`` is its ctypes binding.
Importing the package does not load the library; ``paper_conf_hpdc_xietfl17_b200.mf`` does.
"""
__all__ = ["mf", "synth"]
