"""B200 (sm_100a) hmmsearch hot path: HMMER 3.0 MSV filter + Viterbi filter (Lazy-F).

Jiang & Ganesan, "Fine-Grained Acceleration of HMMER 3.0 via Architecture-aware
Optimization on Massively Parallel Processors", IPDPSW 2015.

The compute path is libhmg.so (C ABI, include/hmg.h; CUDA kernels under csrc/).
``hmg`` is its thin ctypes binding, ``dist`` the multi-GPU shard/gather layer,
``synth`` the seeded input generators.  Importing the package does not load the
library; the first call does, and fails loudly if it is missing.
"""
__all__ = ["hmg", "synth", "dist", "build"]
