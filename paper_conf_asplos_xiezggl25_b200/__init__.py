"""Frugal (ASPLOS '25) data-parallel training-step hot path, B200-native.

The product is the C-ABI library ``libfrugal.so`` (include/frugal.h) built from
``csrc/``; ``frugal.py`` is its thin ctypes binding.  ``workload.py`` is the
seeded input generator shared with the test oracle.  Nothing is imported
eagerly here so that importing the generator never loads the CUDA library.
"""
