"""B200-native explicit step of the non-gray phonon BTE (Heisler et al., IPDPS 2024).

The product is the C-ABI library ``libbte.so`` (CUDA, sm_100a) declared in
``include/bte.h``; :mod:`.bte` is its thin ctypes binding and :mod:`.inputs`
the seeded synthetic input generators.  Importing this package does not load
the CUDA library; ``from paper_conf_ipps_heislersdms24_b200 import bte`` does,
and fails loudly if it is missing.
"""
__all__ = ["bte", "inputs"]
