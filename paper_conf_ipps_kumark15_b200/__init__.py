"""B200-native LDDP-Plus table fill (Kumar & Kothapalli, IPDPSW 2015).

The product is the C-ABI library ``liblddp.so`` (include/lddp.h, csrc/); ``lddp`` is its thin
ctypes binding.  Importing this package does not load the library; ``from
paper_conf_ipps_kumark15_b200 import lddp`` does, and fails loudly if it is missing.
"""

__all__ = ["lddp", "inputs"]
