"""B200-native moment-representation regularized LBM (MR-LBM).

Hot path: the fused per-timestep MR-LBM update (Alg. 2)
for D2Q9 / D3Q19 / D3Q27 x projective / recursive regularization, as
hand-written sm_100a CUDA behind the C-ABI library ``libmrlbm.so``
(``include/mrlbm.h``).  ``mrlbm`` is the thin ctypes binding; importing it
loads the native library and fails loudly if it is missing.
"""
__all__ = ["inputs", "configs", "roofline"]
