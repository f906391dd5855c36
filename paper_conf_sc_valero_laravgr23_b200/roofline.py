"""Performance model of the paper (eq 15, Tables 2-3) and the
byte / op accounting the bench reports against.

  MFLUPS_max = B_BW / (10^6 * B/F)                       eq 15
  B/F        = 2 Q w (ST, two lattices)  or  2 M w (MR)  Table 2
"""
from __future__ import annotations

Q_OF = {"D2Q9": 9, "D3Q19": 19, "D3Q27": 27}
M_OF = {"D2Q9": 6, "D3Q19": 10, "D3Q27": 10}
WORD = {"fp64": 8, "fp32": 4}


def bytes_per_lup(lattice: str, pattern: str = "MR", precision: str = "fp64") -> int:
    """Algorithmic HBM bytes per lattice update (Table 2): read + write of the state."""
    n = M_OF[lattice] if pattern == "MR" else Q_OF[lattice]
    return 2 * n * WORD[precision]


def mflups_max(bandwidth_bytes_per_s: float, lattice: str, pattern: str = "MR", precision: str = "fp64") -> float:
    """eq 15"""
    return bandwidth_bytes_per_s / (1e6 * bytes_per_lup(lattice, pattern, precision))


def memory_bytes(nodes: int, lattice: str, pattern: str = "MR", precision: str = "fp64", copies: int = 2) -> int:
    """Footprint of the state (two copies for both patterns)."""
    n = M_OF[lattice] if pattern == "MR" else Q_OF[lattice]
    return copies * nodes * n * WORD[precision]
