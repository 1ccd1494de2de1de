"""B200-native swap-image engine: the data path of SwapServeLLM's model hot-swap.

Checkpoint gathers an inference engine's registered GPU allocations into a packed, pinned
host image with per-chunk CRC-32C/XXH64 checksums and a region manifest; restore scatters
it back to the recorded addresses and verifies it (§4.2, L203 §5.3). The
work runs in libswap.so (C ABI in include/swap.h, CUDA kernels for sm_100a); this package
is the ctypes binding (`swap`) and the multi-GPU coordinator (`dist`).
"""
from .swap import (  # noqa: F401
    MECHANISMS,
    SWAP_CHECKSUM_CRC32C,
    SWAP_CHECKSUM_XXH64,
    SwapError,
    Swapper,
    load,
)

__all__ = ["Swapper", "SwapError", "load", "MECHANISMS", "SWAP_CHECKSUM_CRC32C", "SWAP_CHECKSUM_XXH64"]
