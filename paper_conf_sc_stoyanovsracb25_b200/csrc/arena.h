// arena.h — libswap-internal view of swap_arena (csrc/arena.cpp) used by the restore path.
#pragma once
#include <cstdint>

#include "../../include/swap.h"

namespace swarena {
uint64_t slab_bytes();
uint64_t n_slabs(const swap_arena* a);
uint64_t slab_size(const swap_arena* a, uint64_t i);
bool slab_mapped(const swap_arena* a, uint64_t i);
uint64_t mapped_bytes(const swap_arena* a);
uint64_t slab_of(const swap_arena* a, uint64_t dev);  // dev inside the arena
swap_status map_slab(swap_arena* a, uint64_t i);
swap_status unmap_slab(swap_arena* a, uint64_t i);  // no device work may still use the slab
bool contains(const swap_arena* a, uint64_t lo, uint64_t hi);  // [lo, hi) inside the arena's VA range
bool resident(const swap_arena* a);
int device(const swap_arena* a);
swap_status map_dev_range(swap_arena* a, uint64_t lo, uint64_t hi);  // maps the slabs covering [lo, hi)
}  // namespace swarena
