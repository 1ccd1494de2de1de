// arena.h — libswap-internal view of swap_arena (csrc/arena.cpp) used by the restore path.
#pragma once
#include <cstdint>

#include "../../include/swap.h"

namespace swarena {
bool contains(const swap_arena* a, uint64_t lo, uint64_t hi);  // [lo, hi) inside the arena's VA range
bool resident(const swap_arena* a);
int device(const swap_arena* a);
swap_status map_dev_range(swap_arena* a, uint64_t lo, uint64_t hi);  // maps the slabs covering [lo, hi)
}  // namespace swarena
