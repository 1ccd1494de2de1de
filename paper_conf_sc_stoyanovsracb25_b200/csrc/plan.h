// plan.h — host-side image planning, manifest and shard summary (libswap internal).
//
// Implements the image format DESIGN.md §"Image and manifest" fixes (SURVEY.md §8(c) steps
// 1-3, 6, 7): registration-order layout with A-aligned offsets, per-region chunks of C bytes,
// a little-endian manifest with a trailing CRC-32C, and the 64-B shard summary. Written
// independently of oracle/ (which the tests compare it against).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../../include/swap.h"

namespace swp {

struct RegionPlan {
  swap_region_t r;
  uint64_t off;      // image offset
  uint64_t first;    // global index of its first chunk
  uint64_t nchunks;  // ceil(bytes / C)
};

struct Plan {
  uint32_t kind = 0;
  uint64_t C = 0, A = 0;
  uint32_t rank = 0, world = 1;
  std::vector<RegionPlan> regions;
  uint64_t payload_bytes = 0, n_chunks = 0;
  uint64_t manifest_off = 0, manifest_bytes = 0, image_bytes = 0;
  mutable std::vector<uint8_t> skeleton;  // cached static manifest bytes (c_g = 0, no trailer) for checks
};

constexpr uint64_t kHeaderBytes = 64, kRegionRecBytes = 48, kChunkRecBytes = 32, kTrailerBytes = 8;

// Fills defaults (0 -> default) and validates the config.
swap_status normalize_config(swap_config_t* cfg, std::string* err);
// Validates the table in the documented order and computes the layout.
swap_status build_plan(const swap_region_t* regions, size_t n, const swap_config_t& cfg, Plan* out,
                       std::string* err);
// Writes header, region records and the static fields of every chunk record (c_g = 0).
void write_manifest_skeleton(const Plan& p, uint8_t* man);
// Writes the trailing CRC-32C over the preceding manifest bytes; returns it.
uint32_t seal_manifest(const Plan& p, uint8_t* man);
// 1 if the manifest CRC holds and the manifest describes exactly this plan.
swap_status check_manifest(const Plan& p, const uint8_t* man, std::string* err);
bool manifest_crc_ok(const Plan& p, const uint8_t* man);
void make_summary(const Plan& p, const uint8_t* man, swap_shard_summary_t* out);

// Host CRC-32C, standard init/xorout: SSE4.2 crc32 instruction (3 interleaved streams) when present,
// else slicing-by-8.
uint32_t crc32c_host(const void* data, size_t n, uint32_t crc = 0);

}  // namespace swp
