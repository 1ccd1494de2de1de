// plan.cpp — see plan.h. Validation order (include/swap.h): null/arg -> config -> alignment
// -> overlap -> duplicate id. Overlap and duplicate checks sort (O(n log n)).
#include "plan.h"

#include <algorithm>
#include <cstring>
#if defined(__x86_64__)
#include <cpuid.h>
#include <nmmintrin.h>
#endif

namespace swp {

namespace {
bool pow2_ge(uint64_t v, uint64_t lo) { return v >= lo && (v & (v - 1)) == 0; }
uint64_t round_up(uint64_t v, uint64_t a) { return (v + a - 1) & ~(a - 1); }

inline void le32(uint8_t* p, uint32_t v) { std::memcpy(p, &v, 4); }  // x86-64 / aarch64: little-endian
inline void le64(uint8_t* p, uint64_t v) { std::memcpy(p, &v, 8); }
inline uint32_t rd32(const uint8_t* p) {
  uint32_t v;
  std::memcpy(&v, p, 4);
  return v;
}
inline uint64_t rd64(const uint8_t* p) {
  uint64_t v;
  std::memcpy(&v, p, 8);
  return v;
}

struct Crc8Tables {
  uint32_t t[8][256];
  Crc8Tables() {
    for (uint32_t b = 0; b < 256; ++b) {
      uint32_t c = b;
      for (int k = 0; k < 8; ++k) c = (c >> 1) ^ (0x82F63B78u & (0u - (c & 1u)));
      t[0][b] = c;
    }
    for (int k = 1; k < 8; ++k)
      for (uint32_t b = 0; b < 256; ++b) t[k][b] = (t[k - 1][b] >> 8) ^ t[0][t[k - 1][b] & 0xFF];
  }
};
const Crc8Tables& crc_tables() {
  static const Crc8Tables T;
  return T;
}
}  // namespace

#if defined(__x86_64__)
bool have_crc32_insn() {
  static const bool ok = [] {
    unsigned a, b, c, d;
    return __get_cpuid(1, &a, &b, &c, &d) && (c & bit_SSE4_2);
  }();
  return ok;
}
// The SSE4.2 crc32 instruction implements the CRC-32C register update; three independent streams
// hide its 3-cycle latency and are merged with the GF(2) shift (crc_shift_bytes below).
uint32_t crc_shift_bytes(uint32_t c, uint64_t n);
__attribute__((target("sse4.2"))) uint32_t crc32c_hw(const uint8_t* p, size_t n, uint32_t c32) {
  uint64_t c = c32;
  if (n >= 3 * 4096) {
    const size_t blk = n / 3 / 8 * 8;
    uint64_t c1 = 0, c2 = 0;
    const uint8_t* q1 = p + blk;
    const uint8_t* q2 = p + 2 * blk;
    for (size_t i = 0; i < blk; i += 8) {
      uint64_t w0, w1, w2;
      std::memcpy(&w0, p + i, 8);
      std::memcpy(&w1, q1 + i, 8);
      std::memcpy(&w2, q2 + i, 8);
      c = _mm_crc32_u64(c, w0);
      c1 = _mm_crc32_u64(c1, w1);
      c2 = _mm_crc32_u64(c2, w2);
    }
    // register after stream 0 then stream 1 then stream 2 (streams 1, 2 started from 0: linearity)
    c = crc_shift_bytes((uint32_t)c, blk) ^ (uint32_t)c1;
    c = crc_shift_bytes((uint32_t)c, blk) ^ (uint32_t)c2;
    p += 3 * blk;
    n -= 3 * blk;
  }
  for (; n >= 8; n -= 8, p += 8) {
    uint64_t w;
    std::memcpy(&w, p, 8);
    c = _mm_crc32_u64(c, w);
  }
  uint32_t r = (uint32_t)c;
  for (; n; --n) r = _mm_crc32_u8(r, *p++);
  return r;
}
#endif

// Z^n (n zero bytes) of a register: square-and-multiply with x^(2^k) mod P, reflected.
uint32_t gf2_mul(uint32_t a, uint32_t b) {
  uint32_t p = 0;
  for (int i = 0; i < 32; ++i) {
    if ((a >> (31 - i)) & 1u) p ^= b;
    b = (b & 1u) ? (b >> 1) ^ 0x82F63B78u : (b >> 1);
  }
  return p;
}
uint32_t crc_shift_bytes(uint32_t c, uint64_t n) {
  static const std::vector<uint32_t> x2n = [] {
    std::vector<uint32_t> t(64);
    t[0] = 1u << 30;  // x^1
    for (int k = 1; k < 64; ++k) t[k] = gf2_mul(t[k - 1], t[k - 1]);
    return t;
  }();
  uint32_t x = 1u << 31;  // x^0
  for (unsigned k = 3; n; n >>= 1, ++k)
    if (n & 1) x = gf2_mul(x2n[k & 63], x);
  return gf2_mul(x, c);
}

uint32_t crc32c_host(const void* data, size_t n, uint32_t crc) {
#if defined(__x86_64__)
  if (have_crc32_insn()) return ~crc32c_hw(static_cast<const uint8_t*>(data), n, ~crc);
#endif
  const auto& T = crc_tables().t;
  const uint8_t* p = static_cast<const uint8_t*>(data);
  uint32_t c = ~crc;
  while (n && (reinterpret_cast<uintptr_t>(p) & 7)) {
    c = T[0][(c ^ *p++) & 0xFF] ^ (c >> 8);
    --n;
  }
  while (n >= 8) {
    uint64_t w = rd64(p) ^ c;
    c = T[7][w & 0xFF] ^ T[6][(w >> 8) & 0xFF] ^ T[5][(w >> 16) & 0xFF] ^ T[4][(w >> 24) & 0xFF] ^
        T[3][(w >> 32) & 0xFF] ^ T[2][(w >> 40) & 0xFF] ^ T[1][(w >> 48) & 0xFF] ^ T[0][w >> 56];
    p += 8;
    n -= 8;
  }
  while (n--) c = T[0][(c ^ *p++) & 0xFF] ^ (c >> 8);
  return ~c;
}

static_assert(sizeof(swap_config_t) == 56, "swap_config_t layout (include/swap.h)");

swap_status normalize_config(swap_config_t* c, std::string* err) {
  if (c->chunk_bytes == 0) c->chunk_bytes = 1ull << 20;
  if (c->align == 0) c->align = 4096;
  if (c->checksum == 0) c->checksum = SWAP_CHECKSUM_CRC32C;
  if (!pow2_ge(c->chunk_bytes, 16) || !pow2_ge(c->align, 16)) {
    *err = "chunk_bytes and align must be powers of 2 >= 16";
    return SWAP_EINVAL;
  }
  if (c->checksum != SWAP_CHECKSUM_CRC32C && c->checksum != SWAP_CHECKSUM_XXH64) {
    *err = "checksum must be SWAP_CHECKSUM_CRC32C or SWAP_CHECKSUM_XXH64";
    return SWAP_EINVAL;
  }
  if (c->mechanism >= SWAP_MECH_COUNT) {
    *err = "unknown mechanism";
    return SWAP_EINVAL;
  }
  if (c->world < 1 || c->rank < 0 || c->rank >= c->world || c->device < 0) {
    *err = "need world >= 1, 0 <= rank < world, device >= 0";
    return SWAP_EINVAL;
  }
  if (c->seg_bytes != 0 && !pow2_ge(c->seg_bytes, 4096)) {
    *err = "seg_bytes must be 0 (auto) or a power of 2 >= 4096";
    return SWAP_EINVAL;
  }
  if (c->host_numa < -1) {
    *err = "host_numa must be 0 (auto), -1 (none) or node + 1";
    return SWAP_EINVAL;
  }
  if (c->chunk_bytes > (1ull << 31)) {
    *err = "chunk_bytes > 2 GiB is not supported by the movers";
    return SWAP_EUNSUPPORTED;
  }
  return SWAP_OK;
}

swap_status build_plan(const swap_region_t* regions, size_t n, const swap_config_t& cfg, Plan* out,
                       std::string* err) {
  if (!regions || n == 0 || n > 0xFFFFFFFFull) {
    *err = "need 1 <= n <= 2^32-1 regions";
    return SWAP_EINVAL;
  }
  for (size_t i = 0; i < n; ++i)
    if (regions[i].kind > SWAP_KIND_OTHER) {
      *err = "region kind must be 0..3";
      return SWAP_EINVAL;
    }
  for (size_t i = 0; i < n; ++i) {
    if (regions[i].dev_addr % 16) {
      *err = "region " + std::to_string(i) + " dev_addr is not 16-B aligned";
      return SWAP_EINVAL;
    }
    if (regions[i].bytes && regions[i].bytes - 1 > UINT64_MAX - regions[i].dev_addr) {
      *err = "region " + std::to_string(i) + " wraps the address space";
      return SWAP_EINVAL;
    }
  }
  std::vector<size_t> order;
  for (size_t i = 0; i < n; ++i)
    if (regions[i].bytes) order.push_back(i);
  std::sort(order.begin(), order.end(),
            [&](size_t a, size_t b) { return regions[a].dev_addr < regions[b].dev_addr; });
  for (size_t k = 1; k < order.size(); ++k) {
    const auto& a = regions[order[k - 1]];
    if (regions[order[k]].dev_addr - a.dev_addr < a.bytes) {
      *err = "regions " + std::to_string(order[k - 1]) + " and " + std::to_string(order[k]) + " overlap";
      return SWAP_EINVAL;
    }
  }
  std::vector<uint32_t> ids(n);
  for (size_t i = 0; i < n; ++i) ids[i] = regions[i].id;
  std::sort(ids.begin(), ids.end());
  if (std::adjacent_find(ids.begin(), ids.end()) != ids.end()) {
    *err = "duplicate region id";
    return SWAP_EINVAL;
  }

  Plan p;
  p.kind = cfg.checksum;
  p.C = cfg.chunk_bytes;
  p.A = cfg.align;
  p.rank = (uint32_t)cfg.rank;
  p.world = (uint32_t)cfg.world;
  p.regions.resize(n);
  uint64_t cursor = 0, chunk = 0;
  for (size_t i = 0; i < n; ++i) {
    RegionPlan& rp = p.regions[i];
    rp.r = regions[i];
    rp.off = i == 0 ? 0 : round_up(cursor, p.A);
    rp.first = chunk;
    rp.nchunks = (rp.r.bytes + p.C - 1) / p.C;
    cursor = rp.off + rp.r.bytes;
    chunk += rp.nchunks;
  }
  if (chunk > 0xFFFFFFFFull) {
    *err = "more than 2^32-1 chunks";
    return SWAP_EUNSUPPORTED;
  }
  p.payload_bytes = cursor;
  p.n_chunks = chunk;
  p.manifest_off = round_up(p.payload_bytes, p.A);
  p.manifest_bytes = kHeaderBytes + kRegionRecBytes * n + kChunkRecBytes * p.n_chunks + kTrailerBytes;
  p.image_bytes = p.manifest_off + p.manifest_bytes;
  *out = std::move(p);
  return SWAP_OK;
}

void write_manifest_skeleton(const Plan& p, uint8_t* man) {
  std::memset(man, 0, p.manifest_bytes);
  std::memcpy(man, "SWAPMAN1", 8);
  le32(man + 8, 1);
  le32(man + 12, p.kind);
  le64(man + 16, p.C);
  le64(man + 24, p.A);
  le64(man + 32, p.regions.size());
  le64(man + 40, p.n_chunks);
  le64(man + 48, p.payload_bytes);
  le32(man + 56, p.rank);
  le32(man + 60, p.world);
  uint8_t* rr = man + kHeaderBytes;
  uint8_t* cr = rr + kRegionRecBytes * p.regions.size();
  for (size_t i = 0; i < p.regions.size(); ++i) {
    const RegionPlan& r = p.regions[i];
    uint8_t* q = rr + kRegionRecBytes * i;
    le32(q, r.r.id);
    le32(q + 4, r.r.kind);
    le64(q + 8, r.r.dev_addr);
    le64(q + 16, r.r.bytes);
    le64(q + 24, r.off);
    le64(q + 32, r.first);
    le64(q + 40, r.nchunks);
    for (uint64_t j = 0; j < r.nchunks; ++j) {
      uint8_t* c = cr + kChunkRecBytes * (r.first + j);
      const uint64_t lo = j * p.C;
      le32(c, (uint32_t)i);
      le64(c + 8, lo);
      le64(c + 16, std::min<uint64_t>(p.C, r.r.bytes - lo));
    }
  }
}

uint32_t seal_manifest(const Plan& p, uint8_t* man) {
  const uint32_t c = crc32c_host(man, p.manifest_bytes - kTrailerBytes);
  le64(man + p.manifest_bytes - kTrailerBytes, c);
  return c;
}

bool manifest_crc_ok(const Plan& p, const uint8_t* man) {
  return rd64(man + p.manifest_bytes - kTrailerBytes) == crc32c_host(man, p.manifest_bytes - kTrailerBytes);
}

swap_status check_manifest(const Plan& p, const uint8_t* man, std::string* err) {
  if (!manifest_crc_ok(p, man)) {
    *err = "manifest CRC-32C mismatch";
    return SWAP_ECORRUPT;
  }
  // The CRC holds: the manifest must also describe this ctx's registered layout.
  if (p.skeleton.size() != p.manifest_bytes) {
    p.skeleton.resize(p.manifest_bytes);
    write_manifest_skeleton(p, p.skeleton.data());
  }
  const std::vector<uint8_t>& want = p.skeleton;
  const uint64_t chunk_base = kHeaderBytes + kRegionRecBytes * p.regions.size();
  if (std::memcmp(want.data(), man, chunk_base) != 0) {
    *err = "manifest header/regions do not match the registered layout";
    return SWAP_ECORRUPT;
  }
  for (uint64_t g = 0; g < p.n_chunks; ++g)
    if (std::memcmp(want.data() + chunk_base + kChunkRecBytes * g, man + chunk_base + kChunkRecBytes * g, 24) != 0) {
      *err = "manifest chunk table does not match the registered layout";
      return SWAP_ECORRUPT;
    }
  return SWAP_OK;
}

void make_summary(const Plan& p, const uint8_t* man, swap_shard_summary_t* s) {
  std::memset(s, 0, sizeof(*s));
  s->rank = p.rank;
  s->world = p.world;
  s->checksum = p.kind;
  s->n_regions = (uint32_t)p.regions.size();
  s->n_chunks = p.n_chunks;
  s->payload_bytes = p.payload_bytes;
  s->image_bytes = p.image_bytes;
  s->manifest_crc = rd64(man + p.manifest_bytes - kTrailerBytes);
  const uint8_t* cr = man + kHeaderBytes + kRegionRecBytes * p.regions.size();
  uint32_t c = 0;
  for (uint64_t g = 0; g < p.n_chunks; ++g) c = crc32c_host(cr + kChunkRecBytes * g + 24, 8, c);
  s->chunk_digest = c;
}

}  // namespace swp
