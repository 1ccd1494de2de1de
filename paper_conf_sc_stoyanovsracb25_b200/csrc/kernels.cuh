// kernels.cuh — device-side data movers of libswap (sm_100a). Internal header.
//
// One persistent kernel family moves bytes between HBM and the mapped pinned host image
// and computes the per-chunk checksum from the same registers (BASELINE.json north_star
// (a)+(b); SURVEY.md §2d K1 gather_ckpt, K2 scatter_restore, K3 verify_hbm):
//   GATHER      HBM -> host image, c_g stored into the manifest chunk record   (checkpoint)
//   SCATTER     host image -> HBM, c_g compared with the manifest               (restore)
//   HASH_STORE  HBM only, c_g stored      (copy-engine checkpoint's hash pass, K4)
//   HASH_CHECK  HBM only, c_g compared    (HBM verify pass K3; copy-engine restore's check)
// Work unit: a "segment" descriptor (32 B). CRC-32C chunks are split into segments of
// seg_bytes whose partial CRCs are combined by the last-arriving warp; XXH64 is not
// combinable, so an XXH64 segment is a whole chunk.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace swk {

struct SegDesc {
  uint64_t dev;    // device address of the segment's first byte
  uint64_t host;   // host (mapped, UVA) address of the segment's first byte in the image
  uint32_t bytes;  // segment length
  uint32_t chunk;  // global chunk index g
  uint32_t seg;    // index of this segment inside chunk g
  uint32_t nseg;   // number of segments of chunk g
};
static_assert(sizeof(SegDesc) == 32, "descriptor is 32 B");

struct DevStatus {
  unsigned long long n_bad, first_bad;          // fused check of the last restore
  unsigned long long hbm_n_bad, hbm_first_bad;  // HBM verify pass
  unsigned int ticket, pad;                     // work counter of the dynamic XXH64 lane kernel
};

enum Mode : int { GATHER = 0, SCATTER = 1, HASH_STORE = 2, HASH_CHECK = 3 };
enum Kind : int { KIND_NONE = 0, KIND_CRC32C = 1, KIND_XXH64 = 2 };

// CRC tables blob, built on the host by build_tables() and uploaded once per ctx.
constexpr int TAB_T16 = 0;          // [16][256] slicing-by-16: T_k[b] = F(0, b . 0^k)
constexpr int TAB_Z496 = 16 * 256;  // [4][256]  Z^496 applied to byte j of a register
constexpr int TAB_LANE = TAB_Z496 + 4 * 256;  // [32] x^(8*16*(31-l)) mod P
constexpr int TAB_X2N = TAB_LANE + 32;        // [32] x^(2^k) mod P
constexpr int TAB_HLANE = TAB_X2N + 32;       // [32] hash kernel: Z^(L1 - end_l) for the common segment length L1
constexpr int TAB_Z96N = TAB_HLANE + 32;       // [8][16] hash kernel: Z^96 of nibble v at position k
constexpr int ZS_N = 1024;
constexpr int TAB_ZS = TAB_Z96N + 128;         // [ZS_N] x^(8*m*seg) mod P: shift by m whole segments
constexpr int TAB_Z96B = TAB_ZS + ZS_N;        // [4][256] hash kernel (ZB variant): Z^96 of byte e at position k
constexpr int TAB_SLANE = TAB_Z96B + 4 * 256;  // [32] strand-staged hash kernel: Z^(L1 - ts_lane_end(L1, l))
constexpr int TAB_WORDS = TAB_SLANE + 32;
constexpr int TAB_SMEM_WORDS = TAB_LANE + 32;  // the part staged in shared memory

struct Params {
  const SegDesc* desc;
  uint32_t n_desc;
  uint32_t seg_bytes;            // CRC split size (all segments but a chunk's last)
  uint32_t* partial;             // [n_desc] partial F(0, segment)
  uint32_t* arrive;              // [n_chunks] arrival counters (kept at 0 between launches)
  uint64_t* cs_out;              // &chunk_record[0].c_g in the mapped manifest; stride 4 u64
  const uint64_t* cs_exp;        // same field, read for compares
  unsigned long long* n_bad;     // mismatch counter
  unsigned long long* first_bad; // atomicMin target
  const uint32_t* tables;        // TAB_WORDS words in device memory
  uint64_t chunk_bytes;          // C
  uint32_t zinit_c;              // Z^C(0xFFFFFFFF): the init term of a full chunk
  uint32_t xseg;                 // x^(8*seg_bytes) mod P
  uint32_t hlane_len;            // L1: the segment length TAB_HLANE was built for
  unsigned int* ticket;          // dynamic XXH64 lane kernel: chunk counter, zeroed before each launch
  const void* tmaps;             // [n_chunks] CUtensorMap of the strand-staged CRC kernel's tensor path, or null
  const unsigned long long* chunk_dev;  // [n_chunks] device address of chunk g's first byte (0: no map)
};

void build_tables(uint32_t* tab /* TAB_WORDS */, uint64_t common_seg_len, uint64_t seg_bytes);
// Quad-line geometry of the CRC-32C HBM hash kernel for a segment of `len` bytes: 8 strands (one per
// lane quad) of hash_strand(len) bytes (a multiple of 128); lane (q = lane/4, j = lane%4) owns the 32-B
// pieces at q*Ls + j*32 + t*128 that start inside its strand and the segment.
__host__ __device__ inline uint64_t hash_strand(uint64_t len) { return ((len + 7) / 8 + 127) / 128 * 128; }
// One past the lane's last byte (0 if the lane owns none).
__host__ __device__ inline uint64_t hash_lane_end(uint64_t len, int lane) {
  const uint64_t Ls = hash_strand(len), q = (uint64_t)(lane >> 2), j = (uint64_t)(lane & 3);
  const uint64_t s0 = q * Ls + j * 32;
  const uint64_t strand_end = (q + 1) * Ls < len ? (q + 1) * Ls : len;
  if (s0 >= strand_end) return 0;
  const uint64_t last = s0 + (strand_end - 1 - s0) / 128 * 128;
  return last + 32 < strand_end ? last + 32 : strand_end;
}
// Strand geometry of the strand-staged CRC-32C hash kernel: a segment of `len` bytes is cut into 32
// contiguous strands of ts_strand(len) bytes (a multiple of 16), one per lane; lane l owns
// [l*Ls, min((l+1)*Ls, len)). ts_lane_end = one past the lane's last byte (0 if it owns none).
__host__ __device__ inline uint64_t ts_strand(uint64_t len) { return ((len + 31) / 32 + 15) / 16 * 16; }
__host__ __device__ inline uint64_t ts_lane_end(uint64_t len, int lane) {
  const uint64_t Ls = ts_strand(len), a0 = (uint64_t)lane * Ls;
  if (a0 >= len) return 0;
  return a0 + Ls < len ? a0 + Ls : len;
}
// Its tensor path: one map per chunk (its whole extent inside the chunk: a scheduler swap-out releases a
// victim's VMM slabs group by group while later groups are still hashed, and a TMA load through a map whose
// tensor reaches into a released slab faults even if the box does not), chunk viewed as rows of L1/32 bytes
// (u8, row pitch L1/32), box {TS_S, 32}; map g at tmaps + 128 * g. out: n * 128 bytes (host); a chunk
// smaller than one row gets a zeroed map. Returns false if the driver entry point is missing or an encode
// fails (the kernel then takes per-lane bulk copies, or launch_hash the quad-line kernel).
constexpr int TS_S = 80;
bool encode_tmaps(void* out, const uint64_t* base, const uint64_t* bytes, int n, uint64_t L1);
uint32_t host_x2nmodp(uint64_t n, unsigned k, const uint32_t* x2n);
uint32_t host_multmodp(uint32_t a, uint32_t b);

// Launch mover kernel <mode, kind> with `grid` CTAs on `stream`.
cudaError_t launch_mover(int mode, int kind, const Params& p, int grid, cudaStream_t stream);
int mover_threads();
// Measures (once per device) where kernels' dynamic shared memory starts; the CRC hash kernel's table
// layout is derived from it. Called by swap_create.
cudaError_t probe_smem_base();
// Grid for the CRC HBM hash kernels: one CTA per SM (never more CTAs than segments).
int hash_grid(int sm_count, uint32_t n_desc);
size_t mover_smem_bytes(int kind);
// XXH64 HBM hash: one warp per chunk, chunk bytes TMA-streamed through a shared-memory ring.
bool hash_xxh_lane_ok(int sm_count, uint32_t n_desc);
cudaError_t launch_xxh_hash(int mode, const Params& p, int sm_count, cudaStream_t stream);
// XXH64 GATHER / SCATTER with the quad-per-chunk kernel (needs p.ticket); enabled unless SWAP_XXH_MOVER=warp.
bool xxh_quad_mover_enabled();
cudaError_t launch_xxh_move(int mode, const Params& p, int sm_count, cudaStream_t stream);

// Zero-fill of a span list (DISCARD regions and masked chunks on the device at restore; stale masked
// chunks of the mapped host image at checkpoint): one launch instead of one cudaMemsetAsync per span.
// dst must be 16-B aligned; bytes arbitrary (split into pieces of <= kZeroPiece by the host).
struct ZSpan {
  uint64_t dst, bytes;
};
constexpr uint64_t kZeroPiece = 1ull << 20;
cudaError_t launch_zero_fill(const ZSpan* spans, uint32_t n, int sm_count, cudaStream_t stream);

}  // namespace swk
