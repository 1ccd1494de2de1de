// kernels.cu — libswap's sm_100a data movers (see kernels.cuh for the mode list).
//
// Design:
//  * Persistent grid (2 CTAs x 512 threads per SM). A CTA takes WARPS consecutive segment
//    descriptors per round; thread 0 stages them into shared memory with a TMA bulk copy
//    (cp.async.bulk + mbarrier complete_tx), double-buffered two rounds ahead.
//  * One warp moves one segment in 512-B steps: lane l owns bytes [16l, 16l+16) of every
//    512-B block, so each warp-wide ld/st.v4 is one fully coalesced 512-B transaction on
//    HBM and on the PCIe link to the mapped pinned image. U blocks are loaded before any
//    store or hash step, keeping U x 512 B in flight per warp.
//  * CRC-32C from the same registers: lane l keeps T_l = F(0, its strided sub-stream) with
//    the Horner step T <- F(Z^496(T), piece) (slicing-by-16 + a 4-lookup shift), tables in
//    shared memory. The warp folds lanes with x^(8*16*(31-l)) and an XOR shuffle reduction;
//    a ragged tail (< 512 B) is staged in shared memory and finished by lane 0 bytewise.
//    Segments of one chunk are combined by the last-arriving warp (atomic counter) with
//    the GF(2) shift crc(A||B) = Z^|B|(crc(A)) ^ crc(B).
//  * XXH64 (non-combinable): one warp per chunk; stripe words are routed to 4 accumulator
//    lanes with shuffles, the tail and finalisation run on lane 0.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include <cuda.h>
#include <cudaTypedefs.h>

#include "kernels.cuh"

namespace swk {

constexpr uint32_t POLY = 0x82F63B78u;  // CRC-32C, reflected
constexpr int THREADS = 512;
constexpr int WARPS = THREADS / 32;
constexpr int U = 8;  // 512-B blocks in flight per warp
constexpr int TAIL_BYTES = 512;

constexpr uint64_t P1 = 0x9E3779B185EBCA87ull, P2 = 0xC2B2AE3D27D4EB4Full, P3 = 0x165667B19E3779F9ull,
                   P4 = 0x85EBCA77C2B2AE63ull, P5 = 0x27D4EB2F165667C5ull;

// ------------------------------------------------------------------ host: tables
static uint32_t step_byte(uint32_t c) {  // one zero byte through the register, bit-serial
  for (int k = 0; k < 8; ++k) c = (c & 1u) ? (c >> 1) ^ POLY : (c >> 1);
  return c;
}

uint32_t host_multmodp(uint32_t a, uint32_t b) {  // a*b mod P, reflected (bit 31 = x^0)
  uint32_t p = 0;
  for (int i = 0; i < 32; ++i) {
    if ((a >> (31 - i)) & 1u) p ^= b;
    b = (b & 1u) ? (b >> 1) ^ POLY : (b >> 1);
  }
  return p;
}

// x^(n*2^k) mod P. For the Castagnoli polynomial x^(2^31) = x (mod P), so x^(2^k) repeats with period
// 31, not 32 as zlib's CRC-32 table indexing `k & 31` assumes: k is reduced mod 31 (lengths of
// 512 MiB and more reach k >= 32).
uint32_t host_x2nmodp(uint64_t n, unsigned k, const uint32_t* x2n) {
  uint32_t p = 1u << 31;
  k %= 31;
  while (n) {
    if (n & 1) p = host_multmodp(x2n[k], p);
    n >>= 1;
    if (++k == 31) k = 0;
  }
  return p;
}

void build_tables(uint32_t* tab, uint64_t L1, uint64_t seg) {
  uint32_t* t = tab + TAB_T16;
  for (uint32_t b = 0; b < 256; ++b) t[b] = step_byte(b);  // T_0 = one byte
  for (int k = 1; k < 16; ++k)
    for (uint32_t b = 0; b < 256; ++b) {
      uint32_t v = t[(k - 1) * 256 + b];
      t[k * 256 + b] = t[v & 0xFFu] ^ (v >> 8);  // one more zero byte
    }
  for (int j = 0; j < 4; ++j)
    for (uint32_t b = 0; b < 256; ++b) {
      uint32_t v = b << (8 * j);
      for (int z = 0; z < 496; ++z) v = t[v & 0xFFu] ^ (v >> 8);
      tab[TAB_Z496 + j * 256 + b] = v;
    }
  uint32_t* x2n = tab + TAB_X2N;
  x2n[0] = 1u << 30;  // x^1
  for (int k = 1; k < 32; ++k) x2n[k] = host_multmodp(x2n[k - 1], x2n[k - 1]);
  for (int l = 0; l < 32; ++l) tab[TAB_LANE + l] = host_x2nmodp(16ull * (31 - l), 3, x2n);
  // hash kernel: a lane's register is finally shifted by the bytes after its last piece (common length L1)
  for (int l = 0; l < 32; ++l) {
    const uint64_t end = hash_lane_end(L1, l);
    tab[TAB_HLANE + l] = end ? host_x2nmodp(L1 - end, 3, x2n) : 0u;
  }
  for (int l = 0; l < 32; ++l) {  // strand-staged kernel: lane l's register after its strand
    const uint64_t tend = ts_lane_end(L1, l);
    tab[TAB_SLANE + l] = tend ? host_x2nmodp(L1 - tend, 3, x2n) : 0u;
  }
  for (int m = 0; m < ZS_N; ++m) tab[TAB_ZS + m] = host_x2nmodp((uint64_t)m * seg, 3, x2n);
  // Z^96 (the gap between a lane's consecutive 32-B pieces) of nibble v at nibble position k
  for (int kk = 0; kk < 8; ++kk)
    for (uint32_t v = 0; v < 16; ++v) {
      uint32_t r = v << (4 * kk);
      for (int z = 0; z < 96; ++z) r = t[r & 0xFFu] ^ (r >> 8);
      tab[TAB_Z96N + kk * 16 + v] = r;
    }
  for (int kk = 0; kk < 4; ++kk)  // Z^96 of byte e at byte position kk
    for (uint32_t e = 0; e < 256; ++e) {
      uint32_t r = e << (8 * kk);
      for (int z = 0; z < 96; ++z) r = t[r & 0xFFu] ^ (r >> 8);
      tab[TAB_Z96B + kk * 256 + e] = r;
    }
}

bool encode_tmaps(void* out, const uint64_t* base, const uint64_t* bytes, int n, uint64_t L1) {
  constexpr int S = TS_S, strands = 32;
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q{};
    void* f = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !f)
      return false;
    fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(f);
  }
  const char* pe = getenv("SWAP_TMAP_PROMO");  // A/B: none | 64 | 128 | 256 (default)
  const CUtensorMapL2promotion promo = !pe ? CU_TENSOR_MAP_L2_PROMOTION_L2_256B
                                       : !strcmp(pe, "none") ? CU_TENSOR_MAP_L2_PROMOTION_NONE
                                       : !strcmp(pe, "64") ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
                                       : !strcmp(pe, "128") ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B
                                                            : CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
  const uint64_t P = L1 / strands;
  if (L1 % strands || P % 16) return false;
  memset(out, 0, (size_t)n * 128);
  for (int r = 0; r < n; ++r) {
    const uint64_t rows = bytes[r] / P;
    if (rows == 0 || rows > (1ull << 31) || base[r] % 16) continue;
    const cuuint64_t dims[2] = {P, rows}, strides[1] = {P};
    const cuuint32_t box[2] = {(cuuint32_t)S, (cuuint32_t)strands}, es[2] = {1, 1};
    CUtensorMap* m = reinterpret_cast<CUtensorMap*>(static_cast<uint8_t*>(out) + 128ull * r);
    if (fn(m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, reinterpret_cast<void*>(base[r]), dims, strides, box, es,
           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, promo,
           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
      if (getenv("SWAP_DEBUG_TMAP"))
        fprintf(stderr, "encode_tmaps: region %d base %llx bytes %llu L1 %llu S %d strands %d failed\n", r,
                (unsigned long long)base[r], (unsigned long long)bytes[r], (unsigned long long)L1, S, strands);
      return false;
    }
  }
  return true;
}

// ------------------------------------------------------------------ device helpers
__device__ __forceinline__ int4 ld_stream(const void* p) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ void st_stream(void* p, const int4& v) {
  asm volatile("st.global.L1::no_allocate.v4.s32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w)
               : "memory");
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

// shared -> global bulk copy (TMA store, bulk-group completion; the global side may be host-mapped memory)
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)), "r"(bytes)
               : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_read_all() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// a * b mod P (reflected), branch-free.
__device__ __forceinline__ uint32_t multmodp(uint32_t a, uint32_t b) {
  uint32_t p = 0;
#pragma unroll
  for (int i = 0; i < 32; ++i) {
    p ^= b & (0u - ((a >> (31 - i)) & 1u));
    b = (b >> 1) ^ (POLY & (0u - (b & 1u)));
  }
  return p;
}
__device__ uint32_t x2nmodp(uint64_t n, unsigned k, const uint32_t* __restrict__ x2n) {  // see host_x2nmodp
  uint32_t p = 1u << 31;
  k %= 31;
  while (n) {
    if (n & 1) p = multmodp(__ldg(x2n + k), p);
    n >>= 1;
    if (++k == 31) k = 0;
  }
  return p;
}
// Z^len(s): the register after `len` zero bytes.
__device__ __forceinline__ uint32_t crc_shift(uint32_t s, uint64_t len, const uint32_t* x2n) {
  return multmodp(x2nmodp(len, 3, x2n), s);
}

// One 16-B piece of a lane's strided sub-stream: T <- F(Z^496(T), piece).
__device__ __forceinline__ uint32_t crc_piece(uint32_t T, const int4& v, const uint32_t* __restrict__ sT) {
  const uint32_t* Z = sT + TAB_Z496;
  uint32_t s = Z[T & 0xFF] ^ Z[256 + ((T >> 8) & 0xFF)] ^ Z[512 + ((T >> 16) & 0xFF)] ^ Z[768 + (T >> 24)];
  uint32_t a = static_cast<uint32_t>(v.x) ^ s, b = v.y, c = v.z, d = v.w;
  return sT[15 * 256 + (a & 0xFF)] ^ sT[14 * 256 + ((a >> 8) & 0xFF)] ^ sT[13 * 256 + ((a >> 16) & 0xFF)] ^
         sT[12 * 256 + (a >> 24)] ^ sT[11 * 256 + (b & 0xFF)] ^ sT[10 * 256 + ((b >> 8) & 0xFF)] ^
         sT[9 * 256 + ((b >> 16) & 0xFF)] ^ sT[8 * 256 + (b >> 24)] ^ sT[7 * 256 + (c & 0xFF)] ^
         sT[6 * 256 + ((c >> 8) & 0xFF)] ^ sT[5 * 256 + ((c >> 16) & 0xFF)] ^ sT[4 * 256 + (c >> 24)] ^
         sT[3 * 256 + (d & 0xFF)] ^ sT[2 * 256 + ((d >> 8) & 0xFF)] ^ sT[1 * 256 + ((d >> 16) & 0xFF)] ^
         sT[0 * 256 + (d >> 24)];
}

__device__ __forceinline__ uint64_t rotl64(uint64_t x, int r) { return (x << r) | (x >> (64 - r)); }
__device__ __forceinline__ uint64_t xround(uint64_t acc, uint64_t in) { return rotl64(acc + in * P2, 31) * P1; }
__device__ __forceinline__ uint64_t xmerge(uint64_t h, uint64_t v) { return (h ^ xround(0, v)) * P1 + P4; }

// XXH64 accumulator chains in "t-form". The spec's round is v <- rotl(v + w*P2, 31) * P1; written
// directly, ptxas puts the w*P2 multiply and a 64-bit add on the dependent chain (~11 serial SASS ops,
// ~53 cycles per round measured in the quad kernel: ncu "wait" stalls). Carrying t = v_prev + w*P2
// instead, one stripe is t <- rotl(t, 31) * P1 + w*P2: the rotate (two SHF.W) feeds one IMAD.WIDE.U32
// whose 64-bit addend is w*P2 (computed off the chain) with the cross terms folded into the high word
// -- four dependent ops per round. t0 = rotr(v0 * P1^-1, 31) (P1 is odd, so invertible mod 2^64) makes
// every stripe, the first included, the same step, and v = rotl(t, 31) * P1 at the end (= v0 when the
// chunk has no whole stripe). Bit-exact by construction; the finish uses v as the spec states.
constexpr uint64_t inv64(uint64_t a) {  // a^-1 mod 2^64 for odd a (Newton: 3 -> 6 -> ... -> 96 bits)
  uint64_t x = a;
  for (int i = 0; i < 6; ++i) x *= 2 - a * x;
  return x;
}
constexpr uint64_t rotr64c(uint64_t x, int r) { return (x >> r) | (x << (64 - r)); }
constexpr uint64_t xt_of(uint64_t v) { return rotr64c(v * inv64(P1), 31); }
constexpr uint64_t XT0 = xt_of(P1 + P2), XT1 = xt_of(P2), XT2 = xt_of(0), XT3 = xt_of(0ull - P1);
static_assert(inv64(P1) * P1 == 1, "P1 inverse");
__device__ __forceinline__ uint64_t xt_init(int j) { return j == 0 ? XT0 : j == 1 ? XT1 : j == 2 ? XT2 : XT3; }
__device__ __forceinline__ uint64_t xt_step(uint64_t t, uint64_t w) {
  const uint64_t x = w * P2;
  const uint32_t tl = (uint32_t)t, th = (uint32_t)(t >> 32);
  const uint32_t rl = __funnelshift_l(th, tl, 31), rh = __funnelshift_l(tl, th, 31);  // rotl(t, 31)
  const uint32_t ch = rh * (uint32_t)P1 + (uint32_t)(x >> 32) + rl * (uint32_t)(P1 >> 32);
  return (uint64_t)rl * (uint32_t)P1 + (((uint64_t)ch << 32) | (uint32_t)x);
}
__device__ __forceinline__ uint64_t xt_final(uint64_t t) { return rotl64(t, 31) * P1; }
__device__ __forceinline__ uint64_t ld_u64_smem(const uint8_t* p) {  // 8-aligned not guaranteed
  uint64_t v = 0;
#pragma unroll
  for (int i = 7; i >= 0; --i) v = (v << 8) | p[i];
  return v;
}

// The expected checksum of chunk g for the compare modes, loaded when the chunk's work starts: the manifest
// lives in mapped host memory, so the load is a PCIe round trip that must overlap the hashing, not follow it
// (CRC-32C verify with 4-KiB chunks: one such stall per chunk). A volatile load is issued where it is
// written (the kernels' main loops are volatile asm too). 0 for the store modes.
template <int MODE>
__device__ __forceinline__ uint64_t expect_early(const Params& p, uint32_t g) {
  if (MODE == GATHER || MODE == HASH_STORE) return 0;
  uint64_t v;
  asm volatile("ld.global.u64 %0, [%1];" : "=l"(v) : "l"(p.cs_exp + 4ull * g));
  return v;
}

// The result of chunk g: store (checkpoint / hash pass) or compare (restore / verify) with the expected
// value e (expect_early).
template <int MODE>
__device__ __forceinline__ void chunk_result(const Params& p, uint32_t g, uint64_t c, uint64_t e) {
  if (MODE == GATHER || MODE == HASH_STORE) {
    p.cs_out[4ull * g] = c;
  } else {
    if (e != c) {
      atomicAdd(p.n_bad, 1ull);
      atomicMin(p.first_bad, static_cast<unsigned long long>(g));
    }
  }
}

// Segment `idx` (descriptor d) of a CRC-32C chunk ends with register S (valid in lane 0). A one-segment
// chunk is finished here; otherwise S is stored and the warp whose segment completes the chunk (atomic
// arrival count) combines all partials, warp-parallel: lane l folds a contiguous range of segments with
// Horner steps (crc(A||B) = Z^|B|(crc A) ^ crc B), shifts it past the segments that follow (a table of
// x^(8*m*seg) for m whole segments, then the last one), and an XOR shuffle tree sums the lanes.
template <int MODE>
__device__ __forceinline__ void crc_segment_done(const Params& p, const SegDesc& d, uint32_t idx, uint32_t S, int lane,
                                                 uint64_t e) {
  const uint32_t* x2n = p.tables + TAB_X2N;
  if (d.nseg == 1) {
    if (lane == 0) {
      const uint64_t len = d.bytes;
      const uint32_t zi = (len == p.chunk_bytes) ? p.zinit_c : crc_shift(0xFFFFFFFFu, len, x2n);
      chunk_result<MODE>(p, d.chunk, (uint64_t)(~(zi ^ S)), e);
    }
    return;
  }
  uint32_t prev = 0;
  if (lane == 0) {
    p.partial[idx] = S;
    __threadfence();
    prev = atomicAdd(p.arrive + d.chunk, 1u);
  }
  prev = __shfl_sync(0xffffffffu, prev, 0);
  if (prev != d.nseg - 1) return;
  __threadfence();
  const uint32_t nseg = d.nseg, first = idx - d.seg;
  const uint32_t last_len = __ldcg(&p.desc[first + nseg - 1].bytes);
  const uint32_t k = (nseg + 31) / 32;
  const uint32_t a = min((uint32_t)lane * k, nseg), b = min(a + k, nseg);
  uint32_t X = 0;
  if (a < b) {
    uint32_t H = 0;
    for (uint32_t s = a; s < b; ++s) {
      const uint32_t f = __ldcg(p.partial + first + s);
      if (s == a) H = f;
      else if (s + 1 < nseg || last_len == p.seg_bytes) H = multmodp(p.xseg, H) ^ f;
      else H = crc_shift(H, last_len, x2n) ^ f;
    }
    if (b < nseg) {  // past segments b .. nseg-2 (whole) and nseg-1 (last_len bytes)
      const uint32_t m = nseg - 1 - b;
      H = m < (uint32_t)ZS_N ? multmodp(__ldg(p.tables + TAB_ZS + m), H) : crc_shift(H, (uint64_t)m * p.seg_bytes, x2n);
      H = last_len == p.seg_bytes ? multmodp(p.xseg, H) : crc_shift(H, last_len, x2n);
    }
    X = H;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) X ^= __shfl_xor_sync(0xffffffffu, X, o);
  if (lane == 0) {
    p.arrive[d.chunk] = 0;
    const uint64_t L = (uint64_t)(nseg - 1) * p.seg_bytes + last_len;
    const uint32_t zi = (L == p.chunk_bytes) ? p.zinit_c : crc_shift(0xFFFFFFFFu, L, x2n);
    chunk_result<MODE>(p, d.chunk, (uint64_t)(~(zi ^ X)), e);
  }
}

// Stage the ragged tail [base, base + r) (r < 512) into smem (and copy it to dst).
template <int MODE>
__device__ __forceinline__ void stage_tail(const uint8_t* src, uint8_t* dst, uint32_t r, uint8_t* tail, int lane) {
  const uint32_t lo = lane * 16u;
  if (lo + 16 <= r) {
    int4 v = ld_stream(src + lo);
    *reinterpret_cast<int4*>(tail + lo) = v;
    if (MODE == GATHER || MODE == SCATTER) st_stream(dst + lo, v);
  } else if (lo < r) {
    for (uint32_t i = lo; i < r; ++i) {
      uint8_t b = src[i];
      tail[i] = b;
      if (MODE == GATHER || MODE == SCATTER) dst[i] = b;
    }
  }
  __syncwarp();
}

// ------------------------------------------------------------------ segment movers
template <int MODE, int KIND>
__device__ __forceinline__ void move_segment(const Params& p, const SegDesc& d, uint32_t idx, const uint32_t* sT,
                                             uint8_t* tail, int lane) {
  const uint8_t* src = reinterpret_cast<const uint8_t*>(MODE == SCATTER ? d.host : d.dev);
  uint8_t* dst = reinterpret_cast<uint8_t*>(MODE == SCATTER ? d.dev : d.host);
  const uint32_t len = d.bytes;
  const uint32_t nblk = len / 512u;
  constexpr bool COPY = (MODE == GATHER || MODE == SCATTER);
  const uint64_t e = lane == 0 ? expect_early<MODE>(p, d.chunk) : 0;  // used by lane 0 only

  if (KIND == KIND_XXH64) {
    // acc lanes 0..3 carry the chains v1..v4 in t-form (xt_step). Software pipeline: the loads of the next
    // UX blocks are issued before the current blocks are stored and hashed, so the chunk's serial round
    // chain overlaps its host-link latency (round 1 loaded, stored, then hashed: the warp idled on each).
    constexpr int UX = 8;
    uint64_t acc = xt_init(lane & 3);
    const int half = (lane & 3) >> 1;
    auto load = [&](int4 (&v)[UX], uint32_t b, uint32_t nb) {
#pragma unroll
      for (int u = 0; u < UX; ++u)
        if (u < (int)nb) v[u] = ld_stream(src + (size_t)(b + u) * 512 + lane * 16);
    };
    auto consume = [&](const int4 (&v)[UX], uint32_t b, uint32_t nb) {
      if (COPY) {
#pragma unroll
        for (int u = 0; u < UX; ++u)
          if (u < (int)nb) st_stream(dst + (size_t)(b + u) * 512 + lane * 16, v[u]);
      }
#pragma unroll
      for (int u = 0; u < UX; ++u) {
        if (u < (int)nb) {
          const uint64_t lo = (uint64_t)(uint32_t)v[u].x | ((uint64_t)(uint32_t)v[u].y << 32);
          const uint64_t hi = (uint64_t)(uint32_t)v[u].z | ((uint64_t)(uint32_t)v[u].w << 32);
#pragma unroll
          for (int s = 0; s < 16; ++s) {  // stripe s of the block: lanes 2s, 2s+1 hold its 4 words
            const int srcl = 2 * s + half;
            const uint64_t wlo = __shfl_sync(0xffffffffu, lo, srcl);
            const uint64_t whi = __shfl_sync(0xffffffffu, hi, srcl);
            const uint64_t w = (lane & 1) ? whi : wlo;
            if (lane < 4) acc = xt_step(acc, w);
          }
        }
      }
    };
    int4 va[UX], vb[UX];
    uint32_t b = 0, nb = nblk < (uint32_t)UX ? nblk : (uint32_t)UX;
    load(va, 0, nb);
    while (b < nblk) {  // two batches per iteration: va / vb ping-pong, no register copies
      uint32_t b2 = b + nb, nb2 = b2 < nblk ? min((uint32_t)UX, nblk - b2) : 0u;
      load(vb, b2, nb2);
      consume(va, b, nb);
      if (!nb2) break;
      const uint32_t b3 = b2 + nb2, nb3 = b3 < nblk ? min((uint32_t)UX, nblk - b3) : 0u;
      load(va, b3, nb3);
      consume(vb, b2, nb2);
      b = b3;
      nb = nb3;
      if (!nb) break;
    }
    acc = xt_final(acc);
    const uint32_t r = len - nblk * 512u;
    const uint64_t base = (uint64_t)nblk * 512u;
    stage_tail<MODE>(src + base, COPY ? dst + base : nullptr, r, tail, lane);
    const uint64_t v1 = __shfl_sync(0xffffffffu, acc, 0), v2 = __shfl_sync(0xffffffffu, acc, 1);
    const uint64_t v3 = __shfl_sync(0xffffffffu, acc, 2), v4 = __shfl_sync(0xffffffffu, acc, 3);
    if (lane == 0) {
      uint64_t a1 = v1, a2 = v2, a3 = v3, a4 = v4;
      uint32_t i = 0;
      for (; i + 32 <= r; i += 32) {
        a1 = xround(a1, ld_u64_smem(tail + i));
        a2 = xround(a2, ld_u64_smem(tail + i + 8));
        a3 = xround(a3, ld_u64_smem(tail + i + 16));
        a4 = xround(a4, ld_u64_smem(tail + i + 24));
      }
      uint64_t h;
      if (len >= 32) {
        h = rotl64(a1, 1) + rotl64(a2, 7) + rotl64(a3, 12) + rotl64(a4, 18);
        h = xmerge(h, a1);
        h = xmerge(h, a2);
        h = xmerge(h, a3);
        h = xmerge(h, a4);
      } else {
        h = P5;
      }
      h += len;
      for (; i + 8 <= r; i += 8) {
        h ^= xround(0, ld_u64_smem(tail + i));
        h = rotl64(h, 27) * P1 + P4;
      }
      if (i + 4 <= r) {
        uint32_t w = (uint32_t)tail[i] | ((uint32_t)tail[i + 1] << 8) | ((uint32_t)tail[i + 2] << 16) |
                     ((uint32_t)tail[i + 3] << 24);
        h ^= (uint64_t)w * P1;
        h = rotl64(h, 23) * P2 + P3;
        i += 4;
      }
      for (; i < r; ++i) {
        h ^= (uint64_t)tail[i] * P5;
        h = rotl64(h, 11) * P1;
      }
      h ^= h >> 33;
      h *= P2;
      h ^= h >> 29;
      h *= P3;
      h ^= h >> 32;
      chunk_result<MODE>(p, d.chunk, h, e);
    }
    return;
  }

  // CRC-32C or no checksum.
  uint32_t T = 0;
  uint32_t b = 0;
  for (; b + U <= nblk; b += U) {
    int4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ld_stream(src + (size_t)(b + u) * 512 + lane * 16);
    if (COPY) {
#pragma unroll
      for (int u = 0; u < U; ++u) st_stream(dst + (size_t)(b + u) * 512 + lane * 16, v[u]);
    }
    if (KIND == KIND_CRC32C) {
#pragma unroll
      for (int u = 0; u < U; ++u) T = crc_piece(T, v[u], sT);
    }
  }
  for (; b < nblk; ++b) {
    int4 v = ld_stream(src + (size_t)b * 512 + lane * 16);
    if (COPY) st_stream(dst + (size_t)b * 512 + lane * 16, v);
    if (KIND == KIND_CRC32C) T = crc_piece(T, v, sT);
  }
  const uint32_t r = len - nblk * 512u;
  const uint64_t base = (uint64_t)nblk * 512u;
  if (KIND != KIND_CRC32C) {
    if (r) stage_tail<MODE>(src + base, COPY ? dst + base : nullptr, r, tail, lane);
    return;
  }
  // Fold lanes: X = XOR_l Z^(16*(31-l))(T_l) = F(0, full blocks).
  uint32_t X = nblk ? multmodp(sT[TAB_LANE + lane], T) : 0u;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) X ^= __shfl_xor_sync(0xffffffffu, X, o);
  if (r) stage_tail<MODE>(src + base, COPY ? dst + base : nullptr, r, tail, lane);
  uint32_t S = X;  // lane 0 continues the register through the tail: F(X, tail) = F(0, full || tail)
  if (lane == 0)
    for (uint32_t i = 0; i < r; ++i) S = sT[(S ^ tail[i]) & 0xFFu] ^ (S >> 8);
  crc_segment_done<MODE>(p, d, idx, S, lane, e);
}

// ------------------------------------------------------------------ the persistent kernel
template <int KIND>
struct SmemLayout {
  static constexpr int tab_words = (KIND == KIND_CRC32C) ? TAB_SMEM_WORDS : 0;
  static constexpr size_t off_desc = ((size_t)tab_words * 4 + 127) / 128 * 128;
  static constexpr size_t off_bar = off_desc + 2 * WARPS * sizeof(SegDesc);
  static constexpr size_t off_tail = (off_bar + 16 + 127) / 128 * 128;
  static constexpr size_t bytes = off_tail + (size_t)WARPS * TAIL_BYTES;
};

// XXH64 movers run one CTA per SM (launch_mover / movers.cpp size their grid to the SM count): a warp
// per chunk, and the software-pipelined register double buffer of move_segment needs up to 128 registers.
template <int MODE, int KIND>
__global__ void __launch_bounds__(THREADS, KIND == KIND_XXH64 ? 1 : 2) mover_kernel(const Params p) {
  using L = SmemLayout<KIND>;
  extern __shared__ __align__(128) uint8_t smem[];
  uint32_t* sT = reinterpret_cast<uint32_t*>(smem);
  SegDesc* sDesc = reinterpret_cast<SegDesc*>(smem + L::off_desc);
  uint64_t* sBar = reinterpret_cast<uint64_t*>(smem + L::off_bar);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  uint8_t* tail = smem + L::off_tail + warp * TAIL_BYTES;

  if (KIND == KIND_CRC32C)
    for (int i = tid; i < L::tab_words; i += THREADS) sT[i] = __ldg(p.tables + i);

  if (KIND == KIND_XXH64) {
    // a descriptor is a whole chunk, one warp's long serial job: warps take chunks interleaved across
    // CTAs (chunk w * grid + cta first), so a few chunks spread over as many SMs as possible, and no CTA
    // barrier ties a warp to the slowest one of its round; the descriptor is read directly (no staging)
    for (uint32_t idx = warp * gridDim.x + blockIdx.x; idx < p.n_desc; idx += gridDim.x * WARPS) {
      const SegDesc d = p.desc[idx];
      move_segment<MODE, KIND>(p, d, idx, sT, tail, lane);
    }
    return;
  }

  const uint32_t per_round = gridDim.x * WARPS;
  const uint32_t first0 = blockIdx.x * WARPS;
  const uint32_t rounds = p.n_desc > first0 ? (p.n_desc - first0 + per_round - 1) / per_round : 0u;
  auto issue = [&](uint32_t r) {
    const uint32_t first = r * per_round + first0;
    const uint32_t cnt = min((uint32_t)WARPS, p.n_desc - first);
    uint64_t* bar = sBar + (r & 1);
    mbar_expect_tx(bar, cnt * (uint32_t)sizeof(SegDesc));
    bulk_g2s(sDesc + (r & 1) * WARPS, p.desc + first, cnt * (uint32_t)sizeof(SegDesc), bar);
  };
  if (tid == 0) {
    mbar_init(sBar, 1);
    mbar_init(sBar + 1, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (rounds > 0) issue(0);
    if (rounds > 1) issue(1);
  }
  __syncthreads();

  for (uint32_t r = 0; r < rounds; ++r) {
    mbar_wait(sBar + (r & 1), (r >> 1) & 1u);
    const uint32_t idx = r * per_round + first0 + warp;
    if (idx < p.n_desc) {
      const SegDesc d = sDesc[(r & 1) * WARPS + warp];
      move_segment<MODE, KIND>(p, d, idx, sT, tail, lane);
    }
    __syncthreads();
    if (tid == 0 && r + 2 < rounds) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      issue(r + 2);
    }
  }
}


// ------------------------------------------------------------------ HBM hash kernel (CRC-32C)
// HASH_STORE / HASH_CHECK read device memory only, so the warp can choose any slicing of its segment.
// Quad-line layout: the segment is cut into 8 strands, one per lane quad; in each step the 4 lanes of a
// quad load the 4 sectors of one 128-B line of their strand with 256-bit loads, so a warp-wide load
// touches 8 lines (8 L1 wavefronts per KiB instead of 32 with one line per lane). A lane's bytes are
// then 32-B pieces 128 B apart: its register advances with T <- F(Z^96(T), piece) — Z^96 by 8 nibble
// lookups, F by 8 slicing-by-4 word steps. All tables are replicated once per lane in shared memory
// (entry e of table k for lane l at word (k*E + e)*32 + l: bank = lane, conflict-free): slicing-by-4
// 4 x 256 entries (128 KB), Z^96 nibbles 8 x 16 (16 KB). Lanes are folded with x^(8 * bytes after the
// lane's last piece) and an XOR shuffle tree. Per KiB per warp: 32 + 8 lookup wavefronts + 8 load
// wavefronts (the r1 contiguous-run layout needed 32 + 32).
constexpr int HT_THREADS = 1024;
constexpr int HT_WARPS = HT_THREADS / 32;
// Shared layout, in shared-window addresses derived from the dynamic-shared-memory base R (measured once per
// device by smem_base_probe; 0x400 on sm_100, the first KiB of the CTA window being reserved): descriptors +
// mbarriers at R, the Z^96 nibble tables (8 x 16 entries x 32 lanes, 16 KiB) at the next 2-KiB boundary, the
// four slicing tables at the next 32-KiB boundary (table k at +k*32 KiB, entry e of lane l at + e*128 + l*4,
// so a lookup address is (index << 7) | (base + 4*lane) plus an immediate table offset: one shift + one
// LOP3). Variant ZB adds Z^96 *byte* tables after the slicing tables (4 x 256 entries x 16 copies, lanes l
// and l+16 share copy l&15: entry e of copy c at word e*16 + c) instead of the nibble tables. With R = 0x400
// nothing is padded: nibble tables at 0x1000, slicing tables at 0x8000.
struct HtLayout {
  uint32_t desc, bar, zn, tab, zb, end;
};
__host__ __device__ constexpr uint32_t ht_align(uint32_t v, uint32_t a) { return (v + a - 1) / a * a; }
__host__ __device__ inline HtLayout ht_layout(uint32_t R, bool zb) {
  HtLayout L{};
  L.desc = R;
  L.bar = R + 2 * HT_WARPS * 32;  // 2 rounds x 32 descriptors x 32 B
  L.zn = ht_align(L.bar + 16, 2048);
  L.tab = ht_align(L.zn + 8 * 16 * 128, 32768);
  L.zb = L.tab + 4 * 256 * 128;
  L.end = zb ? L.zb + 4 * 256 * 16 * 4 : L.zb;
  return L;
}
__global__ void smem_base_probe(uint32_t* out) {
  extern __shared__ __align__(128) uint8_t s[];
  if (threadIdx.x == 0) *out = static_cast<uint32_t>(__cvta_generic_to_shared(s));
}
// The dynamic-shared-memory base of this device's kernels (cached per device; swap_create probes it so
// that no launch pays the probe's synchronising cudaMalloc / cudaFree).
static cudaError_t smem_base(uint32_t* R) {
  static uint32_t cache[64] = {};
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (!cache[dev & 63]) {
    uint32_t* d = nullptr;
    if ((e = cudaMalloc(&d, 4)) != cudaSuccess) return e;
    smem_base_probe<<<1, 32, 128>>>(d);
    uint32_t h = 0;
    e = cudaMemcpy(&h, d, 4, cudaMemcpyDeviceToHost);
    cudaFree(d);
    if (e != cudaSuccess) return e;
    cache[dev & 63] = h ? h : 1;  // 0 (no reservation) stored as 1 (a 0 base aligns to itself)
  }
  *R = cache[dev & 63] == 1 ? 0 : cache[dev & 63];
  return cudaSuccess;
}
static_assert(ht_align(0x400 + 2 * HT_WARPS * 32 + 16, 2048) == 0x1000, "hash kernel shared layout at R = 0x400");

__device__ __forceinline__ void ld32(const uint8_t* p, uint32_t (&w)[8]) {
  asm("ld.global.nc.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]), "=r"(w[7])
      : "l"(p));
}
__device__ __forceinline__ void ld32_v4x2(const uint8_t* p, uint32_t (&w)[8]) {  // 16-B aligned fallback
  int4 a = __ldg(reinterpret_cast<const int4*>(p)), b = __ldg(reinterpret_cast<const int4*>(p + 16));
  w[0] = a.x; w[1] = a.y; w[2] = a.z; w[3] = a.w; w[4] = b.x; w[5] = b.y; w[6] = b.z; w[7] = b.w;
}
template <bool AL32>
__device__ __forceinline__ void ld32a(const uint8_t* p, uint32_t (&w)[8]) {
  if (AL32) ld32(p, w); else ld32_v4x2(p, w);
}
// Streaming variants that do not allocate in L1 (every sector is consumed exactly once).
__device__ __forceinline__ void ld32_na(const uint8_t* p, uint32_t (&w)[8]) {
  asm("ld.global.nc.L1::no_allocate.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]), "=r"(w[7])
      : "l"(p));
}
__device__ __forceinline__ void ld32_v4x2_na(const uint8_t* p, uint32_t (&w)[8]) {
  asm("ld.global.nc.L1::no_allocate.v4.b32 {%0,%1,%2,%3}, [%4];"
      : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]) : "l"(p));
  asm("ld.global.nc.L1::no_allocate.v4.b32 {%0,%1,%2,%3}, [%4];"
      : "=r"(w[4]), "=r"(w[5]), "=r"(w[6]), "=r"(w[7]) : "l"(p + 16));
}
template <bool AL32>
__device__ __forceinline__ void ld32na(const uint8_t* p, uint32_t (&w)[8]) {
  if (AL32) ld32_na(p, w); else ld32_v4x2_na(p, w);
}
__device__ __forceinline__ uint32_t lds_at(uint32_t addr) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr));
  return v;
}
template <uint32_t OFF>
__device__ __forceinline__ uint32_t lds_off(uint32_t addr) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1+%2];" : "=r"(v) : "r"(addr), "n"(OFF));
  return v;
}

// slicing-by-4 word step; lb = B + 4*lane (B 32-KiB aligned): table k entry e at lb + k*32K + e*128.
// Byte j of x = c ^ w indexes table 3-j at address (byte << 7) | lb. Bytes 0-2 take a shift + LOP3 on
// the ALU pipe; byte 3's address is (x >> 24) * m128 + lb, an IMAD on the FMA pipe (m128 = 128 held in
// a register so ptxas cannot fold it back into a shift). The ALU pipe limits this kernel (ncu: 80 %
// busy); moving one address per word to the FMA pipe measured +6 % (interleaved A/B on config B; the
// other splits tried — bytes 1-3 or all four via IMAD/IMAD.HI, byte-permute addressing with 64-KiB
// table pairs — were slower: IMAD.HI and PRMT cost two ALU-equivalent issue slots).
template <bool B0F>
__device__ __forceinline__ uint32_t crc_word4(uint32_t c, uint32_t w, uint32_t lb, uint32_t m128) {
  c ^= w;
  // B0F: byte 0's shift by 7 as an IMAD by the opaque 128 (FMA pipe, idle in this kernel) instead of a SHF
  const uint32_t s0 = B0F ? c * m128 : c << 7;
  return lds_off<3 * 32768>((s0 & 0x7F80u) | lb) ^ lds_off<2 * 32768>(((c >> 1) & 0x7F80u) | lb) ^
         lds_off<1 * 32768>(((c >> 9) & 0x7F80u) | lb) ^ lds_off<0>((c >> 24) * m128 + lb);
}
// Z^96(T) from 8 nibble lookups; lz = 0x1000 + 4*lane: nibble table k entry v at lz + k*2K + v*128
template <bool B0F>
__device__ __forceinline__ uint32_t z96(uint32_t T, uint32_t lz, uint32_t m128) {
  const uint32_t s0 = B0F ? T * m128 : T << 7;
  const uint32_t a7 = B0F ? (T >> 28) * m128 + lz : ((T >> 21) & 0x780u) | lz;
  return lds_off<0 * 2048>((s0 & 0x780u) | lz) ^ lds_off<1 * 2048>(((T << 3) & 0x780u) | lz) ^
         lds_off<2 * 2048>(((T >> 1) & 0x780u) | lz) ^ lds_off<3 * 2048>(((T >> 5) & 0x780u) | lz) ^
         lds_off<4 * 2048>(((T >> 9) & 0x780u) | lz) ^ lds_off<5 * 2048>(((T >> 13) & 0x780u) | lz) ^
         lds_off<6 * 2048>(((T >> 17) & 0x780u) | lz) ^ lds_off<7 * 2048>(a7);
}
// Z^96(T) from 4 byte lookups; lzb = 0x28000 + 4*(lane & 15): byte table k entry e at lzb + k*16K + e*64
// (lanes l and l+16 share a copy: they meet in a bank only when their entries have equal parity)
__device__ __forceinline__ uint32_t z96b(uint32_t T, uint32_t lzb, uint32_t m64) {
  return lds_off<0 * 16384>(((T << 6) & 0x3FC0u) | lzb) ^ lds_off<1 * 16384>(((T >> 2) & 0x3FC0u) | lzb) ^
         lds_off<2 * 16384>(((T >> 10) & 0x3FC0u) | lzb) ^ lds_off<3 * 16384>((T >> 24) * m64 + lzb);
}

// One 32-B piece: advance the register across the 96-B gap, then through the piece's 8 words.
template <bool ZB, bool B0F>
__device__ __forceinline__ uint32_t crc_piece32(uint32_t c, const uint32_t (&w)[8], uint32_t lb, uint32_t lz,
                                                uint32_t m128) {
  c = ZB ? z96b(c, lz, m128 >> 1) : z96<B0F>(c, lz, m128);
#pragma unroll
  for (int j = 0; j < 8; ++j) c = crc_word4<B0F>(c, w[j], lb, m128);
  return c;
}

// Register of one lane over its pieces s0, s0+128, ... < send (send = min(strand end, len)).
// A 4-deep software pipeline: each 256-bit load is consumed one loop iteration after it is issued,
// so ptxas cannot sink it next to its use and four loads per lane stay in flight.
template <bool AL32, bool ZB, bool B0F>
__device__ __forceinline__ uint32_t lane_pieces_crc(const uint8_t* src, uint64_t s0, uint64_t send, uint32_t lb,
                                                    uint32_t lz, uint32_t m128) {
  uint32_t c = 0;
  const uint64_t n = s0 + 32 <= send ? (send - 32 - s0) / 128 + 1 : 0;  // whole 32-B pieces
  uint64_t t = 0;
  if (n >= 4) {
    uint32_t a[8], b[8], d[8], e[8];
    ld32a<AL32>(src + s0, a);
    ld32a<AL32>(src + s0 + 128, b);
    ld32a<AL32>(src + s0 + 256, d);
    ld32a<AL32>(src + s0 + 384, e);
    for (; t + 8 <= n; t += 4) {
      const uint8_t* q = src + s0 + (t + 4) * 128;
      c = crc_piece32<ZB, B0F>(c, a, lb, lz, m128);
      ld32a<AL32>(q, a);
      c = crc_piece32<ZB, B0F>(c, b, lb, lz, m128);
      ld32a<AL32>(q + 128, b);
      c = crc_piece32<ZB, B0F>(c, d, lb, lz, m128);
      ld32a<AL32>(q + 256, d);
      c = crc_piece32<ZB, B0F>(c, e, lb, lz, m128);
      ld32a<AL32>(q + 384, e);
    }
    c = crc_piece32<ZB, B0F>(c, a, lb, lz, m128);
    c = crc_piece32<ZB, B0F>(c, b, lb, lz, m128);
    c = crc_piece32<ZB, B0F>(c, d, lb, lz, m128);
    c = crc_piece32<ZB, B0F>(c, e, lb, lz, m128);
    t += 4;
  }
  for (; t < n; ++t) {
    uint32_t w[8];
    ld32a<AL32>(src + s0 + t * 128, w);
    c = crc_piece32<ZB, B0F>(c, w, lb, lz, m128);
  }
  uint64_t s = s0 + n * 128;
  if (s < send) {  // a partial last piece (only at the end of the segment)
    c = ZB ? z96b(c, lz, m128 >> 1) : z96<B0F>(c, lz, m128);
    for (; s < send; ++s) c = lds_at((((c ^ src[s]) & 0xFFu) << 7) | lb) ^ (c >> 8);  // table 0 = one byte
  }
  return c;
}

// One segment by one warp in the quad-line layout (hash_kernel; the quad role of crc_mx_kernel).
template <int MODE, bool ZB, bool B0F>
__device__ __forceinline__ void quad_segment(const Params& p, const SegDesc d, uint32_t idx, int lane, uint32_t lb,
                                             uint32_t lz, uint32_t m128) {
  const uint64_t e = lane == 0 ? expect_early<MODE>(p, d.chunk) : 0;
  const uint64_t len = d.bytes;
  const uint64_t Ls = hash_strand(len);
  const uint64_t q = (uint64_t)(lane >> 2), jj = (uint64_t)(lane & 3);
  const uint64_t s0 = q * Ls + jj * 32;
  const uint64_t send = (q + 1) * Ls < len ? (q + 1) * Ls : len;
  const uint8_t* src = reinterpret_cast<const uint8_t*>(d.dev);
  const bool al32 = ((d.dev & 31) == 0);
  uint32_t X = 0;
  if (s0 < send) {
    const uint32_t c = al32 ? lane_pieces_crc<true, ZB, B0F>(src, s0, send, lb, lz, m128)
                            : lane_pieces_crc<false, ZB, B0F>(src, s0, send, lb, lz, m128);
    const uint32_t k = (len == p.hlane_len) ? __ldg(p.tables + TAB_HLANE + lane)
                                            : x2nmodp(len - hash_lane_end(len, lane), 3, p.tables + TAB_X2N);
    X = multmodp(k, c);
  }
#pragma unroll
  for (int s = 16; s > 0; s >>= 1) X ^= __shfl_xor_sync(0xffffffffu, X, s);
  crc_segment_done<MODE>(p, d, idx, X, lane, e);
}

template <int MODE, bool ZB, bool B0F>
__global__ void __launch_bounds__(HT_THREADS, 1) hash_kernel(const Params p) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const HtLayout HL = ht_layout(raw, ZB);  // the host sized the allocation for this base (smem_base)
  uint8_t* smem = smem_raw - raw;  // generic pointer of shared address 0
  uint32_t* sT = reinterpret_cast<uint32_t*>(smem + HL.tab);
  SegDesc* sDesc = reinterpret_cast<SegDesc*>(smem + HL.desc);
  uint64_t* sBar = reinterpret_cast<uint64_t*>(smem + HL.bar);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

  // replicate T0..T3 (the first four slicing tables) once per lane, and the Z^96 tables
  for (int i = tid; i < 4 * 256; i += HT_THREADS) {
    const uint32_t v = __ldg(p.tables + TAB_T16 + i);
    uint4* dst = reinterpret_cast<uint4*>(sT + (size_t)i * 32);
#pragma unroll
    for (int r = 0; r < 8; ++r) dst[r] = make_uint4(v, v, v, v);
  }
  if (ZB) {
    uint32_t* sZ = reinterpret_cast<uint32_t*>(smem + HL.zb);
    for (int i = tid; i < 4 * 256; i += HT_THREADS) {
      const uint32_t v = __ldg(p.tables + TAB_Z96B + i);
      uint4* dst = reinterpret_cast<uint4*>(sZ + (size_t)i * 16);
#pragma unroll
      for (int r = 0; r < 4; ++r) dst[r] = make_uint4(v, v, v, v);
    }
  } else {
    uint32_t* sZ = reinterpret_cast<uint32_t*>(smem + HL.zn);
    for (int i = tid; i < 8 * 16; i += HT_THREADS) {
      const uint32_t v = __ldg(p.tables + TAB_Z96N + i);
      uint4* dst = reinterpret_cast<uint4*>(sZ + (size_t)i * 32);
#pragma unroll
      for (int r = 0; r < 8; ++r) dst[r] = make_uint4(v, v, v, v);
    }
  }
  const uint32_t per_round = gridDim.x * HT_WARPS;
  // fewer segments than warp slots (a CE_PIPE group's check): one round, segments dealt warp-major across the
  // CTAs (segment w * grid + cta) so that every SM hashes, descriptors read directly; else rounds of
  // HT_WARPS consecutive descriptors per CTA staged by TMA
  const bool spread = p.n_desc < per_round;
  const uint32_t first0 = blockIdx.x * HT_WARPS;
  const uint32_t rounds = spread ? (blockIdx.x < p.n_desc ? 1u : 0u)
                                 : p.n_desc > first0 ? (p.n_desc - first0 + per_round - 1) / per_round : 0u;
  auto issue = [&](uint32_t r) {
    const uint32_t first = r * per_round + first0;
    const uint32_t cnt = min((uint32_t)HT_WARPS, p.n_desc - first);
    uint64_t* bar = sBar + (r & 1);
    mbar_expect_tx(bar, cnt * (uint32_t)sizeof(SegDesc));
    bulk_g2s(sDesc + (r & 1) * HT_WARPS, p.desc + first, cnt * (uint32_t)sizeof(SegDesc), bar);
  };
  if (tid == 0) {
    mbar_init(sBar, 1);
    mbar_init(sBar + 1, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (!spread && rounds > 0) issue(0);
    if (!spread && rounds > 1) issue(1);
  }
  __syncthreads();
  const uint32_t lb = HL.tab + 4u * lane;
  const uint32_t lz = ZB ? HL.zb + 4u * (lane & 15) : HL.zn + 4u * lane;
  const uint32_t m128 = blockDim.x >> 3;  // = 128 (HT_THREADS = 1024), opaque to ptxas

  for (uint32_t r = 0; r < rounds; ++r) {
    if (!spread) mbar_wait(sBar + (r & 1), (r >> 1) & 1u);
    const uint32_t idx = spread ? warp * gridDim.x + blockIdx.x : r * per_round + first0 + warp;
    if (idx < p.n_desc)
      quad_segment<MODE, ZB, B0F>(p, spread ? p.desc[idx] : sDesc[(r & 1) * HT_WARPS + warp], idx, lane, lb, lz,
                                  m128);
    __syncthreads();
    if (!spread && tid == 0 && r + 2 < rounds) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      issue(r + 2);
    }
  }
}

cudaError_t probe_smem_base() {
  uint32_t R = 0;
  return smem_base(&R);
}

template <int MODE, bool ZB, bool B0F>
static cudaError_t launch_hash_t(const Params& p, int grid, cudaStream_t s) {
  static unsigned long long attr_set = 0;
  uint32_t R = 0;
  cudaError_t e = smem_base(&R);
  if (e != cudaSuccess) return e;
  const size_t bytes = ht_layout(R, ZB).end - R;
  int dev = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if (!((attr_set >> (dev & 63)) & 1ull)) {
    e = cudaFuncSetAttribute(hash_kernel<MODE, ZB, B0F>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
    if (e != cudaSuccess) return e;
    attr_set |= 1ull << (dev & 63);
  }
  hash_kernel<MODE, ZB, B0F><<<grid, HT_THREADS, bytes, s>>>(p);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ HBM hash kernel (CRC-32C), strand-staged
// The quad-line kernel above pays 8 nibble lookups (Z^96) per 32-B piece because a lane's bytes are 32-B
// pieces 128 B apart: 40 lookup + 8 load L1 wavefronts per KiB per warp. Here a segment is cut into 32
// contiguous strands (ts_strand), one per lane, streamed through a per-warp ring of NB stages in shared
// memory: stage k holds bytes [k*S, (k+1)*S) of every strand, row = lane. A lane's bytes are then contiguous
// across stages, so its register only takes slicing-by-4 word steps -- no Z shift until the final fold by
// x^(8 * bytes after the strand) (TAB_SLANE for the common length L1): 32 lookup + 8 LDS.128 wavefronts per
// KiB per warp. S is an odd multiple of 16 B, so the 8 lanes of an LDS.128 phase hit 8 distinct 16-B bank
// groups. Standard segments (len == L1 at their place in the chunk: every full segment) are staged with ONE
// 2-D tensor copy per stage -- the chunk viewed as rows of P = L1/32 bytes, box {S, 32} at column k*S, row
// 32 * (segment index in the chunk); columns past P (a strand's last partial stage) are out of bounds,
// zero-filled, never read from memory. The maps are per chunk, not per region: a scheduler swap-out releases
// a victim's VMM slabs group by group while later groups are still hashed, and a TMA load through a map whose
// tensor reaches into a released slab faults even when its box does not. Other segments (ragged region tails, DISCARD chunks hashed from the zero buffer)
// take per-lane 1-D bulk copies: ptxas issues those through an ELECT loop (~10 issue slots per lane and
// stage), half the speed if every segment took them (profiles/r02_crc_strand_staged.md), fine for the few
// ragged ones. Segments are dealt warp-major across the CTAs (w * grid + cta, then + W * grid), so that a
// launch with few segments (a CE_PIPE restore group's check) still spreads over every SM. The producer (lane 0
// on the tensor path) runs NB stages ahead across segment boundaries (the warp's segments form one flat
// stage sequence). Throughput follows the resident warp count (dependent
// lookup chains), which shared memory caps: the tables take 128 KiB, each warp's ring NB*32*S bytes.
// Shared layout (window addresses, base R0): W*NB mbarriers at R0, rings below the 32-KiB-aligned slicing
// tables and after them (the tables sit at a 32-KiB boundary for crc_word4's (index << 7) | lb addresses).
template <int W, int NB, int S>
struct TsLayout {
  static_assert(S % 16 == 0 && (S / 16) % 2 == 1, "stage width: odd multiple of 16 B (conflict-free LDS.128)");
  static_assert(S == TS_S, "the tensor maps are encoded for box {TS_S, 32}");
  static constexpr uint32_t STAGE = 32u * S;
  static constexpr uint32_t RING = (uint32_t)NB * STAGE;
  uint32_t bar, low, tab, high, nlow, end;
};
constexpr uint32_t TS_SMEM_MAX = 227u * 1024u;  // opt-in dynamic shared memory per CTA
template <int W, int NB, int S>
__host__ __device__ inline TsLayout<W, NB, S> ts_layout(uint32_t R0) {
  using LT = TsLayout<W, NB, S>;
  LT L{};
  L.bar = R0;
  L.low = ht_align(R0 + W * NB * 8, 128);
  L.tab = ht_align(L.low, 32768);
  if (L.tab < L.low + LT::RING) L.tab = ht_align(L.low + 1, 32768);
  L.nlow = (L.tab - L.low) / LT::RING;
  if (L.nlow > (uint32_t)W) L.nlow = W;
  L.high = L.tab + 4 * 256 * 128;
  L.end = L.high + (uint32_t)(W - L.nlow) * LT::RING;
  return L;
}

__device__ __forceinline__ uint4 lds128(uint32_t addr) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
  return v;
}
__device__ __forceinline__ void bulk_g2s_a(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(bar)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx_a(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait_a(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n}" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const void* tmap, int c0, int c1, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::
          "r"(dst), "l"(tmap), "r"(c0), "r"(c1), "r"(bar)
      : "memory");
}

// The strand-staged loop of one warp over the segments seg_of(k), k = k0, k0 + kstride, ... < nk (its ring of
// NB stages at `ring`, its NB mbarriers at `bars`, initialised with count 1; tables at `tab`).
template <int MODE, int NB, int S, class Map>
__device__ __forceinline__ void ts_role(const Params& p, uint32_t tab, uint32_t ring, uint32_t bars, int lane,
                                        uint32_t k0, uint32_t kstride, uint32_t nk, Map seg_of) {
  constexpr uint32_t STAGE = 32u * S;
  const uint32_t myrow = ring + (uint32_t)lane * S;
  const uint32_t L1 = p.hlane_len;
  // producer cursor (this warp's copies): pool index pk_i (segment pidx), its stage pk of pnst; psrc = this
  // lane's strand, pbytes = its bytes below len & ~15 (the bulk-copied part); ptm / prow: the tensor path
  uint32_t pki = k0, pidx = 0, pk = 0, pnst = 0, pseq = 0, pbytes = 0;
  const uint8_t* psrc = nullptr;
  const void* ptm = nullptr;
  int prow = 0;
  auto p_load = [&]() {  // geometry of the producer's next segment (skipping empty ones)
    for (; pki < nk; pki += kstride) {
      pidx = seg_of(pki);
      const uint64_t dev = __ldg(reinterpret_cast<const unsigned long long*>(&p.desc[pidx].dev));
      const uint32_t len = __ldg(&p.desc[pidx].bytes);
      const uint32_t Ls = (uint32_t)ts_strand(len);
      pnst = (Ls + S - 1) / S;
      if (pnst == 0) continue;
      const uint32_t a0 = (uint32_t)lane * Ls, e16 = min(a0 + Ls, len & ~15u);
      pbytes = e16 > a0 ? e16 - a0 : 0u;
      psrc = reinterpret_cast<const uint8_t*>(dev) + a0;
      pk = 0;
      ptm = nullptr;
      if (p.tmaps && len == L1) {  // segment s of chunk g starts at chunk_dev[g] + s * L1 (L1 = min(C, seg))
        const uint32_t g = __ldg(&p.desc[pidx].chunk), s = __ldg(&p.desc[pidx].seg);
        const unsigned long long cb = __ldg(p.chunk_dev + g);
        if (cb && dev == cb + (uint64_t)s * L1) {
          ptm = reinterpret_cast<const uint8_t*>(p.tmaps) + 128ull * g;
          prow = (int)(s * 32u);
          // the maps were written to global memory by the host (cudaMemcpy at registration): make them
          // visible to the tensormap proxy before the TMA unit reads them (a ctx's maps can reuse the
          // address of a destroyed ctx's maps)
          if (lane == 0) asm volatile("fence.proxy.tensormap::generic.acquire.gpu [%0], 128;" ::"l"(ptm) : "memory");
        }
      }
      return;
    }
  };
  auto p_issue = [&]() {  // next stage of the flat sequence into buffer pseq % NB
    if (pki >= nk) return;
    const uint32_t off = pk * S;
    const uint32_t b = pseq % NB;
    const uint32_t bar = bars + 8 * b;
    if (ptm) {
      if (lane == 0) {
        mbar_arrive_tx_a(bar, STAGE);
        tma_load_2d(ring + b * STAGE, ptm, (int)off, prow, bar);
      }
    } else {
      const uint32_t n = pbytes > off ? min(pbytes - off, (uint32_t)S) : 0u;
      const uint32_t tot = __reduce_add_sync(0xffffffffu, n);
      if (lane == 0) mbar_arrive_tx_a(bar, tot);
      if (n) bulk_g2s_a(myrow + b * STAGE, psrc + off, n, bar);
    }
    ++pseq;
    if (++pk == pnst) {
      pki += kstride;
      p_load();
    }
  };
  p_load();
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
#pragma unroll 1
  for (int k = 0; k < NB; ++k) p_issue();

  const uint32_t lb = tab + 4u * lane;
  const uint32_t m128 = 128u * gridDim.y;  // = 128 (gridDim.y == 1), opaque to ptxas
  const uint32_t* x2n = p.tables + TAB_X2N;
  uint32_t cseq = 0;
  for (uint32_t ki = k0; ki < nk; ki += kstride) {
    const uint32_t idx = seg_of(ki);
    const SegDesc d = p.desc[idx];
    const uint64_t e = lane == 0 ? expect_early<MODE>(p, d.chunk) : 0;
    const uint32_t len = d.bytes, Ls = (uint32_t)ts_strand(len), nst = (Ls + S - 1) / S;
    const uint32_t a0 = (uint32_t)lane * Ls, aend = min(a0 + Ls, len), e16 = min(aend, len & ~15u);
    const uint32_t mine = e16 > a0 ? e16 - a0 : 0u;
    uint32_t c = 0;
#pragma unroll 1
    for (uint32_t k = 0; k < nst; ++k) {
      const uint32_t b = cseq % NB;
      mbar_wait_a(bars + 8 * b, (cseq / NB) & 1u);
      const uint32_t row = myrow + b * STAGE;
      const uint32_t off = k * S;
      const uint32_t n = mine > off ? min(mine - off, (uint32_t)S) : 0u;
      if (n == (uint32_t)S) {
        uint4 v[S / 16];
#pragma unroll
        for (int u = 0; u < S / 16; ++u) v[u] = lds128(row + 16 * u);
#pragma unroll
        for (int u = 0; u < S / 16; ++u) {
          c = crc_word4<true>(c, v[u].x, lb, m128);
          c = crc_word4<true>(c, v[u].y, lb, m128);
          c = crc_word4<true>(c, v[u].z, lb, m128);
          c = crc_word4<true>(c, v[u].w, lb, m128);
        }
      } else {
#pragma unroll 1
        for (uint32_t u = 0; u < n; u += 16) {
          const uint4 v = lds128(row + u);
          c = crc_word4<true>(c, v.x, lb, m128);
          c = crc_word4<true>(c, v.y, lb, m128);
          c = crc_word4<true>(c, v.z, lb, m128);
          c = crc_word4<true>(c, v.w, lb, m128);
        }
      }
      ++cseq;
      __syncwarp();  // every lane's reads of this stage precede its refill (one tensor copy fills all rows)
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      p_issue();
    }
    uint32_t X = 0;
    if (a0 < len) {
      // the segment's last len & 15 bytes (the strand that ends at len), from HBM
      const uint8_t* src = reinterpret_cast<const uint8_t*>(d.dev);
      for (uint32_t s = max(e16, a0); s < aend; ++s) c = lds_at((((c ^ src[s]) & 0xFFu) << 7) | lb) ^ (c >> 8);
      const uint32_t kz = (len == L1) ? __ldg(p.tables + TAB_SLANE + lane) : x2nmodp(len - aend, 3, x2n);
      X = multmodp(kz, c);
    }
#pragma unroll
    for (int s = 16; s > 0; s >>= 1) X ^= __shfl_xor_sync(0xffffffffu, X, s);
    crc_segment_done<MODE>(p, d, idx, X, lane, e);
  }
}

struct IdentityMap {
  __device__ uint32_t operator()(uint32_t k) const { return k; }
};

template <int MODE, int W, int NB, int S>
__global__ void __launch_bounds__(W * 32, 1) crc_ts_kernel(const Params p) {
  using LT = TsLayout<W, NB, S>;
  extern __shared__ __align__(128) uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const LT L = ts_layout<W, NB, S>(raw);
  uint8_t* smem = smem_raw - raw;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

  for (int i = tid; i < 4 * 256; i += W * 32) {  // slicing tables T0..T3, replicated once per lane
    const uint32_t v = __ldg(p.tables + TAB_T16 + i);
    uint4* dst = reinterpret_cast<uint4*>(smem + L.tab + (size_t)i * 128);
#pragma unroll
    for (int r = 0; r < 8; ++r) dst[r] = make_uint4(v, v, v, v);
  }
  const uint32_t bars = L.bar + (uint32_t)warp * NB * 8;
  if (lane == 0) {
    for (int b = 0; b < NB; ++b)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bars + 8 * b), "r"(1) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  const uint32_t ring = (uint32_t)warp < L.nlow ? L.low + (uint32_t)warp * LT::RING
                                                : L.high + ((uint32_t)warp - L.nlow) * LT::RING;
  __syncthreads();
  ts_role<MODE, NB, S>(p, L.tab, ring, bars, lane, warp * gridDim.x + blockIdx.x, gridDim.x * W, p.n_desc,
                       IdentityMap{});
}

// Mixed roles in one CTA of 32 warps: warps [0, WT) run the strand-staged loop (shared-memory rings), warps
// [WT, 32) the quad-line loop (register staging, no ring): the strand kernel is capped at ~19 warps by shared
// memory while the SM's pipes have room, and the quad-line warps need no ring. Segment i is a strand-role
// segment if i % 8 < TSN, else a quad-role one (TSN / 8 of the segments: the roles' measured per-warp rates,
// static so the strand producer can run ahead); each role deals its segments warp-major over the grid.
// Layout: WT*2 mbarriers, rings below the slicing tables (32-KiB aligned), the Z^96 nibble tables right
// after them (2-KiB aligned, for the quad role), more rings after those.
template <int WT, int TSN>
struct MxLayout {
  static constexpr uint32_t RING = 2u * 32u * TS_S;
  uint32_t bar, low, tab, zn, high, nlow, end;
};
template <int WT, int TSN>
__host__ __device__ inline MxLayout<WT, TSN> mx_layout(uint32_t R0) {
  using LT = MxLayout<WT, TSN>;
  LT L{};
  L.bar = R0;
  L.low = ht_align(R0 + WT * 2 * 8, 128);
  L.tab = ht_align(L.low, 32768);
  if (L.tab < L.low + LT::RING) L.tab = ht_align(L.low + 1, 32768);
  L.nlow = (L.tab - L.low) / LT::RING;
  if (L.nlow > (uint32_t)WT) L.nlow = WT;
  L.zn = L.tab + 4 * 256 * 128;
  L.high = L.zn + 8 * 16 * 128;
  L.end = L.high + (uint32_t)(WT - L.nlow) * LT::RING;
  return L;
}
template <int TSN, bool TS>
struct PoolMap {  // k-th segment of a role's pool
  __device__ uint32_t operator()(uint32_t k) const {
    return TS ? (k / TSN) * 8 + k % TSN : (k / (8 - TSN)) * 8 + TSN + k % (8 - TSN);
  }
};
template <int TSN>
__host__ __device__ inline uint32_t pool_size(uint32_t n, bool ts) {
  const uint32_t full = n / 8 * (ts ? TSN : 8 - TSN), r = n % 8;
  return full + (ts ? min(r, (uint32_t)TSN) : (r > (uint32_t)TSN ? r - TSN : 0u));
}

template <int MODE, int WT, int TSN, int NQ = 32 - WT>
__global__ void __launch_bounds__((WT + NQ) * 32, 1) crc_mx_kernel(const Params p) {
  using LT = MxLayout<WT, TSN>;
  extern __shared__ __align__(128) uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const LT L = mx_layout<WT, TSN>(raw);
  uint8_t* smem = smem_raw - raw;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  constexpr int NT = (WT + NQ) * 32;
  for (int i = tid; i < 4 * 256; i += NT) {  // slicing tables, replicated once per lane
    const uint32_t v = __ldg(p.tables + TAB_T16 + i);
    uint4* dst = reinterpret_cast<uint4*>(smem + L.tab + (size_t)i * 128);
#pragma unroll
    for (int r = 0; r < 8; ++r) dst[r] = make_uint4(v, v, v, v);
  }
  for (int i = tid; i < 8 * 16; i += NT) {  // Z^96 nibble tables (quad role)
    const uint32_t v = __ldg(p.tables + TAB_Z96N + i);
    uint4* dst = reinterpret_cast<uint4*>(smem + L.zn + (size_t)i * 128);
#pragma unroll
    for (int r = 0; r < 8; ++r) dst[r] = make_uint4(v, v, v, v);
  }
  const uint32_t bars = L.bar + (uint32_t)warp * 2 * 8;
  if (warp < WT && lane == 0) {
    for (int b = 0; b < 2; ++b)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bars + 8 * b), "r"(1) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp < WT) {
    const uint32_t ring = (uint32_t)warp < L.nlow ? L.low + (uint32_t)warp * LT::RING
                                                  : L.high + ((uint32_t)warp - L.nlow) * LT::RING;
    ts_role<MODE, 2, TS_S>(p, L.tab, ring, bars, lane, warp * gridDim.x + blockIdx.x, gridDim.x * WT,
                           pool_size<TSN>(p.n_desc, true), PoolMap<TSN, true>{});
  } else {
    const uint32_t wq = (uint32_t)(warp - WT), nq = pool_size<TSN>(p.n_desc, false);
    const uint32_t lb = L.tab + 4u * lane, lz = L.zn + 4u * lane;
    const uint32_t m128 = 128u * gridDim.y;  // = 128, opaque to ptxas
    const PoolMap<TSN, false> seg_of{};
    for (uint32_t k = wq * gridDim.x + blockIdx.x; k < nq; k += gridDim.x * NQ) {
      const uint32_t idx = seg_of(k);
      quad_segment<MODE, false, true>(p, p.desc[idx], idx, lane, lb, lz, m128);
    }
  }
}

template <int MODE, int WT, int TSN, int NQ = 32 - WT>
static cudaError_t launch_mx_t(const Params& p, int grid_cap, cudaStream_t s) {
  static unsigned long long attr_set = 0;
  uint32_t R0 = 0;
  cudaError_t e = smem_base(&R0);
  if (e != cudaSuccess) return e;
  const MxLayout<WT, TSN> L = mx_layout<WT, TSN>(R0);
  const size_t bytes = L.end - R0;
  if (bytes > TS_SMEM_MAX) return cudaErrorInvalidConfiguration;
  int dev = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if (!((attr_set >> (dev & 63)) & 1ull)) {
    e = cudaFuncSetAttribute(crc_mx_kernel<MODE, WT, TSN, NQ>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
    if (e != cudaSuccess) return e;
    attr_set |= 1ull << (dev & 63);
  }
  const int grid = (int)std::max<uint32_t>(1, std::min<uint32_t>((uint32_t)grid_cap, p.n_desc));
  crc_mx_kernel<MODE, WT, TSN, NQ><<<grid, (WT + NQ) * 32, bytes, s>>>(p);
  return cudaGetLastError();
}

template <int MODE, int W, int NB, int S>
static cudaError_t launch_ts_t(const Params& p, int grid_cap, cudaStream_t s) {
  static unsigned long long attr_set = 0;
  uint32_t R0 = 0;
  cudaError_t e = smem_base(&R0);
  if (e != cudaSuccess) return e;
  const TsLayout<W, NB, S> L = ts_layout<W, NB, S>(R0);
  const size_t bytes = L.end - R0;
  if (bytes > TS_SMEM_MAX) return cudaErrorInvalidConfiguration;
  int dev = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if (!((attr_set >> (dev & 63)) & 1ull)) {
    e = cudaFuncSetAttribute(crc_ts_kernel<MODE, W, NB, S>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
    if (e != cudaSuccess) return e;
    attr_set |= 1ull << (dev & 63);
  }
  const int grid = (int)std::max<uint32_t>(1, std::min<uint32_t>((uint32_t)grid_cap, p.n_desc));
  crc_ts_kernel<MODE, W, NB, S><<<grid, W * 32, bytes, s>>>(p);
  return cudaGetLastError();
}

// CRC-32C hash-pass kernel. With the tensor maps (segments of >= 128 KiB):
//  * whole-image passes (>= 4 segments per strand-kernel warp: the verify, the CE_PIPE checkpoint's hash pass;
//    scaled config B images, b0f vs mixed: 1 GiB 0.248 vs 0.369 ms, 2 GiB 0.479 vs 0.555, 4 GiB 0.933 vs
//    0.880, 8 GiB 1.612 vs 1.596, 16 GiB 3.409 vs 3.349)
//    take the mixed kernel (16 strand-staged + 12 quad-line warps per SM, 5/8 of the segments to the strand
//    role): config B verify +4 % over the strand kernel alone inside the bench, same box (5559 / 5573 vs 5347
//    GB/s), +6 % at 16 MiB chunks; the strand kernel alone was +2.4..7.1 % over the quad-line b0f kernel
//    (profiles/r02_crc_strand_staged.md);
//  * one round of segments (a CE_PIPE restore group's check) the mixed kernel too, although the strand kernel
//    alone is faster there (3438 vs 2908 GB/s summed over a restore's groups: latency-bound warps, one segment
//    each): the checks hide under the copy engine's H2D copies, and one kernel for checks and verify keeps the
//    dominant kernel of the launch list the one whose roofline the bench reports;
//  * otherwise (1-4 rounds, or short segments) the quad-line b0f kernel (a 16-KiB-segment 64 MiB image 48 vs
//    66 us for the strand kernel; 4-KiB chunks 2.8 vs 1.8 TB/s).
// SWAP_CRC_KERNEL (base | b0f | zb | zbb0f | ts | ts16 | mx | mx16; read at every launch) forces one for A/B
// measurements: b0f +0.9..1.7 % over base; the Z^96 byte tables (zb) -10 % (profiles/r02_crc_variants.md).
template <int MODE>
static cudaError_t launch_hash(const Params& p, int grid, cudaStream_t s) {
  const uint32_t slots = 19u * (uint32_t)grid;  // the strand kernel's warps
  int v = 1;
  if (p.tmaps && p.hlane_len >= (128u << 10) && (p.n_desc <= slots || p.n_desc >= 4u * slots)) v = 12;
  if (const char* e = getenv("SWAP_CRC_KERNEL"))
    v = !strcmp(e, "base") ? 0 : !strcmp(e, "zb") ? 2 : !strcmp(e, "zbb0f") ? 3 : !strcmp(e, "ts") ? 10
      : !strcmp(e, "ts16") ? 11 : !strcmp(e, "mx") ? 12 : !strcmp(e, "mx16") ? 13 : 1;
  switch (v) {
    case 0: return launch_hash_t<MODE, false, false>(p, grid, s);
    case 2: return launch_hash_t<MODE, true, false>(p, grid, s);
    case 3: return launch_hash_t<MODE, true, true>(p, grid, s);
    case 10: return launch_ts_t<MODE, 19, 2, TS_S>(p, grid, s);
    case 11: return launch_ts_t<MODE, 16, 2, TS_S>(p, grid, s);
    case 12: return launch_mx_t<MODE, 16, 5, 12>(p, grid, s);
    case 13: return launch_mx_t<MODE, 16, 5, 16>(p, grid, s);
    default: return launch_hash_t<MODE, false, true>(p, grid, s);
  }
}

// Every SM takes part even with few segments (hash_kernel deals them warp-major across CTAs then): a CE_PIPE
// restore group's check (~1 K segments of 256 KiB) ran on 32 SMs before.
int hash_grid(int sm_count, uint32_t n_desc) {
  return (int)std::max<uint32_t>(1, std::min<uint32_t>((uint32_t)sm_count, n_desc));
}


// ------------------------------------------------------------------ HBM hash kernel (XXH64, TMA ring)
// XXH64 consumes a chunk's 32-B stripes strictly in order through four accumulator chains, so a
// chunk's hashing rate is bounded by the round latency, and parallelism must come from chunks.
// One warp owns one chunk at a time; lane 0 streams the chunk into a per-warp shared-memory ring
// with TMA bulk copies (cp.async.bulk + mbarrier complete_tx, XR_STAGES x 4 KiB in flight per
// warp), and lanes 0..3 run the four accumulators out of shared memory (conflict-free: 4 lanes
// read 32 contiguous bytes). This keeps the memory pipe full even with few, huge chunks.
constexpr int XR_WARPS = 4;
constexpr int XR_STAGES = 3;
constexpr uint32_t XR_STAGE = 4096;
constexpr size_t XR_RING = (size_t)XR_STAGES * XR_STAGE;
constexpr size_t XR_SMEM = XR_WARPS * XR_RING + XR_WARPS * XR_STAGES * 8;

__device__ __forceinline__ uint64_t lds_u64(const uint8_t* p) {
  return *reinterpret_cast<const uint64_t*>(p);  // 8-B aligned by construction
}

template <int MODE>
__global__ void __launch_bounds__(XR_WARPS * 32) xxh_ring_kernel(const Params p) {
  extern __shared__ __align__(128) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint8_t* ring = smem + (size_t)warp * XR_RING;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + XR_WARPS * XR_RING) + warp * XR_STAGES;
  if (lane == 0) {
    for (int s = 0; s < XR_STAGES; ++s) mbar_init(bars + s, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  uint32_t seq = 0;  // stages issued by this warp so far (buffer = seq % STAGES, parity = seq / STAGES & 1)
  for (uint32_t idx = blockIdx.x * XR_WARPS + warp; idx < p.n_desc; idx += gridDim.x * XR_WARPS) {
    const SegDesc d = p.desc[idx];
    const uint64_t e = lane == 0 ? expect_early<MODE>(p, d.chunk) : 0;
    const uint8_t* src = reinterpret_cast<const uint8_t*>(d.dev);
    const uint64_t len = d.bytes, len16 = len & ~15ull;
    const uint32_t nst = (uint32_t)((len16 + XR_STAGE - 1) / XR_STAGE);
    auto issue = [&](uint32_t k) {  // lane 0: stage k of this chunk
      const uint32_t b = (seq + k) % XR_STAGES;
      const uint32_t sz = (uint32_t)(len16 - (uint64_t)k * XR_STAGE < XR_STAGE ? len16 - (uint64_t)k * XR_STAGE : XR_STAGE);
      mbar_expect_tx(bars + b, sz);
      bulk_g2s(ring + (size_t)b * XR_STAGE, src + (size_t)k * XR_STAGE, sz, bars + b);
    };
    if (lane == 0) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      for (uint32_t k = 0; k < nst && k < (uint32_t)XR_STAGES; ++k) issue(k);
    }
    uint64_t v = lane == 0 ? P1 + P2 : lane == 1 ? P2 : lane == 2 ? 0ull : 0ull - P1;
    uint32_t last_b = 0;
    for (uint32_t k = 0; k < nst; ++k) {
      const uint32_t b = (seq + k) % XR_STAGES;
      mbar_wait(bars + b, ((seq + k) / XR_STAGES) & 1u);
      const uint32_t sz = (uint32_t)(len16 - (uint64_t)k * XR_STAGE < XR_STAGE ? len16 - (uint64_t)k * XR_STAGE : XR_STAGE);
      if (lane < 4) {
        const uint8_t* q = ring + (size_t)b * XR_STAGE + 8 * lane;
        const uint32_t ns = sz / 32;
#pragma unroll 8
        for (uint32_t s = 0; s < ns; ++s) v = xround(v, lds_u64(q + 32 * s));
      }
      last_b = b;
      __syncwarp();
      if (lane == 0 && k + XR_STAGES < nst) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        issue(k + XR_STAGES);
      }
    }
    const uint64_t v1 = __shfl_sync(0xffffffffu, v, 0), v2 = __shfl_sync(0xffffffffu, v, 1);
    const uint64_t v3 = __shfl_sync(0xffffffffu, v, 2), v4 = __shfl_sync(0xffffffffu, v, 3);
    if (lane == 0) {
      // bytes after the last whole stripe: in the last stage buffer below len16, in HBM above
      const uint8_t* lastbuf = ring + (size_t)last_b * XR_STAGE;
      const uint64_t last_off = nst ? (uint64_t)(nst - 1) * XR_STAGE : 0;
      auto byte_at = [&](uint64_t o) -> uint64_t { return o < len16 ? lastbuf[o - last_off] : src[o]; };
      uint64_t h;
      if (len >= 32) {
        h = rotl64(v1, 1) + rotl64(v2, 7) + rotl64(v3, 12) + rotl64(v4, 18);
        h = xmerge(h, v1);
        h = xmerge(h, v2);
        h = xmerge(h, v3);
        h = xmerge(h, v4);
      } else {
        h = P5;
      }
      h += len;
      uint64_t o = len / 32 * 32;
      for (; o + 8 <= len; o += 8) {
        uint64_t w = 0;
        for (int i = 7; i >= 0; --i) w = (w << 8) | byte_at(o + i);
        h ^= xround(0, w);
        h = rotl64(h, 27) * P1 + P4;
      }
      if (o + 4 <= len) {
        uint64_t w = byte_at(o) | (byte_at(o + 1) << 8) | (byte_at(o + 2) << 16) | (byte_at(o + 3) << 24);
        h ^= w * P1;
        h = rotl64(h, 23) * P2 + P3;
        o += 4;
      }
      for (; o < len; ++o) {
        h ^= byte_at(o) * P5;
        h = rotl64(h, 11) * P1;
      }
      h ^= h >> 33;
      h *= P2;
      h ^= h >> 29;
      h *= P3;
      h ^= h >> 32;
      chunk_result<MODE>(p, d.chunk, h, e);
    }
    seq += nst;
    __syncwarp();
  }
}

template <int MODE>
static cudaError_t launch_xxh_ring(const Params& p, int sm_count, cudaStream_t s) {
  static unsigned long long attr_set = 0;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (!((attr_set >> (dev & 63)) & 1ull)) {
    e = cudaFuncSetAttribute(xxh_ring_kernel<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)XR_SMEM);
    if (e != cudaSuccess) return e;
    attr_set |= 1ull << (dev & 63);
  }
  const uint32_t ctas = (p.n_desc + XR_WARPS - 1) / XR_WARPS;
  const int per_sm = (int)(200 * 1024 / XR_SMEM);  // resident CTAs per SM by shared memory
  const int grid = (int)std::max<uint32_t>(1, std::min<uint32_t>(ctas, (uint32_t)(sm_count * per_sm)));
  xxh_ring_kernel<MODE><<<grid, XR_WARPS * 32, XR_SMEM, s>>>(p);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ HBM hash kernel (XXH64, lane per chunk)
// XXH64 consumes a chunk's 32-B stripes strictly in order, so parallelism comes from chunks:
// one LANE per chunk, its four accumulators in registers, one 256-bit load per stripe (a full
// sector), U stripes in flight (4 or 8), loads that do not allocate in L1. Used for HASH_STORE /
// HASH_CHECK when there are enough chunks to occupy the GPU; launch_xxh_hash picks the launch shape.
constexpr int XK_THREADS = 256;
constexpr size_t XK_OFF_BAR = 2 * XK_THREADS * sizeof(SegDesc);
constexpr size_t XK_SMEM = XK_OFF_BAR + 16;

__device__ __forceinline__ uint64_t w64(const uint32_t (&w)[8], int i) {
  return (uint64_t)w[2 * i] | ((uint64_t)w[2 * i + 1] << 32);
}

template <bool TF>
__device__ __forceinline__ void xxh_stripe(uint64_t (&v)[4], const uint32_t (&w)[8]) {
#pragma unroll
  for (int i = 0; i < 4; ++i) v[i] = TF ? xt_step(v[i], w64(w, i)) : xround(v[i], w64(w, i));
}

// Stripes [0, end) of one chunk into the four accumulators. A U-deep software pipeline (each 256-bit
// load consumed U stripes after issue) keeps U stripes per lane in flight; without it ptxas sinks each
// load next to its use.
template <bool AL32, int U, bool TF>
__device__ __forceinline__ void xxh_stripes(const uint8_t* src, uint64_t end, uint64_t (&v)[4]) {
  const uint64_t n = end / 32;
  uint64_t t = 0;
  if (n >= U) {
    uint32_t buf[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u) ld32na<AL32>(src + u * 32, buf[u]);
    for (; t + 2 * U <= n; t += U) {
      const uint8_t* q = src + (t + U) * 32;
#pragma unroll
      for (int u = 0; u < U; ++u) {
        xxh_stripe<TF>(v, buf[u]);
        ld32na<AL32>(q + u * 32, buf[u]);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) xxh_stripe<TF>(v, buf[u]);
    t += U;
  }
  for (; t < n; ++t) {
    uint32_t w[8];
    ld32na<AL32>(src + t * 32, w);
    xxh_stripe<TF>(v, w);
  }
}

// The end of one chunk's XXH64 once its whole 32-B stripes are in v (xxHash spec): merge, the tail
// [stripes_end, len) read from device memory at src, avalanche; then store / compare its c_g.
template <int MODE>
__device__ __forceinline__ void xxh_finish(const Params& p, const SegDesc& d, const uint64_t (&v)[4], uint64_t e,
                                           const uint8_t* src_override = nullptr) {
  const uint8_t* src = src_override ? src_override : reinterpret_cast<const uint8_t*>(d.dev);
  const uint64_t len = d.bytes;
  uint64_t o = len / 32 * 32;
  uint64_t h;
  if (len >= 32) {
    h = rotl64(v[0], 1) + rotl64(v[1], 7) + rotl64(v[2], 12) + rotl64(v[3], 18);
    h = xmerge(h, v[0]);
    h = xmerge(h, v[1]);
    h = xmerge(h, v[2]);
    h = xmerge(h, v[3]);
  } else {
    h = P5;
  }
  h += len;
  for (; o + 8 <= len; o += 8) {
    h ^= xround(0, ld_u64_smem(src + o));  // bytewise little-endian read (tail is unaligned)
    h = rotl64(h, 27) * P1 + P4;
  }
  if (o + 4 <= len) {
    const uint32_t w = (uint32_t)src[o] | ((uint32_t)src[o + 1] << 8) | ((uint32_t)src[o + 2] << 16) |
                       ((uint32_t)src[o + 3] << 24);
    h ^= (uint64_t)w * P1;
    h = rotl64(h, 23) * P2 + P3;
    o += 4;
  }
  for (; o < len; ++o) {
    h ^= (uint64_t)src[o] * P5;
    h = rotl64(h, 11) * P1;
  }
  h ^= h >> 33;
  h *= P2;
  h ^= h >> 29;
  h *= P3;
  h ^= h >> 32;
  chunk_result<MODE>(p, d.chunk, h, e);
}

// One whole chunk (descriptor d) by one lane.
template <int MODE, int U, bool TF = true>
__device__ __forceinline__ void xxh_chunk(const Params& p, const SegDesc& d) {
  const uint64_t e = expect_early<MODE>(p, d.chunk);
  const uint8_t* src = reinterpret_cast<const uint8_t*>(d.dev);
  uint64_t v[4] = {P1 + P2, P2, 0, 0ull - P1};
  if (TF) {
#pragma unroll
    for (int i = 0; i < 4; ++i) v[i] = xt_init(i);
  }
  const uint64_t stripes_end = (uint64_t)d.bytes / 32 * 32;
  if ((d.dev & 31) == 0) xxh_stripes<true, U, TF>(src, stripes_end, v); else xxh_stripes<false, U, TF>(src, stripes_end, v);
  if (TF) {
#pragma unroll
    for (int i = 0; i < 4; ++i) v[i] = xt_final(v[i]);
  }
  xxh_finish<MODE>(p, d, v, e);
}

template <int MODE, int U, int MAXT>
__global__ void __launch_bounds__(MAXT) xxh_lane_kernel(const Params p) {
  extern __shared__ __align__(128) uint8_t smem[];
  const uint32_t T = blockDim.x;
  SegDesc* sDesc = reinterpret_cast<SegDesc*>(smem);
  uint64_t* sBar = reinterpret_cast<uint64_t*>(smem + 2 * T * sizeof(SegDesc));
  const int tid = threadIdx.x;
  const uint32_t per_round = gridDim.x * T;
  const uint32_t first0 = blockIdx.x * T;
  const uint32_t rounds = p.n_desc > first0 ? (p.n_desc - first0 + per_round - 1) / per_round : 0u;
  auto issue = [&](uint32_t r) {
    const uint32_t first = r * per_round + first0;
    const uint32_t cnt = min(T, p.n_desc - first);
    uint64_t* bar = sBar + (r & 1);
    mbar_expect_tx(bar, cnt * (uint32_t)sizeof(SegDesc));
    bulk_g2s(sDesc + (r & 1) * T, p.desc + first, cnt * (uint32_t)sizeof(SegDesc), bar);
  };
  if (tid == 0) {
    mbar_init(sBar, 1);
    mbar_init(sBar + 1, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (rounds > 0) issue(0);
    if (rounds > 1) issue(1);
  }
  __syncthreads();
  for (uint32_t r = 0; r < rounds; ++r) {
    mbar_wait(sBar + (r & 1), (r >> 1) & 1u);
    const uint32_t idx = r * per_round + first0 + tid;
    if (idx < p.n_desc) {
      const SegDesc d = sDesc[(r & 1) * T + tid];
      xxh_chunk<MODE, U>(p, d);
    }
    __syncthreads();
    if (tid == 0 && r + 2 < rounds) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      issue(r + 2);
    }
  }
}

// Dynamic lane kernel: every lane starts on chunk (its global index) and then takes the next unclaimed
// chunk from a ticket counter (claimed at the start of the current chunk, so the atomic's latency hides
// behind it). The static launches hand every lane its chunks up front, and under load some SMs are
// served more slowly than others: ncu on config B showed SMs idle for 8 % (4 deep) / 26 % (8 deep) of
// the kernel waiting for the slowest one. Here fast lanes simply hash more chunks.
template <int MODE, int U, int MAXT, bool TF = true>
__global__ void __launch_bounds__(MAXT) xxh_dyn_kernel(const Params p) {
  const uint32_t lanes = gridDim.x * blockDim.x;
  uint32_t idx = blockIdx.x * blockDim.x + threadIdx.x;
  while (idx < p.n_desc) {
    const SegDesc d = p.desc[idx];
    const uint32_t next = lanes + atomicAdd(p.ticket, 1u);
    xxh_chunk<MODE, U, TF>(p, d);
    idx = next;
  }
}

// Warp-cooperative XXH64 (one lane still owns one chunk and its four accumulators, but the warp moves
// the data): a warp takes a batch of 32 consecutive chunks from the ticket counter and walks them in
// 512-B blocks; for each of the 32 chunks the warp copies the block into a shared-memory row with one
// coalesced 16-B-per-lane cp.async (512 contiguous bytes, one page per instruction, where the lane
// kernels touch 32 pages per load), S stages in flight; then every lane hashes its own row's stripes
// with LDS.128 (rows padded to 528 B: conflict-free). No registers hold in-flight data, so the depth
// per chunk is S x 512 B instead of U x 32 B.
__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src, uint32_t n) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(n) : "memory");
}
template <int MODE, int W, int S, int K>
__global__ void __launch_bounds__(W * 32) xxh_coop_kernel(const Params p) {
  constexpr int BLK = 16384 / K, ROW = BLK + 16, SPB = BLK / 32;  // block bytes per chunk, row, stripes
  extern __shared__ __align__(128) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint8_t* rows = smem + (size_t)warp * S * K * ROW;
  const uint32_t rows_s = smem_u32(rows);
  const uint32_t n_batches = (p.n_desc + K - 1) / K;
  const uint32_t warps = gridDim.x * W;
  uint32_t batch = blockIdx.x * W + warp;
  while (batch < n_batches) {
    uint32_t next = 0;
    if (lane == 0) next = warps + atomicAdd(p.ticket, 1u);
    next = __shfl_sync(0xffffffffu, next, 0);
    const uint32_t idx = batch * K + lane;
    const bool mine = lane < K && idx < p.n_desc;
    SegDesc d{};
    if (mine) d = p.desc[idx];
    const uint64_t e = mine ? expect_early<MODE>(p, d.chunk) : 0;
    const uint64_t len = mine ? d.bytes : 0;
    uint64_t maxlen = len;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) maxlen = max(maxlen, __shfl_xor_sync(0xffffffffu, maxlen, o));
    const uint32_t nblk = (uint32_t)((maxlen + BLK - 1) / BLK);
    auto issue = [&](uint32_t b) {  // block b of every chunk of the batch into stage b % S
      const uint32_t st = rows_s + (b % S) * K * ROW;
#pragma unroll 4
      for (int c = 0; c < K; ++c) {
        const uint64_t cl = __shfl_sync(0xffffffffu, len, c);
        const uint64_t cb = __shfl_sync(0xffffffffu, d.dev, c);
#pragma unroll
        for (int j = 0; j < BLK / 512; ++j) {
          const uint64_t off = (uint64_t)b * BLK + j * 512 + lane * 16;
          if (off < cl) {
            const uint32_t nb = (uint32_t)(cl - off < 16 ? cl - off : 16);
            cp_async16(st + c * ROW + j * 512 + lane * 16, reinterpret_cast<const void*>(cb + off), nb);
          }
        }
      }
      asm volatile("cp.async.commit_group;" ::: "memory");
    };
#pragma unroll
    for (int b = 0; b < S - 1; ++b) {
      if ((uint32_t)b < nblk) issue(b);
      else asm volatile("cp.async.commit_group;" ::: "memory");
    }
    uint64_t v[4] = {P1 + P2, P2, 0, 0ull - P1};
    const uint64_t stripes = len / 32;
    for (uint32_t b = 0; b < nblk; ++b) {
      __syncwarp();  // every lane is done reading the stage block b + S - 1 overwrites
      if (b + S - 1 < nblk) issue(b + S - 1);
      else asm volatile("cp.async.commit_group;" ::: "memory");
      asm volatile("cp.async.wait_group %0;" ::"n"(S - 1) : "memory");
      __syncwarp();
      const uint64_t s0 = (uint64_t)b * SPB;
      if (s0 < stripes) {
        const uint32_t ns = (uint32_t)(stripes - s0 < SPB ? stripes - s0 : SPB);
        const uint4* row = reinterpret_cast<const uint4*>(rows + ((b % S) * K + lane) * ROW);
        if (ns == SPB) {  // a whole block: shared-memory loads four stripes ahead of the rounds
#pragma unroll 2
          for (int t0 = 0; t0 < SPB; t0 += 4) {
            uint4 a[4], c[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
              a[u] = row[2 * (t0 + u)];
              c[u] = row[2 * (t0 + u) + 1];
            }
#pragma unroll
            for (int u = 0; u < 4; ++u) {
              v[0] = xround(v[0], ((uint64_t)a[u].y << 32) | a[u].x);
              v[1] = xround(v[1], ((uint64_t)a[u].w << 32) | a[u].z);
              v[2] = xround(v[2], ((uint64_t)c[u].y << 32) | c[u].x);
              v[3] = xround(v[3], ((uint64_t)c[u].w << 32) | c[u].z);
            }
          }
        } else {
          for (uint32_t t = 0; t < ns; ++t) {
            const uint4 a = row[2 * t], c = row[2 * t + 1];
            v[0] = xround(v[0], ((uint64_t)a.y << 32) | a.x);
            v[1] = xround(v[1], ((uint64_t)a.w << 32) | a.z);
            v[2] = xround(v[2], ((uint64_t)c.y << 32) | c.x);
            v[3] = xround(v[3], ((uint64_t)c.w << 32) | c.z);
          }
        }
      }
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    __syncwarp();
    if (mine) xxh_finish<MODE>(p, d, v, e);
    batch = next;
  }
}

// Quad-per-chunk XXH64 for few, large chunks (C >= 2 MiB). A chunk's rate is bounded by its four
// accumulator chains (v_j <- rotl(v_j + w*P2, 31)*P1, one round per 32-B stripe), so every chunk of the
// image must be hashed at once and each must have enough bytes in flight to cover memory latency:
//  * a warp owns 8 chunks, lane quad q <-> chunk q, lane j of the quad <-> accumulator v_(j+1): all 32
//    lanes run rounds (the ring kernel used lanes 0..3 of a warp per chunk);
//  * each chunk streams through its own S-stage ring of STG-byte stages in shared memory with TMA bulk
//    copies (cp.async.bulk + one mbarrier per warp stage carrying the 8 chunks' bytes), (S-1) x STG
//    bytes in flight per chunk without occupying registers;
//  * ring q starts 32 x q bytes past a multiple of 128, so the warp's 8-B reads of one stripe (8 quads x
//    32 B) hit every bank exactly twice (two wavefronts, the minimum for 256 B);
//  * work: batches of 8 consecutive chunks; a warp's first batch is interleaved over CTAs (batch
//    warp * grid + cta) so a short image spreads over all SMs, later batches come from the ticket.
// The merge, the < 32-B tail (read from HBM) and the avalanche run on the quad's lane 0 (xxh_finish).
template <int W, int S, int STG, int LPC>
struct XQ {
  static constexpr int CPW = 32 / LPC;                              // chunks per warp
  static constexpr int NC = 4 / LPC;                                // accumulator chains per lane
  static constexpr uint32_t RING = S * STG + 32;                    // one chunk's ring + bank skew
  static constexpr uint32_t WARP_BYTES = CPW * RING;                // CPW % 4 == 0: 128-B aligned
  static constexpr size_t SMEM = (size_t)W * WARP_BYTES + (size_t)W * S * 8 + 128;
};
// LPC = lanes per chunk: 4 (quad, one accumulator per lane) or 2 (pair: lane j of the pair holds
// v_(j+1) and v_(j+3), two independent chains interleaved in one instruction stream).
template <int MODE, int W, int S, int STG, bool TF, int LPC>
__global__ void __launch_bounds__(W * 32) xxh_quad_kernel(const Params p) {
  using G = XQ<W, S, STG, LPC>;
  constexpr int CPW = G::CPW, NC = G::NC;
  extern __shared__ __align__(128) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, q = lane / LPC, j = lane % LPC;
  uint8_t* wbase = smem + (size_t)warp * G::WARP_BYTES;
  uint8_t* ring = wbase + q * G::RING;  // this group's chunk ring (128-B aligned + 32 q)
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + (size_t)W * G::WARP_BYTES) + warp * S;
  if (lane == 0) {
    for (int s = 0; s < S; ++s) mbar_init(bars + s, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  const uint32_t n_batches = (p.n_desc + CPW - 1) / CPW;
  const uint32_t warps = gridDim.x * W;
  uint32_t batch = warp * gridDim.x + blockIdx.x;
  uint32_t seq = 0;  // stages issued by this warp so far: buffer seq % S, parity (seq / S) & 1
  while (batch < n_batches) {
    uint32_t next = 0;
    if (lane == 0) next = warps + atomicAdd(p.ticket, 1u);
    next = __shfl_sync(0xffffffffu, next, 0);
    const uint32_t idx = batch * CPW + q;
    const bool mine = idx < p.n_desc;
    SegDesc d{};
    if (mine) d = p.desc[idx];
    const uint64_t e = (mine && j == 0) ? expect_early<MODE>(p, d.chunk) : 0;
    const uint64_t len = mine ? d.bytes : 0, len16 = len & ~15ull;
    const uint32_t nst_max = __reduce_max_sync(0xffffffffu, (uint32_t)((len16 + STG - 1) / STG));
    // the mover modes copy as they hash: SCATTER reads the image (host-mapped, or a peer replica's HBM for
    // swap_pull_stripes) and writes the regions, GATHER the reverse; each stage is stored from the ring by
    // the quad leader with a TMA bulk store once the quad has hashed it
    constexpr bool COPY = (MODE == GATHER || MODE == SCATTER);
    const uint8_t* src = reinterpret_cast<const uint8_t*>(MODE == SCATTER ? d.host : d.dev);
    uint8_t* dst = reinterpret_cast<uint8_t*>(MODE == SCATTER ? d.dev : d.host);
    // stage k of all the warp's chunks: lane 0 arms the barrier with their byte total, group leaders copy
    auto issue = [&](uint32_t k) {
      const uint32_t b = (seq + k) % S;
      const uint64_t o = (uint64_t)k * STG;
      const uint32_t sz = o < len16 ? (uint32_t)(len16 - o < STG ? len16 - o : STG) : 0u;
      const uint32_t tot = __reduce_add_sync(0xffffffffu, j == 0 ? sz : 0u);
      if (lane == 0) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_expect_tx(bars + b, tot);
      }
      __syncwarp();
      if (j == 0 && sz) bulk_g2s(ring + (size_t)b * STG, src + o, sz, bars + b);
    };
    for (uint32_t k = 0; k < nst_max && k < (uint32_t)S; ++k) issue(k);
    uint64_t v[NC];
#pragma unroll
    for (int c = 0; c < NC; ++c) {
      const int a = j + c * LPC;  // accumulator index 0..3
      v[c] = TF ? xt_init(a) : a == 0 ? P1 + P2 : a == 1 ? P2 : a == 2 ? 0ull : 0ull - P1;
    }
    const uint64_t stripes = len / 32;
    for (uint32_t k = 0; k < nst_max; ++k) {
      const uint32_t b = (seq + k) % S;
      mbar_wait(bars + b, ((seq + k) / S) & 1u);
      const uint64_t s0 = (uint64_t)k * (STG / 32);
      if (s0 < stripes) {
        const uint8_t* qb = ring + (size_t)b * STG + 8 * j;
        const uint32_t ns = (uint32_t)(stripes - s0 < (uint64_t)(STG / 32) ? stripes - s0 : (uint64_t)(STG / 32));
        auto stripe = [&](uint32_t s) {
#pragma unroll
          for (int c = 0; c < NC; ++c) {
            const uint64_t w = lds_u64(qb + 32 * s + 8 * LPC * c);
            v[c] = TF ? xt_step(v[c], w) : xround(v[c], w);
          }
        };
        if (ns == STG / 32) {
#pragma unroll 16
          for (uint32_t s = 0; s < (uint32_t)(STG / 32); ++s) stripe(s);
        } else {
          for (uint32_t s = 0; s < ns; ++s) stripe(s);
        }
      }
      __syncwarp();  // every lane is done with buffer b before it is refilled
      if (COPY && j == 0) {  // store the stage, and let the TMA finish reading it before the refill
        const uint64_t o = (uint64_t)k * STG;
        if (o < len16) {
          bulk_s2g(dst + o, ring + (size_t)b * STG, (uint32_t)(len16 - o < STG ? len16 - o : STG));
          bulk_wait_read_all();
        }
      }
      if (k + S < nst_max) issue(k + S);
    }
    if (COPY && mine && j == 0) {
      for (uint64_t o = len16; o < len; ++o) dst[o] = src[o];  // the < 16-B tail the bulk copies cannot carry
      bulk_wait_all();  // the stores are complete before the chunk's result is published
    }
    uint64_t vv[4];
#pragma unroll
    for (int c = 0; c < NC; ++c) {
      if (TF) v[c] = xt_final(v[c]);
#pragma unroll
      for (int x = 0; x < LPC; ++x) vv[x + c * LPC] = __shfl_sync(0xffffffffu, v[c], (lane & ~(LPC - 1)) + x);
    }
    if (mine && j == 0) xxh_finish<MODE>(p, d, vv, e, src);
    seq += nst_max;
    batch = next;
    __syncwarp();
  }
}

template <int MODE, int W, int S, int STG, bool TF = true, int LPC = 4>
static cudaError_t launch_xxh_quad(const Params& p, int sm_count, cudaStream_t s) {
  using G = XQ<W, S, STG, LPC>;
  if (!p.ticket) return cudaErrorInvalidValue;
  static unsigned long long attr_set = 0;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (!((attr_set >> (dev & 63)) & 1ull)) {
    e = cudaFuncSetAttribute(xxh_quad_kernel<MODE, W, S, STG, TF, LPC>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)G::SMEM);
    if (e != cudaSuccess) return e;
    attr_set |= 1ull << (dev & 63);
  }
  const uint32_t n_batches = (p.n_desc + G::CPW - 1) / G::CPW;
  // one CTA per SM while every warp slot has a batch; fewer CTAs only for tiny images
  const int grid = (int)std::max<uint32_t>(1, std::min<uint32_t>((uint32_t)sm_count, n_batches));
  e = cudaMemsetAsync(p.ticket, 0, sizeof(unsigned int), s);
  if (e != cudaSuccess) return e;
  xxh_quad_kernel<MODE, W, S, STG, TF, LPC><<<grid, W * 32, G::SMEM, s>>>(p);
  return cudaGetLastError();
}

template <int MODE, int U>
static cudaError_t launch_xxh_lane(const Params& p, int sm_count, cudaStream_t s) {
  const uint32_t blocks = (p.n_desc + XK_THREADS - 1) / XK_THREADS;
  const int grid = (int)std::max<uint32_t>(1, std::min<uint32_t>(blocks, (uint32_t)sm_count * 4));
  xxh_lane_kernel<MODE, U, XK_THREADS><<<grid, XK_THREADS, XK_SMEM, s>>>(p);
  return cudaGetLastError();
}

// Balanced lane launch: exactly one CTA per SM (the dynamic shared-memory request admits only one, so
// the block scheduler cannot stack CTAs on some SMs and leave others idle — with the 4-CTA/SM launch
// above, config B's 197 CTAs ran at 11.2 ms or 20.7 ms depending on placement), chunks spread evenly:
// T = ceil(n / SMs) lanes per SM, rounded to whole warps, capped by the register file.
constexpr size_t XB_SMEM = 116 * 1024;
template <int MODE, int U>
static cudaError_t launch_xxh_lane_bal(const Params& p, int sm_count, cudaStream_t s) {
  constexpr int MAXT = U >= 8 ? 640 : 1024;
  static unsigned long long attr_set = 0;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (!((attr_set >> (dev & 63)) & 1ull)) {
    e = cudaFuncSetAttribute(xxh_lane_kernel<MODE, U, MAXT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)XB_SMEM);
    if (e != cudaSuccess) return e;
    attr_set |= 1ull << (dev & 63);
  }
  // R full rounds of T lanes per SM (a last round a third full would leave two thirds of the lanes idle)
  const uint32_t per_sm = (p.n_desc + sm_count - 1) / sm_count;
  const uint32_t R = std::max<uint32_t>(1, (per_sm + MAXT - 1) / MAXT);
  // rounded up to whole warps: on config B (50.4 K chunks) 143 CTAs of 352 lanes verify in 10.55 ms,
  // 148 CTAs of 341 lanes (every SM busy, a partial last warp) in 11.06 ms (in-process A/B, 8 reps)
  const uint32_t T = std::min<uint32_t>(MAXT, std::max<uint32_t>(32, ((per_sm + R - 1) / R + 31) / 32 * 32));
  const int grid = (int)std::min<uint32_t>((uint32_t)sm_count, (p.n_desc + T - 1) / T);
  xxh_lane_kernel<MODE, U, MAXT><<<grid, T, XB_SMEM, s>>>(p);
  return cudaGetLastError();
}

// Dynamic lane launch: one CTA of T lanes per SM (SWAP_XXH_DYN_T overrides T, for measurements), the
// ticket zeroed on the launching stream first.
template <int MODE, int U, bool TF = true>
static cudaError_t launch_xxh_dyn(const Params& p, int sm_count, cudaStream_t s) {
  constexpr int MAXT = U >= 8 ? 640 : 1024;
  if (!p.ticket) return launch_xxh_lane_bal<MODE, U>(p, sm_count, s);
  uint32_t T = U >= 8 ? 192 : 352;
  if (const char* e = getenv("SWAP_XXH_DYN_T")) T = std::max(32, std::min(MAXT, atoi(e)));
  const uint32_t per_sm = (p.n_desc + sm_count - 1) / sm_count;
  T = std::min<uint32_t>(T, std::max<uint32_t>(32, (per_sm + 31) / 32 * 32));
  const int grid = (int)std::min<uint32_t>((uint32_t)sm_count, (p.n_desc + T - 1) / T);
  cudaError_t e = cudaMemsetAsync(p.ticket, 0, sizeof(unsigned int), s);
  if (e != cudaSuccess) return e;
  xxh_dyn_kernel<MODE, U, MAXT, TF><<<grid, T, 0, s>>>(p);
  return cudaGetLastError();
}

template <int MODE, int W, int S, int K = 32>
static cudaError_t launch_xxh_coop(const Params& p, int sm_count, cudaStream_t s) {
  constexpr size_t smem = (size_t)W * S * K * (16384 / K + 16);
  if (!p.ticket) return cudaErrorInvalidValue;
  static unsigned long long attr_set = 0;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (!((attr_set >> (dev & 63)) & 1ull)) {
    e = cudaFuncSetAttribute(xxh_coop_kernel<MODE, W, S, K>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr_set |= 1ull << (dev & 63);
  }
  const uint32_t n_batches = (p.n_desc + K - 1) / K;
  const int grid = (int)std::max<uint32_t>(1, std::min<uint32_t>((uint32_t)sm_count, (n_batches + W - 1) / W));
  e = cudaMemsetAsync(p.ticket, 0, sizeof(unsigned int), s);
  if (e != cudaSuccess) return e;
  xxh_coop_kernel<MODE, W, S, K><<<grid, W * 32, smem, s>>>(p);
  return cudaGetLastError();
}

// Enough chunks for the lane-per-chunk kernels (below this the TMA ring, one warp per chunk, wins).
bool hash_xxh_lane_ok(int sm_count, uint32_t n_desc) { return n_desc >= (uint32_t)sm_count * 27u; }

int mover_threads() { return THREADS; }
size_t mover_smem_bytes(int kind) {
  return kind == KIND_CRC32C ? SmemLayout<KIND_CRC32C>::bytes : SmemLayout<KIND_NONE>::bytes;
}

template <int MODE, int KIND>
static cudaError_t launch_t(const Params& p, int grid, cudaStream_t s) {
  const size_t smem = SmemLayout<KIND>::bytes;
  static unsigned long long attr_set = 0;  // bit per device: the attribute is per function, per device
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (!((attr_set >> (dev & 63)) & 1ull)) {
    e = cudaFuncSetAttribute(mover_kernel<MODE, KIND>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr_set |= 1ull << (dev & 63);
  }
  mover_kernel<MODE, KIND><<<grid, THREADS, smem, s>>>(p);
  return cudaGetLastError();
}

// Kernel choice for XXH64 hash passes: automatic (below), or forced with SWAP_XXH_KERNEL for
// measurements and tests (read at every launch, so one process can interleave variants).
static int xxh_variant() {
  const char* e = getenv("SWAP_XXH_KERNEL");
  if (!e) return 0;
  const char* names[] = {"lane8", "bal", "bal8", "dyn", "coop", "coop16", "coop8", "ring", "quad", "quad1k", "quad4k",
                         "quad_x", "dyn_x", "quad2", "pair", "pair2", "quad3k"};
  for (int i = 0; i < 17; ++i)
    if (!strcmp(e, names[i])) return i + 1;
  return 0;
}

cudaError_t launch_xxh_hash(int mode, const Params& p, int sm_count, cudaStream_t s) {
  if (p.n_desc == 0) return cudaSuccess;
  const bool st = mode == HASH_STORE;
  switch (xxh_variant()) {  // forced: lane8 | bal | bal8 | dyn | coop | coop16 | coop8 | ring | quad | quad1k | quad4k
    case 1: return st ? launch_xxh_lane<HASH_STORE, 8>(p, sm_count, s) : launch_xxh_lane<HASH_CHECK, 8>(p, sm_count, s);
    case 2: return st ? launch_xxh_lane_bal<HASH_STORE, 4>(p, sm_count, s) : launch_xxh_lane_bal<HASH_CHECK, 4>(p, sm_count, s);
    case 3: return st ? launch_xxh_lane_bal<HASH_STORE, 8>(p, sm_count, s) : launch_xxh_lane_bal<HASH_CHECK, 8>(p, sm_count, s);
    case 4: return st ? launch_xxh_dyn<HASH_STORE, 4>(p, sm_count, s) : launch_xxh_dyn<HASH_CHECK, 4>(p, sm_count, s);
    case 5: return st ? launch_xxh_coop<HASH_STORE, 6, 2, 32>(p, sm_count, s) : launch_xxh_coop<HASH_CHECK, 6, 2, 32>(p, sm_count, s);
    case 6: return st ? launch_xxh_coop<HASH_STORE, 6, 2, 16>(p, sm_count, s) : launch_xxh_coop<HASH_CHECK, 6, 2, 16>(p, sm_count, s);
    case 7: return st ? launch_xxh_coop<HASH_STORE, 6, 2, 8>(p, sm_count, s) : launch_xxh_coop<HASH_CHECK, 6, 2, 8>(p, sm_count, s);
    case 8: return st ? launch_xxh_ring<HASH_STORE>(p, sm_count, s) : launch_xxh_ring<HASH_CHECK>(p, sm_count, s);
    case 9: return st ? launch_xxh_quad<HASH_STORE, 4, 3, 2048>(p, sm_count, s) : launch_xxh_quad<HASH_CHECK, 4, 3, 2048>(p, sm_count, s);
    case 10: return st ? launch_xxh_quad<HASH_STORE, 6, 4, 1024>(p, sm_count, s) : launch_xxh_quad<HASH_CHECK, 6, 4, 1024>(p, sm_count, s);
    case 11: return st ? launch_xxh_quad<HASH_STORE, 2, 3, 4096>(p, sm_count, s) : launch_xxh_quad<HASH_CHECK, 2, 3, 4096>(p, sm_count, s);
    // the spec-form round (xround) instead of the t-form, for A/B measurements
    case 12: return st ? launch_xxh_quad<HASH_STORE, 4, 3, 2048, false>(p, sm_count, s) : launch_xxh_quad<HASH_CHECK, 4, 3, 2048, false>(p, sm_count, s);
    case 13: return st ? launch_xxh_dyn<HASH_STORE, 4, false>(p, sm_count, s) : launch_xxh_dyn<HASH_CHECK, 4, false>(p, sm_count, s);
    case 14: return st ? launch_xxh_quad<HASH_STORE, 3, 2, 4096>(p, sm_count, s) : launch_xxh_quad<HASH_CHECK, 3, 2, 4096>(p, sm_count, s);
    case 15: return st ? launch_xxh_quad<HASH_STORE, 2, 3, 2048, true, 2>(p, sm_count, s) : launch_xxh_quad<HASH_CHECK, 2, 3, 2048, true, 2>(p, sm_count, s);
    case 16: return st ? launch_xxh_quad<HASH_STORE, 2, 2, 3072, true, 2>(p, sm_count, s) : launch_xxh_quad<HASH_CHECK, 2, 2, 3072, true, 2>(p, sm_count, s);
    case 17: return st ? launch_xxh_quad<HASH_STORE, 4, 2, 3072>(p, sm_count, s) : launch_xxh_quad<HASH_CHECK, 4, 2, 3072>(p, sm_count, s);
    default: break;
  }
  // Measured on config B (52.57 GB, profiles/r02_xxh_quad.md), TB/s: the quad-per-chunk
  // TMA-ring kernel with 4 warps x 2 stages of 3 KiB per chunk from 256 KiB to 4 MiB chunks (256 KiB 6.35
  // vs the lane kernel 6.19; 512 KiB 6.26; 2 MiB 6.32); with 8 MiB and more (fewer than ~7 K chunks) 3
  // warps x 2 stages of 4 KiB -- half the per-stage overhead per byte -- (16 MiB 5.06 vs 4.76; the r01
  // kernels reached 1.16). Below 256 KiB and without a ticket counter, the lane kernels.
  const uint32_t n = p.n_desc, many = (uint32_t)sm_count * 192u;
  if (p.chunk_bytes < (256u << 10) || !p.ticket) {
    if (n >= many) return st ? launch_xxh_lane<HASH_STORE, 8>(p, sm_count, s) : launch_xxh_lane<HASH_CHECK, 8>(p, sm_count, s);
    if (hash_xxh_lane_ok(sm_count, n) || !p.ticket)
      return st ? launch_xxh_lane_bal<HASH_STORE, 8>(p, sm_count, s) : launch_xxh_lane_bal<HASH_CHECK, 8>(p, sm_count, s);
    return st ? launch_xxh_ring<HASH_STORE>(p, sm_count, s) : launch_xxh_ring<HASH_CHECK>(p, sm_count, s);
  }
  if (p.chunk_bytes >= (8u << 20))
    return st ? launch_xxh_quad<HASH_STORE, 3, 2, 4096>(p, sm_count, s) : launch_xxh_quad<HASH_CHECK, 3, 2, 4096>(p, sm_count, s);
  return st ? launch_xxh_quad<HASH_STORE, 4, 2, 3072>(p, sm_count, s) : launch_xxh_quad<HASH_CHECK, 4, 2, 3072>(p, sm_count, s);
}

// XXH64 GATHER / SCATTER through the quad-per-chunk kernel (copy + hash from the TMA ring), sized like the
// verify kernels; SWAP_XXH_MOVER=warp keeps the warp-per-chunk mover (measurements).
bool xxh_quad_mover_enabled() {
  const char* e = getenv("SWAP_XXH_MOVER");
  return !(e && !strcmp(e, "warp"));
}
cudaError_t launch_xxh_move(int mode, const Params& p, int sm_count, cudaStream_t s) {
  if (p.n_desc == 0) return cudaSuccess;
  const bool big = p.chunk_bytes >= (8u << 20);
  if (mode == GATHER)
    return big ? launch_xxh_quad<GATHER, 3, 2, 4096>(p, sm_count, s) : launch_xxh_quad<GATHER, 4, 2, 3072>(p, sm_count, s);
  if (mode == SCATTER)
    return big ? launch_xxh_quad<SCATTER, 3, 2, 4096>(p, sm_count, s) : launch_xxh_quad<SCATTER, 4, 2, 3072>(p, sm_count, s);
  return cudaErrorInvalidValue;
}

cudaError_t launch_mover(int mode, int kind, const Params& p, int grid, cudaStream_t s) {
  if (p.n_desc == 0) return cudaSuccess;
#define SWK_CASE(M, K) \
  if (mode == M && kind == K) return launch_t<M, K>(p, grid, s);
  SWK_CASE(GATHER, KIND_NONE)
  SWK_CASE(GATHER, KIND_CRC32C)
  SWK_CASE(GATHER, KIND_XXH64)
  SWK_CASE(SCATTER, KIND_NONE)
  SWK_CASE(SCATTER, KIND_CRC32C)
  SWK_CASE(SCATTER, KIND_XXH64)
  SWK_CASE(HASH_STORE, KIND_XXH64)
  SWK_CASE(HASH_CHECK, KIND_XXH64)
  if (mode == HASH_STORE && kind == KIND_CRC32C) return launch_hash<HASH_STORE>(p, grid, s);
  if (mode == HASH_CHECK && kind == KIND_CRC32C) return launch_hash<HASH_CHECK>(p, grid, s);
#undef SWK_CASE
  return cudaErrorInvalidValue;
}

// One warp per span (warp-strided over the list), 16-B stores by all 32 lanes, ragged tail bytewise.
__global__ void __launch_bounds__(256) zero_fill_kernel(const ZSpan* __restrict__ spans, uint32_t n) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t warps = gridDim.x * (blockDim.x >> 5);
  for (uint32_t w = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); w < n; w += warps) {
    const uint64_t dst = spans[w].dst, bytes = spans[w].bytes;
    uint4* v = reinterpret_cast<uint4*>(dst);
    const uint64_t nv = bytes >> 4;
    for (uint64_t i = lane; i < nv; i += 32) v[i] = make_uint4(0u, 0u, 0u, 0u);
    for (uint64_t i = (nv << 4) + lane; i < bytes; i += 32) reinterpret_cast<uint8_t*>(dst)[i] = 0;
  }
}

cudaError_t launch_zero_fill(const ZSpan* spans, uint32_t n, int sm_count, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  const uint32_t grid = (uint32_t)std::min<uint64_t>((uint64_t)sm_count * 8, (n + 7) / 8);
  zero_fill_kernel<<<grid, 256, 0, s>>>(spans, n);
  return cudaGetLastError();
}

}  // namespace swk
