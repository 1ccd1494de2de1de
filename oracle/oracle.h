/*
 * oracle.h — plain CPU oracle for the swap-image hot path.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library. The product path
 * (paper_conf_sc_stoyanovsracb25_b200/) never includes, links or calls it, and
 * shares no code, table or constant generator with it.
 *
 * What it computes (SURVEY.md §8(c) "Definition, step by step", which DESIGN.md
 * adopts as the reading of the paper's in-memory GPU snapshot
 * §3.2 "in-memory snapshot of the GPU state" and L171 §4.2 "saves the amount of
 * GPU memory in use ... creates an in-memory snapshot"):
 *   1 validate, 2 layout, 3 chunks, 4 pack, 5 checksums, 6 manifest,
 *   7 shard summary, 8 unpack (restore), 9 verify.
 * The paper prints no image, checksum or manifest value (its mechanism is the
 * closed cuda-checkpoint driver path), so every pin is external:
 * CRC-32C test vectors (RFC 3720 §B.4), the xxHash spec vectors, the CRC
 * combine algebra, brute force and round-trip identities (tests/test_oracle_*.py).
 *
 * Memory model: device memory is stood in for by a host byte array `mem`;
 * region i's bytes live at mem + (addr_i - mem_base).
 * Return codes mirror the product's swap_status numerically (0 OK, -1 EINVAL,
 * -5 ECORRUPT) but are defined here independently.
 */
#ifndef SWAP_ORACLE_H
#define SWAP_ORACLE_H
#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ORACLE_OK 0
#define ORACLE_EINVAL (-1)
#define ORACLE_ECORRUPT (-5)

#define ORACLE_CRC32C 1u
#define ORACLE_XXH64 2u

typedef struct {
  uint64_t addr;  /* device virtual address of the region (16-B aligned) */
  uint64_t bytes; /* region size, any value >= 0 */
  uint32_t id;    /* caller id, unique */
  uint32_t kind;  /* 0 weights, 1 kv, 2 workspace, 3 other */
} oracle_region;

/* ---- checksums (step 5) ---- */
uint32_t oracle_crc32c_bitwise(const uint8_t* p, uint64_t n);  /* definition: shift register */
uint32_t oracle_crc32c_table(const uint8_t* p, uint64_t n);    /* Sarwate byte table */
uint32_t oracle_crc32c_sse42(const uint8_t* p, uint64_t n);    /* x86 crc32 instruction */
int oracle_have_sse42(void);
/* crc(A||B) from crc(A), crc(B), |B| — zlib GF(2) matrix algebra. */
uint32_t oracle_crc32c_combine(uint32_t crc_a, uint32_t crc_b, uint64_t len_b);
uint64_t oracle_xxh64(const uint8_t* p, uint64_t n, uint64_t seed);
uint64_t oracle_chunk_hash(uint32_t kind, const uint8_t* p, uint64_t n); /* H_K, zero-extended */

/* ---- plan (steps 1-3) ---- */
/* Fills off[n], first[n], nchunks[n] (caller-allocated) and the totals. */
int oracle_plan(const oracle_region* r, uint64_t n, uint64_t chunk_bytes, uint64_t align,
                uint64_t* off, uint64_t* first, uint64_t* nchunks,
                uint64_t* payload_bytes, uint64_t* n_chunks);
uint64_t oracle_manifest_bytes(uint64_t n_regions, uint64_t n_chunks);
/* image_bytes = align_up(payload_bytes, A) + manifest_bytes; also returns the manifest offset. */
int oracle_image_layout(const oracle_region* r, uint64_t n, uint64_t chunk_bytes, uint64_t align,
                        uint64_t* image_bytes, uint64_t* manifest_off);

/* ---- checkpoint (steps 4-6): writes payload + zero padding + manifest into image ---- */
int oracle_checkpoint(const oracle_region* r, uint64_t n, const uint8_t* mem, uint64_t mem_base,
                      uint64_t mem_len, uint32_t kind, uint64_t chunk_bytes, uint64_t align,
                      uint32_t rank, uint32_t world, uint8_t* image, uint64_t image_cap,
                      int threads);

/* ---- shard summary (step 7): 64 B ---- */
int oracle_summary(const uint8_t* manifest, uint64_t manifest_len, uint64_t image_bytes,
                   uint8_t out[64]);
uint32_t oracle_global_digest(const uint8_t* summaries, uint64_t world);

/* ---- restore (step 8) and verify (step 9) ---- */
/* Checks the manifest CRC first (ECORRUPT, nothing written); then writes every
 * region byte and counts chunks whose hash over the moved bytes != recorded. */
int oracle_restore(const uint8_t* image, uint64_t manifest_off, uint8_t* mem, uint64_t mem_base,
                   uint64_t mem_len, uint64_t* n_bad, uint64_t* first_bad, int threads);
/* Same as oracle_restore with CRC-32C from the SSE4.2 instruction: the "fast" CPU timing of the bench. */
int oracle_restore_fast(const uint8_t* image, uint64_t manifest_off, uint8_t* mem, uint64_t mem_base,
                        uint64_t mem_len, uint64_t* n_bad, uint64_t* first_bad, int threads);
int oracle_verify(const uint8_t* manifest, uint8_t* mem, uint64_t mem_base, uint64_t mem_len,
                  uint64_t* n_bad, uint64_t* first_bad, int threads);
/* Manifest CRC check alone: 1 = intact. */
int oracle_manifest_ok(const uint8_t* manifest);

#ifdef __cplusplus
}
#endif
#endif
