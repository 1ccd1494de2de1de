/*
 * swap.h — C ABI of libswap: B200-native checkpoint/restore of an inference engine's
 * GPU memory state (the data path of SwapServeLLM's model hot-swap).
 *
 * Paper: Stoyanov et al., "Engine-Agnostic Model Hot-Swapping for Cost-Effective LLM
 * Inference", SC Workshops '25 (/root/reference/PAPER.md, "P:Lnnn" = line nnn).
 *   - preempt = "saves the amount of GPU memory in use. It then creates an in-memory
 *     snapshot ... thus freeing GPU capacity" (§4.2)      -> swap_checkpoint + swap_sync
 *   - snapshot taken once after initialisation, restored many times (§3, §3.2)
 *                                                                  -> REGISTERED -> CHECKPOINTED -> RESTORED*
 *   - swap-in = reserve memory, restore GPU state, check the engine (§3.3, §3.4);
 *     its time "primarily depends on the GPU memory utilized" (§5.3)
 *                                                                  -> swap_restore + swap_verify
 *   - per-GPU topology fixed at init, per-GPU reservations (§6) -> one ctx per (process, device, rank)
 * The paper's mechanism is the closed cuda-checkpoint driver path; the image
 * layout, chunk checksums and manifest below are this library's (DESIGN.md §"Readings",
 * SURVEY.md §8(c)), identical to the CPU oracle's definition in oracle/oracle.c.
 *
 * Conventions (all entry points):
 *   - Every call returns swap_status: 0 = OK, < 0 = error. Nothing aborts or throws.
 *   - Argument checks run in a fixed order: null/arg -> config -> alignment -> overlap ->
 *     duplicate id -> state -> CUDA; the first failing check's code is returned.
 *   - CUDA failures return SWAP_ECUDA; swap_last_error(ctx) holds the text.
 *   - Streams are cudaStream_t values passed as swap_stream_t (NULL = legacy default stream).
 *   - Calls on one ctx are NOT thread-safe; the caller serialises them (the paper's
 *     per-backend write lock, §3.5). Distinct ctxs are independent.
 *   - There is no CPU fallback: with no usable sm_100 device, swap_create returns SWAP_ECUDA.
 */
#ifndef SWAP_H
#define SWAP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define SWAP_API __attribute__((visibility("default")))
#else
#define SWAP_API
#endif

typedef int32_t swap_status;
#define SWAP_OK 0
#define SWAP_EINVAL (-1)       /* bad argument, config or region table */
#define SWAP_ENOMEM (-2)       /* host pinning or device allocation failed */
#define SWAP_ECUDA (-3)        /* CUDA runtime error; see swap_last_error */
#define SWAP_ESTATE (-4)       /* call not valid in the ctx's current state */
#define SWAP_ECORRUPT (-5)     /* manifest CRC bad, or >= 1 chunk checksum mismatch */
#define SWAP_ENCCL (-6)        /* inconsistent global manifest (rank/world mismatch) */
#define SWAP_EUNSUPPORTED (-7) /* valid but unsupported here (e.g. chunk_bytes > 2 GiB) */
#define SWAP_EINTERNAL (-8)

/* Chunk checksum H_K (reading 1-3): */
#define SWAP_CHECKSUM_CRC32C 1u /* CRC-32C/ISCSI (RFC 3720), zero-extended to u64 */
#define SWAP_CHECKSUM_XXH64 2u  /* XXH64, seed 0 for every chunk */

/* Data mover for checkpoint/restore (the image bytes are identical for all of them): */
#define SWAP_MECH_AUTO 0u        /* default, resolved per call from the measured crossover: restore
                                    SM < 2 GiB, else CE_PIPE; checkpoint SM < 1 GiB, else CE_PIPE; XXH64 with
                                    chunks > 4 MiB: restore CE_BATCH from 2 GiB (SM below) */
#define SWAP_MECH_SM 1u          /* one SM kernel: 16-B vector loads/stores to mapped pinned host memory with the
                                    chunk checksum fused from the same registers (one pass, bytes checked in flight) */
#define SWAP_MECH_CE_REGION 2u   /* copy engine: cudaMemcpyAsync per region + separate HBM hash pass */
#define SWAP_MECH_CE_CHUNK 3u    /* copy engine: cudaMemcpyAsync per chunk + HBM hash pass */
#define SWAP_MECH_CE_BATCH 4u    /* copy engine: the per-chunk copies coalesced into maximal runs contiguous on
                                    both sides, one cudaMemcpyAsync per run, + HBM hash pass */
#define SWAP_MECH_CE_PIPE 5u     /* copy engine moves the image in groups of ~pipe_mib MiB on the caller's stream
                                    while the hash kernel checks (restore) / hashes (checkpoint) each group from
                                    HBM on a second, library-owned stream; the caller's stream joins at the end */
#define SWAP_MECH_SM_NOCHECK 6u  /* diagnostic: the SM kernel with the checksum compiled out. Checkpoint leaves
                                    c_g unspecified; restore reports no mismatches. Only for measuring the
                                    fused-checksum overhead (BASELINE.json north_star: <= 5 %). */
#define SWAP_MECH_COUNT 7u

/* Region kinds (manifest only; movement is kind-agnostic) */
#define SWAP_KIND_WEIGHTS 0u
#define SWAP_KIND_KV 1u
#define SWAP_KIND_WORKSPACE 2u
#define SWAP_KIND_OTHER 3u

/* One registered device allocation. dev_addr must be 16-B aligned; bytes may be any
 * value (0 allowed: a region record with no chunks). Non-empty regions must not
 * overlap; ids must be unique. Regions are laid out in the image in the order given. */
typedef struct {
  uint64_t dev_addr;
  uint64_t bytes;
  uint32_t id;
  uint32_t kind; /* SWAP_KIND_* (0..3) */
} swap_region_t;

typedef struct {
  uint64_t chunk_bytes; /* checksum granule C: power of 2, >= 16, <= 2^31; 0 -> 1 MiB */
  uint64_t align;       /* image offset alignment A: power of 2, >= 16; 0 -> 4096 */
  uint32_t checksum;    /* SWAP_CHECKSUM_*; 0 -> CRC32C */
  uint32_t mechanism;   /* SWAP_MECH_*; default SWAP_MECH_AUTO */
  int32_t device;       /* CUDA device ordinal the regions live on */
  int32_t rank;         /* 0 <= rank < world (tensor-parallel shard index) */
  int32_t world;        /* >= 1 */
  uint32_t grid_ctas;   /* SM mover grid; 0 -> auto (2 CTAs per SM) */
  uint32_t seg_bytes;   /* CRC32C work split inside a chunk: power of 2, >= 4096; 0 -> auto (at registration:
                           one segment per warp slot of the GPU, 4 KiB .. 256 KiB) */
  uint32_t pipe_mib;    /* SWAP_MECH_CE_PIPE group size in MiB (rounded up to whole chunks); 0 -> auto: payload/32
                           clamped to [16, 512] MiB */
  int32_t host_numa;    /* host NUMA placement of the image (per-GPU topology fixed at init):
                           0 -> auto: the node sysfs reports for the device's PCI function
                           (/sys/bus/pci/devices/<bus id>/numa_node), preferred policy (mbind
                           MPOL_PREFERRED) and zero-filling threads pinned to that node's CPUs;
                           n >= 1 -> node n-1; -1 -> no placement (first touch by unbound threads).
                           A single-node host or an unknown node means no placement. */
  uint32_t reserved0;   /* 0 */
} swap_config_t;

typedef struct {
  uint64_t n_bad;           /* chunks whose checksum over the bytes moved by the last restore
                               differs from the manifest (fused check) */
  uint64_t first_bad_chunk; /* lowest such global chunk index, or UINT64_MAX */
  uint64_t hbm_n_bad;       /* same, recomputed from device memory by the HBM pass (if run) */
  uint64_t hbm_first_bad;   /* lowest such chunk, or UINT64_MAX */
  uint32_t manifest_ok;     /* 1 if the manifest CRC holds */
  uint32_t hbm_checked;     /* 1 if the HBM pass ran in this call */
} swap_verify_result_t;

/* Exactly 64 bytes, little-endian; the unit of the multi-GPU all-gather. */
typedef struct {
  uint32_t rank, world, checksum, n_regions;
  uint64_t n_chunks, payload_bytes, image_bytes;
  uint64_t manifest_crc; /* the manifest's trailing CRC-32C */
  uint64_t chunk_digest; /* CRC-32C over the n_chunks little-endian u64 chunk checksums */
  uint64_t reserved;     /* 0 */
} swap_shard_summary_t;

/* Opaque per-(process, device, rank) context. */
typedef struct swap_ctx swap_ctx_t;
/* A cudaStream_t (struct CUstream_st*) without pulling CUDA headers into this file. */
typedef struct CUstream_st* swap_stream_t;

/* Fills *cfg with the defaults above (device 0, rank 0, world 1). */
SWAP_API void swap_config_default(swap_config_t* cfg);

/* Validates cfg and binds the ctx to cfg->device. EINVAL on a bad cfg; ECUDA when the
 * device is missing or not sm_100. *out receives a ctx the caller frees with swap_destroy. */
SWAP_API swap_status swap_create(const swap_config_t* cfg, swap_ctx_t** out);

/* Copies the table (caller keeps ownership of `regions` and of the device memory),
 * validates it, plans the image (offsets, chunks), allocates the library-owned
 * pinned + mapped host image (zero-filled, so padding is 0), builds and uploads the
 * work descriptors. Allowed once per ctx. State -> REGISTERED. The caller must keep
 * every region allocated at the same address until swap_destroy. */
SWAP_API swap_status swap_register_regions(swap_ctx_t* ctx, const swap_region_t* regions, size_t n);

/* Enqueues the gather of every region into the image plus the chunk checksums (written
 * into the manifest's chunk records) on `stream`. Needs REGISTERED or RESTORED (or
 * CHECKPOINTED: re-snapshot). The caller must not write the regions until the stream
 * reaches this point. State -> CHECKPOINT_PENDING; swap_sync completes it. */
SWAP_API swap_status swap_checkpoint(swap_ctx_t* ctx, swap_stream_t stream);

/* Synchronises `stream`, then finalises the manifest (header, region records, trailing
 * CRC-32C). State CHECKPOINT_PENDING -> CHECKPOINTED; a no-op in other states. */
SWAP_API swap_status swap_sync(swap_ctx_t* ctx, swap_stream_t stream);

/* Needs CHECKPOINTED or RESTORED (restore many times). Checks on the host, before
 * anything is enqueued, that the manifest CRC holds and that the manifest describes the
 * registered layout (else ECORRUPT, nothing written). Then enqueues the scatter of the image
 * to the recorded device addresses with the fused per-chunk compare. Mismatches do not stop
 * the scatter: every byte is written and the result is reported by swap_verify.
 * The caller must not read the regions until the stream reaches this point. State -> RESTORED. */
SWAP_API swap_status swap_restore(swap_ctx_t* ctx, swap_stream_t stream);

/* Needs RESTORED. If hbm_pass != 0, first enqueues the HBM re-read of every region with
 * checksums recomputed against the manifest. Synchronises `stream` and fills *res.
 * Returns ECORRUPT iff a mismatch was found or the manifest is bad, else OK. */
SWAP_API swap_status swap_verify(swap_ctx_t* ctx, swap_stream_t stream, int hbm_pass, swap_verify_result_t* res);

/* Engine-aware state reduction (NEXT-3; "engine-specific optimizations, such as vLLM's sleep
 * API ... reduce both GPU state size and checkpoint/restore latency"). Per-region swap policy: */
#define SWAP_POLICY_SAVE 0u      /* default: gathered by every checkpoint, scattered by every restore */
#define SWAP_POLICY_SAVE_ONCE 1u /* immutable after registration (weights): gathered by the first checkpoint
                                    only; later checkpoints keep its image bytes and chunk checksums */
#define SWAP_POLICY_DISCARD 2u   /* never saved (a KV pool the engine rebuilds, vLLM sleep level 2): captured
                                    as zeros (image bytes 0, c_g = checksum of a zero chunk), restored by
                                    zero-filling the device bytes, checked by the HBM pass like any region */
/* Sets region `region_index`'s policy (index in registration order). Only between
 * swap_register_regions and the first checkpoint (ESTATE otherwise). */
SWAP_API swap_status swap_set_region_policy(swap_ctx_t* ctx, uint32_t region_index, uint32_t policy);
/* Touched-block masks (NEXT-3, "move only touched KV blocks"; reading 25): keep[j] = 0 marks
 * chunk j of SAVE region `region_index` as holding no state the engine needs (an unused KV block). The
 * mask takes effect at the NEXT checkpoint, which captures such chunks as zeros exactly like DISCARD —
 * image bytes 0 (zero-filled in stream order if an earlier checkpoint left data there), c_g = checksum of
 * a zero chunk — and moves only the kept chunks; the restore of that checkpoint moves only the kept chunks
 * and zero-fills the others on the device; the HBM pass checks every chunk. keep = NULL keeps all.
 * n must equal the region's chunk count ceil(bytes / C) (EINVAL otherwise, or if the region's policy is
 * not SAVE; changing the policy resets the mask). Any state after registration except a checkpoint
 * that is not yet synced (ESTATE). swap_import/swap_load restore the whole imported image and re-apply
 * the mask at the next checkpoint. The array is copied. */
SWAP_API swap_status swap_set_chunk_mask(swap_ctx_t* ctx, uint32_t region_index, const uint8_t* keep, uint64_t n);

/* Selects the data mover for later calls (SWAP_MECH_*). The image format is unchanged. */
SWAP_API swap_status swap_set_mechanism(swap_ctx_t* ctx, uint32_t mechanism);
/* The mechanism the next restore will use (SWAP_MECH_AUTO resolved; REGISTERED+). */
SWAP_API swap_status swap_get_mechanism(const swap_ctx_t* ctx, uint32_t* effective);
/* The mechanism the next call of one direction will use: direction 0 = checkpoint, 1 = restore
 * (AUTO resolves per direction, so the two can differ; REGISTERED+; EINVAL for another direction). */
SWAP_API swap_status swap_get_mechanism_dir(const swap_ctx_t* ctx, int direction, uint32_t* effective);

/* Data-parallel replicas (NEXT-2, "swap-in time depends on the GPU memory utilized", P:L230 one
 * backend per GPU set): k replicas hold the same engine image, each in its own ctx/process. Instead of
 * every replica pulling the whole image over its own PCIe link, replica r restores only the copy-engine
 * restore groups g with g % n_stripes == stripe (copy engine H2D + the fused per-group hash check, as
 * SWAP_MECH_CE_PIPE does), and the replicas then exchange their stripes over NVLink (the caller's
 * collective: dist.restore_replicas broadcasts each span from its owner with NCCL). Until that exchange
 * the other stripes' bytes on this device are stale; swap_verify(hbm_pass = 1) afterwards checks every
 * chunk against this ctx's manifest. Zero chunks (DISCARD, masks) are zero-filled in full on every replica.
 * n_stripes == 1 is exactly swap_restore (AUTO mechanism). EINVAL: stripe >= n_stripes, n_stripes == 0, or
 * helper devices are set together with n_stripes > 1.
 * State as swap_restore (-> RESTORED). */
SWAP_API swap_status swap_restore_stripe(swap_ctx_t* ctx, uint32_t stripe, uint32_t n_stripes, swap_stream_t stream);

/* DP replicas, fused NVLink pull (NEXT-2): after swap_restore_stripe(ctx, stripe, n_stripes, ...), moves
 * every chunk of the other stripes from the replica that restored it, reading that replica's HBM directly
 * (over NVLink; the peer memory mapped into this process, e.g. by swap_ipc_import) with the SM mover kernel,
 * which checks each chunk's checksum from the same registers: the all-gather and the chunk check are one
 * kernel; mismatches add to the restore's n_bad / first_bad_chunk. peer_delta[o] for o != stripe =
 * (this process's address of replica o's copy of a region byte) - (address of this ctx's copy): the
 * replicas' regions must have one layout up to a constant shift per replica (e.g. one arena each, same
 * offsets). The peers must have completed their stripe restores (caller's barrier). ESTATE unless
 * RESTORED; EINVAL for n_stripes < 2, stripe >= n_stripes or no deltas. */
SWAP_API swap_status swap_pull_stripes(swap_ctx_t* ctx, uint32_t stripe, uint32_t n_stripes, const int64_t* peer_delta,
                                       swap_stream_t stream);
/* CUDA IPC of a device range (for swap_pull_stripes across processes). export: 64-B handle of the
 * cudaMalloc allocation holding dev_ptr and dev_ptr's offset in it (ECUDA for memory IPC cannot export,
 * e.g. VMM arenas). import (in another process, device = the importer's): *base = the mapped allocation
 * (pass to swap_ipc_close), *mapped = *base + offset. Opening a handle in its own process fails (ECUDA). */
SWAP_API swap_status swap_ipc_export(int device, const void* dev_ptr, uint8_t* handle, uint64_t* offset);
SWAP_API swap_status swap_ipc_import(int device, const uint8_t* handle, uint64_t offset, void** base, void** mapped);
SWAP_API swap_status swap_ipc_close(int device, void* base);

/* One coalesced copy of a restore group: `bytes` at device address dev_addr <- image[image_offset ..). */
typedef struct {
  uint32_t group;        /* restore group index (the striping unit of swap_restore_stripe) */
  uint32_t reserved;     /* 0 */
  uint64_t dev_addr;
  uint64_t image_offset;
  uint64_t bytes;
} swap_span_t;
/* The restore spans in group order (REGISTERED+). Writes min(cap, total) spans to out (out may be NULL
 * when cap == 0) and the total count to *n. Replicas with the same region layout get the same list. */
SWAP_API swap_status swap_get_restore_spans(const swap_ctx_t* ctx, swap_span_t* out, size_t cap, size_t* n);

/* Borrowed views, valid until swap_destroy. The manifest is final only after swap_sync.
 * The image is writable: a caller may load a stored image into it and call swap_import. */
SWAP_API swap_status swap_get_manifest(const swap_ctx_t* ctx, const void** bytes, size_t* n);
SWAP_API swap_status swap_get_image(const swap_ctx_t* ctx, void** host, size_t* n);
SWAP_API swap_status swap_get_summary(const swap_ctx_t* ctx, swap_shard_summary_t* out);

/* Storage tier (NEXT-4): persist a sealed image to a file and load it back. swap_save needs a sealed
 * checkpoint (ESTATE otherwise) and writes image_bytes bytes (O_DIRECT, several threads; buffered if
 * the filesystem refuses O_DIRECT). swap_load reads a file of exactly image_bytes bytes into the image
 * buffer (ECORRUPT if the size differs) and then behaves as swap_import (manifest CRC and layout
 * checks; state -> CHECKPOINTED). I/O errors return EINVAL (open/read) or ENOMEM (write/space). */
SWAP_API swap_status swap_save(const swap_ctx_t* ctx, const char* path);
SWAP_API swap_status swap_load(swap_ctx_t* ctx, const char* path);

/* Declares that the image buffer now holds a complete image (e.g. loaded from storage):
 * checks the manifest CRC and that it describes the registered layout (ECORRUPT if not).
 * Needs REGISTERED, CHECKPOINTED or RESTORED. State -> CHECKPOINTED. */
SWAP_API swap_status swap_import(swap_ctx_t* ctx);

/* After the all-gather of every rank's summary (rank order): checks world and that entry r
 * has rank r and this ctx's own entry equals its summary (ENCCL otherwise), stores the
 * global manifest and writes the global digest (CRC-32C of the world*64 bytes). */
SWAP_API swap_status swap_set_global(swap_ctx_t* ctx, const swap_shard_summary_t* all, int world, uint64_t* global_digest);

/* Ctx-free host planning (needs no GPU): the layout and the sealed manifest libswap produces for a
 * region table under cfg (same validation as swap_register_regions). swap_plan_manifest writes the
 * manifest (header, region and chunk records with the given chunk checksums, CRC trailer) into out
 * (cap >= manifest bytes, else EINVAL with *manifest_bytes set). chunk_checksums may be NULL (zeros). */
SWAP_API swap_status swap_plan_layout(const swap_region_t* regions, size_t n, const swap_config_t* cfg,
                                      uint64_t* payload_bytes, uint64_t* n_chunks, uint64_t* manifest_off,
                                      uint64_t* image_bytes);
SWAP_API swap_status swap_plan_manifest(const swap_region_t* regions, size_t n, const swap_config_t* cfg,
                                        const uint64_t* chunk_checksums, void* out, size_t cap,
                                        size_t* manifest_bytes);

/* Ctx-free half of swap_set_global, usable without a GPU: checks that `all` holds `world`
 * summaries with all[r].rank == r and all[r].world == world (ENCCL otherwise) and writes
 * the global digest = CRC-32C of the world*64 summary bytes. */
SWAP_API swap_status swap_merge_global(const swap_shard_summary_t* all, int world, uint64_t* global_digest);

/* Device time (CUDA events recorded on the caller's stream right before and after the
 * movers) of the last checkpoint (updated by swap_sync), and of the last restore and HBM
 * verify pass (updated by swap_verify). 0 if the phase has not run. */
typedef struct {
  float checkpoint_ms; /* gather kernel, or hash pass + copy-engine copies */
  float restore_ms;    /* scatter kernel, or copy-engine copies + hash pass */
  float verify_ms;     /* HBM verify pass */
  float check_ms;      /* CE_PIPE restore: summed device time of its per-group HASH_CHECK launches on the side
                        * stream (CUDA events around each launch; they overlap the copy engine's H2D copies,
                        * off the critical path); 0 for other mechanisms and for helper groups */
} swap_timings_t;
SWAP_API swap_status swap_get_timings(const swap_ctx_t* ctx, swap_timings_t* out);

/* Where the pinned image lives (REGISTERED+): *node = the NUMA node placement targeted (-1 none),
 * *local_fraction = share of the image's pages found on that node (256 pages sampled with
 * get_mempolicy(MPOL_F_NODE | MPOL_F_ADDR); 1.0 when no placement was targeted). */
SWAP_API swap_status swap_get_numa(const swap_ctx_t* ctx, int32_t* node, double* local_fraction);

/* Number of libswap kernels this ctx has launched in total (for the bench's gpu_launches). */
SWAP_API swap_status swap_get_launch_count(const swap_ctx_t* ctx, uint64_t* launches);

/* ---------------------------------------------------------------------------------------------
 * Device arena with releasable HBM (NEXT-1; "freeing GPU capacity for other workloads",
 * P:L142 swap-in "requesting the required GPU memory"). An engine allocates the state it wants
 * swappable inside an arena; after swap_checkpoint + swap_sync, swap_arena_release returns the
 * arena's physical HBM to the device while its virtual addresses stay reserved; before
 * swap_restore, swap_arena_reacquire maps fresh HBM at the same addresses (contents undefined
 * until the restore). Built on CUDA virtual memory management (reserve VA once; 1-GiB physical
 * slabs created, mapped and released). One arena belongs to one device; calls are not
 * thread-safe per arena.
 * ------------------------------------------------------------------------------------------- */
typedef struct swap_arena swap_arena_t;
/* Reserves VA for `bytes` (rounded up to the allocation granularity) and maps physical memory.
 * ENOMEM if the device cannot back it; EUNSUPPORTED if the driver lacks VMM entry points. */
SWAP_API swap_status swap_arena_create(int device, uint64_t bytes, swap_arena_t** out);
SWAP_API swap_status swap_arena_info(const swap_arena_t* a, uint64_t* dev_addr, uint64_t* bytes, int* resident);
/* Synchronises the device, unmaps and frees all mapped physical memory. ESTATE if nothing is mapped. */
SWAP_API swap_status swap_arena_release(swap_arena_t* a);
/* Maps new physical memory at the original addresses. ESTATE if resident; ENOMEM if HBM is short. */
SWAP_API swap_status swap_arena_reacquire(swap_arena_t* a);
/* Maps only the slabs covering [offset, offset + bytes) (idempotent); the arena is resident once all are. */
SWAP_API swap_status swap_arena_reacquire_range(swap_arena_t* a, uint64_t offset, uint64_t bytes);
/* Binds an arena holding (some of) ctx's regions. Then swap_restore re-acquires the arena's HBM
 * itself if it is released: with SWAP_MECH_CE_PIPE group by group, just before each group's copies are
 * enqueued, so the host-side mapping overlaps the copy engine; with other movers all at once first.
 * NULL unbinds. The arena must outlive the binding. */
SWAP_API swap_status swap_bind_arena(swap_ctx_t* ctx, swap_arena_t* a);

/* NVLink-assisted restore (NEXT-2): with SWAP_MECH_CE_PIPE, restore groups are striped round-robin over
 * this device and the `n` helper devices; a helper copies its groups' image range from the pinned host
 * image into its own HBM staging buffer over its own PCIe link, and then this device's SM mover kernel
 * pulls the group from the helper's staging over NVLink (peer access this device -> helper) into the
 * regions and checks every chunk from the same registers (the transfer and the check are one kernel).
 * With SWAP_ASSIST=copy in the environment (read when the helpers are set) the helper instead copies the
 * group to this device with peer copies (copy engines) and this device re-reads it for the hash check.
 * Helpers should be idle GPUs of the node; peer access is enabled both ways. A helper equal to this
 * device degenerates to an on-device staging buffer (used by the one-GPU tests). n = 0 removes them.
 * Needs REGISTERED+ (staging is sized from the restore groups). The checkpoint path is unchanged. */
SWAP_API swap_status swap_set_helpers(swap_ctx_t* ctx, const int* devices, int n);

/* Full-duplex exchange on one device (NEXT-1; §3.4-3.5 swap-out of victims then swap-in of the
 * requested backend, here overlapped on the duplex PCIe link): checkpoints + seals + releases every victim
 * (each with a bound, mapped arena) on s_out while scattering `incoming` (bound, released arena; sealed
 * image) on s_in. Incoming HBM is mapped slab by slab just before each pipeline group, and only while
 * (victim HBM still mapped + incoming HBM mapped) <= (victim HBM at the start + headroom): victim slabs are
 * released as soon as the last group reading them has left the device. Either side may be empty
 * (nv == 0 or incoming == NULL). Victims end CHECKPOINTED, incoming RESTORED (call swap_verify on it).
 * *peak_extra (optional) = the most HBM held above the victims' starting amount (<= headroom). ENOMEM if
 * the incoming arena cannot fit. The device is synchronised first; calls on the ctxs are serialised. */
SWAP_API swap_status swap_exchange(swap_ctx_t* const* victims, size_t n_victims, swap_ctx_t* incoming,
                                   swap_stream_t s_out, swap_stream_t s_in, uint64_t headroom,
                                   uint64_t* peak_extra);
SWAP_API const char* swap_arena_last_error(const swap_arena_t* a);
SWAP_API void swap_arena_destroy(swap_arena_t* a);
/* Peer mapping of arenas (data-parallel replicas, NEXT-2): swap_arena_export writes one POSIX file
 * descriptor per slab (the caller owns them: pass them to another process, e.g. over a Unix socket with
 * SCM_RIGHTS, then close them) and the slab size; with fds == NULL it only reports *n. Every slab must be
 * mapped (ESTATE otherwise); the descriptors stay valid for the slabs' current physical memory, so a
 * released and re-acquired arena must be exported again. swap_arena_import maps such a set of slabs (total
 * bytes = the exporter's arena size) into a fresh VA range on `device` with read-write access and returns it
 * (the fds may be closed afterwards); swap_arena_unimport unmaps it. This is how swap_pull_stripes reads a
 * replica's VMM arena. */
typedef struct swap_arena_view swap_arena_view_t;
SWAP_API swap_status swap_arena_export(swap_arena_t* a, int* fds, size_t cap, size_t* n, uint64_t* slab_bytes);
SWAP_API swap_status swap_arena_import(int device, const int* fds, size_t n, uint64_t slab_bytes, uint64_t total_bytes,
                                       swap_arena_view_t** out, uint64_t* dev_addr);
SWAP_API void swap_arena_unimport(swap_arena_view_t* v);

/* ---------------------------------------------------------------------------------------------
 * Task manager (NEXT-1): memory reservations and demand-aware preemption, host-only.
 * PAPER.md §3.3-3.5 (L136-148) and §6 (L230): swap-in requests are reservations served from a
 * priority queue (several granted at once when memory suffices); when memory is short, running
 * backends are evicted one at a time in the order (shorter request queue, older last access),
 * re-checking after each; a write-locked backend is not a candidate; a backend's per-GPU needs are
 * fixed at init and acquired/released together. All sizes are bytes; GPUs are indices
 * 0..n_gpus-1. Not thread-safe: the caller serialises calls (the paper's task manager is one actor).
 * ------------------------------------------------------------------------------------------- */
typedef struct swap_sched swap_sched_t;
SWAP_API swap_status swap_sched_create(uint32_t n_gpus, const uint64_t* capacity, swap_sched_t** out);
/* need[n_gpus]: bytes on each GPU (0 = not placed there). EINVAL: duplicate id, no GPU, or a need
 * above capacity; ENOMEM: `resident` but it does not fit next to the current residents. */
SWAP_API swap_status swap_sched_add_backend(swap_sched_t* s, uint32_t id, const uint64_t* need, int resident);
/* Request-handler bookkeeping: current queue length and last-accessed time. */
SWAP_API swap_status swap_sched_touch(swap_sched_t* s, uint32_t id, uint32_t queue_len, double last_access);
SWAP_API swap_status swap_sched_lock(swap_sched_t* s, uint32_t id, int locked);
/* Victims (eviction order) that would let `id` become resident now; *n = 0 if none needed.
 * ENOMEM if infeasible; EINVAL if more than `cap` victims (then *n holds the count). */
SWAP_API swap_status swap_sched_plan(const swap_sched_t* s, uint32_t id, uint32_t* victims, uint32_t cap, uint32_t* n);
/* Queues a reservation (lower priority value = served first; ties in arrival order). ESTATE if
 * `id` is resident or already queued. */
SWAP_API swap_status swap_sched_reserve(swap_sched_t* s, uint32_t id, double priority);
SWAP_API swap_status swap_sched_cancel(swap_sched_t* s, uint32_t id);
/* Serves the head reservation: *id = the granted backend (UINT32_MAX if the queue is empty) and its
 * victims, which are marked swapped out while `id` is marked resident. ENOMEM: the head cannot be
 * satisfied now (it stays queued; *id names it). The caller then swaps the victims out and `id` in. */
SWAP_API swap_status swap_sched_grant(swap_sched_t* s, uint32_t* id, uint32_t* victims, uint32_t cap, uint32_t* n);
/* Voluntary swap-out: releases the backend's reservations on all its GPUs. */
SWAP_API swap_status swap_sched_release(swap_sched_t* s, uint32_t id);
SWAP_API swap_status swap_sched_query(const swap_sched_t* s, uint32_t id, int* resident, int* queued);
SWAP_API swap_status swap_sched_free(const swap_sched_t* s, uint32_t gpu, uint64_t* free_bytes);
SWAP_API void swap_sched_destroy(swap_sched_t* s);

SWAP_API const char* swap_status_str(swap_status s);
SWAP_API const char* swap_last_error(const swap_ctx_t* ctx);

/* Frees the pinned image, descriptors and device scratch. NULL is a no-op. */
SWAP_API void swap_destroy(swap_ctx_t* ctx);

#ifdef __cplusplus
}
#endif
#endif /* SWAP_H */
