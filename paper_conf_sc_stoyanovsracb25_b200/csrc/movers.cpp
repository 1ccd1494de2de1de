// movers.cpp — libswap internals: kernel launches, copy-engine movers, the CE_PIPE pipeline, the
// descriptor sets of the region policies, CRC tables and context teardown (see ctx.h).
#include <sys/mman.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "ctx.h"

namespace swc {
swap_status cuda_fail(swap_ctx* c, cudaError_t e, const char* what) {
  c->err = std::string(what) + ": " + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ")";
  return SWAP_ECUDA;
}

uint8_t* manifest_ptr(swap_ctx* c) { return c->image + c->plan.manifest_off; }

swk::Params base_params(swap_ctx* c, const DescSet& S) {
  swk::Params p{};
  p.desc = S.d_desc;
  p.n_desc = S.n_desc;
  p.seg_bytes = c->seg;
  p.partial = c->d_partial;
  p.arrive = c->d_arrive;
  const uint64_t cs_off = c->plan.manifest_off + swp::kHeaderBytes + swp::kRegionRecBytes * c->plan.regions.size() + 24;
  p.cs_out = reinterpret_cast<uint64_t*>(c->image_dev + cs_off);
  p.cs_exp = c->exp_valid ? reinterpret_cast<const uint64_t*>(c->d_exp + 24) : p.cs_out;
  p.n_bad = &c->d_status->n_bad;
  p.first_bad = &c->d_status->first_bad;
  p.tables = c->d_tables;
  p.chunk_bytes = c->plan.C;
  p.zinit_c = c->zinit_c;
  p.xseg = c->xseg;
  p.hlane_len = (uint32_t)std::min<uint64_t>(c->plan.C, c->seg);
  p.ticket = &c->d_status->ticket;
  p.tmaps = c->d_tmaps;
  p.chunk_dev = c->d_chunk_dev;
  return p;
}

int grid_of(swap_ctx* c) { return c->cfg.grid_ctas ? (int)c->cfg.grid_ctas : 2 * c->sm_count; }

// The mechanism a call uses. AUTO resolves per direction from the measured crossover (DESIGN.md §6,
// `profiles/r01_crossover_v2.md`): the copy engines reach a higher link rate than SM-issued accesses, but
// per-copy and per-launch costs make the single fused SM pass faster for small images (swap-in GB/s,
// SM / CE_PIPE: 256 MiB 50.2 / 41.2, 1 GiB 50.7 / 50.6, 4 GiB 50.9 / 53.7).
//   restore:    < 2 GiB SM;  else CE_PIPE
//   checkpoint: < 1 GiB SM;  else CE_PIPE
// XXH64 is not combinable: with chunks > 4 MiB a pipeline group holds too few chunks for the side-stream
// hash to keep up with the link (config B, 16 MiB: CE_PIPE swap-in 15 GB/s), so restores from 2 GiB take
// the coalesced CE_BATCH copies plus one hash pass (50.2 vs SM 48.7). Checkpoints follow the CRC rule: the
// one whole-image hash pass overlaps every D2H copy (config B, 16 MiB: CE_PIPE 57.2 vs SM 51.5 GB/s,
// `profiles/r01_bench_B_xxh64_16MiB_v2.json`). Up to 4 MiB the restore rule is the CRC one too (config B,
// 2 / 4 MiB: CE_PIPE 54.6 / 54.2 vs SM 50.8 / 50.6).
// XXH64 with chunks of 1 MiB and more on images below the CRC crossover (round 2, config A 64 MiB): a chunk
// is one serial hash job, so with few chunks every path is bound by per-chunk round chains. Restores keep
// the SM mover -- the quad-per-chunk kernel copies and hashes from its TMA ring: 1 MiB restore 50.7 GB/s,
// swap-in 31.0 (CE_BATCH 23.1); 4 MiB 21.1 / 10.7 (9.0) -- checkpoints take CE_PIPE, whose hash pass runs
// beside the D2H copies (1 MiB 53.5 vs SM 45.7 GB/s).
uint32_t resolve_mech(const swap_ctx* c, int dir) {
  if (c->cfg.mechanism != SWAP_MECH_AUTO) return c->cfg.mechanism;
  const uint64_t S = c->plan.payload_bytes;
  const bool xxh = c->plan.kind == SWAP_CHECKSUM_XXH64;
  if (dir == 1 && xxh && c->plan.C > (4ull << 20) && S >= (2ull << 30)) return SWAP_MECH_CE_BATCH;
  if (dir == 0 && xxh && c->plan.C >= (1ull << 20)) return SWAP_MECH_CE_PIPE;
  if (dir == 0) return S < (1ull << 30) ? SWAP_MECH_SM : SWAP_MECH_CE_PIPE;
  return S < (2ull << 30) ? SWAP_MECH_SM : SWAP_MECH_CE_PIPE;
}
uint32_t mech(const swap_ctx* c) { return c->cur_mech; }

// Stages the manifest's chunk records (expected checksums at +24 of each 32-B record) into HBM on `s`, at
// every copy-engine restore (after its manifest check); the verify that follows reads the same copy.
swap_status stage_expected(swap_ctx* c, cudaStream_t s) {
  const uint64_t n = c->plan.n_chunks;
  if (n == 0) return SWAP_OK;
  if (!c->d_exp) CUDA_TRY(c, cudaMalloc(&c->d_exp, n * swp::kChunkRecBytes));
  const uint64_t off = c->plan.manifest_off + swp::kHeaderBytes + swp::kRegionRecBytes * c->plan.regions.size();
  CUDA_TRY(c, cudaMemcpyAsync(c->d_exp, c->image + off, n * swp::kChunkRecBytes, cudaMemcpyHostToDevice, s));
  c->exp_valid = true;
  return SWAP_OK;
}
int kind_of(swap_ctx* c) {
  if (mech(c) == SWAP_MECH_SM_NOCHECK) return swk::KIND_NONE;
  return c->plan.kind == SWAP_CHECKSUM_XXH64 ? swk::KIND_XXH64 : swk::KIND_CRC32C;
}
int hash_kind(swap_ctx* c) { return c->plan.kind == SWAP_CHECKSUM_XXH64 ? swk::KIND_XXH64 : swk::KIND_CRC32C; }

swap_status launch(swap_ctx* c, int mode, int kind, const swk::Params& p, cudaStream_t s) {
  if (p.n_desc == 0) return SWAP_OK;
  // never more CTAs than descriptor batches (idle CTAs would only load tables)
  int want = (int)std::min<uint64_t>((uint64_t)grid_of(c), (p.n_desc + 15) / 16);
  if ((mode == swk::HASH_STORE || mode == swk::HASH_CHECK) && kind == swk::KIND_CRC32C)
    want = c->cfg.grid_ctas ? std::min<int>(want, (int)c->cfg.grid_ctas) : swk::hash_grid(c->sm_count, p.n_desc);
  // XXH64 movers: one resident CTA per SM (kernels.cu: a warp per chunk, up to 128 registers per thread),
  // as many CTAs as chunks up to the SM count (chunks are dealt to warps interleaved across CTAs)
  if ((mode == swk::GATHER || mode == swk::SCATTER) && kind == swk::KIND_XXH64 && !c->cfg.grid_ctas)
    want = (int)std::min<uint64_t>((uint64_t)c->sm_count, p.n_desc);
  cudaError_t e;
  if ((mode == swk::HASH_STORE || mode == swk::HASH_CHECK) && kind == swk::KIND_XXH64 && !c->cfg.grid_ctas)
    e = swk::launch_xxh_hash(mode, p, c->sm_count, s);
  else if ((mode == swk::GATHER || mode == swk::SCATTER) && kind == swk::KIND_XXH64 && !c->cfg.grid_ctas &&
           p.ticket && swk::xxh_quad_mover_enabled())
    e = swk::launch_xxh_move(mode, p, c->sm_count, s);
  else
    e = swk::launch_mover(mode, kind, p, std::max(1, want), s);
  if (e != cudaSuccess) return cuda_fail(c, e, "mover kernel launch");
  ++c->launches;
  return SWAP_OK;
}

// Merges consecutive spans whose device and image ranges both continue where the previous one ends.
std::vector<Span> coalesce(const std::vector<Span>& spans) {
  std::vector<Span> out;
  out.reserve(spans.size());
  for (const Span& sp : spans) {
    if (!sp.bytes) continue;
    if (!out.empty()) {
      Span& b = out.back();
      if (b.dev + b.bytes == sp.dev && b.host + b.bytes == sp.host) {
        b.bytes += sp.bytes;
        continue;
      }
    }
    out.push_back(sp);
  }
  return out;
}

swap_status memcpy_dir(swap_ctx* c, const Span& sp, int dir, cudaStream_t s) {
  void* dev = reinterpret_cast<void*>(sp.dev);
  CUDA_TRY(c, dir == 0 ? cudaMemcpyAsync(sp.host, dev, sp.bytes, cudaMemcpyDeviceToHost, s)
                       : cudaMemcpyAsync(dev, sp.host, sp.bytes, cudaMemcpyHostToDevice, s));
  return SWAP_OK;
}

// Copy-engine data movement for CE_REGION / CE_CHUNK / CE_BATCH: dir 0 = device -> image, 1 = image -> device.
swap_status ce_copy(swap_ctx* c, DescSet& S, int dir, cudaStream_t s) {
  const uint32_t m = mech(c);
  if (m == SWAP_MECH_CE_REGION) {
    for (const Span& sp : S.region_spans) {
      swap_status st = memcpy_dir(c, sp, dir, s);
      if (st != SWAP_OK) return st;
    }
    return SWAP_OK;
  }
  if (m == SWAP_MECH_CE_CHUNK) {
    for (size_t i = 0; i < S.ce_bytes.size(); ++i) {
      Span sp{reinterpret_cast<uint64_t>(S.ce_dev[i]), static_cast<uint8_t*>(S.ce_host[i]), S.ce_bytes[i]};
      swap_status st = memcpy_dir(c, sp, dir, s);
      if (st != SWAP_OK) return st;
    }
    return SWAP_OK;
  }
  // CE_BATCH: the per-chunk copies coalesced into maximal runs contiguous on both sides, one
  // cudaMemcpyAsync per run (a masked chunk or a region boundary with padding ends a run).
  std::vector<Span> runs;
  runs.reserve(S.ce_bytes.size());
  for (size_t i = 0; i < S.ce_bytes.size(); ++i)
    runs.push_back(Span{reinterpret_cast<uint64_t>(S.ce_dev[i]), static_cast<uint8_t*>(S.ce_host[i]), S.ce_bytes[i]});
  for (const Span& sp : coalesce(runs)) {
    swap_status st = memcpy_dir(c, sp, dir, s);
    if (st != SWAP_OK) return st;
  }
  return SWAP_OK;
}

// Re-acquires the bound arena's slabs under `spans` (no-op without an arena or when resident).
swap_status map_spans(swap_ctx* c, const std::vector<Span>& spans) {
  if (!c->arena || swarena::resident(c->arena)) return SWAP_OK;
  for (const Span& sp : spans) {
    if (!sp.bytes || !swarena::contains(c->arena, sp.dev, sp.dev + sp.bytes)) continue;
    bool mapped = true;  // skip the driver round trip for spans on slabs already mapped
    for (uint64_t k = swarena::slab_of(c->arena, sp.dev); mapped && k <= swarena::slab_of(c->arena, sp.dev + sp.bytes - 1); ++k)
      mapped = swarena::slab_mapped(c->arena, k);
    if (mapped) continue;
    swap_status st = swarena::map_dev_range(c->arena, sp.dev, sp.dev + sp.bytes);
    if (st != SWAP_OK) {
      c->err = "re-acquiring arena HBM failed";
      return st;
    }
  }
  return SWAP_OK;
}

// The copies of one pipeline group: spans contiguous on both sides (consecutive chunks of a region, a
// region and its successor with no padding between) are coalesced, one cudaMemcpyAsync per run.
swap_status copy_spans(swap_ctx* c, const std::vector<Span>& spans, int dir, cudaStream_t s) {
  for (const Span& sp : coalesce(spans)) {
    swap_status st = memcpy_dir(c, sp, dir, s);
    if (st != SWAP_OK) return st;
  }
  return SWAP_OK;
}

// CE_PIPE. Checkpoint (dir 0): the hash pass over HBM runs on the side stream concurrently with the
// D2H copies (both only read HBM). Restore (dir 1): group g's H2D copies are followed by an event;
// the side stream waits for it and checks group g from HBM while the copy engine moves group g+1.
swap_status ce_pipe(swap_ctx* c, DescSet& S, int dir, const swk::Params& base, cudaStream_t s) {
  CUDA_TRY(c, cudaEventRecord(c->ev_fork, s));
  CUDA_TRY(c, cudaStreamWaitEvent(c->side, c->ev_fork, 0));
  swap_status st;
  if (dir == 0 && (st = launch(c, swk::HASH_STORE, hash_kind(c), base, c->side)) != SWAP_OK) return st;
  const size_t H = dir == 1 ? c->helpers.size() : 0;
  if (dir == 1) c->n_chk = 0;
  for (auto& h : c->helpers)
    if (H) CUDA_TRY(c, cudaStreamWaitEvent(h.s, c->ev_fork, 0));
  for (size_t g = 0; g < S.groups.size(); ++g) {
    const Group& G = S.groups[g];
    if (dir == 1 && (st = map_spans(c, G.spans)) != SWAP_OK) return st;  // lazy HBM re-acquire
    if (dir == 1 && c->n_stripes > 1 && g % c->n_stripes != c->stripe) continue;  // another replica's stripe
    const size_t k = H ? g % (H + 1) : 0;
    if (k > 0) {
      // helper k-1: H2D of the group's image range into its staging over its own PCIe link, then
      // NVLink peer copies of each span to this device; the side stream checks it as usual
      auto& h = c->helpers[k - 1];
      const int slot = (int)((g / (H + 1)) % 2);  // the same slot the fused descriptors were built for
      uint8_t* lo = G.spans.front().host;
      uint8_t* hi = G.spans.back().host + G.spans.back().bytes;
      if ((uint64_t)(hi - lo) > h.staging_bytes) {  // groups rebuilt without re-sizing the helpers
        c->err = "restore group larger than the helper staging buffer (call swap_set_helpers again)";
        return SWAP_EINTERNAL;
      }
      CUDA_TRY(c, cudaSetDevice(h.dev));
      // the slot is free once this device has pulled the group that used it before (fused mode; in copy
      // mode the helper's own stream orders the reuse)
      CUDA_TRY(c, cudaStreamWaitEvent(h.s, h.consumed[slot], 0));
      CUDA_TRY(c, cudaMemcpyAsync(h.staging[slot], lo, (size_t)(hi - lo), cudaMemcpyHostToDevice, h.s));
      if (c->assist_copy || !c->d_assist)  // copy-engine peer copies, then the usual HBM hash check
        for (const Span& sp : G.spans)
          CUDA_TRY(c, cudaMemcpyPeerAsync(reinterpret_cast<void*>(sp.dev), c->cfg.device,
                                          h.staging[slot] + (sp.host - lo), h.dev, sp.bytes, h.s));
      CUDA_TRY(c, cudaEventRecord(h.ev, h.s));
      CUDA_TRY(c, cudaSetDevice(c->cfg.device));
      CUDA_TRY(c, cudaStreamWaitEvent(c->side, h.ev, 0));
      swk::Params p = base;
      p.partial = base.partial + G.d0;
      p.n_desc = G.d1 - G.d0;
      if (c->assist_copy || !c->d_assist) {
        p.desc = base.desc + G.d0;
        if ((st = launch(c, swk::HASH_CHECK, hash_kind(c), p, c->side)) != SWAP_OK) return st;
      } else {  // fused: this device's SM mover pulls the group from the helper's staging over NVLink and
                // checks every chunk from the same registers (no peer copy, no HBM re-read)
        p.desc = c->d_assist + G.d0;
        if ((st = launch(c, swk::SCATTER, hash_kind(c), p, c->side)) != SWAP_OK) return st;
        CUDA_TRY(c, cudaEventRecord(h.consumed[slot], c->side));
      }
      continue;
    }
    if ((st = copy_spans(c, G.spans, dir, s)) != SWAP_OK) return st;
    if (dir == 1) {
      CUDA_TRY(c, cudaEventRecord(S.group_ev[g], s));
      CUDA_TRY(c, cudaStreamWaitEvent(c->side, S.group_ev[g], 0));
      swk::Params p = base;
      p.desc = base.desc + G.d0;
      p.partial = base.partial + G.d0;
      p.n_desc = G.d1 - G.d0;
      while (c->chk_ev.size() < 2ull * (c->n_chk + 1)) {
        cudaEvent_t e = nullptr;
        CUDA_TRY(c, cudaEventCreate(&e));
        c->chk_ev.push_back(e);
      }
      CUDA_TRY(c, cudaEventRecord(c->chk_ev[2 * c->n_chk], c->side));
      if ((st = launch(c, swk::HASH_CHECK, hash_kind(c), p, c->side)) != SWAP_OK) return st;
      CUDA_TRY(c, cudaEventRecord(c->chk_ev[2 * c->n_chk + 1], c->side));
      ++c->n_chk;
    }
  }
  for (auto& h : c->helpers) {
    if (!H) break;
    CUDA_TRY(c, cudaSetDevice(h.dev));
    CUDA_TRY(c, cudaEventRecord(h.done, h.s));
    CUDA_TRY(c, cudaSetDevice(c->cfg.device));
    CUDA_TRY(c, cudaStreamWaitEvent(s, h.done, 0));
  }
  CUDA_TRY(c, cudaEventRecord(c->ev_join, c->side));
  CUDA_TRY(c, cudaStreamWaitEvent(s, c->ev_join, 0));
  return SWAP_OK;
}

// Phase p: 0 checkpoint, 1 restore, 2 verify. Call after the stream has been synchronised.
swap_status collect_timing(swap_ctx* c, int p) {
  if (!c->pending[p]) return SWAP_OK;
  CUDA_TRY(c, cudaEventElapsedTime(&c->ms[p], c->ev[2 * p], c->ev[2 * p + 1]));
  c->pending[p] = false;
  if (p == 1) {  // the per-group checks of a CE_PIPE restore (n_chk = 0 for other movers)
    c->chk_ms = 0.f;
    for (uint32_t i = 0; i < c->n_chk; ++i) {
      float ms = 0.f;
      CUDA_TRY(c, cudaEventElapsedTime(&ms, c->chk_ev[2 * i], c->chk_ev[2 * i + 1]));
      c->chk_ms += ms;
    }
    c->n_chk = 0;
  }
  return SWAP_OK;
}

bool is_ce(uint32_t m) { return m == SWAP_MECH_CE_REGION || m == SWAP_MECH_CE_CHUNK || m == SWAP_MECH_CE_BATCH; }

void free_set(DescSet& S) {
  if (S.owned) {
    if (S.d_desc) cudaFree(S.d_desc);
    for (auto& e : S.group_ev)
      if (e) cudaEventDestroy(e);
  }
  S = DescSet();
}

// CRC tables for the ctx's chunk and segment sizes (the hash kernels fold lanes with constants that
// depend on min(C, seg)); uploads them and derives the init / segment shift constants.
swap_status upload_tables(swap_ctx* c) {
  std::vector<uint32_t> tab(swk::TAB_WORDS);
  swk::build_tables(tab.data(), std::min<uint64_t>(c->cfg.chunk_bytes, c->seg), c->seg);
  if (!c->d_tables) CUDA_TRY(c, cudaMalloc(&c->d_tables, tab.size() * 4));
  CUDA_TRY(c, cudaMemcpy(c->d_tables, tab.data(), tab.size() * 4, cudaMemcpyHostToDevice));
  const uint32_t* x2n = tab.data() + swk::TAB_X2N;
  c->zinit_c = swk::host_multmodp(swk::host_x2nmodp(c->cfg.chunk_bytes, 3, x2n), 0xFFFFFFFFu);
  c->xseg = swk::host_x2nmodp(c->seg, 3, x2n);
  // strand-staged CRC kernel's tensor path (only used for segments of >= 128 KiB): a map per chunk
  const uint64_t L1 = std::min<uint64_t>(c->plan.C, c->seg);
  const uint64_t nc = c->plan.n_chunks;
  if (c->plan.kind == SWAP_CHECKSUM_CRC32C && nc && L1 >= (128u << 10) && !c->d_tmaps) {
    std::vector<uint64_t> base(nc), bytes(nc);
    for (const auto& R : c->plan.regions)
      for (uint64_t j = 0; j < R.nchunks; ++j) {
        base[R.first + j] = R.r.dev_addr + j * c->plan.C;
        bytes[R.first + j] = std::min<uint64_t>(c->plan.C, R.r.bytes - j * c->plan.C);
      }
    std::vector<uint8_t> maps(nc * 128);
    if (swk::encode_tmaps(maps.data(), base.data(), bytes.data(), (int)nc, L1)) {
      for (uint64_t g = 0; g < nc; ++g)  // a chunk without a map (shorter than one row) never takes the tensor path
        if (std::all_of(maps.begin() + g * 128, maps.begin() + (g + 1) * 128, [](uint8_t v) { return v == 0; }))
          base[g] = 0;
      CUDA_TRY(c, cudaMalloc(&c->d_tmaps, maps.size()));
      CUDA_TRY(c, cudaMemcpy(c->d_tmaps, maps.data(), maps.size(), cudaMemcpyHostToDevice));
      CUDA_TRY(c, cudaMalloc(&c->d_chunk_dev, nc * 8));
      CUDA_TRY(c, cudaMemcpy(c->d_chunk_dev, base.data(), nc * 8, cudaMemcpyHostToDevice));
    }
  }
  return SWAP_OK;
}

// Auto segment size: the smallest power of 2 that gives every warp slot of the GPU (SMs x 32) at most one
// CRC work item -- one round of the hash kernel -- between 4 KiB and 256 KiB (large images keep 256 KiB; a
// 64 MiB image gets 16 KiB: its verify pass 45 us vs 50 us with 8 KiB, 74 / 54 / 80 us with 4 / 32 / 64 KiB,
// tools/seg_ab.py).
uint32_t auto_seg(const swap_ctx* c, uint64_t payload) {
  const uint64_t per = payload / ((uint64_t)c->sm_count * 32 + 1);
  uint64_t s = 4096;
  while (s < per && s < (256u << 10)) s *= 2;
  return (uint32_t)s;
}

void free_helpers(swap_ctx* c) {
  int cur = -1;
  cudaGetDevice(&cur);
  if (c->side) {  // the side stream may still be pulling from the staging buffers
    cudaSetDevice(c->cfg.device);
    cudaStreamSynchronize(c->side);
  }
  for (auto& h : c->helpers) {
    cudaSetDevice(h.dev);
    if (h.s) cudaStreamSynchronize(h.s);
    for (int k = 0; k < 2; ++k) {
      if (h.staging[k]) cudaFree(h.staging[k]);
      if (h.consumed[k]) cudaEventDestroy(h.consumed[k]);
    }
    if (h.ev) cudaEventDestroy(h.ev);
    if (h.done) cudaEventDestroy(h.done);
    if (h.s) cudaStreamDestroy(h.s);
  }
  c->helpers.clear();
  if (cur >= 0) cudaSetDevice(cur);
  if (c->d_assist) cudaFree(c->d_assist);
  c->d_assist = nullptr;
}

void release(swap_ctx* c) {
  free_helpers(c);
  free_set(c->s_move);
  free_set(c->s_save);
  free_set(c->s_zero);
  free_set(c->s_all);
  if (c->d_zero) cudaFree(c->d_zero);
  c->d_zero = nullptr;
  if (c->d_zspans) cudaFree(c->d_zspans);
  c->d_zspans = nullptr;
  if (c->d_partial) cudaFree(c->d_partial);
  if (c->d_pull) cudaFree(c->d_pull);
  c->d_pull = nullptr;
  c->pull_cap = 0;
  if (c->ev_pull) cudaEventDestroy(c->ev_pull);
  c->ev_pull = nullptr;
  if (c->d_arrive) cudaFree(c->d_arrive);
  if (c->d_status) cudaFree(c->d_status);
  if (c->h_status) cudaFreeHost(c->h_status);
  if (c->d_tables) cudaFree(c->d_tables);
  if (c->d_exp) cudaFree(c->d_exp);
  if (c->d_tmaps) cudaFree(c->d_tmaps);
  if (c->d_chunk_dev) cudaFree(c->d_chunk_dev);
  for (auto& e : c->ev)
    if (e) cudaEventDestroy(e);
  for (auto& e : c->chk_ev)
    if (e) cudaEventDestroy(e);
  c->chk_ev.clear();
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  if (c->ev_join) cudaEventDestroy(c->ev_join);
  if (c->side) cudaStreamDestroy(c->side);
  if (c->host_registered) cudaHostUnregister(c->image);
  if (c->image) munmap(c->image, c->map_bytes);
  c->d_partial = nullptr;
  c->image = nullptr;
}

// Builds the descriptor set of the regions `pick` selects. zero_src: segment sources point into
// the zero buffer instead of the region (hashing DISCARD chunks as zeros).
template <class Pick>
static swap_status build_set(swap_ctx* c, DescSet* S, Pick pick, bool zero_src) {
  const swp::Plan& P = c->plan;
  const uint64_t seg = P.kind == SWAP_CHECKSUM_XXH64 ? P.C : std::min<uint64_t>(P.C, c->seg);
  std::vector<swk::SegDesc> desc;
  // group size: cfg.pipe_mib, or auto = payload / 32 clamped to [16 MiB, 512 MiB] (smaller groups cost
  // more in per-copy and per-launch overhead than they gain in overlap; config B, profiles/r02_pipe_groups.md:
  // swap-in 54.76-54.90 GB/s for 256 MiB - 1 GiB groups, the side-stream group checks 2.05 / 3.40 / 4.33 TB/s
  // at 256 / 512 / 1024 MiB -- more segments per launch; 512 keeps ~12 groups per replica for 8 DP stripes)
  uint64_t target = (uint64_t)c->cfg.pipe_mib << 20;
  if (!target) target = std::min<uint64_t>(512ull << 20, std::max<uint64_t>(16ull << 20, c->plan.payload_bytes / 32));
  Group cur{0, 0, {}};
  uint64_t cur_bytes = 0;
  for (size_t i = 0; i < P.regions.size(); ++i) {
    const auto& r = P.regions[i];
    if (r.r.bytes == 0) continue;
    for (uint64_t j = 0; j < r.nchunks; ++j) {
      if (!pick(i, r.first + j)) continue;
      const uint64_t lo = j * P.C, len = std::min<uint64_t>(P.C, r.r.bytes - lo);
      // CE_REGION spans: runs of picked chunks (a whole region unless chunk masks cut it)
      if (!S->region_spans.empty() && S->region_spans.back().dev + S->region_spans.back().bytes == r.r.dev_addr + lo &&
          S->region_spans.back().host + S->region_spans.back().bytes == c->image + r.off + lo)
        S->region_spans.back().bytes += len;
      else
        S->region_spans.push_back(Span{r.r.dev_addr + lo, c->image + r.off + lo, len});
      const uint32_t nseg = (uint32_t)((len + seg - 1) / seg);
      for (uint32_t s = 0; s < nseg; ++s) {
        swk::SegDesc d;
        d.dev = zero_src ? reinterpret_cast<uint64_t>(c->d_zero) + s * seg : r.r.dev_addr + lo + s * seg;
        d.host = reinterpret_cast<uint64_t>(c->image_dev + r.off + lo + s * seg);
        d.bytes = (uint32_t)std::min<uint64_t>(seg, len - s * seg);
        d.chunk = (uint32_t)(r.first + j);
        d.seg = s;
        d.nseg = nseg;
        desc.push_back(d);
      }
      S->ce_dev.push_back(reinterpret_cast<void*>(r.r.dev_addr + lo));
      S->ce_host.push_back(c->image + r.off + lo);
      S->ce_bytes.push_back(len);
      // CE_PIPE groups: consecutive whole chunks up to ~pipe_mib MiB; spans merge contiguous chunks
      Span sp{r.r.dev_addr + lo, c->image + r.off + lo, len};
      if (!cur.spans.empty() && cur.spans.back().dev + cur.spans.back().bytes == sp.dev &&
          cur.spans.back().host + cur.spans.back().bytes == sp.host)
        cur.spans.back().bytes += len;
      else
        cur.spans.push_back(sp);
      cur.d1 = (uint32_t)desc.size();
      cur_bytes += len;
      if (cur_bytes >= target) {
        S->groups.push_back(std::move(cur));
        cur = Group{(uint32_t)desc.size(), (uint32_t)desc.size(), {}};
        cur_bytes = 0;
      }
    }
  }
  if (!cur.spans.empty()) S->groups.push_back(std::move(cur));
  if (desc.size() > 0xFFFFFFFFull) {
    c->err = "too many segments";
    return SWAP_EUNSUPPORTED;
  }
  S->owned = true;
  S->n_desc = (uint32_t)desc.size();
  CUDA_TRY(c, cudaMalloc(&S->d_desc, std::max<size_t>(1, desc.size()) * sizeof(swk::SegDesc)));
  if (!desc.empty())
    CUDA_TRY(c, cudaMemcpy(S->d_desc, desc.data(), desc.size() * sizeof(swk::SegDesc), cudaMemcpyHostToDevice));
  S->group_ev.assign(S->groups.size(), nullptr);
  for (auto& e : S->group_ev) CUDA_TRY(c, cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  S->h_desc = std::make_shared<const std::vector<swk::SegDesc>>(std::move(desc));
  return SWAP_OK;
}

static DescSet alias_of(const DescSet& S) {
  DescSet a = S;
  a.owned = false;
  return a;
}

static void cut_pieces(uint64_t dst, uint64_t bytes, std::vector<swk::ZSpan>* out) {
  for (uint64_t o = 0; o < bytes; o += swk::kZeroPiece)
    out->push_back(swk::ZSpan{dst + o, std::min<uint64_t>(swk::kZeroPiece, bytes - o)});
}

// Zero-fills every DISCARD region and masked chunk on the device: one kernel launch.
swap_status zero_fill_device(swap_ctx* c, cudaStream_t s) {
  if (!c->n_zspans) return SWAP_OK;
  CUDA_TRY(c, swk::launch_zero_fill(c->d_zspans, c->n_zspans, c->sm_count, s));
  ++c->launches;
  return SWAP_OK;
}

// (Re)builds every set from the current policies and chunk masks (c->keep).
swap_status build_sets(swap_ctx* c) {
  free_set(c->s_move);
  free_set(c->s_save);
  free_set(c->s_zero);
  free_set(c->s_all);
  if (c->d_zero) {
    cudaFree(c->d_zero);
    c->d_zero = nullptr;
  }
  const auto& pol = c->policy;
  const auto& P = c->plan;
  bool any_once = false, any_zero = false;
  uint64_t zero_bytes = 0;
  c->zero_spans.clear();
  for (size_t i = 0; i < pol.size(); ++i) {
    const auto& r = P.regions[i];
    any_once |= pol[i] == SWAP_POLICY_SAVE_ONCE;
    for (uint64_t j = 0; j < r.nchunks; ++j) {
      if (pol[i] != SWAP_POLICY_DISCARD && c->keep[r.first + j]) continue;
      // a zero chunk: DISCARD region or masked-out chunk — restored by zero-filling, hashed from d_zero
      any_zero = true;
      const uint64_t lo = j * P.C, len = std::min<uint64_t>(P.C, r.r.bytes - lo);
      zero_bytes = std::max<uint64_t>(zero_bytes, len);
      std::vector<Span>& z = c->zero_spans;
      if (!z.empty() && z.back().dev + z.back().bytes == r.r.dev_addr + lo)
        z.back().bytes += len;
      else
        z.push_back(Span{r.r.dev_addr + lo, c->image + r.off + lo, len});
    }
  }
  auto keep = [&](size_t i, uint64_t g) { return pol[i] != SWAP_POLICY_DISCARD && c->keep[g]; };
  swap_status st = build_set(c, &c->s_all, [](size_t, uint64_t) { return true; }, false);
  if (st != SWAP_OK) return st;
  if (!any_once && !any_zero) {
    c->s_move = alias_of(c->s_all);
    c->s_save = alias_of(c->s_all);
  } else {
    st = build_set(c, &c->s_move, keep, false);
    if (st != SWAP_OK) return st;
    if (any_once) {
      st = build_set(c, &c->s_save, [&](size_t i, uint64_t g) { return pol[i] == SWAP_POLICY_SAVE && keep(i, g); },
                     false);
      if (st != SWAP_OK) return st;
    } else {
      c->s_save = alias_of(c->s_move);
    }
  }
  if (any_zero) {
    CUDA_TRY(c, cudaMalloc(&c->d_zero, std::max<uint64_t>(16, (zero_bytes + 31) & ~31ull)));
    CUDA_TRY(c, cudaMemset(c->d_zero, 0, std::max<uint64_t>(16, (zero_bytes + 31) & ~31ull)));
    st = build_set(c, &c->s_zero, [&](size_t i, uint64_t g) { return !keep(i, g); }, true);
    if (st != SWAP_OK) return st;
  }
  if (c->d_zspans) cudaFree(c->d_zspans);
  c->d_zspans = nullptr;
  std::vector<swk::ZSpan> pieces;
  for (const Span& z : c->zero_spans) cut_pieces(z.dev, z.bytes, &pieces);
  c->n_zspans = (uint32_t)pieces.size();
  if (!pieces.empty()) {
    CUDA_TRY(c, cudaMalloc(&c->d_zspans, pieces.size() * sizeof(swk::ZSpan)));
    CUDA_TRY(c, cudaMemcpy(c->d_zspans, pieces.data(), pieces.size() * sizeof(swk::ZSpan), cudaMemcpyHostToDevice));
  }
  if (c->d_partial) cudaFree(c->d_partial);
  c->d_partial = nullptr;
  CUDA_TRY(c, cudaMalloc(&c->d_partial, std::max<size_t>(1, c->s_all.n_desc) * 4));
  return SWAP_OK;
}

// Chunk masks (swap_set_chunk_mask) take effect at the next checkpoint: rebuilds the sets for the new
// mask and zero-fills, in stream order, the image bytes of chunks that are masked now but hold data from
// an earlier checkpoint (their image bytes must read as zeros, reading 25). *hash_zero: the zero chunks'
// checksums must be (re)written by this checkpoint.
swap_status apply_mask(swap_ctx* c, cudaStream_t s, bool* hash_zero) {
  *hash_zero = !c->first_ckpt_done;
  if (!c->mask_dirty) return SWAP_OK;
  const auto& P = c->plan;
  std::vector<swk::ZSpan> pieces;  // image bytes of chunks masked now that still hold older data
  for (size_t i = 0; i < P.regions.size(); ++i) {
    const auto& r = P.regions[i];
    uint64_t run_lo = 0, run_len = 0;
    for (uint64_t j = 0; j < r.nchunks; ++j) {
      const uint64_t g = r.first + j, lo = j * P.C, len = std::min<uint64_t>(P.C, r.r.bytes - lo);
      if (c->next_keep[g] || c->img_zero[g]) continue;
      if (run_len && run_lo + run_len != lo) {
        pieces.push_back(swk::ZSpan{reinterpret_cast<uint64_t>(c->image_dev + r.off + run_lo), run_len});
        run_len = 0;
      }
      if (!run_len) run_lo = lo;
      run_len += len;
      c->img_zero[g] = 1;
    }
    if (run_len) pieces.push_back(swk::ZSpan{reinterpret_cast<uint64_t>(c->image_dev + r.off + run_lo), run_len});
  }
  // zeros to the mapped image, in stream order: one cudaMemsetAsync per run of chunks. (A single
  // zero_fill_kernel launch over the same pieces was measured slower here: config-B scale checkpoints
  // 0.85-0.97 s vs 0.32-0.57 s, tools/mask_probe.py — SM-issued writes to host memory.)
  for (const swk::ZSpan& z : pieces)
    CUDA_TRY(c, cudaMemsetAsync(reinterpret_cast<void*>(z.dst), 0, z.bytes, s));
  c->keep = c->next_keep;
  c->mask_dirty = false;
  swap_status st = build_sets(c);
  if (st != SWAP_OK) return st;
  *hash_zero = true;
  if (!c->helpers.empty()) {  // restore groups changed: re-size the helpers' staging
    std::vector<int> devs;
    for (auto& h : c->helpers) devs.push_back(h.dev);
    return swap_set_helpers(c, devs.data(), (int)devs.size());
  }
  return SWAP_OK;
}

// After a checkpoint has been enqueued: the chunks it gathered now hold data in the image.
void note_gathered(swap_ctx* c, const DescSet& S) {
  (void)S;
  const auto& P = c->plan;
  for (size_t i = 0; i < P.regions.size(); ++i) {
    if (c->policy[i] == SWAP_POLICY_DISCARD) continue;
    const auto& r = P.regions[i];
    for (uint64_t j = 0; j < r.nchunks; ++j)
      if (c->keep[r.first + j]) c->img_zero[r.first + j] = 0;
  }
}

}  // namespace swc
