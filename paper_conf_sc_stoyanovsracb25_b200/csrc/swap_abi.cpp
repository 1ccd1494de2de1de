// swap_abi.cpp — the extern "C" boundary of libswap (declared and documented in include/swap.h).
//
// Context state machine (include/swap.h; the paper's snapshot-once / restore-many model,
// P:L115):
//   CREATED --register--> REGISTERED --checkpoint--> CKPT_PENDING --sync--> CHECKPOINTED
//   CHECKPOINTED|RESTORED --restore--> RESTORED;   REGISTERED|CHECKPOINTED|RESTORED --checkpoint--> CKPT_PENDING
#include <sys/mman.h>
#include <unistd.h>

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "arena.h"
#include "kernels.cuh"
#include "plan.h"

namespace {

enum class St { CREATED, REGISTERED, CKPT_PENDING, CHECKPOINTED, RESTORED };

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

}  // namespace

struct Span {  // one copy-engine transfer: contiguous on the device and in the image
  uint64_t dev;
  uint8_t* host;
  uint64_t bytes;
};
struct Group {  // CE_PIPE unit: whole chunks, descriptor range [d0, d1)
  uint32_t d0, d1;
  std::vector<Span> spans;
};

// The work of one pass over a subset of the regions (selected by their swap policy): segment
// descriptors on the device plus the copy-engine views of the same bytes. A chunk's segments are
// always contiguous, so per-chunk CRC combining works on any set.
struct DescSet {
  swk::SegDesc* d_desc = nullptr;
  uint32_t n_desc = 0;
  std::vector<Span> region_spans;         // CE_REGION
  std::vector<void*> ce_dev, ce_host;     // CE_CHUNK / CE_BATCH, one entry per chunk
  std::vector<size_t> ce_bytes;
  std::vector<Group> groups;              // CE_PIPE
  std::vector<cudaEvent_t> group_ev;
  bool owned = false;                     // false: an alias of another set
};

struct swap_ctx {
  swap_config_t cfg{};
  St st = St::CREATED;
  int sm_count = 0;
  swp::Plan plan;
  // host image: mmap'd, pinned + mapped with cudaHostRegister (library-owned)
  uint8_t* image = nullptr;
  size_t map_bytes = 0;
  bool host_registered = false;
  uint8_t* image_dev = nullptr;  // device (UVA) view of the image
  // device-side work state; sets: all regions (verify), SAVE|SAVE_ONCE (first checkpoint, restore),
  // SAVE (later checkpoints), DISCARD chunks hashed from a zero buffer (their c_g)
  std::vector<uint32_t> policy;
  DescSet s_all, s_move, s_save, s_zero;
  bool first_ckpt_done = false;
  uint8_t* d_zero = nullptr;
  uint32_t* d_partial = nullptr;
  uint32_t* d_arrive = nullptr;
  swk::DevStatus* d_status = nullptr;
  swk::DevStatus* h_status = nullptr;  // pinned
  uint32_t* d_tables = nullptr;
  uint32_t zinit_c = 0, xseg = 0;
  uint32_t seg = 0;  // CRC-32C segment size in use (cfg.seg_bytes, or chosen at registration when 0)
  uint32_t cur_mech = SWAP_MECH_SM;  // mechanism of the call in progress (resolve_mech)
  cudaEvent_t ev[6] = {};  // checkpoint, restore, verify: begin/end pairs
  bool pending[3] = {false, false, false};
  float ms[3] = {0.f, 0.f, 0.f};
  uint64_t launches = 0;
  std::string err;
  std::vector<swap_shard_summary_t> global;
  // CE_PIPE
  cudaStream_t side = nullptr;
  swap_arena* arena = nullptr;  // bound arena: restore re-acquires its HBM (swap_bind_arena)
  // NVLink-assisted restore (swap_set_helpers): peers pull groups over their own PCIe links into
  // HBM staging and copy them to this device over NVLink
  struct Helper {
    int dev = -1;
    cudaStream_t s = nullptr;
    uint8_t* staging = nullptr;
    cudaEvent_t ev = nullptr, done = nullptr;
  };
  std::vector<Helper> helpers;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
};

namespace {

swap_status cuda_fail(swap_ctx* c, cudaError_t e, const char* what) {
  c->err = std::string(what) + ": " + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ")";
  return SWAP_ECUDA;
}
#define CUDA_TRY(ctx, expr)                                    \
  do {                                                         \
    cudaError_t e_ = (expr);                                   \
    if (e_ != cudaSuccess) return cuda_fail((ctx), e_, #expr); \
  } while (0)

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
  p.cs_exp = p.cs_out;
  p.n_bad = &c->d_status->n_bad;
  p.first_bad = &c->d_status->first_bad;
  p.tables = c->d_tables;
  p.chunk_bytes = c->plan.C;
  p.zinit_c = c->zinit_c;
  p.xseg = c->xseg;
  p.hlane_len = (uint32_t)std::min<uint64_t>(c->plan.C, c->seg);
  return p;
}

int grid_of(swap_ctx* c) { return c->cfg.grid_ctas ? (int)c->cfg.grid_ctas : 2 * c->sm_count; }

// The mechanism a call uses. AUTO resolves per direction from the measured crossover (DESIGN.md §6,
// `profiles/r01_crossover.md`): the copy engines reach a higher link rate than SM-issued accesses, but
// per-copy and per-launch costs make the single fused SM pass faster for small images.
//   restore:    < 128 MiB SM;  < 2 GiB CE_BATCH (needs a non-default stream, else SM);  else CE_PIPE
//   checkpoint: < 1 GiB SM;    else CE_PIPE
// XXH64 is not combinable: with chunks > 1 MiB a pipeline group holds too few chunks for the side-stream
// hash to keep up with the link, while the fused SM pass hashes every chunk in flight — SM then.
uint32_t resolve_mech(const swap_ctx* c, int dir, bool default_stream) {
  if (c->cfg.mechanism != SWAP_MECH_AUTO) return c->cfg.mechanism;
  const uint64_t S = c->plan.payload_bytes;
  if (c->plan.kind == SWAP_CHECKSUM_XXH64 && c->plan.C > (1ull << 20)) return SWAP_MECH_SM;
  if (dir == 0) return S < (1ull << 30) ? SWAP_MECH_SM : SWAP_MECH_CE_PIPE;
  if (S < (128ull << 20)) return SWAP_MECH_SM;
  if (S < (2ull << 30)) return default_stream ? SWAP_MECH_SM : SWAP_MECH_CE_BATCH;
  return SWAP_MECH_CE_PIPE;
}
uint32_t mech(const swap_ctx* c) { return c->cur_mech; }
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
  cudaError_t e;
  if ((mode == swk::HASH_STORE || mode == swk::HASH_CHECK) && kind == swk::KIND_XXH64 && !c->cfg.grid_ctas)
    e = swk::launch_xxh_hash(mode, p, c->sm_count, s);
  else
    e = swk::launch_mover(mode, kind, p, std::max(1, want), s);
  if (e != cudaSuccess) return cuda_fail(c, e, "mover kernel launch");
  ++c->launches;
  return SWAP_OK;
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
  // CE_BATCH: one cudaMemcpyBatchAsync over every chunk.
  if (s == nullptr) {
    c->err = "SWAP_MECH_CE_BATCH needs a non-default stream (cudaMemcpyBatchAsync restriction)";
    return SWAP_EUNSUPPORTED;
  }
  if (S.ce_bytes.empty()) return SWAP_OK;
  cudaMemcpyAttributes attr;
  std::memset(&attr, 0, sizeof(attr));
  attr.srcAccessOrder = cudaMemcpySrcAccessOrderStream;
  attr.srcLocHint.type = dir == 0 ? cudaMemLocationTypeDevice : cudaMemLocationTypeHost;
  attr.srcLocHint.id = dir == 0 ? c->cfg.device : 0;
  attr.dstLocHint.type = dir == 0 ? cudaMemLocationTypeHost : cudaMemLocationTypeDevice;
  attr.dstLocHint.id = dir == 0 ? 0 : c->cfg.device;
  size_t attr_idx = 0, fail_idx = 0;
  std::vector<void*>& dst = dir == 0 ? S.ce_host : S.ce_dev;
  std::vector<void*>& src = dir == 0 ? S.ce_dev : S.ce_host;
  CUDA_TRY(c, cudaMemcpyBatchAsync(dst.data(), src.data(), S.ce_bytes.data(), S.ce_bytes.size(), &attr, &attr_idx, 1,
                                   &fail_idx, s));
  return SWAP_OK;
}

// Re-acquires the bound arena's slabs under `spans` (no-op without an arena or when resident).
swap_status map_spans(swap_ctx* c, const std::vector<Span>& spans) {
  if (!c->arena || swarena::resident(c->arena)) return SWAP_OK;
  for (const Span& sp : spans) {
    if (!swarena::contains(c->arena, sp.dev, sp.dev + sp.bytes)) continue;
    swap_status st = swarena::map_dev_range(c->arena, sp.dev, sp.dev + sp.bytes);
    if (st != SWAP_OK) {
      c->err = "re-acquiring arena HBM failed";
      return st;
    }
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
  for (auto& h : c->helpers)
    if (H) CUDA_TRY(c, cudaStreamWaitEvent(h.s, c->ev_fork, 0));
  for (size_t g = 0; g < S.groups.size(); ++g) {
    const Group& G = S.groups[g];
    if (dir == 1 && (st = map_spans(c, G.spans)) != SWAP_OK) return st;  // lazy HBM re-acquire
    const size_t k = H ? g % (H + 1) : 0;
    if (k > 0) {
      // helper k-1: H2D of the group's image range into its staging over its own PCIe link, then
      // NVLink peer copies of each span to this device; the side stream checks it as usual
      auto& h = c->helpers[k - 1];
      uint8_t* lo = G.spans.front().host;
      uint8_t* hi = G.spans.back().host + G.spans.back().bytes;
      CUDA_TRY(c, cudaSetDevice(h.dev));
      CUDA_TRY(c, cudaMemcpyAsync(h.staging, lo, (size_t)(hi - lo), cudaMemcpyHostToDevice, h.s));
      for (const Span& sp : G.spans)
        CUDA_TRY(c, cudaMemcpyPeerAsync(reinterpret_cast<void*>(sp.dev), c->cfg.device, h.staging + (sp.host - lo), h.dev,
                                        sp.bytes, h.s));
      CUDA_TRY(c, cudaEventRecord(h.ev, h.s));
      CUDA_TRY(c, cudaSetDevice(c->cfg.device));
      CUDA_TRY(c, cudaStreamWaitEvent(c->side, h.ev, 0));
      swk::Params p = base;
      p.desc = base.desc + G.d0;
      p.partial = base.partial + G.d0;
      p.n_desc = G.d1 - G.d0;
      if ((st = launch(c, swk::HASH_CHECK, hash_kind(c), p, c->side)) != SWAP_OK) return st;
      continue;
    }
    for (const Span& sp : G.spans)
      if ((st = memcpy_dir(c, sp, dir, s)) != SWAP_OK) return st;
    if (dir == 1) {
      CUDA_TRY(c, cudaEventRecord(S.group_ev[g], s));
      CUDA_TRY(c, cudaStreamWaitEvent(c->side, S.group_ev[g], 0));
      swk::Params p = base;
      p.desc = base.desc + G.d0;
      p.partial = base.partial + G.d0;
      p.n_desc = G.d1 - G.d0;
      if ((st = launch(c, swk::HASH_CHECK, hash_kind(c), p, c->side)) != SWAP_OK) return st;
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
  return SWAP_OK;
}

// Auto segment size: enough CRC work items to give every warp slot of the GPU (SMs x 32) one, between
// 4 KiB and 256 KiB (large images keep 256 KiB; a 64 MiB image gets 8 KiB).
uint32_t auto_seg(const swap_ctx* c, uint64_t payload) {
  const uint64_t per = payload / ((uint64_t)c->sm_count * 32 + 1);
  uint64_t s = 4096;
  while (s * 2 <= per && s < (256u << 10)) s *= 2;
  return (uint32_t)s;
}

void free_helpers(swap_ctx* c) {
  int cur = -1;
  cudaGetDevice(&cur);
  for (auto& h : c->helpers) {
    cudaSetDevice(h.dev);
    if (h.s) cudaStreamSynchronize(h.s);
    if (h.staging) cudaFree(h.staging);
    if (h.ev) cudaEventDestroy(h.ev);
    if (h.done) cudaEventDestroy(h.done);
    if (h.s) cudaStreamDestroy(h.s);
  }
  c->helpers.clear();
  if (cur >= 0) cudaSetDevice(cur);
}

void release(swap_ctx* c) {
  free_helpers(c);
  free_set(c->s_move);
  free_set(c->s_save);
  free_set(c->s_zero);
  free_set(c->s_all);
  if (c->d_zero) cudaFree(c->d_zero);
  c->d_zero = nullptr;
  if (c->d_partial) cudaFree(c->d_partial);
  if (c->d_arrive) cudaFree(c->d_arrive);
  if (c->d_status) cudaFree(c->d_status);
  if (c->h_status) cudaFreeHost(c->h_status);
  if (c->d_tables) cudaFree(c->d_tables);
  for (auto& e : c->ev)
    if (e) cudaEventDestroy(e);
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
swap_status build_set(swap_ctx* c, DescSet* S, Pick pick, bool zero_src) {
  const swp::Plan& P = c->plan;
  const uint64_t seg = P.kind == SWAP_CHECKSUM_XXH64 ? P.C : std::min<uint64_t>(P.C, c->seg);
  std::vector<swk::SegDesc> desc;
  // group size: cfg.pipe_mib, or auto = payload / 32 clamped to [16 MiB, 256 MiB] (smaller groups cost
  // more in per-copy and per-launch overhead than they gain in overlap)
  uint64_t target = (uint64_t)c->cfg.pipe_mib << 20;
  if (!target) target = std::min<uint64_t>(256ull << 20, std::max<uint64_t>(16ull << 20, c->plan.payload_bytes / 32));
  Group cur{0, 0, {}};
  uint64_t cur_bytes = 0;
  for (size_t i = 0; i < P.regions.size(); ++i) {
    const auto& r = P.regions[i];
    if (!pick(i) || r.r.bytes == 0) continue;
    S->region_spans.push_back(Span{r.r.dev_addr, c->image + r.off, r.r.bytes});
    for (uint64_t j = 0; j < r.nchunks; ++j) {
      const uint64_t lo = j * P.C, len = std::min<uint64_t>(P.C, r.r.bytes - lo);
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
  return SWAP_OK;
}

DescSet alias_of(const DescSet& S) {
  DescSet a = S;
  a.owned = false;
  return a;
}

// (Re)builds every set from the current policies.
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
  bool any_once = false, any_discard = false;
  uint64_t zero_bytes = 0;
  for (size_t i = 0; i < pol.size(); ++i) {
    any_once |= pol[i] == SWAP_POLICY_SAVE_ONCE;
    if (pol[i] == SWAP_POLICY_DISCARD) {
      any_discard = true;
      zero_bytes = std::max<uint64_t>(zero_bytes, std::min<uint64_t>(c->plan.C, c->plan.regions[i].r.bytes));
    }
  }
  swap_status st = build_set(c, &c->s_all, [](size_t) { return true; }, false);
  if (st != SWAP_OK) return st;
  if (!any_once && !any_discard) {
    c->s_move = alias_of(c->s_all);
    c->s_save = alias_of(c->s_all);
  } else {
    st = build_set(c, &c->s_move, [&](size_t i) { return pol[i] != SWAP_POLICY_DISCARD; }, false);
    if (st != SWAP_OK) return st;
    if (any_once) {
      st = build_set(c, &c->s_save, [&](size_t i) { return pol[i] == SWAP_POLICY_SAVE; }, false);
      if (st != SWAP_OK) return st;
    } else {
      c->s_save = alias_of(c->s_move);
    }
  }
  if (any_discard) {
    CUDA_TRY(c, cudaMalloc(&c->d_zero, std::max<uint64_t>(16, (zero_bytes + 31) & ~31ull)));
    CUDA_TRY(c, cudaMemset(c->d_zero, 0, std::max<uint64_t>(16, (zero_bytes + 31) & ~31ull)));
    st = build_set(c, &c->s_zero, [&](size_t i) { return pol[i] == SWAP_POLICY_DISCARD; }, true);
    if (st != SWAP_OK) return st;
  }
  if (c->d_partial) cudaFree(c->d_partial);
  c->d_partial = nullptr;
  CUDA_TRY(c, cudaMalloc(&c->d_partial, std::max<size_t>(1, c->s_all.n_desc) * 4));
  return SWAP_OK;
}

}  // namespace

extern "C" {

void swap_config_default(swap_config_t* cfg) {
  if (!cfg) return;
  std::memset(cfg, 0, sizeof(*cfg));
  cfg->chunk_bytes = 1ull << 20;
  cfg->align = 4096;
  cfg->checksum = SWAP_CHECKSUM_CRC32C;
  cfg->mechanism = SWAP_MECH_AUTO;
  cfg->world = 1;
  cfg->seg_bytes = 0;  // auto
  cfg->pipe_mib = 0;  // auto
}

swap_status swap_create(const swap_config_t* cfg_in, swap_ctx_t** out) {
  if (!cfg_in || !out) return SWAP_EINVAL;
  *out = nullptr;
  auto* c = new (std::nothrow) swap_ctx();
  if (!c) return SWAP_ENOMEM;
  c->cfg = *cfg_in;
  swap_status st = swp::normalize_config(&c->cfg, &c->err);
  if (st != SWAP_OK) {
    fprintf(stderr, "libswap: swap_create: %s\n", c->err.c_str());
    delete c;
    return st;
  }
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || c->cfg.device >= ndev) {
    fprintf(stderr, "libswap: swap_create: no CUDA device %d (%s)\n", c->cfg.device,
            e != cudaSuccess ? cudaGetErrorString(e) : "ordinal out of range");
    delete c;
    return SWAP_ECUDA;
  }
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, c->cfg.device) != cudaSuccess || prop.major != 10 || !prop.canMapHostMemory) {
    fprintf(stderr, "libswap: swap_create: device %d is not an sm_100 GPU with mapped host memory\n",
            c->cfg.device);
    delete c;
    return SWAP_ECUDA;
  }
  c->sm_count = prop.multiProcessorCount;
  DeviceGuard g(c->cfg.device);
  if ((e = cudaMalloc(&c->d_status, sizeof(swk::DevStatus))) != cudaSuccess ||
      (e = cudaMemset(c->d_status, 0, sizeof(swk::DevStatus))) != cudaSuccess ||
      (e = cudaHostAlloc(&c->h_status, sizeof(swk::DevStatus), cudaHostAllocDefault)) != cudaSuccess ||
      (e = cudaEventCreate(&c->ev[0])) != cudaSuccess || (e = cudaEventCreate(&c->ev[1])) != cudaSuccess ||
      (e = cudaEventCreate(&c->ev[2])) != cudaSuccess || (e = cudaEventCreate(&c->ev[3])) != cudaSuccess ||
      (e = cudaEventCreate(&c->ev[4])) != cudaSuccess || (e = cudaEventCreate(&c->ev[5])) != cudaSuccess) {
    cuda_fail(c, e, "swap_create");
    fprintf(stderr, "libswap: %s\n", c->err.c_str());
    release(c);
    delete c;
    return SWAP_ECUDA;
  }
  *out = c;
  return SWAP_OK;
}

swap_status swap_register_regions(swap_ctx_t* c, const swap_region_t* regions, size_t n) {
  if (!c) return SWAP_EINVAL;
  swp::Plan plan;
  swap_status st = swp::build_plan(regions, n, c->cfg, &plan, &c->err);
  if (st != SWAP_OK) return st;
  if (c->st != St::CREATED || c->image) {  // registered, or a failed registration left its image
    c->err = "regions already registered";
    return SWAP_ESTATE;
  }
  DeviceGuard g(c->cfg.device);
  c->plan = std::move(plan);
  const swp::Plan& P = c->plan;

  // Library-owned image: anonymous mapping (zero-filled, so padding is 0), huge pages when
  // available, pinned and mapped into the device address space.
  const size_t page = 2u << 20;
  c->map_bytes = (P.image_bytes + page - 1) / page * page;
  void* m = mmap(nullptr, c->map_bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  if (m == MAP_FAILED) {
    c->err = "mmap of " + std::to_string(c->map_bytes) + " B failed";
    c->map_bytes = 0;
    return SWAP_ENOMEM;
  }
  c->image = static_cast<uint8_t*>(m);
  madvise(m, c->map_bytes, MADV_HUGEPAGE);
  cudaError_t e = cudaHostRegister(m, c->map_bytes, cudaHostRegisterMapped | cudaHostRegisterPortable);
  if (e != cudaSuccess) {
    cudaGetLastError();
    munmap(m, c->map_bytes);
    c->image = nullptr;
    c->map_bytes = 0;
    c->err = std::string("cudaHostRegister (pinning the image) failed: ") + cudaGetErrorString(e);
    return SWAP_ENOMEM;
  }
  c->host_registered = true;
  void* dview = nullptr;
  CUDA_TRY(c, cudaHostGetDevicePointer(&dview, m, 0));
  c->image_dev = static_cast<uint8_t*>(dview);
  swp::write_manifest_skeleton(P, manifest_ptr(c));

  CUDA_TRY(c, cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming));
  CUDA_TRY(c, cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming));
  CUDA_TRY(c, cudaStreamCreateWithFlags(&c->side, cudaStreamNonBlocking));
  CUDA_TRY(c, cudaMalloc(&c->d_arrive, std::max<uint64_t>(1, P.n_chunks) * 4));
  CUDA_TRY(c, cudaMemset(c->d_arrive, 0, std::max<uint64_t>(1, P.n_chunks) * 4));
  c->seg = c->cfg.seg_bytes ? c->cfg.seg_bytes : auto_seg(c, P.payload_bytes);
  if ((st = upload_tables(c)) != SWAP_OK) return st;
  c->policy.assign(P.regions.size(), SWAP_POLICY_SAVE);
  st = build_sets(c);
  if (st != SWAP_OK) return st;
  c->st = St::REGISTERED;
  return SWAP_OK;
}

swap_status swap_checkpoint(swap_ctx_t* c, swap_stream_t stream) {
  if (!c) return SWAP_EINVAL;
  if (c->st == St::CREATED || c->st == St::CKPT_PENDING) {
    c->err = c->st == St::CREATED ? "checkpoint before swap_register_regions" : "previous checkpoint not synced";
    return SWAP_ESTATE;
  }
  DeviceGuard g(c->cfg.device);
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  c->cur_mech = resolve_mech(c, 0, s == nullptr);
  // SAVE_ONCE regions are gathered by the first checkpoint only; DISCARD regions never (their image
  // bytes stay zero and their c_g are the checksums of zero chunks, hashed once from a zero buffer).
  DescSet& S = c->first_ckpt_done ? c->s_save : c->s_move;
  swk::Params p = base_params(c, S);
  CUDA_TRY(c, cudaEventRecord(c->ev[0], s));
  swap_status st;
  if (!c->first_ckpt_done && c->s_zero.n_desc &&
      (st = launch(c, swk::HASH_STORE, hash_kind(c), base_params(c, c->s_zero), s)) != SWAP_OK)
    return st;
  if (mech(c) == SWAP_MECH_CE_PIPE) {
    if ((st = ce_pipe(c, S, 0, p, s)) != SWAP_OK) return st;
  } else if (is_ce(mech(c))) {
    if ((st = launch(c, swk::HASH_STORE, hash_kind(c), p, s)) != SWAP_OK) return st;
    if ((st = ce_copy(c, S, 0, s)) != SWAP_OK) return st;
  } else {
    if ((st = launch(c, swk::GATHER, kind_of(c), p, s)) != SWAP_OK) return st;
  }
  CUDA_TRY(c, cudaEventRecord(c->ev[1], s));
  c->first_ckpt_done = true;
  c->pending[0] = true;
  c->st = St::CKPT_PENDING;
  return SWAP_OK;
}

swap_status swap_sync(swap_ctx_t* c, swap_stream_t stream) {
  if (!c) return SWAP_EINVAL;
  DeviceGuard g(c->cfg.device);
  CUDA_TRY(c, cudaStreamSynchronize(reinterpret_cast<cudaStream_t>(stream)));
  if (c->pending[0]) {
    CUDA_TRY(c, cudaEventSynchronize(c->ev[1]));
    swap_status ts = collect_timing(c, 0);
    if (ts != SWAP_OK) return ts;
  }
  if (c->st == St::CKPT_PENDING) {
    swp::seal_manifest(c->plan, manifest_ptr(c));
    c->st = St::CHECKPOINTED;
  }
  return SWAP_OK;
}

swap_status swap_restore(swap_ctx_t* c, swap_stream_t stream) {
  if (!c) return SWAP_EINVAL;
  if (c->st != St::CHECKPOINTED && c->st != St::RESTORED) {
    c->err = "restore needs a completed checkpoint (swap_sync) or an imported image";
    return SWAP_ESTATE;
  }
  swap_status st = swp::check_manifest(c->plan, manifest_ptr(c), &c->err);
  if (st != SWAP_OK) return st;
  DeviceGuard g(c->cfg.device);
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  c->cur_mech = resolve_mech(c, 1, s == nullptr);
  DescSet& S = c->s_move;
  swk::Params p = base_params(c, S);
  CUDA_TRY(c, cudaMemsetAsync(&c->d_status->n_bad, 0, 8, s));
  CUDA_TRY(c, cudaMemsetAsync(&c->d_status->first_bad, 0xFF, 8, s));
  CUDA_TRY(c, cudaEventRecord(c->ev[2], s));
  if (c->arena && !swarena::resident(c->arena)) {
    // DISCARD regions (zero-filled below) and, for movers other than CE_PIPE, everything, need HBM now
    std::vector<Span> now;
    for (size_t i = 0; i < c->policy.size(); ++i)
      if (mech(c) != SWAP_MECH_CE_PIPE || c->policy[i] == SWAP_POLICY_DISCARD)
        now.push_back(Span{c->plan.regions[i].r.dev_addr, nullptr, c->plan.regions[i].r.bytes});
    if ((st = map_spans(c, now)) != SWAP_OK) return st;
  }
  for (size_t i = 0; i < c->policy.size(); ++i)  // DISCARD regions come back as zeros
    if (c->policy[i] == SWAP_POLICY_DISCARD && c->plan.regions[i].r.bytes)
      CUDA_TRY(c, cudaMemsetAsync(reinterpret_cast<void*>(c->plan.regions[i].r.dev_addr), 0,
                                  c->plan.regions[i].r.bytes, s));
  if (mech(c) == SWAP_MECH_CE_PIPE) {
    if ((st = ce_pipe(c, S, 1, p, s)) != SWAP_OK) return st;
  } else if (is_ce(mech(c))) {
    if ((st = ce_copy(c, S, 1, s)) != SWAP_OK) return st;
    if ((st = launch(c, swk::HASH_CHECK, hash_kind(c), p, s)) != SWAP_OK) return st;
  } else {
    if ((st = launch(c, swk::SCATTER, kind_of(c), p, s)) != SWAP_OK) return st;
  }
  CUDA_TRY(c, cudaEventRecord(c->ev[3], s));
  c->pending[1] = true;
  c->st = St::RESTORED;
  return SWAP_OK;
}

swap_status swap_verify(swap_ctx_t* c, swap_stream_t stream, int hbm_pass, swap_verify_result_t* res) {
  if (!c || !res) return SWAP_EINVAL;
  if (c->st != St::RESTORED) {
    c->err = "verify needs a restore";
    return SWAP_ESTATE;
  }
  DeviceGuard g(c->cfg.device);
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  if (hbm_pass) {
    swk::Params p = base_params(c, c->s_all);
    p.n_bad = &c->d_status->hbm_n_bad;
    p.first_bad = &c->d_status->hbm_first_bad;
    CUDA_TRY(c, cudaMemsetAsync(&c->d_status->hbm_n_bad, 0, 8, s));
    CUDA_TRY(c, cudaMemsetAsync(&c->d_status->hbm_first_bad, 0xFF, 8, s));
    CUDA_TRY(c, cudaEventRecord(c->ev[4], s));
    swap_status st = launch(c, swk::HASH_CHECK, hash_kind(c), p, s);
    if (st != SWAP_OK) return st;
    CUDA_TRY(c, cudaEventRecord(c->ev[5], s));
    c->pending[2] = true;
  }
  CUDA_TRY(c, cudaMemcpyAsync(c->h_status, c->d_status, sizeof(swk::DevStatus), cudaMemcpyDeviceToHost, s));
  CUDA_TRY(c, cudaStreamSynchronize(s));
  for (int ph = 1; ph < 3; ++ph) {
    swap_status ts = collect_timing(c, ph);
    if (ts != SWAP_OK) return ts;
  }
  res->n_bad = c->h_status->n_bad;
  res->first_bad_chunk = c->h_status->first_bad;
  res->hbm_checked = hbm_pass ? 1u : 0u;
  res->hbm_n_bad = hbm_pass ? c->h_status->hbm_n_bad : 0;
  res->hbm_first_bad = hbm_pass ? c->h_status->hbm_first_bad : UINT64_MAX;
  res->manifest_ok = swp::manifest_crc_ok(c->plan, manifest_ptr(c)) ? 1u : 0u;
  if (res->n_bad || res->hbm_n_bad || !res->manifest_ok) {
    c->err = "verification failed: " + std::to_string(res->n_bad) + " bad chunk(s) in restore, " +
             std::to_string(res->hbm_n_bad) + " in HBM pass, manifest_ok=" + std::to_string(res->manifest_ok);
    return SWAP_ECORRUPT;
  }
  return SWAP_OK;
}

swap_status swap_set_region_policy(swap_ctx_t* c, uint32_t region_index, uint32_t policy) {
  if (!c || policy > SWAP_POLICY_DISCARD) return SWAP_EINVAL;
  if (c->st != St::REGISTERED) {
    c->err = "region policies can only change between swap_register_regions and the first checkpoint";
    return SWAP_ESTATE;
  }
  if (region_index >= c->policy.size()) return SWAP_EINVAL;
  if (c->policy[region_index] == policy) return SWAP_OK;
  c->policy[region_index] = policy;
  DeviceGuard g(c->cfg.device);
  swap_status st = build_sets(c);
  if (st != SWAP_OK || c->helpers.empty()) return st;
  std::vector<int> devs;  // restore groups changed: re-size the helpers' staging
  for (auto& h : c->helpers) devs.push_back(h.dev);
  return swap_set_helpers(c, devs.data(), (int)devs.size());
}

// Full-duplex exchange (see include/swap.h). Victims are gathered group by group on s_out (hash pass of
// the group, then its D2H copies, then an event); a victim slab is released once the last group touching
// it has completed. The incoming image is scattered group by group on s_in; before a group is enqueued its
// slabs are mapped, first waiting for victim events (and releasing their slabs) while the mapping would
// exceed the victims' initial HBM plus `headroom`.
swap_status swap_exchange(swap_ctx_t* const* victims, size_t nv, swap_ctx_t* in, swap_stream_t s_out_,
                          swap_stream_t s_in_, uint64_t headroom, uint64_t* peak_extra) {
  if ((!victims && nv) || (!in && nv == 0)) return SWAP_EINVAL;
  swap_ctx* any = nv ? victims[0] : in;
  const int dev = any->cfg.device;
  for (size_t i = 0; i < nv; ++i) {
    swap_ctx* v = victims[i];
    if (!v || v->cfg.device != dev || !v->arena || v == in) return SWAP_EINVAL;
    if (v->st == St::CREATED || v->st == St::CKPT_PENDING) return SWAP_ESTATE;
  }
  if (in) {
    if (in->cfg.device != dev || !in->arena) return SWAP_EINVAL;
    if (in->st != St::CHECKPOINTED && in->st != St::RESTORED) return SWAP_ESTATE;
    swap_status st = swp::check_manifest(in->plan, manifest_ptr(in), &in->err);
    if (st != SWAP_OK) return st;
  }
  DeviceGuard g(dev);
  cudaStream_t so = reinterpret_cast<cudaStream_t>(s_out_), si = reinterpret_cast<cudaStream_t>(s_in_);
  if (cudaDeviceSynchronize() != cudaSuccess) return cuda_fail(any, cudaGetLastError(), "swap_exchange sync");

  // ---- victims: enqueue every group's hash + D2H copies, remember which slabs each event frees
  struct Release {
    cudaEvent_t ev;
    swap_arena* arena;
    std::vector<uint64_t> slabs;
  };
  std::vector<Release> rel;
  uint64_t held = 0;  // victim HBM still mapped
  std::vector<DescSet*> vsets(nv);
  swap_status st;
  for (size_t i = 0; i < nv; ++i) {
    swap_ctx* v = victims[i];
    DescSet& S = v->first_ckpt_done ? v->s_save : v->s_move;
    vsets[i] = &S;
    swap_arena* A = v->arena;
    held += swarena::mapped_bytes(A);
    std::vector<int64_t> last(swarena::n_slabs(A), -1);  // last group touching each slab
    for (size_t gi = 0; gi < S.groups.size(); ++gi)
      for (const Span& sp : S.groups[gi].spans)
        if (sp.bytes && swarena::contains(A, sp.dev, sp.dev + sp.bytes))
          for (uint64_t s = swarena::slab_of(A, sp.dev); s <= swarena::slab_of(A, sp.dev + sp.bytes - 1); ++s)
            last[s] = (int64_t)gi;
    std::vector<uint64_t> idle;  // slabs no saved group reads: free them right away
    for (uint64_t s = 0; s < last.size(); ++s)
      if (last[s] < 0 && swarena::slab_mapped(A, s)) idle.push_back(s);
    for (uint64_t s : idle) {
      held -= swarena::slab_size(A, s);
      if ((st = swarena::unmap_slab(A, s)) != SWAP_OK) return cuda_fail(v, cudaErrorUnknown, "slab release");
    }
    CUDA_TRY(v, cudaEventRecord(v->ev[0], so));
    if (!v->first_ckpt_done && v->s_zero.n_desc &&
        (st = launch(v, swk::HASH_STORE, hash_kind(v), base_params(v, v->s_zero), so)) != SWAP_OK)
      return st;
    for (size_t gi = 0; gi < S.groups.size(); ++gi) {
      const Group& G = S.groups[gi];
      swk::Params p = base_params(v, S);
      p.desc = S.d_desc + G.d0;
      p.partial = v->d_partial + G.d0;
      p.n_desc = G.d1 - G.d0;
      if ((st = launch(v, swk::HASH_STORE, hash_kind(v), p, so)) != SWAP_OK) return st;
      for (const Span& sp : G.spans)
        if ((st = memcpy_dir(v, sp, 0, so)) != SWAP_OK) return st;
      CUDA_TRY(v, cudaEventRecord(S.group_ev[gi], so));
      Release r{S.group_ev[gi], A, {}};
      for (uint64_t s = 0; s < last.size(); ++s)
        if (last[s] == (int64_t)gi) r.slabs.push_back(s);
      rel.push_back(std::move(r));
    }
    CUDA_TRY(v, cudaEventRecord(v->ev[1], so));
    v->pending[0] = true;
    v->first_ckpt_done = true;
    v->st = St::CKPT_PENDING;
  }
  const uint64_t budget = held + headroom;
  uint64_t acquired = 0, peak = 0;
  size_t next_rel = 0;
  auto release_next = [&]() -> swap_status {
    Release& r = rel[next_rel++];
    CUDA_TRY(any, cudaEventSynchronize(r.ev));
    for (uint64_t s : r.slabs) {
      if (!swarena::slab_mapped(r.arena, s)) continue;
      held -= swarena::slab_size(r.arena, s);
      if (swarena::unmap_slab(r.arena, s) != SWAP_OK) return cuda_fail(any, cudaErrorUnknown, "slab release");
    }
    return SWAP_OK;
  };
  const uint64_t base_held = held;
  // map one incoming slab, first waiting for victim releases while the mapping would exceed the budget
  auto acquire_slab = [&](uint64_t s) -> swap_status {
    swap_arena* A = in->arena;
    if (swarena::slab_mapped(A, s)) return SWAP_OK;
    const uint64_t need = swarena::slab_size(A, s);
    while (held + acquired + need > budget) {
      if (next_rel == rel.size()) {
        in->err = "swap_exchange: the incoming image does not fit in the victims' HBM plus headroom";
        return SWAP_ENOMEM;
      }
      swap_status rs = release_next();
      if (rs != SWAP_OK) return rs;
    }
    swap_status ms = swarena::map_slab(A, s);
    if (ms != SWAP_OK) return ms;
    acquired += need;
    if (held + acquired > base_held) peak = std::max(peak, held + acquired - base_held);
    return SWAP_OK;
  };
  auto acquire = [&](uint64_t lo, uint64_t hi) -> swap_status {
    swap_arena* A = in->arena;
    if (hi <= lo || !swarena::contains(A, lo, hi)) return SWAP_OK;
    for (uint64_t s = swarena::slab_of(A, lo); s <= swarena::slab_of(A, hi - 1); ++s) {
      swap_status as = acquire_slab(s);
      if (as != SWAP_OK) return as;
    }
    return SWAP_OK;
  };

  // ---- incoming: scatter group by group, each mapped just in time under the budget
  if (in) {
    DescSet& S = in->s_move;
    swk::Params base = base_params(in, S);
    CUDA_TRY(in, cudaMemsetAsync(&in->d_status->n_bad, 0, 8, si));
    CUDA_TRY(in, cudaMemsetAsync(&in->d_status->first_bad, 0xFF, 8, si));
    CUDA_TRY(in, cudaEventRecord(in->ev[2], si));
    for (size_t i = 0; i < in->policy.size(); ++i)
      if (in->policy[i] == SWAP_POLICY_DISCARD && in->plan.regions[i].r.bytes) {
        const auto& r = in->plan.regions[i].r;
        if ((st = acquire(r.dev_addr, r.dev_addr + r.bytes)) != SWAP_OK) return st;
        CUDA_TRY(in, cudaMemsetAsync(reinterpret_cast<void*>(r.dev_addr), 0, r.bytes, si));
      }
    CUDA_TRY(in, cudaEventRecord(in->ev_fork, si));
    CUDA_TRY(in, cudaStreamWaitEvent(in->side, in->ev_fork, 0));
    for (size_t gi = 0; gi < S.groups.size(); ++gi) {
      const Group& G = S.groups[gi];
      for (const Span& sp : G.spans)
        if ((st = acquire(sp.dev, sp.dev + sp.bytes)) != SWAP_OK) return st;
      for (const Span& sp : G.spans)
        if ((st = memcpy_dir(in, sp, 1, si)) != SWAP_OK) return st;
      CUDA_TRY(in, cudaEventRecord(S.group_ev[gi], si));
      CUDA_TRY(in, cudaStreamWaitEvent(in->side, S.group_ev[gi], 0));
      swk::Params p = base;
      p.desc = base.desc + G.d0;
      p.partial = base.partial + G.d0;
      p.n_desc = G.d1 - G.d0;
      if ((st = launch(in, swk::HASH_CHECK, hash_kind(in), p, in->side)) != SWAP_OK) return st;
    }
    // slabs holding no restored bytes (guards, padding) are mapped too: the arena is whole again
    for (uint64_t s = 0; s < swarena::n_slabs(in->arena); ++s)
      if ((st = acquire_slab(s)) != SWAP_OK) return st;
    CUDA_TRY(in, cudaEventRecord(in->ev_join, in->side));
    CUDA_TRY(in, cudaStreamWaitEvent(si, in->ev_join, 0));
    CUDA_TRY(in, cudaEventRecord(in->ev[3], si));
    in->pending[1] = true;
    in->st = St::RESTORED;
  }
  // ---- drain the victims, release the rest, seal their manifests
  while (next_rel < rel.size())
    if ((st = release_next()) != SWAP_OK) return st;
  CUDA_TRY(any, cudaStreamSynchronize(so));
  for (size_t i = 0; i < nv; ++i) {
    swap_ctx* v = victims[i];
    for (uint64_t s = 0; s < swarena::n_slabs(v->arena); ++s)
      if (swarena::slab_mapped(v->arena, s)) {
        held -= swarena::slab_size(v->arena, s);
        swarena::unmap_slab(v->arena, s);
      }
    swap_status ts = collect_timing(v, 0);
    if (ts != SWAP_OK) return ts;
    swp::seal_manifest(v->plan, manifest_ptr(v));
    v->st = St::CHECKPOINTED;
  }
  if (peak_extra) *peak_extra = peak;
  return SWAP_OK;
}

swap_status swap_set_helpers(swap_ctx_t* c, const int* devices, int n) {
  if (!c || n < 0 || (n && !devices)) return SWAP_EINVAL;
  if (c->st == St::CREATED) return SWAP_ESTATE;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess) return SWAP_ECUDA;
  for (int i = 0; i < n; ++i)
    if (devices[i] < 0 || devices[i] >= ndev) return SWAP_EINVAL;
  DeviceGuard g(c->cfg.device);
  free_helpers(c);
  uint64_t stage = 0;  // largest image range of one restore group
  for (const Group& G : c->s_move.groups)
    stage = std::max<uint64_t>(stage, (uint64_t)(G.spans.back().host + G.spans.back().bytes - G.spans.front().host));
  for (int i = 0; i < n; ++i) {
    swap_ctx::Helper h;
    h.dev = devices[i];
    CUDA_TRY(c, cudaSetDevice(h.dev));
    if (h.dev != c->cfg.device) {
      cudaError_t e = cudaDeviceEnablePeerAccess(c->cfg.device, 0);  // NVLink P2P to the target
      if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return cuda_fail(c, e, "peer access");
      cudaGetLastError();
    }
    CUDA_TRY(c, cudaStreamCreateWithFlags(&h.s, cudaStreamNonBlocking));
    CUDA_TRY(c, cudaEventCreateWithFlags(&h.ev, cudaEventDisableTiming));
    CUDA_TRY(c, cudaEventCreateWithFlags(&h.done, cudaEventDisableTiming));
    CUDA_TRY(c, cudaMalloc(&h.staging, std::max<uint64_t>(stage, 16)));
    c->helpers.push_back(h);
  }
  CUDA_TRY(c, cudaSetDevice(c->cfg.device));
  return SWAP_OK;
}

swap_status swap_bind_arena(swap_ctx_t* c, swap_arena_t* a) {
  if (!c) return SWAP_EINVAL;
  if (a && swarena::device(a) != c->cfg.device) {
    c->err = "arena and ctx are on different devices";
    return SWAP_EINVAL;
  }
  c->arena = a;
  return SWAP_OK;
}

swap_status swap_set_mechanism(swap_ctx_t* c, uint32_t mechanism) {
  if (!c || mechanism >= SWAP_MECH_COUNT) return SWAP_EINVAL;
  c->cfg.mechanism = mechanism;
  return SWAP_OK;
}

swap_status swap_get_mechanism(const swap_ctx_t* c, uint32_t* effective) {
  if (!c || !effective) return SWAP_EINVAL;
  if (c->st == St::CREATED) return SWAP_ESTATE;
  *effective = resolve_mech(c, 1, false);
  return SWAP_OK;
}

swap_status swap_get_manifest(const swap_ctx_t* c, const void** bytes, size_t* n) {
  if (!c || !bytes || !n) return SWAP_EINVAL;
  if (!c->image) return SWAP_ESTATE;
  *bytes = c->image + c->plan.manifest_off;
  *n = c->plan.manifest_bytes;
  return SWAP_OK;
}

swap_status swap_get_image(const swap_ctx_t* c, void** host, size_t* n) {
  if (!c || !host || !n) return SWAP_EINVAL;
  if (!c->image) return SWAP_ESTATE;
  *host = c->image;
  *n = c->plan.image_bytes;
  return SWAP_OK;
}

swap_status swap_get_summary(const swap_ctx_t* c, swap_shard_summary_t* out) {
  if (!c || !out) return SWAP_EINVAL;
  if (c->st != St::CHECKPOINTED && c->st != St::RESTORED) return SWAP_ESTATE;
  swp::make_summary(c->plan, c->image + c->plan.manifest_off, out);
  return SWAP_OK;
}

swap_status swap_import(swap_ctx_t* c) {
  if (!c) return SWAP_EINVAL;
  if (c->st == St::CREATED || c->st == St::CKPT_PENDING) return SWAP_ESTATE;
  swap_status st = swp::check_manifest(c->plan, manifest_ptr(c), &c->err);
  if (st != SWAP_OK) return st;
  c->st = St::CHECKPOINTED;
  c->first_ckpt_done = true;  // the imported image already holds SAVE_ONCE bytes and DISCARD checksums
  return SWAP_OK;
}

swap_status swap_plan_layout(const swap_region_t* regions, size_t n, const swap_config_t* cfg_in, uint64_t* payload,
                             uint64_t* n_chunks, uint64_t* manifest_off, uint64_t* image_bytes) {
  if (!cfg_in) return SWAP_EINVAL;
  swap_config_t cfg = *cfg_in;
  std::string err;
  swap_status st = swp::normalize_config(&cfg, &err);
  if (st != SWAP_OK) return st;
  swp::Plan P;
  if ((st = swp::build_plan(regions, n, cfg, &P, &err)) != SWAP_OK) return st;
  if (payload) *payload = P.payload_bytes;
  if (n_chunks) *n_chunks = P.n_chunks;
  if (manifest_off) *manifest_off = P.manifest_off;
  if (image_bytes) *image_bytes = P.image_bytes;
  return SWAP_OK;
}

swap_status swap_plan_manifest(const swap_region_t* regions, size_t n, const swap_config_t* cfg_in,
                               const uint64_t* cs, void* out, size_t cap, size_t* manifest_bytes) {
  if (!cfg_in || !manifest_bytes) return SWAP_EINVAL;
  swap_config_t cfg = *cfg_in;
  std::string err;
  swap_status st = swp::normalize_config(&cfg, &err);
  if (st != SWAP_OK) return st;
  swp::Plan P;
  if ((st = swp::build_plan(regions, n, cfg, &P, &err)) != SWAP_OK) return st;
  *manifest_bytes = P.manifest_bytes;
  if (!out || cap < P.manifest_bytes) return SWAP_EINVAL;
  uint8_t* man = static_cast<uint8_t*>(out);
  swp::write_manifest_skeleton(P, man);
  if (cs) {
    uint8_t* cr = man + swp::kHeaderBytes + swp::kRegionRecBytes * P.regions.size();
    for (uint64_t g = 0; g < P.n_chunks; ++g) std::memcpy(cr + swp::kChunkRecBytes * g + 24, cs + g, 8);
  }
  swp::seal_manifest(P, man);
  return SWAP_OK;
}

swap_status swap_merge_global(const swap_shard_summary_t* all, int world, uint64_t* digest) {
  if (!all || world < 1) return SWAP_EINVAL;
  for (int r = 0; r < world; ++r)
    if ((int)all[r].rank != r || (int)all[r].world != world || all[r].reserved != 0) return SWAP_ENCCL;
  if (digest) *digest = swp::crc32c_host(all, sizeof(swap_shard_summary_t) * (size_t)world);
  return SWAP_OK;
}

swap_status swap_set_global(swap_ctx_t* c, const swap_shard_summary_t* all, int world, uint64_t* digest) {
  if (!c || !all || world < 1) return SWAP_EINVAL;
  if (c->st != St::CHECKPOINTED && c->st != St::RESTORED) return SWAP_ESTATE;
  if (world != c->cfg.world) {
    c->err = "world mismatch in global manifest";
    return SWAP_ENCCL;
  }
  if (swap_merge_global(all, world, nullptr) != SWAP_OK) {
    c->err = "global manifest entries are not rank-ordered summaries of this world";
    return SWAP_ENCCL;
  }
  swap_shard_summary_t mine;
  swp::make_summary(c->plan, c->image + c->plan.manifest_off, &mine);
  if (std::memcmp(&mine, &all[c->cfg.rank], sizeof(mine)) != 0) {
    c->err = "own entry of the global manifest differs from the local summary";
    return SWAP_ENCCL;
  }
  c->global.assign(all, all + world);
  if (digest) *digest = swp::crc32c_host(all, sizeof(swap_shard_summary_t) * (size_t)world);
  return SWAP_OK;
}

swap_status swap_get_timings(const swap_ctx_t* c, swap_timings_t* out) {
  if (!c || !out) return SWAP_EINVAL;
  out->checkpoint_ms = c->ms[0];
  out->restore_ms = c->ms[1];
  out->verify_ms = c->ms[2];
  out->reserved = 0.f;
  return SWAP_OK;
}

swap_status swap_get_launch_count(const swap_ctx_t* c, uint64_t* n) {
  if (!c || !n) return SWAP_EINVAL;
  *n = c->launches;
  return SWAP_OK;
}

const char* swap_status_str(swap_status s) {
  switch (s) {
    case SWAP_OK: return "SWAP_OK";
    case SWAP_EINVAL: return "SWAP_EINVAL";
    case SWAP_ENOMEM: return "SWAP_ENOMEM";
    case SWAP_ECUDA: return "SWAP_ECUDA";
    case SWAP_ESTATE: return "SWAP_ESTATE";
    case SWAP_ECORRUPT: return "SWAP_ECORRUPT";
    case SWAP_ENCCL: return "SWAP_ENCCL";
    case SWAP_EUNSUPPORTED: return "SWAP_EUNSUPPORTED";
    case SWAP_EINTERNAL: return "SWAP_EINTERNAL";
    default: return "SWAP_UNKNOWN";
  }
}

const char* swap_last_error(const swap_ctx_t* c) { return c ? c->err.c_str() : "null ctx"; }

void swap_destroy(swap_ctx_t* c) {
  if (!c) return;
  {
    DeviceGuard g(c->cfg.device);
    release(c);
  }
  delete c;
}

}  // extern "C"
