// ctx.h — libswap-internal context (the opaque swap_ctx of include/swap.h) and the helpers shared by
// the ABI (swap_abi.cpp), the movers (movers.cpp) and the exchange / assisted restore (exchange.cpp).
#pragma once
#include <cstdint>
#include <memory>
#include <string>
#include <vector>

#include "arena.h"
#include "kernels.cuh"
#include "plan.h"

namespace swc {
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
}  // namespace swc

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
  // host copy of d_desc (the fused pulls rewrite sources); shared, so aliases of a set do not copy it
  std::shared_ptr<const std::vector<swk::SegDesc>> h_desc;
  bool owned = false;                     // false: an alias of another set
};

struct swap_ctx {
  swap_config_t cfg{};
  swc::St st = swc::St::CREATED;
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
  // chunk masks (swap_set_chunk_mask, NEXT-3): keep = the mask of the sets in use (last checkpoint's),
  // next_keep = the mask the next checkpoint applies; img_zero = the chunk's image bytes are known zero
  std::vector<uint8_t> keep, next_keep, img_zero;
  bool mask_dirty = false;
  std::vector<Span> zero_spans;  // device ranges a restore zero-fills (DISCARD regions, masked chunks)
  swk::ZSpan* d_zspans = nullptr;  // the same ranges cut into <= 1 MiB pieces for launch_zero_fill
  uint32_t n_zspans = 0;
  DescSet s_all, s_move, s_save, s_zero;
  bool first_ckpt_done = false;
  uint8_t* d_zero = nullptr;
  uint32_t* d_partial = nullptr;
  uint32_t* d_arrive = nullptr;
  swk::DevStatus* d_status = nullptr;
  swk::DevStatus* h_status = nullptr;  // pinned
  uint32_t* d_tables = nullptr;
  // device copy of the manifest's chunk records, staged by copy-engine restores so that the hash kernels
  // read the expected checksums from HBM, not over a host link saturated by the restore's own copies
  uint8_t* d_exp = nullptr;
  bool exp_valid = false;  // d_exp matches the manifest (cleared by checkpoint / import)
  void* d_tmaps = nullptr;                      // strand-staged CRC kernel: per-chunk tensor maps (null: none)
  unsigned long long* d_chunk_dev = nullptr;    // [n_chunks] chunk g's device address (0: no map)
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
    uint8_t* staging[2] = {nullptr, nullptr};  // ping-pong: the helper's i-th group of a restore uses slot i % 2
    uint64_t staging_bytes = 0;  // the largest restore group's image range when the helpers were set
    cudaEvent_t ev = nullptr, done = nullptr;
    cudaEvent_t consumed[2] = {nullptr, nullptr};  // this device has finished reading the slot (fused pull)
  };
  std::vector<Helper> helpers;
  // fused helper pull: s_move's descriptors with the sources of helper groups rewritten to the helper's
  // staging (read over NVLink by this device's SM mover); assist_copy = use copy-engine peer copies + hash
  swk::SegDesc* d_assist = nullptr;
  bool assist_copy = false;
  uint32_t stripe = 0, n_stripes = 1;  // CE_PIPE restore groups this restore moves (swap_restore_stripe)
  swk::SegDesc* d_pull = nullptr;      // descriptors of the last swap_pull_stripes (sources in peer HBM)
  size_t pull_cap = 0;
  cudaEvent_t ev_pull = nullptr;       // recorded after the last pull kernel (d_pull reuse waits for it)
  int numa_node = -1;         // NUMA node the image placement targeted (-1: none)
  double numa_local = 1.0;    // sampled share of image pages on numa_node
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  // per-group check timing of the last CE_PIPE restore (swap_timings_t.check_ms): event pairs, reused
  std::vector<cudaEvent_t> chk_ev;
  uint32_t n_chk = 0;
  float chk_ms = 0.f;
};

namespace swc {

#define CUDA_TRY(ctx, expr)                                    \
  do {                                                         \
    cudaError_t e_ = (expr);                                   \
    if (e_ != cudaSuccess) return cuda_fail((ctx), e_, #expr); \
  } while (0)

swap_status cuda_fail(swap_ctx* c, cudaError_t e, const char* what);
uint8_t* manifest_ptr(swap_ctx* c);
swk::Params base_params(swap_ctx* c, const DescSet& S);
int grid_of(swap_ctx* c);
uint32_t resolve_mech(const swap_ctx* c, int dir);
uint32_t mech(const swap_ctx* c);
swap_status stage_expected(swap_ctx* c, cudaStream_t s);
int kind_of(swap_ctx* c);
int hash_kind(swap_ctx* c);
swap_status launch(swap_ctx* c, int mode, int kind, const swk::Params& p, cudaStream_t s);
swap_status memcpy_dir(swap_ctx* c, const Span& sp, int dir, cudaStream_t s);
swap_status ce_copy(swap_ctx* c, DescSet& S, int dir, cudaStream_t s);
swap_status copy_spans(swap_ctx* c, const std::vector<Span>& spans, int dir, cudaStream_t s);
std::vector<Span> coalesce(const std::vector<Span>& spans);
swap_status map_spans(swap_ctx* c, const std::vector<Span>& spans);
swap_status ce_pipe(swap_ctx* c, DescSet& S, int dir, const swk::Params& base, cudaStream_t s);
swap_status collect_timing(swap_ctx* c, int p);
bool is_ce(uint32_t m);
void free_set(DescSet& S);
swap_status upload_tables(swap_ctx* c);
uint32_t auto_seg(const swap_ctx* c, uint64_t payload);
void free_helpers(swap_ctx* c);
void release(swap_ctx* c);
swap_status build_sets(swap_ctx* c);
swap_status apply_mask(swap_ctx* c, cudaStream_t s, bool* hash_zero);
void note_gathered(swap_ctx* c, const DescSet& S);
swap_status zero_fill_device(swap_ctx* c, cudaStream_t s);

}  // namespace swc
