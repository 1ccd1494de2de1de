// swap_abi.cpp — the extern "C" boundary of libswap (declared and documented in include/swap.h).
//
// Context state machine (include/swap.h; the paper's snapshot-once / restore-many model,
// P:L115):
//   CREATED --register--> REGISTERED --checkpoint--> CKPT_PENDING --sync--> CHECKPOINTED
//   CHECKPOINTED|RESTORED --restore--> RESTORED;   REGISTERED|CHECKPOINTED|RESTORED --checkpoint--> CKPT_PENDING
#include <sched.h>
#include <sys/mman.h>
#include <sys/syscall.h>
#include <unistd.h>

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <fstream>
#include <string>
#include <thread>
#include <vector>

#include "ctx.h"

using namespace swc;

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
      (e = cudaEventCreate(&c->ev[4])) != cudaSuccess || (e = cudaEventCreate(&c->ev[5])) != cudaSuccess ||
      (e = swk::probe_smem_base()) != cudaSuccess) {
    cuda_fail(c, e, "swap_create");
    fprintf(stderr, "libswap: %s\n", c->err.c_str());
    release(c);
    delete c;
    return SWAP_ECUDA;
  }
  *out = c;
  return SWAP_OK;
}

// ---- host NUMA placement of the image (swap_config_t.host_numa; P:L230 per-GPU topology at init)
static std::string read_line(const std::string& path) {
  std::ifstream f(path);
  std::string s;
  std::getline(f, s);
  return s;
}
// "0-7,16-23" -> {0..7, 16..23}
static std::vector<int> parse_list(const std::string& s) {
  std::vector<int> out;
  size_t i = 0;
  while (i < s.size()) {
    size_t j = s.find(',', i);
    if (j == std::string::npos) j = s.size();
    const std::string t = s.substr(i, j - i);
    int a = -1, b = -1;
    if (sscanf(t.c_str(), "%d-%d", &a, &b) == 2) {
      for (int x = a; x <= b; ++x) out.push_back(x);
    } else if (sscanf(t.c_str(), "%d", &a) == 1) {
      out.push_back(a);
    }
    i = j + 1;
  }
  return out;
}
static int numa_nodes_online() { return (int)parse_list(read_line("/sys/devices/system/node/online")).size(); }
// The NUMA node sysfs reports for the device's PCI function, or -1.
static int device_numa_node(int dev) {
  char bus[64] = {0};
  if (cudaDeviceGetPCIBusId(bus, sizeof bus, dev) != cudaSuccess) return -1;
  unsigned dom = 0, b = 0, d = 0, fn = 0;
  if (sscanf(bus, "%x:%x:%x.%x", &dom, &b, &d, &fn) != 4) return -1;
  char path[128];
  snprintf(path, sizeof path, "/sys/bus/pci/devices/%04x:%02x:%02x.%x/numa_node", dom, b, d, fn);
  const std::string v = read_line(path);
  return v.empty() ? -1 : atoi(v.c_str());
}
constexpr int kMpolPreferred = 1, kMpolFNode = 1, kMpolFAddr = 2;
static bool mbind_preferred(void* p, size_t n, int node) {
  if (node < 0 || node >= 1024) return false;
  unsigned long mask[16] = {0};
  mask[node / 64] = 1ul << (node % 64);
  return syscall(SYS_mbind, p, n, kMpolPreferred, mask, 1025ul, 0u) == 0;
}
// Share of `samples` evenly spaced pages of [p, p+n) that reside on `node`.
static double local_share(const uint8_t* p, size_t n, int node, int samples = 256) {
  int hit = 0, seen = 0;
  for (int i = 0; i < samples; ++i) {
    const uint8_t* a = p + (n / samples) * (size_t)i;
    int where = -1;
    if (syscall(SYS_get_mempolicy, &where, nullptr, 0ul, a, (unsigned long)(kMpolFNode | kMpolFAddr)) != 0) continue;
    ++seen;
    hit += where == node;
  }
  return seen ? (double)hit / seen : 0.0;
}

// Faults the image's pages in (the kernel zero-fills them) from several threads before pinning:
// cudaHostRegister would otherwise fault and zero every page from the calling thread alone. With a
// NUMA node, the threads run on that node's CPUs (first touch + the preferred policy keep the pages there).
static void prefault(uint8_t* p, size_t n, int node) {
  const size_t page = 2u << 20;
  std::vector<int> cpus;
  if (node >= 0) cpus = parse_list(read_line("/sys/devices/system/node/node" + std::to_string(node) + "/cpulist"));
  const unsigned hw = cpus.empty() ? std::thread::hardware_concurrency() : (unsigned)cpus.size();
  const size_t k = std::max<size_t>(1, std::min<size_t>({hw ? hw : 1u, 32u, n / page}));
  const size_t per = (n / k + page - 1) / page * page;
  std::vector<std::thread> th;
  for (size_t t = 0; t < k; ++t) {
    const size_t lo = t * per, hi = std::min(n, lo + per);
    if (lo >= hi) break;
    th.emplace_back([p, lo, hi, &cpus] {
      if (!cpus.empty()) {
        cpu_set_t set;
        CPU_ZERO(&set);
        for (int c : cpus)
          if (c >= 0 && c < CPU_SETSIZE) CPU_SET(c, &set);
        sched_setaffinity(0, sizeof set, &set);  // this thread only
      }
      volatile uint8_t* q = p;
      for (size_t o = lo; o < hi; o += 4096) q[o] = 0;  // a write: a read would map the shared zero page
    });
  }
  for (auto& x : th) x.join();
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
  int node = -1;
  if (c->cfg.host_numa != -1 && numa_nodes_online() > 1) {
    node = c->cfg.host_numa > 0 ? c->cfg.host_numa - 1 : device_numa_node(c->cfg.device);
    if (node >= 0 && !mbind_preferred(m, c->map_bytes, node)) node = -1;
  }
  prefault(c->image, c->map_bytes, node);
  c->numa_node = node;
  c->numa_local = node >= 0 ? local_share(c->image, c->map_bytes, node) : 1.0;
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
  c->keep.assign(P.n_chunks, 1);
  c->next_keep.assign(P.n_chunks, 1);
  c->img_zero.assign(P.n_chunks, 1);  // the image is zero-filled at allocation
  c->mask_dirty = false;
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
  c->exp_valid = false;  // the chunk records are rewritten
  c->cur_mech = resolve_mech(c, 0);
  CUDA_TRY(c, cudaEventRecord(c->ev[0], s));
  bool hash_zero = false;
  swap_status st = apply_mask(c, s, &hash_zero);  // a new chunk mask: sets rebuilt, stale image bytes zeroed
  if (st != SWAP_OK) return st;
  // SAVE_ONCE regions are gathered by the first checkpoint only; DISCARD regions and masked chunks never
  // (their image bytes are zero and their c_g the checksums of zero chunks, hashed from a zero buffer
  // whenever the set of zero chunks changes).
  DescSet& S = c->first_ckpt_done ? c->s_save : c->s_move;
  swk::Params p = base_params(c, S);
  if (hash_zero && c->s_zero.n_desc &&
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
  note_gathered(c, S);
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

// The restore (swap_restore), or with n_stripes > 1 only the CE_PIPE groups g with g % n_stripes == stripe
// (swap_restore_stripe: DP replicas each pull one stripe over their own link, NEXT-2).
static swap_status restore_impl(swap_ctx* c, swap_stream_t stream, uint32_t stripe, uint32_t n_stripes) {
  if (c->st != St::CHECKPOINTED && c->st != St::RESTORED) {
    c->err = "restore needs a completed checkpoint (swap_sync) or an imported image";
    return SWAP_ESTATE;
  }
  swap_status st = swp::check_manifest(c->plan, manifest_ptr(c), &c->err);
  if (st != SWAP_OK) return st;
  DeviceGuard g(c->cfg.device);
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  c->cur_mech = n_stripes > 1 ? (uint32_t)SWAP_MECH_CE_PIPE : resolve_mech(c, 1);
  c->stripe = stripe;
  c->n_stripes = n_stripes;
  DescSet& S = c->s_move;
  if (mech(c) == SWAP_MECH_CE_PIPE || is_ce(mech(c)))  // the copies will saturate the host link
    if ((st = stage_expected(c, s)) != SWAP_OK) return st;
  swk::Params p = base_params(c, S);
  CUDA_TRY(c, cudaMemsetAsync(&c->d_status->n_bad, 0, 8, s));
  CUDA_TRY(c, cudaMemsetAsync(&c->d_status->first_bad, 0xFF, 8, s));
  CUDA_TRY(c, cudaEventRecord(c->ev[2], s));
  if (c->arena && !swarena::resident(c->arena)) {
    // zero chunks (filled below) and, for movers other than CE_PIPE, everything, need HBM now
    std::vector<Span> now = c->zero_spans;
    if (mech(c) != SWAP_MECH_CE_PIPE)
      for (size_t i = 0; i < c->policy.size(); ++i)
        now.push_back(Span{c->plan.regions[i].r.dev_addr, nullptr, c->plan.regions[i].r.bytes});
    if ((st = map_spans(c, now)) != SWAP_OK) return st;
  }
  // DISCARD regions and masked chunks come back as zeros; under CE_PIPE on the side stream, overlapped
  // with the first group's copies (ce_pipe joins the side stream back into `s` at the end)
  cudaStream_t zs = s;
  if (mech(c) == SWAP_MECH_CE_PIPE && !c->zero_spans.empty()) {
    CUDA_TRY(c, cudaEventRecord(c->ev_fork, s));
    CUDA_TRY(c, cudaStreamWaitEvent(c->side, c->ev_fork, 0));
    zs = c->side;
  }
  if ((st = zero_fill_device(c, zs)) != SWAP_OK) return st;
  if (mech(c) == SWAP_MECH_CE_PIPE) {
    st = ce_pipe(c, S, 1, p, s);
    c->stripe = 0;
    c->n_stripes = 1;
    if (st != SWAP_OK) return st;
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

swap_status swap_restore(swap_ctx_t* c, swap_stream_t stream) {
  if (!c) return SWAP_EINVAL;
  return restore_impl(c, stream, 0, 1);
}

swap_status swap_restore_stripe(swap_ctx_t* c, uint32_t stripe, uint32_t n_stripes, swap_stream_t stream) {
  if (!c || n_stripes == 0 || stripe >= n_stripes) return SWAP_EINVAL;
  if (n_stripes > 1 && !c->helpers.empty()) {
    c->err = "stripe restores and helper devices do not combine";
    return SWAP_EINVAL;
  }
  return restore_impl(c, stream, stripe, n_stripes);
}

swap_status swap_get_restore_spans(const swap_ctx_t* c, swap_span_t* out, size_t cap, size_t* n) {
  if (!c || !n || (cap && !out)) return SWAP_EINVAL;
  if (c->st == St::CREATED) return SWAP_ESTATE;
  size_t k = 0;
  const DescSet& S = c->s_move;
  for (size_t g = 0; g < S.groups.size(); ++g)
    for (const Span& sp : coalesce(S.groups[g].spans)) {
      if (k < cap) out[k] = swap_span_t{(uint32_t)g, 0u, sp.dev, (uint64_t)(sp.host - c->image), sp.bytes};
      ++k;
    }
  *n = k;
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
  const auto& r = c->plan.regions[region_index];
  if (policy != SWAP_POLICY_SAVE)  // chunk masks apply to SAVE regions only
    std::fill(c->next_keep.begin() + r.first, c->next_keep.begin() + r.first + r.nchunks, 1);
  c->keep = c->next_keep;
  c->mask_dirty = false;
  DeviceGuard g(c->cfg.device);
  swap_status st = build_sets(c);
  if (st != SWAP_OK || c->helpers.empty()) return st;
  std::vector<int> devs;  // restore groups changed: re-size the helpers' staging
  for (auto& h : c->helpers) devs.push_back(h.dev);
  return swap_set_helpers(c, devs.data(), (int)devs.size());
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
  *effective = resolve_mech(c, 1);
  return SWAP_OK;
}

swap_status swap_get_numa(const swap_ctx_t* c, int32_t* node, double* local_fraction) {
  if (!c || !node || !local_fraction) return SWAP_EINVAL;
  if (!c->image) return SWAP_ESTATE;
  *node = c->numa_node;
  *local_fraction = c->numa_local;
  return SWAP_OK;
}

swap_status swap_get_mechanism_dir(const swap_ctx_t* c, int direction, uint32_t* effective) {
  if (!c || !effective || (direction != 0 && direction != 1)) return SWAP_EINVAL;
  if (c->st == St::CREATED) return SWAP_ESTATE;
  *effective = resolve_mech(c, direction);
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
  c->exp_valid = false;
  c->first_ckpt_done = true;  // the imported image already holds SAVE_ONCE bytes and DISCARD checksums
  // the image came from elsewhere: its zero chunks are unknown, so restores move every chunk a mask
  // does not force to zero by policy, and the next checkpoint re-applies any pending mask in full
  std::fill(c->img_zero.begin(), c->img_zero.end(), 0);
  if (std::find(c->keep.begin(), c->keep.end(), 0) != c->keep.end()) {
    const std::vector<uint8_t> pending = c->next_keep;
    std::fill(c->keep.begin(), c->keep.end(), 1);
    DeviceGuard g(c->cfg.device);
    if ((st = build_sets(c)) != SWAP_OK) return st;
    c->next_keep = pending;
    c->mask_dirty = true;
    if (!c->helpers.empty()) {  // the restore groups changed: re-size the helpers' staging
      std::vector<int> devs;
      for (auto& h : c->helpers) devs.push_back(h.dev);
      return swap_set_helpers(c, devs.data(), (int)devs.size());
    }
  }
  return SWAP_OK;
}

swap_status swap_set_chunk_mask(swap_ctx_t* c, uint32_t region_index, const uint8_t* keep, uint64_t n) {
  if (!c) return SWAP_EINVAL;
  if (c->st == St::CREATED || c->st == St::CKPT_PENDING) {
    c->err = c->st == St::CREATED ? "chunk mask before swap_register_regions" : "previous checkpoint not synced";
    return SWAP_ESTATE;
  }
  if (region_index >= c->policy.size()) return SWAP_EINVAL;
  const auto& r = c->plan.regions[region_index];
  if (n != r.nchunks) {
    c->err = "chunk mask length differs from the region's chunk count";
    return SWAP_EINVAL;
  }
  if (c->policy[region_index] != SWAP_POLICY_SAVE) {
    c->err = "chunk masks apply to SAVE regions only";
    return SWAP_EINVAL;
  }
  for (uint64_t j = 0; j < n; ++j) {
    const uint8_t k = keep ? (keep[j] ? 1 : 0) : 1;
    if (c->next_keep[r.first + j] != k) c->mask_dirty = true;
    c->next_keep[r.first + j] = k;
  }
  if (c->next_keep == c->keep) c->mask_dirty = false;
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
  out->check_ms = c->ms[1] > 0.f ? c->chk_ms : 0.f;
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
