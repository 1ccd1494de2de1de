// exchange.cpp — the two multi-stream data paths of libswap (include/swap.h):
//   swap_exchange     full-duplex swap: victims out (D2H) while the requested backend comes in (H2D),
//                     HBM handed over slab by slab within the victims' memory + headroom (NEXT-1);
//   swap_set_helpers  NVLink-assisted restore: peers pull restore groups over their own PCIe links into
//                     HBM staging and copy them to the target over NVLink (NEXT-2).
#include <cuda.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "ctx.h"

using namespace swc;

extern "C" {

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
    bool hash_zero = false;
    if ((st = apply_mask(v, so, &hash_zero)) != SWAP_OK) return st;
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
    if (hash_zero && v->s_zero.n_desc &&
        (st = launch(v, swk::HASH_STORE, hash_kind(v), base_params(v, v->s_zero), so)) != SWAP_OK)
      return st;
    for (size_t gi = 0; gi < S.groups.size(); ++gi) {
      const Group& G = S.groups[gi];
      swk::Params p = base_params(v, S);
      p.desc = S.d_desc + G.d0;
      p.partial = v->d_partial + G.d0;
      p.n_desc = G.d1 - G.d0;
      if ((st = launch(v, swk::HASH_STORE, hash_kind(v), p, so)) != SWAP_OK) return st;
      if ((st = copy_spans(v, G.spans, 0, so)) != SWAP_OK) return st;
      CUDA_TRY(v, cudaEventRecord(S.group_ev[gi], so));
      Release r{S.group_ev[gi], A, {}};
      for (uint64_t s = 0; s < last.size(); ++s)
        if (last[s] == (int64_t)gi) r.slabs.push_back(s);
      rel.push_back(std::move(r));
    }
    CUDA_TRY(v, cudaEventRecord(v->ev[1], so));
    v->pending[0] = true;
    note_gathered(v, S);
    v->first_ckpt_done = true;
    v->st = St::CKPT_PENDING;
    v->exp_valid = false;
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
    for (const Span& z : in->zero_spans)  // DISCARD regions and masked chunks come back as zeros
      if ((st = acquire(z.dev, z.dev + z.bytes)) != SWAP_OK) return st;
    if ((st = zero_fill_device(in, si)) != SWAP_OK) return st;
    CUDA_TRY(in, cudaEventRecord(in->ev_fork, si));
    CUDA_TRY(in, cudaStreamWaitEvent(in->side, in->ev_fork, 0));
    for (size_t gi = 0; gi < S.groups.size(); ++gi) {
      const Group& G = S.groups[gi];
      for (const Span& sp : G.spans)
        if ((st = acquire(sp.dev, sp.dev + sp.bytes)) != SWAP_OK) return st;
      if ((st = copy_spans(in, G.spans, 1, si)) != SWAP_OK) return st;
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
    v->exp_valid = false;
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
    h.staging_bytes = std::max<uint64_t>(stage, 16);
    c->helpers.push_back(h);  // owned by the ctx from here on (free_helpers releases whatever was made)
    auto& hh = c->helpers.back();
    for (int k = 0; k < 2; ++k) CUDA_TRY(c, cudaMalloc(&hh.staging[k], hh.staging_bytes));
  }
  CUDA_TRY(c, cudaSetDevice(c->cfg.device));
  for (auto& h : c->helpers)  // recorded on this device's side stream, so created on this device
    for (int k = 0; k < 2; ++k) CUDA_TRY(c, cudaEventCreateWithFlags(&h.consumed[k], cudaEventDisableTiming));
  if (n == 0) return SWAP_OK;
  // the fused pull: this device reads the helpers' staging (peer access target -> helper), with s_move's
  // descriptors of every helper group rewritten to source from the staging copy of its image range
  for (const auto& h : c->helpers)
    if (h.dev != c->cfg.device) {
      cudaError_t e = cudaDeviceEnablePeerAccess(h.dev, 0);
      if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return cuda_fail(c, e, "peer access to helper");
      cudaGetLastError();
    }
  const DescSet& S = c->s_move;
  std::vector<swk::SegDesc> d = S.h_desc ? *S.h_desc : std::vector<swk::SegDesc>();
  const size_t H = c->helpers.size();
  for (size_t gi = 0; gi < S.groups.size(); ++gi) {
    const size_t k = gi % (H + 1);
    if (k == 0) continue;
    const Group& G = S.groups[gi];
    const uint64_t lo_dev = reinterpret_cast<uint64_t>(c->image_dev + (G.spans.front().host - c->image));
    const int slot = (int)((gi / (H + 1)) % 2);  // ping-pong staging (movers.cpp ce_pipe)
    for (uint32_t i = G.d0; i < G.d1; ++i)
      d[i].host = reinterpret_cast<uint64_t>(c->helpers[k - 1].staging[slot]) + (d[i].host - lo_dev);
  }
  if (!d.empty()) {
    CUDA_TRY(c, cudaMalloc(&c->d_assist, d.size() * sizeof(swk::SegDesc)));
    CUDA_TRY(c, cudaMemcpy(c->d_assist, d.data(), d.size() * sizeof(swk::SegDesc), cudaMemcpyHostToDevice));
  }
  const char* mode = getenv("SWAP_ASSIST");
  c->assist_copy = mode && !strcmp(mode, "copy");
  return SWAP_OK;
}

// ---- DP replicas, fused NVLink pull (NEXT-2; include/swap.h). After swap_restore_stripe, every chunk of
// the other replicas' stripes is moved by the SM mover kernel (SCATTER) from the replica that restored it:
// the descriptors' source field points into that replica's HBM (mapped into this process by CUDA IPC, read
// over NVLink), so the chunk checksum is computed from the same registers that carry the bytes -- the
// all-gather and the check are one kernel.
swap_status swap_pull_stripes(swap_ctx_t* c, uint32_t stripe, uint32_t n_stripes, const int64_t* peer_delta,
                              swap_stream_t stream) {
  if (!c || !peer_delta || n_stripes < 2 || stripe >= n_stripes) return SWAP_EINVAL;
  if (c->st != St::RESTORED) {
    c->err = "swap_pull_stripes needs this replica's stripe restored first (swap_restore_stripe)";
    return SWAP_ESTATE;
  }
  DeviceGuard g(c->cfg.device);
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  const DescSet& S = c->s_move;
  std::vector<swk::SegDesc> d;
  if (!S.h_desc) return SWAP_OK;
  d.reserve(S.h_desc->size());
  for (size_t gi = 0; gi < S.groups.size(); ++gi) {
    const uint32_t o = (uint32_t)(gi % n_stripes);
    if (o == stripe) continue;
    for (uint32_t i = S.groups[gi].d0; i < S.groups[gi].d1; ++i) {
      swk::SegDesc x = (*S.h_desc)[i];
      x.host = (uint64_t)((int64_t)x.dev + peer_delta[o]);
      d.push_back(x);
    }
  }
  if (d.empty()) return SWAP_OK;
  if (c->ev_pull) CUDA_TRY(c, cudaStreamWaitEvent(s, c->ev_pull, 0));  // a previous pull may still read d_pull
  if (d.size() > c->pull_cap) {
    if (c->d_pull) {
      CUDA_TRY(c, cudaStreamSynchronize(s));
      cudaFree(c->d_pull);
    }
    c->d_pull = nullptr;
    c->pull_cap = 0;
    CUDA_TRY(c, cudaMalloc(&c->d_pull, d.size() * sizeof(swk::SegDesc)));
    c->pull_cap = d.size();
  }
  // pageable source: the call returns once the bytes are staged, so `d` may go out of scope
  CUDA_TRY(c, cudaMemcpyAsync(c->d_pull, d.data(), d.size() * sizeof(swk::SegDesc), cudaMemcpyHostToDevice, s));
  swk::Params p = base_params(c, S);
  p.desc = c->d_pull;
  p.n_desc = (uint32_t)d.size();
  swap_status st = launch(c, swk::SCATTER, hash_kind(c), p, s);
  if (st != SWAP_OK) return st;
  if (!c->ev_pull) CUDA_TRY(c, cudaEventCreateWithFlags(&c->ev_pull, cudaEventDisableTiming));
  CUDA_TRY(c, cudaEventRecord(c->ev_pull, s));
  return SWAP_OK;
}

namespace {
using GetRange = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);
GetRange get_range() {
  static GetRange f = [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      return (GetRange) nullptr;
    return reinterpret_cast<GetRange>(p);
  }();
  return f;
}
}  // namespace

swap_status swap_ipc_export(int device, const void* dev_ptr, uint8_t* handle, uint64_t* offset) {
  if (!dev_ptr || !handle || !offset) return SWAP_EINVAL;
  DeviceGuard g(device);
  GetRange f = get_range();
  CUdeviceptr base = 0;
  size_t size = 0;
  if (!f || f(&base, &size, reinterpret_cast<CUdeviceptr>(dev_ptr)) != CUDA_SUCCESS) return SWAP_ECUDA;
  cudaIpcMemHandle_t h;
  if (cudaIpcGetMemHandle(&h, reinterpret_cast<void*>(base)) != cudaSuccess) {
    cudaGetLastError();
    return SWAP_ECUDA;  // not a cudaMalloc allocation (e.g. a VMM arena)
  }
  static_assert(sizeof(h) == 64, "cudaIpcMemHandle_t is 64 B");
  memcpy(handle, &h, 64);
  *offset = reinterpret_cast<uint64_t>(dev_ptr) - (uint64_t)base;
  return SWAP_OK;
}

swap_status swap_ipc_import(int device, const uint8_t* handle, uint64_t offset, void** base, void** mapped) {
  if (!handle || !base || !mapped) return SWAP_EINVAL;
  DeviceGuard g(device);
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, 64);
  void* b = nullptr;
  if (cudaIpcOpenMemHandle(&b, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
    cudaGetLastError();
    return SWAP_ECUDA;
  }
  *base = b;
  *mapped = static_cast<uint8_t*>(b) + offset;
  return SWAP_OK;
}

swap_status swap_ipc_close(int device, void* base) {
  if (!base) return SWAP_EINVAL;
  DeviceGuard g(device);
  return cudaIpcCloseMemHandle(base) == cudaSuccess ? SWAP_OK : SWAP_ECUDA;
}

}  // extern "C"
