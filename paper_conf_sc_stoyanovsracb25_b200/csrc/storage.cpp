// storage.cpp — storage tier for swap images (NEXT-4; §3.2 keeps the snapshot in host
// memory — a persistent copy lets a snapshot outlive the process and avoids the cold start P:L105
// describes). swap_save writes the pinned image (payload + padding + manifest) to a file; swap_load
// reads it back into the image buffer and runs swap_import's checks (manifest CRC + layout).
//
// I/O: the image buffer is 2-MiB aligned, so the file is written/read with O_DIRECT in large aligned
// slices by several threads (pwrite/pread), bypassing the page cache; the file is then truncated to
// image_bytes. Filesystems that refuse O_DIRECT (tmpfs) get buffered I/O — the same bytes either way.
#include <fcntl.h>
#include <sys/stat.h>
#include <unistd.h>

#include <atomic>
#include <cerrno>
#include <cstring>
#include <string>
#include <thread>
#include <vector>

#include "../../include/swap.h"
#include "ctx.h"

namespace {

constexpr uint64_t kAlign = 4096;
constexpr uint64_t kSlice = 64ull << 20;

// Reads/writes buf[0, bytes) at file offset file_base + [0, bytes) in kSlice pieces from `threads` threads.
bool io_all(int fd, uint8_t* buf, uint64_t bytes, bool write, unsigned threads, uint64_t file_base = 0) {
  std::atomic<uint64_t> next{0};
  std::atomic<bool> ok{true};
  auto worker = [&] {
    for (;;) {
      const uint64_t off = next.fetch_add(kSlice);
      if (off >= bytes || !ok) return;
      uint64_t len = bytes - off < kSlice ? bytes - off : kSlice;
      uint64_t done = 0;
      while (done < len) {
        const off_t fo = (off_t)(file_base + off + done);
        ssize_t r = write ? pwrite(fd, buf + off + done, len - done, fo) : pread(fd, buf + off + done, len - done, fo);
        if (r < 0 && errno == EINTR) continue;
        if (r <= 0) {
          ok = false;
          return;
        }
        done += (uint64_t)r;
      }
    }
  };
  std::vector<std::thread> pool;
  for (unsigned t = 0; t < threads; ++t) pool.emplace_back(worker);
  for (auto& t : pool) t.join();
  return ok;
}

unsigned io_threads() {
  const unsigned n = std::thread::hardware_concurrency();
  return n == 0 ? 4 : (n > 16 ? 16 : n);
}

}  // namespace

extern "C" {

swap_status swap_save(const swap_ctx_t* ctx, const char* path) {
  if (!ctx || !path) return SWAP_EINVAL;
  void* img = nullptr;
  size_t n = 0;
  swap_status st = swap_get_image(ctx, &img, &n);
  if (st != SWAP_OK) return st;
  swap_shard_summary_t sum;
  if (swap_get_summary(ctx, &sum) != SWAP_OK) return SWAP_ESTATE;  // no sealed checkpoint yet
  const uint64_t padded = (n + kAlign - 1) / kAlign * kAlign;   // the image buffer is 2-MiB padded
  int fd = open(path, O_WRONLY | O_CREAT | O_TRUNC | O_DIRECT, 0644);
  bool direct = fd >= 0;
  if (fd < 0) fd = open(path, O_WRONLY | O_CREAT | O_TRUNC, 0644);
  if (fd < 0) return SWAP_EINVAL;
  bool ok = io_all(fd, static_cast<uint8_t*>(img), direct ? padded : n, true, io_threads());
  if (!ok && direct) {  // O_DIRECT accepted at open but refused on write: retry buffered
    close(fd);
    fd = open(path, O_WRONLY | O_CREAT | O_TRUNC, 0644);
    if (fd < 0) return SWAP_EINVAL;
    ok = io_all(fd, static_cast<uint8_t*>(img), n, true, io_threads());
  }
  ok = ok && ftruncate(fd, (off_t)n) == 0 && fsync(fd) == 0;
  close(fd);
  return ok ? SWAP_OK : SWAP_ENOMEM;
}

swap_status swap_load(swap_ctx_t* ctx, const char* path) {
  if (!ctx || !path) return SWAP_EINVAL;
  // the image is overwritten below: refuse before touching it while a checkpoint may still be writing
  // it, and let any restore still reading it finish first
  if (ctx->st == swc::St::CREATED || ctx->st == swc::St::CKPT_PENDING) {
    ctx->err = ctx->st == swc::St::CREATED ? "swap_load before swap_register_regions" : "previous checkpoint not synced";
    return SWAP_ESTATE;
  }
  {
    swc::DeviceGuard g(ctx->cfg.device);
    const cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) return swc::cuda_fail(ctx, e, "swap_load sync");
  }
  void* img = nullptr;
  size_t n = 0;
  swap_status st = swap_get_image(ctx, &img, &n);
  if (st != SWAP_OK) return st;
  struct stat sb;
  if (stat(path, &sb) != 0) return SWAP_EINVAL;
  if ((uint64_t)sb.st_size != n) return SWAP_ECORRUPT;  // not an image of this layout
  int fd = open(path, O_RDONLY | O_DIRECT);
  bool direct = fd >= 0;
  if (fd < 0) fd = open(path, O_RDONLY);
  if (fd < 0) return SWAP_EINVAL;
  // O_DIRECT reads past EOF return short counts; read the aligned prefix directly, the tail buffered
  const uint64_t head = direct ? n / kAlign * kAlign : n;
  bool ok = io_all(fd, static_cast<uint8_t*>(img), head, false, io_threads());
  if (ok && head < n) {
    int fd2 = open(path, O_RDONLY);
    ok = fd2 >= 0 && io_all(fd2, static_cast<uint8_t*>(img) + head, n - head, false, 1, head);
    if (fd2 >= 0) close(fd2);
  }
  if (!ok && direct) {
    close(fd);
    fd = open(path, O_RDONLY);
    ok = fd >= 0 && io_all(fd, static_cast<uint8_t*>(img), n, false, io_threads());
  }
  if (fd >= 0) close(fd);
  if (!ok) return SWAP_EINVAL;
  return swap_import(ctx);
}

}  // extern "C"
