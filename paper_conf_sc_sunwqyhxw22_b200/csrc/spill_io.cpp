// NEXT-2 secondary-storage tier I/O ("asynchronous bulk read/write requests" between
// the secondary storage and the CPU memory): O_DIRECT transfers between a layer's spill file and
// page-locked host buffers, issued through io_uring (raw syscalls; no liburing in this image) with
// several large requests in flight, falling back to synchronous pread/pwrite when io_uring is not
// permitted.  No page cache is involved: the RAM the tier uses is the pinned staging it is given.
//
// Each calling thread owns its own ring (thread_local): the H2D issuer reads fetches, the spill I/O
// thread reads a layer's optimizer state before its CPU update and writes it back afterwards.
#include <fcntl.h>
#include <linux/io_uring.h>
#include <sys/mman.h>
#include <sys/syscall.h>
#include <unistd.h>

#include <atomic>
#include <cerrno>
#include <cstdint>
#include <cstring>

#include "sh_internal.hpp"

namespace sh {
namespace spill {

namespace {

constexpr unsigned kDepth = 16;            // requests in flight
constexpr size_t kChunk = 8u << 20;        // bytes per request

int sys_setup(unsigned entries, io_uring_params* p) { return (int)syscall(__NR_io_uring_setup, entries, p); }
int sys_enter(int fd, unsigned to_submit, unsigned min_complete, unsigned flags) {
  return (int)syscall(__NR_io_uring_enter, fd, to_submit, min_complete, flags, nullptr, 0);
}

class Ring {
 public:
  ~Ring() { close_ring(); }

  bool ok() {
    if (state_ == 0) state_ = open_ring() ? 1 : -1;
    return state_ == 1;
  }

  // Blocking transfer of [buf, buf + bytes) at file offset off, in kChunk requests, kDepth in flight.
  // Returns 0 or -errno.
  int rw(bool write, int fd, char* buf, size_t bytes, off_t off) {
    size_t next = 0, done = 0;
    unsigned inflight = 0;
    int err = 0;
    while (done < bytes) {
      unsigned queued = 0;
      while (inflight + queued < kDepth && next < bytes && !err) {
        const unsigned tail = *sq_tail_;
        const unsigned idx = tail & *sq_mask_;
        io_uring_sqe* e = &sqes_[idx];
        std::memset(e, 0, sizeof(*e));
        const size_t n = bytes - next < kChunk ? bytes - next : kChunk;
        e->opcode = write ? IORING_OP_WRITE : IORING_OP_READ;
        e->fd = fd;
        e->addr = reinterpret_cast<uint64_t>(buf + next);
        e->len = (unsigned)n;
        e->off = (uint64_t)(off + (off_t)next);
        e->user_data = n;
        sq_array_[idx] = idx;
        std::atomic_thread_fence(std::memory_order_release);
        *sq_tail_ = tail + 1;
        next += n;
        ++queued;
      }
      const int r = sys_enter(fd_, queued, 1, IORING_ENTER_GETEVENTS);
      if (r < 0 && errno != EINTR) return -errno;
      inflight += queued;
      // reap
      unsigned head = *cq_head_;
      std::atomic_thread_fence(std::memory_order_acquire);
      while (head != *cq_tail_) {
        const io_uring_cqe& q = cqes_[head & *cq_mask_];
        if (q.res < 0) err = q.res;
        else if ((size_t)q.res != (size_t)q.user_data) err = -EIO;  // short transfer (O_DIRECT: end of file)
        done += (size_t)q.user_data;
        --inflight;
        ++head;
      }
      std::atomic_thread_fence(std::memory_order_release);
      *cq_head_ = head;
      if (err && inflight == 0) return err;
    }
    return err;
  }

 private:
  bool open_ring() {
    io_uring_params p;
    std::memset(&p, 0, sizeof(p));
    fd_ = sys_setup(kDepth, &p);
    if (fd_ < 0) return false;
    sq_sz_ = p.sq_off.array + p.sq_entries * sizeof(unsigned);
    cq_sz_ = p.cq_off.cqes + p.cq_entries * sizeof(io_uring_cqe);
    sq_ptr_ = mmap(nullptr, sq_sz_, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_POPULATE, fd_, IORING_OFF_SQ_RING);
    cq_ptr_ = mmap(nullptr, cq_sz_, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_POPULATE, fd_, IORING_OFF_CQ_RING);
    sqes_sz_ = p.sq_entries * sizeof(io_uring_sqe);
    sqes_ = static_cast<io_uring_sqe*>(
        mmap(nullptr, sqes_sz_, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_POPULATE, fd_, IORING_OFF_SQES));
    if (sq_ptr_ == MAP_FAILED || cq_ptr_ == MAP_FAILED || sqes_ == MAP_FAILED) {
      close_ring();
      return false;
    }
    char* sq = static_cast<char*>(sq_ptr_);
    char* cq = static_cast<char*>(cq_ptr_);
    sq_tail_ = reinterpret_cast<unsigned*>(sq + p.sq_off.tail);
    sq_mask_ = reinterpret_cast<unsigned*>(sq + p.sq_off.ring_mask);
    sq_array_ = reinterpret_cast<unsigned*>(sq + p.sq_off.array);
    cq_head_ = reinterpret_cast<unsigned*>(cq + p.cq_off.head);
    cq_tail_ = reinterpret_cast<unsigned*>(cq + p.cq_off.tail);
    cq_mask_ = reinterpret_cast<unsigned*>(cq + p.cq_off.ring_mask);
    cqes_ = reinterpret_cast<io_uring_cqe*>(cq + p.cq_off.cqes);
    return true;
  }
  void close_ring() {
    if (sqes_ && sqes_ != MAP_FAILED) munmap(sqes_, sqes_sz_);
    if (sq_ptr_ && sq_ptr_ != MAP_FAILED) munmap(sq_ptr_, sq_sz_);
    if (cq_ptr_ && cq_ptr_ != MAP_FAILED) munmap(cq_ptr_, cq_sz_);
    if (fd_ >= 0) close(fd_);
    sqes_ = nullptr;
    sq_ptr_ = cq_ptr_ = nullptr;
    fd_ = -1;
  }
  int state_ = 0;
  int fd_ = -1;
  void *sq_ptr_ = nullptr, *cq_ptr_ = nullptr;
  size_t sq_sz_ = 0, cq_sz_ = 0, sqes_sz_ = 0;
  io_uring_sqe* sqes_ = nullptr;
  io_uring_cqe* cqes_ = nullptr;
  unsigned *sq_tail_ = nullptr, *sq_mask_ = nullptr, *sq_array_ = nullptr;
  unsigned *cq_head_ = nullptr, *cq_tail_ = nullptr, *cq_mask_ = nullptr;
};

thread_local Ring t_ring;
std::atomic<int> g_force_sync{-1};

bool force_sync() {
  int v = g_force_sync.load();
  if (v < 0) {
    const char* e = getenv("SH_SPILL_SYNC_IO");  // test / fallback: pread/pwrite instead of io_uring
    v = (e && e[0] == '1') ? 1 : 0;
    g_force_sync.store(v);
  }
  return v == 1;
}

int sync_rw(bool write, int fd, char* buf, size_t bytes, off_t off) {
  size_t done = 0;
  while (done < bytes) {
    const size_t n = bytes - done < kChunk ? bytes - done : kChunk;
    const ssize_t r = write ? pwrite(fd, buf + done, n, off + (off_t)done) : pread(fd, buf + done, n, off + (off_t)done);
    if (r < 0) {
      if (errno == EINTR) continue;
      return -errno;
    }
    if (r == 0) return -EIO;
    done += (size_t)r;
  }
  return 0;
}

}  // namespace

bool uring_available() { return !force_sync() && t_ring.ok(); }

int transfer(bool write, int fd, void* buf, size_t bytes, int64_t off) {
  if (bytes == 0) return 0;
  if (((uintptr_t)buf & (kAlign - 1)) || (bytes & (kAlign - 1)) || (off & (int64_t)(kAlign - 1))) return -EINVAL;
  char* b = static_cast<char*>(buf);
  if (!force_sync() && t_ring.ok()) return t_ring.rw(write, fd, b, bytes, (off_t)off);
  return sync_rw(write, fd, b, bytes, (off_t)off);
}

}  // namespace spill
}  // namespace sh
