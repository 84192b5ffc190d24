// ratel_uring.h -- a minimal io_uring (raw syscalls, no liburing) for the SSD
// tier's reader and writer threads: many file reads or writes in flight at
// once (queue depth > 1) instead of one blocking pread/pwrite at a time.
//
// One ring per thread.  transfer() splits every (buffer, bytes, offset)
// request into chunks of at most kChunk bytes, keeps up to `depth` of them
// submitted, reaps completions and resubmits the remainder of short
// transfers; it returns once every byte moved or on the first error.
// O_DIRECT rules (4 KiB-aligned buffer, length and offset) are the caller's,
// exactly as for pread/pwrite.
#pragma once

#include <linux/io_uring.h>
#include <sys/mman.h>
#include <sys/syscall.h>
#include <unistd.h>

#include <cerrno>
#include <cstdint>
#include <cstring>
#include <string>
#include <vector>

namespace ratel {

class IoRing {
 public:
  static constexpr uint64_t kChunk = 4ull << 20;  // bytes per request

  ~IoRing() { close_ring(); }

  // 0 on success, else -errno (the kernel may refuse io_uring).
  int open_ring(unsigned depth) {
    io_uring_params p{};
    const int fd = static_cast<int>(syscall(__NR_io_uring_setup, depth, &p));
    if (fd < 0) return -errno;
    fd_ = fd;
    depth_ = p.sq_entries;
    sq_bytes_ = p.sq_off.array + p.sq_entries * sizeof(uint32_t);
    cq_bytes_ = p.cq_off.cqes + p.cq_entries * sizeof(io_uring_cqe);
    single_ = (p.features & IORING_FEAT_SINGLE_MMAP) != 0;
    if (single_) sq_bytes_ = cq_bytes_ = (sq_bytes_ > cq_bytes_ ? sq_bytes_ : cq_bytes_);
    sq_ = mmap(nullptr, sq_bytes_, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_POPULATE, fd_, IORING_OFF_SQ_RING);
    if (sq_ == MAP_FAILED) return fail();
    cq_ = single_ ? sq_ : mmap(nullptr, cq_bytes_, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_POPULATE, fd_,
                               IORING_OFF_CQ_RING);
    if (cq_ == MAP_FAILED) return fail();
    sqes_bytes_ = p.sq_entries * sizeof(io_uring_sqe);
    sqes_ = static_cast<io_uring_sqe*>(
        mmap(nullptr, sqes_bytes_, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_POPULATE, fd_, IORING_OFF_SQES));
    if (sqes_ == MAP_FAILED) return fail();
    char* sq = static_cast<char*>(sq_);
    char* cq = static_cast<char*>(cq_);
    sq_head_ = reinterpret_cast<unsigned*>(sq + p.sq_off.head);
    sq_tail_ = reinterpret_cast<unsigned*>(sq + p.sq_off.tail);
    sq_mask_ = *reinterpret_cast<unsigned*>(sq + p.sq_off.ring_mask);
    sq_array_ = reinterpret_cast<unsigned*>(sq + p.sq_off.array);
    cq_head_ = reinterpret_cast<unsigned*>(cq + p.cq_off.head);
    cq_tail_ = reinterpret_cast<unsigned*>(cq + p.cq_off.tail);
    cq_mask_ = *reinterpret_cast<unsigned*>(cq + p.cq_off.ring_mask);
    cqes_ = reinterpret_cast<io_uring_cqe*>(cq + p.cq_off.cqes);
    return 0;
  }

  bool is_open() const { return fd_ >= 0; }
  unsigned depth() const { return depth_; }

  struct Req {
    void* buf;
    uint64_t bytes, off;
  };

  // Reads (rd = true) or writes every request in full.  RATEL-style status:
  // 0 on success, else -errno or -EIO for an unexpected end of file; `msg`
  // describes the failure.
  int transfer(bool rd, int fd, const std::vector<Req>& reqs, std::string& msg) {
    struct Piece {
      char* buf;
      uint64_t left, off;
    };
    std::vector<Piece> todo;
    for (const Req& r : reqs)
      for (uint64_t o = 0; o < r.bytes; o += kChunk)
        todo.push_back({static_cast<char*>(r.buf) + o, r.bytes - o < kChunk ? r.bytes - o : kChunk, r.off + o});
    std::vector<Piece> inflight(depth_);
    std::vector<unsigned> free_slots;
    for (unsigned i = 0; i < depth_; ++i) free_slots.push_back(depth_ - 1 - i);
    size_t next = 0;
    unsigned busy = 0;
    int err = 0;
    while ((next < todo.size() && err == 0) || busy > 0) {
      unsigned queued = 0;
      while (err == 0 && next < todo.size() && !free_slots.empty()) {  // fill the submission queue
        const unsigned slot = free_slots.back();
        free_slots.pop_back();
        inflight[slot] = todo[next++];
        push(rd, fd, inflight[slot], slot);
        ++queued;
      }
      busy += queued;
      const int r = static_cast<int>(
          syscall(__NR_io_uring_enter, fd_, queued, busy > 0 ? 1u : 0u, IORING_ENTER_GETEVENTS, nullptr, 0));
      if (r < 0 && errno != EINTR) {
        msg = std::string("io_uring_enter: ") + strerror(errno);
        return -errno;
      }
      unsigned head = *cq_head_;
      const unsigned tail = __atomic_load_n(cq_tail_, __ATOMIC_ACQUIRE);
      for (; head != tail; ++head) {
        const io_uring_cqe& c = cqes_[head & cq_mask_];
        const unsigned slot = static_cast<unsigned>(c.user_data);
        Piece& pc = inflight[slot];
        --busy;
        if (c.res < 0 || (c.res == 0 && pc.left > 0)) {
          if (err == 0) {
            err = c.res < 0 ? c.res : -EIO;
            msg = std::string(rd ? "io_uring read" : "io_uring write") + " of the SSD state file failed at offset " +
                  std::to_string(pc.off) + ": " + (c.res < 0 ? strerror(-c.res) : "unexpected end of file");
          }
          free_slots.push_back(slot);
          continue;
        }
        pc.buf += c.res;
        pc.left -= static_cast<uint64_t>(c.res);
        pc.off += static_cast<uint64_t>(c.res);
        if (pc.left > 0 && err == 0) {  // short transfer: the rest goes right back in
          push(rd, fd, pc, slot);
          ++busy;
          syscall(__NR_io_uring_enter, fd_, 1u, 0u, 0u, nullptr, 0);
        } else {
          free_slots.push_back(slot);
        }
      }
      __atomic_store_n(cq_head_, head, __ATOMIC_RELEASE);
    }
    return err;
  }

 private:
  template <class Piece>
  void push(bool rd, int fd, const Piece& pc, unsigned slot) {
    const unsigned tail = *sq_tail_;
    const unsigned idx = tail & sq_mask_;
    io_uring_sqe& e = sqes_[idx];
    memset(&e, 0, sizeof e);
    e.opcode = rd ? IORING_OP_READ : IORING_OP_WRITE;
    e.fd = fd;
    e.addr = reinterpret_cast<uint64_t>(pc.buf);
    e.len = static_cast<uint32_t>(pc.left);
    e.off = pc.off;
    e.user_data = slot;
    sq_array_[idx] = idx;
    __atomic_store_n(sq_tail_, tail + 1, __ATOMIC_RELEASE);
  }

  int fail() {
    const int e = -errno;
    close_ring();
    return e;
  }

  void close_ring() {
    if (sqes_ != nullptr && sqes_ != MAP_FAILED) munmap(sqes_, sqes_bytes_);
    if (cq_ != nullptr && cq_ != MAP_FAILED && !single_) munmap(cq_, cq_bytes_);
    if (sq_ != nullptr && sq_ != MAP_FAILED) munmap(sq_, sq_bytes_);
    if (fd_ >= 0) ::close(fd_);
    sqes_ = nullptr;
    sq_ = cq_ = nullptr;
    fd_ = -1;
  }

  int fd_ = -1;
  unsigned depth_ = 0;
  bool single_ = false;
  size_t sq_bytes_ = 0, cq_bytes_ = 0, sqes_bytes_ = 0;
  void *sq_ = nullptr, *cq_ = nullptr;
  io_uring_sqe* sqes_ = nullptr;
  unsigned *sq_head_ = nullptr, *sq_tail_ = nullptr, *sq_array_ = nullptr, *cq_head_ = nullptr, *cq_tail_ = nullptr;
  unsigned sq_mask_ = 0, cq_mask_ = 0;
  io_uring_cqe* cqes_ = nullptr;
};

}  // namespace ratel
