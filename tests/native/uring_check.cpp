// CPU check of the SSD tier's io_uring helper (csrc/ratel_uring.h): O_DIRECT
// write of a pattern through the ring, read back through the ring at queue
// depth > 1 and with more requests than the depth, compare; then a read past
// the end of the file must report an error.  Exit 0 = all good.
#include <fcntl.h>
#include <stdlib.h>
#include <unistd.h>

#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "ratel_uring.h"

int main(int argc, char** argv) {
  if (argc < 2) return 2;
  const char* path = argv[1];
  const uint64_t n = 3 * ratel::IoRing::kChunk + 8192;  // several chunks + a ragged tail
  void *a = nullptr, *b = nullptr;
  if (posix_memalign(&a, 4096, 3 * n) || posix_memalign(&b, 4096, 3 * n)) return 3;
  for (uint64_t i = 0; i < 3 * n; ++i) static_cast<unsigned char*>(a)[i] = static_cast<unsigned char>(i * 131 + 7);
  memset(b, 0, 3 * n);
  int fd = open(path, O_RDWR | O_CREAT | O_TRUNC | O_DIRECT, 0600);
  if (fd < 0) fd = open(path, O_RDWR | O_CREAT | O_TRUNC, 0600);  // tmpfs has no O_DIRECT
  if (fd < 0) return 4;
  ratel::IoRing ring;
  if (int e = ring.open_ring(4); e != 0) {
    printf("io_uring unavailable: %s\n", strerror(-e));
    return 77;
  }
  std::string msg;
  std::vector<ratel::IoRing::Req> w, r;
  for (int k = 0; k < 3; ++k) {  // three arrays at offsets 0, n, 2n (like theta, m, v)
    w.push_back({static_cast<char*>(a) + k * n, n, k * n});
    r.push_back({static_cast<char*>(b) + k * n, n, k * n});
  }
  if (ring.transfer(false, fd, w, msg) != 0) { printf("write: %s\n", msg.c_str()); return 5; }
  fsync(fd);
  if (ring.transfer(true, fd, r, msg) != 0) { printf("read: %s\n", msg.c_str()); return 6; }
  if (memcmp(a, b, 3 * n) != 0) { printf("mismatch\n"); return 7; }
  std::vector<ratel::IoRing::Req> past{{b, 8192, 3 * n + 4096}};  // beyond the end: EOF -> error
  if (ring.transfer(true, fd, past, msg) == 0) { printf("no EOF error\n"); return 8; }
  close(fd);
  printf("ok depth=%u %s\n", ring.depth(), msg.c_str());
  return 0;
}
