// CPU test of the host-side helpers of the pipelined host call (csrc/host_stage.h): the
// streaming-store memcpy at every alignment and length class, CopyPool::memcpy_par (split over
// the pool's threads) and CopyPool::for_each (every job exactly once). Built and run by
// tests/test_host_stage.py with g++ (no GPU; no CUDA call is made).
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "../../paper_conf_ipps_wangxc17_b200/csrc/host_stage.h"

static int fail(const char* what, size_t a, size_t b) {
  std::printf("FAIL %s %zu %zu\n", what, a, b);
  return 1;
}

int main() {
  std::vector<unsigned char> src(1 << 22), dst((1 << 22) + 64);
  for (size_t i = 0; i < src.size(); ++i) src[i] = (unsigned char)(i * 2654435761u >> 13);
  // memcpy_stream: 16-byte aligned destinations, any source alignment, lengths around the
  // 64-byte stride and the scalar tail
  alignas(64) static unsigned char d16[8192 + 64];
  for (size_t so = 0; so < 16; ++so)
    for (size_t n : {0ul, 1ul, 15ul, 16ul, 63ul, 64ul, 65ul, 127ul, 128ul, 1000ul, 4096ul, 8191ul}) {
      std::memset(d16, 0xAB, sizeof d16);
      phmm::memcpy_stream(reinterpret_cast<char*>(d16), reinterpret_cast<const char*>(src.data() + so), n);
      if (std::memcmp(d16, src.data() + so, n) != 0) return fail("memcpy_stream", so, n);
      for (size_t i = n; i < sizeof d16; ++i)
        if (d16[i] != 0xAB) return fail("memcpy_stream overrun", so, n);
    }
  // CopyPool: memcpy_par at sizes below and above the 1 MiB threshold, aligned and not
  for (int threads : {1, 3, 8}) {
    phmm::CopyPool pool(threads - 1);
    for (size_t off : {0ul, 3ul, 16ul})
      for (size_t n : {100ul, (size_t)1 << 20, ((size_t)1 << 22) - 77}) {
        std::memset(dst.data(), 0, dst.size());
        pool.memcpy_par(dst.data() + off, src.data(), n - (n + off > dst.size() ? off : 0));
        const size_t m = n - (n + off > dst.size() ? off : 0);
        if (std::memcmp(dst.data() + off, src.data(), m) != 0) return fail("memcpy_par", off, n);
      }
    for (int njobs : {0, 1, 5, 64, 1000}) {
      std::vector<int> hits((size_t)njobs, 0);
      pool.for_each(njobs, [&](int j) { ++hits[(size_t)j]; });
      for (int j = 0; j < njobs; ++j)
        if (hits[(size_t)j] != 1) return fail("for_each", (size_t)njobs, (size_t)j);
    }
    // memcpy_par and for_each interleaved on one pool
    std::vector<int> hits(37, 0);
    pool.memcpy_par(dst.data(), src.data(), (size_t)3 << 20);
    pool.for_each(37, [&](int j) { ++hits[(size_t)j]; });
    for (int h : hits)
      if (h != 1) return fail("interleaved", 0, 0);
    if (std::memcmp(dst.data(), src.data(), (size_t)3 << 20) != 0) return fail("interleaved copy", 0, 0);
  }
  std::printf("ok\n");
  return 0;
}
