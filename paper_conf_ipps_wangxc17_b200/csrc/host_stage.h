// host_stage.h -- host <-> device copies of the host-buffer call (phmm_compute_batch) through
// context-owned pinned staging buffers ("stage into pinned memory, then
// H2D"; the paper's end-to-end times include these transfers, PAPER.md L24@1130, §V-B).
//
// A caller's buffer that is already page-locked (cudaMallocHost / cudaHostRegister) is copied
// by one cudaMemcpyAsync. A pageable buffer is cut into pieces of kStagePiece bytes that cycle
// through a ring of kStageSlots pinned slots: host threads memcpy piece k into its slot while
// the DMA engine moves piece k-1 to the device (one cudaMemcpyAsync per piece, an event per
// slot tells when the slot may be refilled). Results travel back the same way in reverse.
// Host part of libphmm only (no kernels).
#pragma once
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <condition_variable>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <mutex>
#include <thread>
#include <vector>

#include <emmintrin.h>  // SSE2 streaming stores (x86-64 baseline)

namespace phmm {

// memcpy into a page-locked staging slot with non-temporal (streaming) stores, so that the
// slot's lines are not left in CPU caches: the GPU's DMA read of lines a CPU core holds runs at
// 5-20 GB/s instead of ~50 on the GPU hosts (tools/h2d_probe4.py). dst must be 16-byte aligned.
inline void memcpy_stream(char* dst, const char* src, size_t n) {
  size_t i = 0;
  for (; i + 64 <= n; i += 64) {
    const __m128i a = _mm_loadu_si128(reinterpret_cast<const __m128i*>(src + i));
    const __m128i b = _mm_loadu_si128(reinterpret_cast<const __m128i*>(src + i + 16));
    const __m128i c = _mm_loadu_si128(reinterpret_cast<const __m128i*>(src + i + 32));
    const __m128i d = _mm_loadu_si128(reinterpret_cast<const __m128i*>(src + i + 48));
    _mm_stream_si128(reinterpret_cast<__m128i*>(dst + i), a);
    _mm_stream_si128(reinterpret_cast<__m128i*>(dst + i + 16), b);
    _mm_stream_si128(reinterpret_cast<__m128i*>(dst + i + 32), c);
    _mm_stream_si128(reinterpret_cast<__m128i*>(dst + i + 48), d);
  }
  if (i < n) std::memcpy(dst + i, src + i, n - i);
  _mm_sfence();
}

// A fixed pool of host threads for parallel memcpy (one job at a time, split evenly).
class CopyPool {
 public:
  explicit CopyPool(int n) {
    for (int i = 0; i < n; ++i) th_.emplace_back([this, i] { run(i); });
  }
  ~CopyPool() {
    {
      std::lock_guard<std::mutex> g(m_);
      stop_ = true;
    }
    cv_.notify_all();
    for (auto& t : th_) t.join();
  }
  int size() const { return (int)th_.size() + 1; }
  bool stream_stores = true;  // PHMM_STAGE_NT=0: plain memcpy into the staging slots
  // dst[0..n) = src[0..n), split over the pool's threads and the caller's (64-byte aligned parts)
  void memcpy_par(void* dst, const void* src, size_t n) {
    const int parts = size();
    if (n < (size_t)1 << 20 || parts == 1) {
      cpy(static_cast<char*>(dst), static_cast<const char*>(src), n);
      return;
    }
    {
      std::lock_guard<std::mutex> g(m_);
      fn_ = nullptr;
      dst_ = static_cast<char*>(dst);
      src_ = static_cast<const char*>(src);
      n_ = n;
      pending_ = (int)th_.size();
      ++gen_;
    }
    cv_.notify_all();
    part(0, parts);
    std::unique_lock<std::mutex> lk(m_);
    done_cv_.wait(lk, [this] { return pending_ == 0; });
  }
  // fn(j) for j in [0, njobs), job j on participant j % size() (the caller is participant 0)
  void for_each(int njobs, const std::function<void(int)>& fn) {
    if (th_.empty() || njobs <= 1) {
      for (int j = 0; j < njobs; ++j) fn(j);
      return;
    }
    {
      std::lock_guard<std::mutex> g(m_);
      fn_ = &fn;
      njobs_ = njobs;
      pending_ = (int)th_.size();
      ++gen_;
    }
    cv_.notify_all();
    part(0, size());
    std::unique_lock<std::mutex> lk(m_);
    done_cv_.wait(lk, [this] { return pending_ == 0; });
  }

 private:
  void part(int k, int parts) {
    if (fn_) {
      for (int j = k; j < njobs_; j += parts) (*fn_)(j);
      return;
    }
    const size_t per = ((n_ + parts - 1) / parts + 63) & ~(size_t)63;
    const size_t a = std::min(n_, per * (size_t)k), z = std::min(n_, a + per);
    if (z > a) cpy(dst_ + a, src_ + a, z - a);
  }
  void cpy(char* d, const char* s, size_t n) const {
    if (stream_stores && ((uintptr_t)d & 15) == 0) memcpy_stream(d, s, n);
    else std::memcpy(d, s, n);
  }
  void run(int i) {
    uint64_t seen = 0;
    while (true) {
      {
        std::unique_lock<std::mutex> lk(m_);
        cv_.wait(lk, [&] { return stop_ || gen_ != seen; });
        if (stop_) return;
        seen = gen_;
      }
      part(i + 1, size());
      {
        std::lock_guard<std::mutex> g(m_);
        if (--pending_ == 0) done_cv_.notify_one();
      }
    }
  }
  std::vector<std::thread> th_;
  std::mutex m_;
  std::condition_variable cv_, done_cv_;
  bool stop_ = false;
  uint64_t gen_ = 0;
  int pending_ = 0;
  char* dst_ = nullptr;
  const char* src_ = nullptr;
  size_t n_ = 0;
  const std::function<void(int)>* fn_ = nullptr;  // for_each job, else a memcpy_par job
  int njobs_ = 0;
};

constexpr int kStageSlots = 4;
constexpr size_t kStagePiece = (size_t)8 << 20;

struct Stager {
  void* slot[kStageSlots] = {};
  cudaEvent_t ev[kStageSlots] = {};
  bool used[kStageSlots] = {};
  int next = 0;
  CopyPool* pool = nullptr;
  int64_t staged_bytes = 0;  // bytes of the last call that went through the slots

  cudaError_t init(int threads) {
    for (int i = 0; i < kStageSlots; ++i) {
      cudaError_t e = cudaMallocHost(&slot[i], kStagePiece);
      if (e != cudaSuccess) {
        slot[i] = nullptr;
        return e;
      }
      e = cudaEventCreateWithFlags(&ev[i], cudaEventDisableTiming);
      if (e != cudaSuccess) {
        ev[i] = nullptr;
        return e;
      }
    }
    pool = new CopyPool(std::max(0, threads - 1));
    if (const char* e = std::getenv("PHMM_STAGE_NT")) pool->stream_stores = std::atoi(e) != 0;
    return cudaSuccess;
  }
  void release() {
    for (int i = 0; i < kStageSlots; ++i) {
      if (ev[i]) cudaEventSynchronize(ev[i]);
      if (slot[i]) cudaFreeHost(slot[i]);
      if (ev[i]) cudaEventDestroy(ev[i]);
      slot[i] = nullptr;
      ev[i] = nullptr;
    }
    delete pool;
    pool = nullptr;
  }

  static bool is_pinned(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
      cudaGetLastError();
      return false;
    }
    return a.type == cudaMemoryTypeHost;
  }

  // the next free slot (waits for its previous DMA)
  cudaError_t take(int* k) {
    *k = next;
    next = (next + 1) % kStageSlots;
    if (used[*k]) {
      cudaError_t e = cudaEventSynchronize(ev[*k]);
      if (e != cudaSuccess) return e;
    }
    used[*k] = true;
    return cudaSuccess;
  }

  // host -> device on stream s
  cudaError_t h2d(void* dst, const void* src, size_t n, cudaStream_t s) {
    if (n == 0) return cudaSuccess;
    if (is_pinned(src)) return cudaMemcpyAsync(dst, src, n, cudaMemcpyHostToDevice, s);
    for (size_t off = 0; off < n; off += kStagePiece) {
      const size_t b = std::min(kStagePiece, n - off);
      int k;
      cudaError_t e = take(&k);
      if (e != cudaSuccess) return e;
      pool->memcpy_par(slot[k], static_cast<const char*>(src) + off, b);
      e = cudaMemcpyAsync(static_cast<char*>(dst) + off, slot[k], b, cudaMemcpyHostToDevice, s);
      if (e != cudaSuccess) return e;
      e = cudaEventRecord(ev[k], s);
      if (e != cudaSuccess) return e;
      staged_bytes += (int64_t)b;
    }
    return cudaSuccess;
  }

  // device -> host on stream s; returns when dst holds the data (a page-locked dst with
  // sync = false: when the copy is queued; the caller synchronises s)
  cudaError_t d2h(void* dst, const void* src, size_t n, cudaStream_t s, bool sync = true) {
    if (n == 0) return cudaSuccess;
    if (is_pinned(dst)) {
      cudaError_t e = cudaMemcpyAsync(dst, src, n, cudaMemcpyDeviceToHost, s);
      return e != cudaSuccess || !sync ? e : cudaStreamSynchronize(s);
    }
    // keep up to kStageSlots pieces in flight; copy each out as soon as it arrived
    const size_t npieces = (n + kStagePiece - 1) / kStagePiece;
    int slot_of[kStageSlots];
    size_t issued = 0, drained = 0;
    while (drained < npieces) {
      while (issued < npieces && issued - drained < (size_t)kStageSlots) {
        const size_t off = issued * kStagePiece, b = std::min(kStagePiece, n - off);
        int k;
        cudaError_t e = take(&k);
        if (e != cudaSuccess) return e;
        e = cudaMemcpyAsync(slot[k], static_cast<const char*>(src) + off, b, cudaMemcpyDeviceToHost, s);
        if (e != cudaSuccess) return e;
        e = cudaEventRecord(ev[k], s);
        if (e != cudaSuccess) return e;
        slot_of[issued % kStageSlots] = k;
        ++issued;
      }
      const int k = slot_of[drained % kStageSlots];
      cudaError_t e = cudaEventSynchronize(ev[k]);
      if (e != cudaSuccess) return e;
      const size_t off = drained * kStagePiece, b = std::min(kStagePiece, n - off);
      pool->memcpy_par(static_cast<char*>(dst) + off, slot[k], b);
      staged_bytes += (int64_t)b;
      ++drained;
    }
    return cudaSuccess;
  }
};

// The host->device side of the pipelined host-buffer call (phmm_lib.cu): a
// context-owned thread that runs one call's copy jobs in order on a copy stream (through the
// Stager, so pageable buffers are staged while earlier pieces are in flight) and records an
// event after each group of jobs. The compute thread waits (on the host) until group k's event
// is recorded and then makes its stream wait on it, so chunk k computes while the copy engine
// moves chunk k+1. One call at a time; the caller finishes every call with wait_all().
struct CopyJob {
  void* dst;
  const void* src;
  size_t n;
};

class Feeder {
 public:
  Feeder() = default;
  Feeder(const Feeder&) = delete;
  ~Feeder() { stop(); }

  cudaError_t init(int device) {
    device_ = device;
    cudaError_t e = cudaStreamCreateWithFlags(&stream_, cudaStreamNonBlocking);
    if (e != cudaSuccess) {
      stream_ = nullptr;
      return e;
    }
    th_ = std::thread([this] { run(); });
    return cudaSuccess;
  }
  cudaStream_t stream() const { return stream_; }
  bool trace = false;
  std::vector<double> job_us;  // trace: host time of each job's issue

  // Start a call: job groups[k] = jobs [group_end[k-1], group_end[k]), event ev[k] recorded
  // on the copy stream after group k. The stager belongs to this thread until wait_all().
  void start(Stager* st, const std::vector<CopyJob>* jobs, const std::vector<size_t>* group_end,
             const std::vector<cudaEvent_t>* ev) {
    std::lock_guard<std::mutex> g(m_);
    st_ = st;
    jobs_ = jobs;
    group_end_ = group_end;
    ev_ = ev;
    recorded_ = 0;
    err_ = cudaSuccess;
    cancel_ = false;
    busy_ = true;
    ++gen_;
    cv_.notify_all();
  }
  // Block until group k's event is recorded (or the feeder failed / was cancelled).
  cudaError_t wait_group(int k) {
    std::unique_lock<std::mutex> lk(m_);
    done_cv_.wait(lk, [&] { return recorded_ > k || err_ != cudaSuccess || !busy_; });
    if (err_ != cudaSuccess) return err_;
    return recorded_ > k ? cudaSuccess : cudaErrorUnknown;
  }
  // Stop issuing further jobs (an error elsewhere in the call).
  void cancel() {
    std::lock_guard<std::mutex> g(m_);
    cancel_ = true;
  }
  // Wait until the thread has issued (or dropped) every job of the call and the copy stream
  // has drained: no copy reads the caller's buffers after this returns.
  cudaError_t wait_all() {
    std::unique_lock<std::mutex> lk(m_);
    done_cv_.wait(lk, [&] { return !busy_; });
    const cudaError_t e = err_;
    lk.unlock();
    const cudaError_t s = stream_ ? cudaStreamSynchronize(stream_) : cudaSuccess;
    return e != cudaSuccess ? e : s;
  }
  void stop() {
    if (th_.joinable()) {
      {
        std::lock_guard<std::mutex> g(m_);
        quit_ = true;
      }
      cv_.notify_all();
      th_.join();
    }
    if (stream_) {
      cudaStreamSynchronize(stream_);
      cudaStreamDestroy(stream_);
      stream_ = nullptr;
    }
  }

 private:
  void run() {
    uint64_t seen = 0;
    bool dev_set = false;
    while (true) {
      {
        std::unique_lock<std::mutex> lk(m_);
        cv_.wait(lk, [&] { return quit_ || gen_ != seen; });
        if (quit_) return;
        seen = gen_;
      }
      if (!dev_set) {
        cudaSetDevice(device_);
        dev_set = true;
      }
      cudaError_t e = cudaSuccess;
      size_t j = 0;
      for (size_t k = 0; k < group_end_->size() && e == cudaSuccess; ++k) {
        for (; j < (*group_end_)[k] && e == cudaSuccess; ++j) {
          {
            std::lock_guard<std::mutex> g(m_);
            if (cancel_) break;
          }
          const CopyJob& c = (*jobs_)[j];
          const auto t0 = std::chrono::steady_clock::now();
          e = st_->h2d(c.dst, c.src, c.n, stream_);
          if (trace) job_us.push_back(std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0).count());
        }
        {
          std::lock_guard<std::mutex> g(m_);
          if (cancel_) break;
        }
        if (e == cudaSuccess) e = cudaEventRecord((*ev_)[k], stream_);
        if (e == cudaSuccess) {
          std::lock_guard<std::mutex> g(m_);
          recorded_ = (int)k + 1;
          done_cv_.notify_all();
        }
      }
      if (e != cudaSuccess) cudaGetLastError();
      std::lock_guard<std::mutex> g(m_);
      err_ = e;
      busy_ = false;
      done_cv_.notify_all();
    }
  }

  int device_ = 0;
  cudaStream_t stream_ = nullptr;
  std::thread th_;
  std::mutex m_;
  std::condition_variable cv_, done_cv_;
  uint64_t gen_ = 0;
  bool quit_ = false, cancel_ = false, busy_ = false;
  int recorded_ = 0;
  cudaError_t err_ = cudaSuccess;
  Stager* st_ = nullptr;
  const std::vector<CopyJob>* jobs_ = nullptr;
  const std::vector<size_t>* group_end_ = nullptr;
  const std::vector<cudaEvent_t>* ev_ = nullptr;
};

}  // namespace phmm
