// FAKE backend: each "stream" is a CPU thread that completes the ops launched on it in FIFO order
// after their profiled duration (scaled), then publishes done = seq + 1. No GPU, no CUDA calls.
#include <time.h>

#include <atomic>
#include <condition_variable>
#include <deque>
#include <mutex>
#include <thread>

#include "backend.h"

namespace orion {

struct StreamHandle {
  std::mutex mu;
  std::condition_variable cv;
  std::deque<std::pair<uint64_t, uint64_t>> q;  // (seq, duration ns)
  alignas(64) std::atomic<uint64_t> done{0};
  bool quit = false;
  std::thread th;
};

static int64_t mono_ns() {
  timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return (int64_t)ts.tv_sec * 1000000000ll + ts.tv_nsec;
}

struct FakeBackend : Backend {
  uint32_t scale_pct;
  explicit FakeBackend(const orion_config& c) : scale_pct(c.fake_time_scale_pct ? c.fake_time_scale_pct : 100) {}
  uint32_t num_sms() override { return 148; }
  int create_stream(int, StreamHandle** out) override {
    StreamHandle* s = new StreamHandle();
    s->th = std::thread([s]() {
      for (;;) {
        std::pair<uint64_t, uint64_t> job;
        {
          std::unique_lock<std::mutex> lk(s->mu);
          s->cv.wait(lk, [s] { return s->quit || !s->q.empty(); });
          if (s->q.empty()) return;
          job = s->q.front();
          s->q.pop_front();
        }
        const int64_t until = mono_ns() + (int64_t)job.second;
        while (mono_ns() < until) std::this_thread::yield();
        s->done.store(job.first + 1, std::memory_order_release);
      }
    });
    *out = s;
    return 0;
  }
  void destroy_stream(StreamHandle* s) override {
    {
      std::lock_guard<std::mutex> lk(s->mu);
      s->quit = true;
    }
    s->cv.notify_all();
    if (s->th.joinable()) s->th.join();
    delete s;
  }
  void* native_stream(StreamHandle*) override { return nullptr; }
  int launch(StreamHandle* s, const orion_op& op, uint64_t seq) override {
    uint64_t d = op.kind == ORION_OP_KERNEL ? op.prof.dur_ns * scale_pct / 100 : 0;
    {
      std::lock_guard<std::mutex> lk(s->mu);
      s->q.emplace_back(seq, d);
    }
    s->cv.notify_one();
    return 0;
  }
  uint64_t read_done(StreamHandle* s) override { return s->done.load(std::memory_order_acquire); }
};

std::unique_ptr<Backend> make_fake_backend(const orion_config& cfg) { return std::unique_ptr<Backend>(new FakeBackend(cfg)); }

int make_backend(const orion_config& cfg, int device, std::unique_ptr<Backend>* out) {
  if (cfg.backend == ORION_BACKEND_FAKE) {
    *out = make_fake_backend(cfg);
    return 0;
  }
  if (cfg.backend == ORION_BACKEND_CUDA) return make_cuda_backend(cfg, device, out);
  return ORION_E_INVAL;
}

}  // namespace orion
