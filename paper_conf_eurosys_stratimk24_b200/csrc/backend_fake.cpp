// FAKE backend: each "stream" is a CPU thread that completes the ops launched on it in FIFO order
// after their profiled duration (scaled), then publishes done = seq + 1. No GPU, no CUDA calls.
// Optional SM-contention model (orion_config.fake_contention, CPU tests of the SM_THRESHOLD
// search): a running kernel occupies min(sm_needed, 148) "SMs"; while the kernels running on all
// streams together ask for more than 148, each progresses at 148 / demand of real time (SMs time-
// shared), so a BE kernel admitted beside the HP slows the HP exactly when the two do not fit.
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
  struct Job { uint64_t seq, dur_ns; uint32_t sm; };
  std::deque<Job> q;
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
  static constexpr int64_t kSms = 148;
  uint32_t scale_pct;
  bool contention;
  std::atomic<int64_t> demand{0};   // SMs asked for by the kernels running now (contention model)
  explicit FakeBackend(const orion_config& c)
      : scale_pct(c.fake_time_scale_pct ? c.fake_time_scale_pct : 100), contention(c.fake_contention != 0) {}
  uint32_t num_sms() override { return (uint32_t)kSms; }
  void run(const StreamHandle::Job& job) {
    if (!contention || job.sm == 0) {
      const int64_t until = mono_ns() + (int64_t)job.dur_ns;
      while (mono_ns() < until) std::this_thread::yield();
      return;
    }
    const int64_t sm = job.sm < kSms ? (int64_t)job.sm : kSms;
    demand.fetch_add(sm);
    double progress = 0.0;
    int64_t t = mono_ns();
    while (progress < (double)job.dur_ns) {
      std::this_thread::yield();
      const int64_t t2 = mono_ns(), d = demand.load();
      progress += (double)(t2 - t) * (d > kSms ? (double)kSms / (double)d : 1.0);
      t = t2;
    }
    demand.fetch_sub(sm);
  }
  int create_stream(int, StreamHandle** out) override {
    StreamHandle* s = new StreamHandle();
    s->th = std::thread([this, s]() {
      for (;;) {
        StreamHandle::Job job;
        {
          std::unique_lock<std::mutex> lk(s->mu);
          s->cv.wait(lk, [s] { return s->quit || !s->q.empty(); });
          if (s->q.empty()) return;
          job = s->q.front();
          s->q.pop_front();
        }
        run(job);
        s->done.store(job.seq + 1, std::memory_order_release);
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
    const bool kern = op.kind == ORION_OP_KERNEL;
    const uint64_t d = kern ? op.prof.dur_ns * scale_pct / 100 : 0;
    {
      std::lock_guard<std::mutex> lk(s->mu);
      s->q.push_back(StreamHandle::Job{seq, d, kern ? op.prof.sm_needed : 0u});
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
