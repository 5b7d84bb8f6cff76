// Device backends of liborion: CUDA (B200: priority streams, green-context BE partition, in-kernel
// completion counters) and FAKE (CPU threads stand in for streams; CPU tests and sanitizers).
#pragma once
#include <cstdint>
#include <memory>
#include "orion.h"

namespace orion {

struct StreamHandle;  // backend-specific

struct Backend {
  virtual ~Backend() {}
  virtual uint32_t num_sms() = 0;
  virtual int create_stream(int prio, StreamHandle** out) = 0;
  virtual void destroy_stream(StreamHandle* s) = 0;
  virtual void* native_stream(StreamHandle* s) = 0;
  // Launch op #seq of the stream's client; when it completes the stream's done counter becomes seq+1.
  virtual int launch(StreamHandle* s, const orion_op& op, uint64_t seq) = 0;
  virtual uint64_t read_done(StreamHandle* s) = 0;  // plain load, no API call
  virtual void thread_init() {}                     // called on the scheduler thread
  virtual void finish() {}
  // live per-kernel tracing (CUDA backend): durations in ms of traced launches, after finish()
  virtual int trace_read(float* ms, uint32_t cap, uint32_t* n) { (void)ms; (void)cap; *n = 0; return 0; }
};

int make_backend(const orion_config& cfg, int device, std::unique_ptr<Backend>* out);
std::unique_ptr<Backend> make_fake_backend(const orion_config& cfg);
int make_cuda_backend(const orion_config& cfg, int device, std::unique_ptr<Backend>* out);

}  // namespace orion
