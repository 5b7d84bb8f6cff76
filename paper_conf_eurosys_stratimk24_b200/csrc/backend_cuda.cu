// CUDA backend (B200): HP stream at the greatest priority, BE streams at the least priority
// (R18), optionally inside a green-context SM partition (Blackwell SM partitioning,
// multiple of 8 SMs, cuda.h:25256-25261). Completion is observed through host-mapped counters
// written by the last CTA of each kernel (kernels/common.cuh: orion_signal) instead of
// cudaEventQuery: a plain load on the scheduler thread. Memory ops are followed by
// cuStreamWriteValue64 on the same stream.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstring>
#include <mutex>
#include <vector>

#include "backend.h"
#include "kernels/common.cuh"

namespace orion {

struct StreamHandle {
  cudaStream_t stream = nullptr;
  CUgreenCtx green = nullptr;
  unsigned long long* done_host = nullptr;  // host-mapped counter (pinned)
  unsigned long long* done_dev = nullptr;   // its device address
  unsigned long long* ticket = nullptr;     // device CTA counter
  unsigned long long ticket_base = 0;       // CTAs launched on this stream so far
};

// Driver entry points resolved at runtime through cudart (the .so never links libcuda directly,
// so it loads on machines without a driver and fails cleanly at orion_create).
struct Drv {
  CUresult (*streamWriteValue64)(CUstream, CUdeviceptr, cuuint64_t, unsigned int) = nullptr;
  CUresult (*deviceGetDevResource)(CUdevice, CUdevResource*, CUdevResourceType) = nullptr;
  CUresult (*devSmResourceSplitByCount)(CUdevResource*, unsigned int*, const CUdevResource*, CUdevResource*, unsigned int,
                                        unsigned int) = nullptr;
  CUresult (*devResourceGenerateDesc)(CUdevResourceDesc*, CUdevResource*, unsigned int) = nullptr;
  CUresult (*greenCtxCreate)(CUgreenCtx*, CUdevResourceDesc, CUdevice, unsigned int) = nullptr;
  CUresult (*greenCtxStreamCreate)(CUstream*, CUgreenCtx, unsigned int, int) = nullptr;
  CUresult (*greenCtxDestroy)(CUgreenCtx) = nullptr;
};

template <class F>
static bool resolve(const char* name, F* fn, int ver) {
  cudaDriverEntryPointQueryResult q;
  void* p = nullptr;
  if (cudaGetDriverEntryPointByVersion(name, &p, ver, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess)
    return false;
  *fn = reinterpret_cast<F>(p);
  return true;
}

struct CudaBackend : Backend {
  int device = 0;
  uint32_t sms = 0;
  int prio_least = 0, prio_greatest = 0;
  uint32_t be_partition = 0;
  uint32_t flags = 0;
  Drv drv;
  unsigned long long* host_counters = nullptr;  // one 64-byte line per stream
  int next_counter = 0;
  // live tracing of one kernel id: event pairs recorded on the launching stream
  uint32_t trace_kid_p1 = 0;
  static constexpr int kTraceCap = 8192;
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> trace_ev;
  int trace_n = 0;

  ~CudaBackend() override {
    for (auto& e : trace_ev) { cudaEventDestroy(e.first); cudaEventDestroy(e.second); }
    if (host_counters) cudaFreeHost(host_counters);
  }
  uint32_t num_sms() override { return sms; }

  int init(const orion_config& cfg, int dev) {
    device = dev;
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess || n <= dev) { cudaGetLastError(); return ORION_E_NODEV; }
    if (cudaSetDevice(dev) != cudaSuccess) return ORION_E_NODEV;
    if (cudaFree(0) != cudaSuccess) return ORION_E_NODEV;
    int v = 0;
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
    sms = (uint32_t)v;
    if (cudaDeviceGetStreamPriorityRange(&prio_least, &prio_greatest) != cudaSuccess) return ORION_E_CUDA;
    if (!resolve("cuStreamWriteValue64", &drv.streamWriteValue64, 12000)) return ORION_E_CUDA;
    be_partition = cfg.be_partition_sms;
    flags = cfg.flags;
    if (be_partition) {
      bool ok = resolve("cuDeviceGetDevResource", &drv.deviceGetDevResource, 12080) &&
                resolve("cuDevSmResourceSplitByCount", &drv.devSmResourceSplitByCount, 12080) &&
                resolve("cuDevResourceGenerateDesc", &drv.devResourceGenerateDesc, 12080) &&
                resolve("cuGreenCtxCreate", &drv.greenCtxCreate, 12080) &&
                resolve("cuGreenCtxStreamCreate", &drv.greenCtxStreamCreate, 12080) &&
                resolve("cuGreenCtxDestroy", &drv.greenCtxDestroy, 12080);
      if (!ok) return ORION_E_CUDA;
    }
    if (cudaHostAlloc((void**)&host_counters, 64 * 8 * 16, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess)
      return ORION_E_CUDA;
    memset(host_counters, 0, 64 * 8 * 16);
    trace_kid_p1 = cfg.trace_kernel_id_plus1;
    if (trace_kid_p1) {
      trace_ev.resize(kTraceCap);
      for (auto& e : trace_ev)
        if (cudaEventCreate(&e.first) != cudaSuccess || cudaEventCreate(&e.second) != cudaSuccess) return ORION_E_CUDA;
    }
    return 0;
  }

  int create_stream(int prio, StreamHandle** out) override {
    if (next_counter >= 16) return ORION_E_INVAL;
    cudaSetDevice(device);
    StreamHandle* s = new StreamHandle();
    if (prio == ORION_BE && be_partition) {
      CUdevice d;
      CUdevResource all, part[1], rem;
      unsigned int nres = 1;
      CUdevResourceDesc desc;
      d = (CUdevice)device;
      if (drv.deviceGetDevResource(d, &all, CU_DEV_RESOURCE_TYPE_SM) != CUDA_SUCCESS ||
          drv.devSmResourceSplitByCount(part, &nres, &all, &rem, 0, be_partition) != CUDA_SUCCESS ||
          drv.devResourceGenerateDesc(&desc, part, 1) != CUDA_SUCCESS ||
          drv.greenCtxCreate(&s->green, desc, d, CU_GREEN_CTX_DEFAULT_STREAM) != CUDA_SUCCESS) {
        delete s;
        return ORION_E_CUDA;
      }
      CUstream cs;
      if (drv.greenCtxStreamCreate(&cs, s->green, CU_STREAM_NON_BLOCKING, prio_least) != CUDA_SUCCESS) {
        drv.greenCtxDestroy(s->green);
        delete s;
        return ORION_E_CUDA;
      }
      s->stream = (cudaStream_t)cs;
    } else {
      const bool hp_prio = prio == ORION_HP && !(flags & ORION_F_NO_PRIORITY);   // NO_PRIORITY: "GPU Streams" baseline
      if (cudaStreamCreateWithPriority(&s->stream, cudaStreamNonBlocking, hp_prio ? prio_greatest : prio_least) != cudaSuccess) {
        delete s;
        return ORION_E_CUDA;
      }
    }
    s->done_host = host_counters + 8 * next_counter++;
    if (cudaHostGetDevicePointer((void**)&s->done_dev, s->done_host, 0) != cudaSuccess) return ORION_E_CUDA;
    if (cudaMalloc((void**)&s->ticket, 256) != cudaSuccess) return ORION_E_CUDA;
    if (cudaMemset(s->ticket, 0, 256) != cudaSuccess) return ORION_E_CUDA;
    if (cudaDeviceSynchronize() != cudaSuccess) return ORION_E_CUDA;
    *out = s;
    return 0;
  }

  void destroy_stream(StreamHandle* s) override {
    if (s->stream) { cudaStreamSynchronize(s->stream); cudaStreamDestroy(s->stream); }
    if (s->green) drv.greenCtxDestroy(s->green);
    if (s->ticket) cudaFree(s->ticket);
    delete s;
  }
  void* native_stream(StreamHandle* s) override { return (void*)s->stream; }

  void thread_init() override { cudaSetDevice(device); }

  int launch(StreamHandle* s, const orion_op& op, uint64_t seq) override {
    if (op.kind == ORION_OP_KERNEL) {
      OrionSig sig{s->ticket, s->done_dev, s->ticket_base, seq + 1};
      unsigned long long ctas = 0;
      const bool tr = trace_kid_p1 && op.prof.kernel_id + 1 == trace_kid_p1 && trace_n < kTraceCap;
      if (tr) cudaEventRecord(trace_ev[trace_n].first, s->stream);
      int r = kernel_launch_sig(op.fn, op.args, op.nargs, sig, s->stream, &ctas);
      if (r) return r;
      if (tr) cudaEventRecord(trace_ev[trace_n++].second, s->stream);
      s->ticket_base += ctas;
      return 0;
    }
    cudaError_t e = cudaSuccess;
    switch (op.kind) {
      case ORION_OP_MEMCPY_H2D: e = cudaMemcpyAsync((void*)op.args[0], (const void*)op.args[1], op.args[2], cudaMemcpyHostToDevice, s->stream); break;
      case ORION_OP_MEMCPY_D2H: e = cudaMemcpyAsync((void*)op.args[0], (const void*)op.args[1], op.args[2], cudaMemcpyDeviceToHost, s->stream); break;
      case ORION_OP_MEMCPY_D2D: e = cudaMemcpyAsync((void*)op.args[0], (const void*)op.args[1], op.args[2], cudaMemcpyDeviceToDevice, s->stream); break;
      case ORION_OP_MEMSET: e = cudaMemsetAsync((void*)op.args[0], (int)op.args[1], op.args[2], s->stream); break;
      default: return ORION_E_INVAL;
    }
    if (e != cudaSuccess) return ORION_E_CUDA;
    if (drv.streamWriteValue64((CUstream)s->stream, (CUdeviceptr)s->done_dev, seq + 1, 0) != CUDA_SUCCESS) return ORION_E_CUDA;
    return 0;
  }

  uint64_t read_done(StreamHandle* s) override {
    return __atomic_load_n(reinterpret_cast<volatile unsigned long long*>(s->done_host), __ATOMIC_ACQUIRE);
  }

  void finish() override {
    cudaSetDevice(device);
    cudaDeviceSynchronize();
  }

  int trace_read(float* ms, uint32_t cap, uint32_t* n) override {
    *n = (uint32_t)trace_n;
    for (int i = 0; i < trace_n && (uint32_t)i < cap; i++) {
      float t = 0.f;
      if (cudaEventElapsedTime(&t, trace_ev[i].first, trace_ev[i].second) != cudaSuccess) return ORION_E_CUDA;
      ms[i] = t;
    }
    return 0;
  }
};

int make_cuda_backend(const orion_config& cfg, int device, std::unique_ptr<Backend>* out) {
  CudaBackend* b = new CudaBackend();
  int r = b->init(cfg, device);
  if (r) { delete b; return r; }
  out->reset(b);
  return 0;
}

}  // namespace orion
