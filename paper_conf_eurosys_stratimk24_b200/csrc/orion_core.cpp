// liborion core: per-client lock-free queues, the scheduler thread running Listing 1 of the paper
// (§5.1.1) with the readings of DESIGN.md §3, the binary decision
// log + observation tape, and the native client drivers.
//
// Independent of oracle/policy.c by construction (no shared code): the log format and the policy
// are implemented here from DESIGN.md; tests compare the two byte for byte.
#include <pthread.h>
#include <sched.h>
#include <time.h>

#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <memory>
#include <new>
#include <thread>
#include <vector>

#include "backend.h"
#include "orion.h"

namespace orion {

static inline int64_t now_ns() {
  timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return (int64_t)ts.tv_sec * 1000000000ll + ts.tv_nsec;
}

static inline void cpu_relax() {
#if defined(__x86_64__)
  __builtin_ia32_pause();
#endif
}

// ------------------------------------------------------------------ SPSC ring (one per client)
struct Ring {
  orion_op* slots = nullptr;
  uint64_t cap = 0, mask = 0;
  alignas(64) std::atomic<uint64_t> tail{0};  // ops published by the producer (visible count)
  alignas(64) std::atomic<uint64_t> head{0};  // ops consumed by the scheduler (popped count)
  alignas(64) uint64_t head_cache = 0;         // producer-side cache of head
};

// Decision kinds / tape record types / reasons
enum { D_HP_LAUNCH = 1, D_PASS = 2, D_ADMIT_IDLE = 3, D_ADMIT_COLOC = 4, D_DEFER_SM = 5, D_DEFER_PROFILE = 6,
       D_DEFER_DUR = 7, D_RESET = 8 };
enum { RSN_NONE = 0, RSN_SM = 1, RSN_PROFILE = 2, RSN_DUR = 3 };
enum { TAPE_VIS = 1, TAPE_DONE = 2 };

struct TapeRec { uint64_t k; uint32_t type, client; uint64_t value; };
struct DecRec { uint64_t k; uint8_t kind, client; uint16_t zero; uint32_t kernel_id; uint64_t seq; int64_t be_dur; };
static_assert(sizeof(TapeRec) == 24, "tape record");
static_assert(sizeof(DecRec) == 32, "decision record");
struct OpRec { uint32_t kernel_id; uint16_t kind; uint8_t opflags, cls; uint32_t sm_needed, zero; uint64_t dur_ns; };
static_assert(sizeof(OpRec) == 24, "op record");

struct Prof { uint8_t cls; uint32_t sm_needed; };

struct Client {
  int id = 0, prio = 0;
  Ring ring;
  std::vector<OpRec> optable;  // producer-appended (logging on)
  uint64_t submitted = 0;      // producer-private
  StreamHandle* stream = nullptr;
};

enum State { CREATED = 0, STARTED = 1, STOPPED = 2 };

struct Instance {
  orion_config cfg{};
  int device = 0;
  uint32_t num_sms = 0, sm_thr = 0;
  uint64_t dur_thr = 0;
  std::unique_ptr<Backend> backend;
  std::vector<std::unique_ptr<Client>> clients;
  int hp = -1;
  std::vector<int> be;  // BE client ids in registration order (R11 round-robin)
  std::atomic<int> state{CREATED};
  std::atomic<int> failed{0};
  std::atomic<int> stop_req{0};
  std::thread sched;

  // scheduler state (scheduler thread only)
  uint64_t vis[16]{}, done[16]{}, popped[16]{};
  Prof hp_ref{0, 0};
  int64_t be_dur = 0;
  uint64_t ld_seq[16];
  uint8_t ld_reason[16];
  bool req_open = false;
  uint64_t req_open_b = 0;
  std::deque<uint64_t> req_closed_end;     // REQ_END seqs of closed requests not yet known done
  std::deque<std::pair<uint64_t, Prof>> hp_inflight;  // (seq, profile) of popped HP ops (HP_REF_ALL)

  // log
  bool logging = false, overflow = false;
  std::vector<TapeRec> tape;
  std::vector<DecRec> decs;
  uint64_t k_end = 0;

  // counters
  std::atomic<uint64_t> st_iters{0}, st_hp{0}, st_admit{0}, st_defer{0}, st_mem{0}, st_reset{0}, st_err{0}, st_launch_ns{0};
};

// ------------------------------------------------------------------ log helpers
static inline void log_tape(Instance* I, uint64_t k, uint32_t type, uint32_t c, uint64_t v) {
  if (!I->logging) return;
  if (I->tape.size() >= I->cfg.log_capacity) { I->overflow = true; return; }
  I->tape.push_back(TapeRec{k, type, c, v});
}
static inline void log_dec(Instance* I, uint64_t k, int kind, int c, uint32_t kid, uint64_t seq) {
  if (!I->logging) return;
  if (I->decs.size() >= I->cfg.log_capacity) { I->overflow = true; return; }
  I->decs.push_back(DecRec{k, (uint8_t)kind, (uint8_t)c, 0, kid, seq, I->be_dur});
}

// ------------------------------------------------------------------ policy pieces (Listing 1)
// different profiles (L28, R1, R4): unknown on either side is compatible
static inline bool profiles_differ(const Instance* I, uint8_t hp_cls, uint8_t be_cls) {
  if (I->cfg.flags & ORION_F_NO_PROFILE_TEST) return true;   // ablation (Fig. 14)
  if (I->cfg.flags & ORION_F_HP_UNKNOWN_STRICT) return be_cls == ORION_CLS_U || (hp_cls != ORION_CLS_U && hp_cls != be_cls);
  return hp_cls == ORION_CLS_U || be_cls == ORION_CLS_U || hp_cls != be_cls;
}
// SM test (L27, R5): sm_needed < SM_THRESHOLD; FREE_SMS: sm_needed + hp.sm_needed <= num_sms
static inline bool sm_fits(const Instance* I, const Prof& h, uint32_t sm_needed) {
  if (I->cfg.flags & ORION_F_NO_SM_TEST) return true;        // ablation (Fig. 14)
  if (I->cfg.flags & ORION_F_FREE_SMS) return (uint64_t)sm_needed + h.sm_needed <= I->num_sms;
  return sm_needed < I->sm_thr;
}

static bool hp_busy(Instance* I) {
  if (I->hp < 0) return false;
  const int h = I->hp;
  if (!(I->cfg.flags & ORION_F_HP_BUSY_REQUEST)) return I->done[h] < I->popped[h];  // R2 (kernel-granular)
  while (!I->req_closed_end.empty() && I->req_closed_end.front() < I->done[h]) I->req_closed_end.pop_front();
  return I->req_open || !I->req_closed_end.empty();
}

// schedule_be (L23-L30) -> reason; RSN_NONE = suitable
static int schedule_be(Instance* I, bool busy, const orion_op& op) {
  if (!busy) return RSN_NONE;  // L25-L26
  const Prof me{op.prof.cls, op.prof.sm_needed};
  if ((I->cfg.flags & ORION_F_HP_REF_ALL) && I->hp >= 0) {
    const int h = I->hp;
    while (!I->hp_inflight.empty() && I->hp_inflight.front().first < I->done[h]) I->hp_inflight.pop_front();
    if (!I->hp_inflight.empty()) {
      bool sm_bad = false, prof_bad = false;
      for (auto& e : I->hp_inflight) {
        if (!sm_fits(I, e.second, me.sm_needed)) sm_bad = true;
        else if (!profiles_differ(I, e.second.cls, me.cls)) prof_bad = true;
      }
      return sm_bad ? RSN_SM : (prof_bad ? RSN_PROFILE : RSN_NONE);
    }
  }
  if (!sm_fits(I, I->hp_ref, me.sm_needed)) return RSN_SM;          // L27
  if (!profiles_differ(I, I->hp_ref.cls, me.cls)) return RSN_PROFILE;  // L28
  return RSN_NONE;
}

static bool be_all_finished(const Instance* I) {  // be_submitted.finished() (L13, R10)
  for (int j : I->be)
    if (I->done[j] != I->popped[j]) return false;
  return true;
}

static void launch_op(Instance* I, Client* c, const orion_op& op, uint64_t seq) {
  int64_t t0 = now_ns();
  int r = I->backend->launch(c->stream, op, seq);
  I->st_launch_ns.fetch_add((uint64_t)(now_ns() - t0), std::memory_order_relaxed);
  if (r != 0) {
    I->st_err.fetch_add(1, std::memory_order_relaxed);
    I->failed.store(1);
  }
}

static void one_iteration(Instance* I, uint64_t k) {
  bool busy = hp_busy(I);  // step 1
  // step 2: HP op present -> launch at once on the dedicated stream (L5, L7-L9)
  if (I->hp >= 0 && I->popped[I->hp] < I->vis[I->hp]) {
    const int h = I->hp;
    Client* c = I->clients[h].get();
    const uint64_t seq = I->popped[h];
    const orion_op& op = c->ring.slots[seq & c->ring.mask];
    const bool kern = op.kind == ORION_OP_KERNEL;
    launch_op(I, c, op, seq);
    log_dec(I, k, kern ? D_HP_LAUNCH : D_PASS, h, op.prof.kernel_id, seq);
    I->hp_ref = kern ? Prof{op.prof.cls, op.prof.sm_needed} : Prof{ORION_CLS_U, 0};
    if (I->cfg.flags & ORION_F_HP_BUSY_REQUEST) {
      if (op.opflags & ORION_OPF_REQ_BEGIN) { I->req_open = true; I->req_open_b = seq; }
      if ((op.opflags & ORION_OPF_REQ_END) && I->req_open) { I->req_open = false; I->req_closed_end.push_back(seq); }
    }
    if (I->cfg.flags & ORION_F_HP_REF_ALL) I->hp_inflight.emplace_back(seq, I->hp_ref);
    I->popped[h] = seq + 1;
    c->ring.head.store(seq + 1, std::memory_order_release);
    busy = true;  // L9
    I->st_hp.fetch_add(1, std::memory_order_relaxed);
  }
  // step 3: BE clients round-robin, rotation j = (k + t) mod n_be (R11)
  const size_t nbe = I->be.size();
  for (size_t t = 0; t < nbe; t++) {
    const int j = I->be[(k + t) % nbe];
    if (I->popped[j] == I->vis[j]) continue;  // L10: nothing queued
    Client* c = I->clients[j].get();
    const uint64_t seq = I->popped[j];
    const orion_op& op = c->ring.slots[seq & c->ring.mask];  // L6 peek (FIFO head only, R13)
    if (op.kind != ORION_OP_KERNEL) {  // memory ops bypass the policy (R14)
      launch_op(I, c, op, seq);
      log_dec(I, k, D_PASS, j, op.prof.kernel_id, seq);
      I->popped[j] = seq + 1;
      c->ring.head.store(seq + 1, std::memory_order_release);
      I->st_mem.fetch_add(1, std::memory_order_relaxed);
      continue;
    }
    int reason = schedule_be(I, busy, op);  // L11
    bool sched = reason == RSN_NONE;
    const bool throttle = !(I->cfg.flags & ORION_F_NO_THROTTLE) && (!(I->cfg.flags & ORION_F_THROTTLE_ONLY_HP_BUSY) || busy);  // R7
    if (throttle && I->be_dur > (int64_t)I->dur_thr) {                                // L12 (R6)
      if (be_all_finished(I)) {                                                       // L13
        I->be_dur = 0;                                                                // L14
        log_dec(I, k, D_RESET, j, 0xFFFFFFFFu, ~0ull);
        I->st_reset.fetch_add(1, std::memory_order_relaxed);
      } else if (sched) {                                                             // L16
        sched = false;
        reason = RSN_DUR;
      }
    }
    if (sched) {  // L17-L21
      launch_op(I, c, op, seq);
      I->be_dur += (int64_t)op.prof.dur_ns;
      log_dec(I, k, busy ? D_ADMIT_COLOC : D_ADMIT_IDLE, j, op.prof.kernel_id, seq);
      I->popped[j] = seq + 1;
      c->ring.head.store(seq + 1, std::memory_order_release);
      I->st_admit.fetch_add(1, std::memory_order_relaxed);
    } else if (!(I->ld_seq[j] == seq && I->ld_reason[j] == reason)) {
      const int kind = reason == RSN_SM ? D_DEFER_SM : (reason == RSN_PROFILE ? D_DEFER_PROFILE : D_DEFER_DUR);
      log_dec(I, k, kind, j, op.prof.kernel_id, seq);
      I->ld_seq[j] = seq;
      I->ld_reason[j] = (uint8_t)reason;
      I->st_defer.fetch_add(1, std::memory_order_relaxed);
    }
  }
}

static void scheduler_main(Instance* I) {
  if (I->cfg.sched_cpu >= 0) {
    cpu_set_t set;
    CPU_ZERO(&set);
    CPU_SET(I->cfg.sched_cpu, &set);
    pthread_setaffinity_np(pthread_self(), sizeof(set), &set);
  }
  I->backend->thread_init();
  const int n = (int)I->clients.size();
  uint64_t k = 0;
  for (;;) {
    // sample every queue tail and completion counter exactly once per iteration (A3)
    for (int c = 0; c < n; c++) {
      uint64_t v = I->clients[c]->ring.tail.load(std::memory_order_acquire);
      if (v != I->vis[c]) { I->vis[c] = v; log_tape(I, k, TAPE_VIS, (uint32_t)c, v); }
    }
    for (int c = 0; c < n; c++) {
      uint64_t d = I->backend->read_done(I->clients[c]->stream);
      if (d != I->done[c]) { I->done[c] = d; log_tape(I, k, TAPE_DONE, (uint32_t)c, d); }
    }
    one_iteration(I, k);
    if (I->failed.load(std::memory_order_relaxed)) break;
    if (I->stop_req.load(std::memory_order_acquire)) {
      bool drained = true;
      for (int c = 0; c < n && drained; c++) {
        uint64_t t = I->clients[c]->ring.tail.load(std::memory_order_acquire);
        drained = I->vis[c] == t && I->popped[c] == t && I->done[c] == t;
      }
      if (drained) { k++; break; }
    }
    k++;
  }
  I->k_end = k;
  I->st_iters.store(k);
}

}  // namespace orion

using namespace orion;

struct orion_s : Instance {};

extern "C" {

const char* orion_strerror(int code) {
  switch (code) {
    case ORION_OK: return "ok";
    case ORION_E_INVAL: return "invalid argument";
    case ORION_E_STATE: return "invalid state";
    case ORION_E_AGAIN: return "queue full";
    case ORION_E_CUDA: return "CUDA failure (handle is failed)";
    case ORION_E_NOMEM: return "out of memory / log capacity";
    case ORION_E_TIMEOUT: return "timeout";
    case ORION_E_NODEV: return "no CUDA device or driver";
  }
  return "unknown error";
}

int64_t orion_now_ns(void) { return now_ns(); }

int orion_create(int cuda_device, const orion_config* cfg, orion_t* out) {
  if (!cfg || !out) return ORION_E_INVAL;
  orion_s* I = new (std::nothrow) orion_s();
  if (!I) return ORION_E_NOMEM;
  I->cfg = *cfg;
  I->device = cuda_device;
  if (I->cfg.queue_capacity == 0) I->cfg.queue_capacity = 4096;
  if (I->cfg.queue_capacity & (I->cfg.queue_capacity - 1)) { delete I; return ORION_E_INVAL; }
  if (I->cfg.be_partition_sms % 8) { delete I; return ORION_E_INVAL; }
  int r = make_backend(I->cfg, cuda_device, &I->backend);
  if (r) { delete I; return r; }
  I->num_sms = I->cfg.num_sms ? I->cfg.num_sms : I->backend->num_sms();
  I->sm_thr = I->cfg.sm_threshold ? I->cfg.sm_threshold : I->num_sms;
  // DUR_THRESHOLD = floor(lat * ppm / 1e6) (R9); unknown HP latency -> no throttle
  if (I->cfg.hp_latency_ns == 0) I->dur_thr = (uint64_t)INT64_MAX;
  else I->dur_thr = (uint64_t)((unsigned __int128)I->cfg.hp_latency_ns * I->cfg.dur_threshold_ppm / 1000000u);
  for (int i = 0; i < 16; i++) { I->ld_seq[i] = ~0ull; I->ld_reason[i] = 0xff; }
  I->logging = I->cfg.log_capacity > 0;
  if (I->logging) {
    try {
      I->tape.reserve(I->cfg.log_capacity);
      I->decs.reserve(I->cfg.log_capacity);
    } catch (...) { delete I; return ORION_E_NOMEM; }
  }
  *out = I;
  return ORION_OK;
}

int orion_register_client(orion_t h, int prio, int* client_id) {
  if (!h || !client_id || (prio != ORION_HP && prio != ORION_BE)) return ORION_E_INVAL;
  if (h->state.load() != CREATED) return ORION_E_STATE;
  if (h->failed.load()) return ORION_E_CUDA;
  if (h->clients.size() >= 16) return ORION_E_INVAL;
  if (prio == ORION_HP && h->hp >= 0) return ORION_E_INVAL;
  auto c = std::make_unique<Client>();
  c->id = (int)h->clients.size();
  c->prio = prio;
  c->ring.cap = h->cfg.queue_capacity;
  c->ring.mask = c->ring.cap - 1;
  c->ring.slots = (orion_op*)aligned_alloc(64, sizeof(orion_op) * c->ring.cap);
  if (!c->ring.slots) return ORION_E_NOMEM;
  int r = h->backend->create_stream(prio, &c->stream);
  if (r) { free(c->ring.slots); if (r == ORION_E_CUDA) h->failed.store(1); return r; }
  if (prio == ORION_HP) h->hp = c->id; else h->be.push_back(c->id);
  *client_id = c->id;
  h->clients.push_back(std::move(c));
  return ORION_OK;
}

int orion_client_stream(orion_t h, int client_id, void** cu_stream) {
  if (!h || !cu_stream || client_id < 0 || client_id >= (int)h->clients.size()) return ORION_E_INVAL;
  *cu_stream = h->backend->native_stream(h->clients[client_id]->stream);
  return ORION_OK;
}

int orion_start(orion_t h) {
  if (!h) return ORION_E_INVAL;
  if (h->failed.load()) return ORION_E_CUDA;
  int expect = CREATED;
  if (!h->state.compare_exchange_strong(expect, STARTED)) return ORION_E_STATE;
  try {
    h->sched = std::thread(scheduler_main, static_cast<Instance*>(h));
  } catch (...) { h->state.store(CREATED); return ORION_E_NOMEM; }
  return ORION_OK;
}

static int submit_impl(orion_t h, int client_id, const orion_op* ops, uint32_t n, uint64_t* first_seq) {
  if (!h || !ops || client_id < 0 || client_id >= (int)h->clients.size()) return ORION_E_INVAL;
  if (h->failed.load(std::memory_order_relaxed)) return ORION_E_CUDA;
  int st = h->state.load(std::memory_order_relaxed);
  if (st == STOPPED) return ORION_E_STATE;
  Client* c = h->clients[client_id].get();
  Ring& R = c->ring;
  const uint64_t t = c->submitted;
  if (t + n - R.head_cache > R.cap) {
    R.head_cache = R.head.load(std::memory_order_acquire);
    if (t + n - R.head_cache > R.cap) return ORION_E_AGAIN;
  }
  for (uint32_t i = 0; i < n; i++) {
    const orion_op& op = ops[i];
    if (op.kind > ORION_OP_MEMCPY_D2D || op.prof.cls > ORION_CLS_M) return ORION_E_INVAL;
  }
  for (uint32_t i = 0; i < n; i++) {
    R.slots[(t + i) & R.mask] = ops[i];
    if (h->logging) {
      const orion_op& op = ops[i];
      const bool kern = op.kind == ORION_OP_KERNEL;
      c->optable.push_back(OpRec{op.prof.kernel_id, op.kind, op.opflags, (uint8_t)(kern ? op.prof.cls : 0),
                                 kern ? op.prof.sm_needed : 0u, 0u, kern ? op.prof.dur_ns : 0ull});
    }
  }
  c->submitted = t + n;
  R.tail.store(t + n, std::memory_order_release);
  if (first_seq) *first_seq = t;
  return ORION_OK;
}

int orion_submit(orion_t h, int client_id, const orion_op* op, uint64_t* seq_out) { return submit_impl(h, client_id, op, 1, seq_out); }
int orion_submit_n(orion_t h, int client_id, const orion_op* ops, uint32_t n, uint64_t* first_seq) {
  return submit_impl(h, client_id, ops, n, first_seq);
}

int orion_done_seq(orion_t h, int client_id, uint64_t* done) {
  if (!h || !done || client_id < 0 || client_id >= (int)h->clients.size()) return ORION_E_INVAL;
  *done = h->backend->read_done(h->clients[client_id]->stream);
  return h->failed.load() ? ORION_E_CUDA : ORION_OK;
}

int orion_synchronize(orion_t h, int client_id, uint64_t timeout_ns) {
  if (!h || client_id < 0 || client_id >= (int)h->clients.size()) return ORION_E_INVAL;
  Client* c = h->clients[client_id].get();
  const uint64_t target = c->submitted;
  const int64_t t0 = now_ns();
  while (h->backend->read_done(c->stream) < target) {
    if (h->failed.load(std::memory_order_relaxed)) return ORION_E_CUDA;
    if (h->state.load(std::memory_order_relaxed) != STARTED && c->ring.head.load() < target) return ORION_E_STATE;
    if (timeout_ns && (uint64_t)(now_ns() - t0) > timeout_ns) return ORION_E_TIMEOUT;
    cpu_relax();
  }
  return ORION_OK;
}

int orion_stop(orion_t h) {
  if (!h) return ORION_E_INVAL;
  if (h->state.load() != STARTED) return ORION_E_STATE;
  h->stop_req.store(1, std::memory_order_release);
  if (h->sched.joinable()) h->sched.join();
  h->state.store(STOPPED);
  h->backend->finish();
  return h->failed.load() ? ORION_E_CUDA : ORION_OK;
}

static void put32(std::vector<uint8_t>& b, uint32_t v) { for (int i = 0; i < 4; i++) b.push_back((uint8_t)(v >> (8 * i))); }
static void put64(std::vector<uint8_t>& b, uint64_t v) { for (int i = 0; i < 8; i++) b.push_back((uint8_t)(v >> (8 * i))); }

int orion_read_log(orion_t h, void* buf, size_t cap, size_t* written) {
  if (!h) return ORION_E_INVAL;
  if (h->state.load() == STARTED) return ORION_E_STATE;
  if (!h->logging) return ORION_E_STATE;
  std::vector<uint8_t> b;
  const uint32_t n = (uint32_t)h->clients.size();
  // header (240 bytes)
  const char magic[8] = {'O', 'R', 'I', 'O', 'N', 'L', 'G', '1'};
  b.insert(b.end(), magic, magic + 8);
  put32(b, 1); put32(b, n); put32(b, h->num_sms); put32(b, h->sm_thr);
  put64(b, h->dur_thr); put32(b, h->cfg.flags); put32(b, (uint32_t)h->hp);
  for (uint32_t i = 0; i < 16; i++) put32(b, i < n ? (uint32_t)h->clients[i]->prio : 0xFFFFFFFFu);
  put64(b, h->k_end);
  for (uint32_t i = 0; i < 16; i++) put64(b, i < n ? (uint64_t)h->clients[i]->optable.size() : 0);
  for (uint32_t i = 0; i < n; i++) {
    const auto& t = h->clients[i]->optable;
    const uint8_t* p = reinterpret_cast<const uint8_t*>(t.data());
    b.insert(b.end(), p, p + t.size() * sizeof(OpRec));
  }
  put64(b, h->tape.size());
  { const uint8_t* p = reinterpret_cast<const uint8_t*>(h->tape.data()); b.insert(b.end(), p, p + h->tape.size() * sizeof(TapeRec)); }
  put64(b, h->decs.size());
  { const uint8_t* p = reinterpret_cast<const uint8_t*>(h->decs.data()); b.insert(b.end(), p, p + h->decs.size() * sizeof(DecRec)); }
  if (written) *written = b.size();
  if (h->overflow) return ORION_E_NOMEM;
  if (!buf || cap < b.size()) return ORION_E_NOMEM;
  memcpy(buf, b.data(), b.size());
  return ORION_OK;
}

int orion_stats(orion_t h, uint64_t* out, uint32_t n) {
  if (!h || !out) return ORION_E_INVAL;
  uint64_t v[8] = {h->st_iters.load(), h->st_hp.load(), h->st_admit.load(), h->st_defer.load(),
                   h->st_mem.load(), h->st_reset.load(), h->st_err.load(), h->st_launch_ns.load()};
  for (uint32_t i = 0; i < n && i < 8; i++) out[i] = v[i];
  return ORION_OK;
}

int orion_trace_read(orion_t h, float* ms_out, uint32_t cap, uint32_t* n) {
  if (!h || !n) return ORION_E_INVAL;
  if (h->state.load() == STARTED) return ORION_E_STATE;
  return h->backend->trace_read(ms_out, ms_out ? cap : 0, n);
}

int orion_destroy(orion_t h) {
  if (!h) return ORION_E_INVAL;
  if (h->state.load() == STARTED) {
    h->stop_req.store(1);
    if (h->sched.joinable()) h->sched.join();
  }
  for (auto& c : h->clients) {
    if (c->stream) h->backend->destroy_stream(c->stream);
    free(c->ring.slots);
  }
  h->clients.clear();
  h->backend.reset();
  delete h;
  return ORION_OK;
}

// ------------------------------------------------------------------ native client drivers
int orion_run_requests(orion_t h, int client_id, const orion_op* ops, uint32_t n_ops, const int64_t* arrivals_ns, uint32_t n_req,
                       uint32_t in_cycle, uint32_t out_cycle, int64_t* t_arrival_ns, int64_t* t_done_ns) {
  if (!h || !ops || !n_ops || !arrivals_ns || client_id < 0 || client_id >= (int)h->clients.size()) return ORION_E_INVAL;
  if (h->state.load() != STARTED) return ORION_E_STATE;
  if (n_ops > h->cfg.queue_capacity) return ORION_E_INVAL;
  if (in_cycle == 0) in_cycle = 1;
  if (out_cycle == 0) out_cycle = 1;
  Client* c = h->clients[client_id].get();
  std::vector<orion_op> buf(ops, ops + n_ops);
  std::vector<uint64_t> end_seq(n_req);
  uint32_t next_done = 0;
  const int64_t start = now_ns();
  auto poll = [&]() {
    uint64_t d = h->backend->read_done(c->stream);
    int64_t t = -1;
    while (next_done < n_req && next_done < (uint32_t)end_seq.size() && end_seq[next_done] != 0 && d >= end_seq[next_done]) {
      if (t < 0) t = now_ns();
      if (t_done_ns) t_done_ns[next_done] = t;
      next_done++;
    }
  };
  for (uint32_t r = 0; r < n_req; r++) {
    const int64_t due = start + arrivals_ns[r];
    while (now_ns() < due) {
      poll();
      if (h->failed.load(std::memory_order_relaxed)) return ORION_E_CUDA;
      cpu_relax();
    }
    for (uint32_t i = 0; i < n_ops; i++) {
      buf[i] = ops[i];
      buf[i].opflags = (uint8_t)(ops[i].opflags | (i == 0 ? ORION_OPF_REQ_BEGIN : 0) | (i + 1 == n_ops ? ORION_OPF_REQ_END : 0));
      if (ops[i].kind == ORION_OP_MEMCPY_H2D) buf[i].args[1] = ops[i].args[1] + (uint64_t)(r % in_cycle) * ops[i].args[2];
      if (ops[i].kind == ORION_OP_MEMCPY_D2H) buf[i].args[0] = ops[i].args[0] + (uint64_t)(r % out_cycle) * ops[i].args[2];
    }
    uint64_t first = 0;
    int rc;
    while ((rc = orion_submit_n(h, client_id, buf.data(), n_ops, &first)) == ORION_E_AGAIN) { poll(); cpu_relax(); }
    if (rc) return rc;
    if (t_arrival_ns) t_arrival_ns[r] = due;
    end_seq[r] = first + n_ops;
    poll();
  }
  while (next_done < n_req) {
    poll();
    if (h->failed.load(std::memory_order_relaxed)) return ORION_E_CUDA;
    cpu_relax();
  }
  return ORION_OK;
}

int orion_run_requests_direct(orion_t h, int client_id, const orion_op* ops, uint32_t n_ops, const int64_t* arrivals_ns, uint32_t n_req,
                              uint32_t in_cycle, uint32_t out_cycle, int64_t* t_arrival_ns, int64_t* t_done_ns) {
  if (!h || !ops || !n_ops || !arrivals_ns || client_id < 0 || client_id >= (int)h->clients.size()) return ORION_E_INVAL;
  if (h->state.load() != CREATED) return ORION_E_STATE;
  if (h->failed.load()) return ORION_E_CUDA;
  if (in_cycle == 0) in_cycle = 1;
  if (out_cycle == 0) out_cycle = 1;
  Client* c = h->clients[client_id].get();
  h->backend->thread_init();
  orion_op op;
  uint32_t next_done = 0;
  std::vector<uint64_t> end_seq(n_req, 0);
  auto poll = [&]() {
    const uint64_t d = h->backend->read_done(c->stream);
    int64_t t = -1;
    while (next_done < n_req && end_seq[next_done] != 0 && d >= end_seq[next_done]) {
      if (t < 0) t = now_ns();
      if (t_done_ns) t_done_ns[next_done] = t;
      next_done++;
    }
  };
  const int64_t start = now_ns();
  for (uint32_t r = 0; r < n_req; r++) {
    const int64_t due = start + arrivals_ns[r];
    while (now_ns() < due) { poll(); cpu_relax(); }
    for (uint32_t i = 0; i < n_ops; i++) {
      op = ops[i];
      if (op.kind == ORION_OP_MEMCPY_H2D) op.args[1] = ops[i].args[1] + (uint64_t)(r % in_cycle) * ops[i].args[2];
      if (op.kind == ORION_OP_MEMCPY_D2H) op.args[0] = ops[i].args[0] + (uint64_t)(r % out_cycle) * ops[i].args[2];
      const uint64_t seq = c->submitted++;
      if (h->backend->launch(c->stream, op, seq) != 0) { h->failed.store(1); return ORION_E_CUDA; }
    }
    if (t_arrival_ns) t_arrival_ns[r] = due;
    end_seq[r] = c->submitted;
    poll();
  }
  while (next_done < n_req) {
    poll();
    if (h->failed.load(std::memory_order_relaxed)) return ORION_E_CUDA;
    cpu_relax();
  }
  return ORION_OK;
}

int orion_run_iterations(orion_t h, int client_id, const orion_op* ops, uint32_t n_ops, uint32_t n_variants, const volatile int32_t* stop,
                         uint64_t max_iters, int64_t* t_end_ns, uint64_t cap_iters, uint64_t* iters_out) {
  if (!h || !ops || !n_ops || client_id < 0 || client_id >= (int)h->clients.size()) return ORION_E_INVAL;
  if (h->state.load() != STARTED) return ORION_E_STATE;
  if (n_variants == 0) n_variants = 1;
  Client* c = h->clients[client_id].get();
  uint64_t it = 0;
  // the stop flag is written by another thread (the controller): an atomic acquire load, not a plain read
  while ((max_iters == 0 || it < max_iters) && !(stop && __atomic_load_n(stop, __ATOMIC_ACQUIRE))) {
    const orion_op* v = ops + (size_t)(it % n_variants) * n_ops;
    for (uint32_t i = 0; i < n_ops; i++) {
      int rc;
      while ((rc = orion_submit(h, client_id, v + i, nullptr)) == ORION_E_AGAIN) {
        if (h->failed.load(std::memory_order_relaxed)) return ORION_E_CUDA;
        cpu_relax();
      }
      if (rc) return rc;
    }
    const uint64_t target = c->submitted;
    while (h->backend->read_done(c->stream) < target) {
      if (h->failed.load(std::memory_order_relaxed)) return ORION_E_CUDA;
      cpu_relax();
    }
    if (t_end_ns && it < cap_iters) t_end_ns[it] = now_ns();
    it++;
  }
  if (iters_out) *iters_out = it;
  return ORION_OK;
}

}  // extern "C"
