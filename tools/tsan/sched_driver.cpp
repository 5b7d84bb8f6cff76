// Host-only stress driver of liborion's scheduler on the FAKE backend, built with
// -fsanitize=thread (or address,undefined) by tests/test_sanitizers_cpu.py. One HP
// producer (open-loop requests through orion_run_requests), two BE producers (closed-loop
// orion_run_iterations and raw orion_submit + orion_synchronize), the scheduler thread and the
// FAKE streams' threads all run at once; the decision log is read back at the end.
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <random>
#include <thread>
#include <vector>

#include "backend.h"
#include "orion.h"

namespace orion {
int make_cuda_backend(const orion_config&, int, std::unique_ptr<Backend>*) { return ORION_E_NODEV; }
}  // namespace orion

static orion_op mk(std::mt19937& rng, uint32_t kid) {
  orion_op op;
  memset(&op, 0, sizeof(op));
  op.kind = (rng() % 13 == 0) ? ORION_OP_MEMCPY_H2D : ORION_OP_KERNEL;
  op.prof.kernel_id = kid;
  op.prof.cls = (uint8_t)(rng() % 3);
  const uint32_t sms[] = {1, 8, 40, 147, 148, 300};
  op.prof.sm_needed = sms[rng() % 6];
  const uint64_t durs[] = {0, 2000, 5000, 20000};
  op.prof.dur_ns = durs[rng() % 4];
  return op;
}

int main(int argc, char** argv) {
  const uint32_t flags = argc > 1 ? (uint32_t)atoi(argv[1]) : 0;
  orion_config cfg;
  memset(&cfg, 0, sizeof(cfg));
  cfg.backend = ORION_BACKEND_FAKE;
  cfg.hp_latency_ns = 500000;
  cfg.dur_threshold_ppm = 25000;
  cfg.queue_capacity = 64;
  cfg.log_capacity = 1 << 20;
  cfg.flags = flags;
  cfg.fake_contention = 1;
  orion_t h;
  if (orion_create(0, &cfg, &h)) return 2;
  int hp, b1, b2;
  if (orion_register_client(h, ORION_HP, &hp) || orion_register_client(h, ORION_BE, &b1) || orion_register_client(h, ORION_BE, &b2)) return 3;
  std::mt19937 rng(7);
  std::vector<orion_op> hp_ops, it_ops, raw_ops;
  for (int i = 0; i < 12; i++) hp_ops.push_back(mk(rng, 100 + i));
  for (int i = 0; i < 20; i++) it_ops.push_back(mk(rng, 1000 + i));
  for (int i = 0; i < 300; i++) raw_ops.push_back(mk(rng, 5000 + i));
  for (auto& o : hp_ops) o.kind = ORION_OP_KERNEL;   // run_requests patches memop args by request; keep kernels
  for (auto& o : it_ops) o.kind = ORION_OP_KERNEL;
  if (orion_start(h)) return 4;
  std::vector<int64_t> arr(40), ta(40), td(40);
  for (int i = 0; i < 40; i++) arr[i] = (int64_t)i * 300000;
  int32_t stop = 0;   // written with an atomic store below, read with atomic loads by the driver
  uint64_t iters = 0;
  std::vector<int64_t> t_end(4096);
  int rc_hp = 0, rc_it = 0, rc_raw = 0;
  std::thread thp([&] { rc_hp = orion_run_requests(h, hp, hp_ops.data(), (uint32_t)hp_ops.size(), arr.data(), 40, 1, 1, ta.data(), td.data()); });
  std::thread tit([&] {
    rc_it = orion_run_iterations(h, b1, it_ops.data(), (uint32_t)it_ops.size(), 1, &stop, 0, t_end.data(), t_end.size(), &iters);
  });
  std::thread traw([&] {
    for (const auto& op : raw_ops) {
      int r;
      while ((r = orion_submit(h, b2, &op, nullptr)) == ORION_E_AGAIN) std::this_thread::yield();
      if (r) { rc_raw = r; return; }
    }
    rc_raw = orion_synchronize(h, b2, 0);
  });
  thp.join();
  traw.join();
  __atomic_store_n(&stop, 1, __ATOMIC_RELEASE);
  tit.join();
  if (orion_stop(h)) return 5;
  size_t need = 0;
  orion_read_log(h, nullptr, 0, &need);
  std::vector<unsigned char> buf(need);
  int rl = orion_read_log(h, buf.data(), buf.size(), &need);
  uint64_t st[8];
  orion_stats(h, st, 8);
  orion_destroy(h);
  printf("hp %d it %d raw %d log %d bytes %zu iters %llu sched_iters %llu admits %llu\n", rc_hp, rc_it, rc_raw, rl, need,
         (unsigned long long)iters, (unsigned long long)st[0], (unsigned long long)st[2]);
  return (rc_hp || rc_it || rc_raw || rl) ? 6 : 0;
}
