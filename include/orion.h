/*
 * orion.h — C ABI of liborion, a B200-native implementation of the hot path of
 * Strati, Ma, Klimovic, "Orion: Interference-aware, Fine-grained GPU Sharing for ML Applications",
 * EuroSys '24 (PAPER.md; citations "P:n" are PAPER.md line numbers).
 *
 * One orion_t per GPU ("a separate instance of Orion runs per GPU device"). Clients
 * register with a priority (one high-priority (HP) client, best-effort (BE) clients),
 * submit operators together with their offline profile (compute/memory class, SM need, duration;
 * P:825-870) into per-client software queues, and synchronize. A pinned
 * scheduler thread runs the policy of Listing 1 with the readings of DESIGN.md §3.
 *
 * Conventions for every call:
 *   - returns int: ORION_OK (0) or a negative ORION_E_* code; no exception crosses the ABI;
 *   - pointers are plain host pointers unless named "device"; sizes are bytes unless stated;
 *   - after any CUDA failure the handle is sticky-failed: every later call returns ORION_E_CUDA;
 *   - thread model: lifecycle calls (create/register/start/stop/read_log/destroy) from one
 *     controller thread; exactly one producer thread per client_id for submit/synchronize.
 */
#ifndef ORION_H
#define ORION_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
  ORION_OK = 0,
  ORION_E_INVAL = -1,   /* bad argument */
  ORION_E_STATE = -2,   /* call not allowed in the current lifecycle state */
  ORION_E_AGAIN = -3,   /* client queue full; retry (submit is non-blocking) */
  ORION_E_CUDA = -4,    /* CUDA failure; handle is sticky-failed */
  ORION_E_NOMEM = -5,   /* allocation or log capacity exhausted */
  ORION_E_TIMEOUT = -6, /* synchronize timed out */
  ORION_E_NODEV = -7    /* CUDA backend requested but no usable GPU / driver */
};

typedef struct orion_s* orion_t;

typedef enum { ORION_HP = 0, ORION_BE = 1 } orion_prio;
typedef enum { ORION_CLS_U = 0, ORION_CLS_C = 1, ORION_CLS_M = 2 } orion_cls;
typedef enum {
  ORION_OP_KERNEL = 0,
  ORION_OP_MEMCPY_H2D = 1, /* args[0]=dst device ptr, args[1]=src host ptr (pinned), args[2]=bytes */
  ORION_OP_MEMCPY_D2H = 2, /* args[0]=dst host ptr (pinned), args[1]=src device ptr, args[2]=bytes */
  ORION_OP_MEMSET = 3,     /* args[0]=dst device ptr, args[1]=byte value, args[2]=bytes */
  ORION_OP_MEMCPY_D2D = 4  /* args[0]=dst device ptr, args[1]=src device ptr, args[2]=bytes */
} orion_kind;
/* Memory operations bypass the policy and are submitted in client FIFO order (R14). */

/* Offline profile of one operator, carried inline in each op record (R15). */
typedef struct {
  uint32_t kernel_id;  /* unique kernel ID: positional id within the model's op list */
  uint8_t cls;         /* orion_cls: compute-bound, memory-bound or unknown */
  uint8_t pad[3];
  uint32_t sm_needed;  /* ceil(num_blocks / blocks_per_sm) */
  uint32_t reserved;
  uint64_t dur_ns;     /* solo execution time */
} orion_profile;

enum { ORION_OPF_REQ_BEGIN = 1, ORION_OPF_REQ_END = 2 }; /* request/iteration boundaries */
#define ORION_MAX_ARGS 24

typedef struct {
  uint32_t fn;      /* index into liborion's kernel table (orion_kernels.h); ignored for memops */
  uint16_t kind;    /* orion_kind */
  uint8_t nargs;    /* number of meaningful args */
  uint8_t opflags;  /* ORION_OPF_* */
  orion_profile prof;
  uint64_t args[ORION_MAX_ARGS]; /* POD: device pointers, dims, scalars (floats bit-cast) */
} orion_op;       /* copied by value into the client's queue at submit */

/* Reading switches (R2-R7). Default 0 = the proposed readings. */
enum {
  ORION_F_HP_BUSY_REQUEST = 1,       /* R2: HP busy from a request's first op until its last completes */
  ORION_F_HP_REF_ALL = 2,            /* R3: profile test against every in-flight HP op */
  ORION_F_HP_UNKNOWN_STRICT = 4,     /* R4: HP-unknown admits only BE-unknown */
  ORION_F_THROTTLE_ONLY_HP_BUSY = 8, /* R7: DUR_THRESHOLD check only while HP is busy */
  ORION_F_FREE_SMS = 16,             /* R5: be.sm_needed + hp.sm_needed <= num_sms */
  /* Policy ablation (Fig. 14) and the Streams baselines: each switch
     removes one component of the policy. NO_PROFILE | NO_SM | NO_THROTTLE admits every BE op
     at once ("Stream Priorities"); adding NO_PRIORITY gives "GPU Streams" (every stream at the
     default priority). NO_SM alone is the "Compute/Mem profiles" bar; NO_PRIORITY alone is
     Orion without stream priorities. */
  ORION_F_NO_PRIORITY = 32,          /* HP stream at the default (least) priority like the BE streams */
  ORION_F_NO_PROFILE_TEST = 64,      /* schedule_be skips the compute/memory profile test (L28) */
  ORION_F_NO_SM_TEST = 128,          /* schedule_be skips the SM-size test (L27) */
  ORION_F_NO_THROTTLE = 256          /* no DUR_THRESHOLD throttle (L12-L16) */
};

enum { ORION_BACKEND_CUDA = 0, ORION_BACKEND_FAKE = 1 };

typedef struct {
  uint32_t num_sms;           /* 0 -> device multiprocessor count (148 on B200) */
  uint32_t sm_threshold;      /* 0 -> num_sms (paper default) */
  uint32_t dur_threshold_ppm; /* DUR_THRESHOLD as ppm of hp_latency_ns; 25000 = 2.5% */
  uint32_t be_partition_sms;  /* 0 = BE streams on the full GPU; else green-context partition of
                                 this many SMs (multiple of 8, cuda.h:25256-25261) */
  uint64_t hp_latency_ns;     /* solo HP request latency; DUR_THR = floor(lat*ppm/1e6) */
  uint32_t flags;             /* ORION_F_* reading switches */
  uint32_t queue_capacity;    /* per-client ring slots, power of two (0 -> 4096) */
  uint32_t backend;           /* ORION_BACKEND_CUDA or ORION_BACKEND_FAKE (CPU threads as streams) */
  int32_t sched_cpu;          /* core to pin the scheduler thread to; -1 = no pinning */
  uint64_t log_capacity;      /* records per section; 0 = logging off */
  uint32_t fake_time_scale_pct; /* FAKE backend: op duration = dur_ns * pct/100 (0 -> 100) */
  uint32_t trace_kernel_id_plus1; /* CUDA backend: 0 = off; else record a CUDA event pair around every
                                     launch of kernel_id (trace_kernel_id_plus1 - 1) on its own stream
                                     (bench roofline: live launch durations, read by orion_trace_read) */
  uint32_t fake_contention;   /* FAKE backend: 1 = model SM contention between concurrently running
                                 kernels (each runs at 148 / total sm_needed of real time while the
                                 running kernels ask for more than 148 SMs); 0 = independent streams */
  uint32_t reserved[5];
} orion_config;

/* Create an instance on `cuda_device` (ignored by the FAKE backend). Returns ORION_E_NODEV if the
 * CUDA backend has no device/driver. `cfg` is copied. */
int orion_create(int cuda_device, const orion_config* cfg, orion_t* out);
/* Register a client before orion_start. At most one ORION_HP client and 15 ORION_BE clients.
 * Client ids are assigned 0,1,2,... in registration order (BE round-robin order, R11). */
int orion_register_client(orion_t h, int prio, int* client_id);
/* The CUstream (cast to void*) ops of this client run on; usable as torch.cuda.ExternalStream. */
int orion_client_stream(orion_t h, int client_id, void** cu_stream);
/* Start the scheduler thread (Listing 1, `run_scheduler`). */
int orion_start(orion_t h);
/* Non-blocking: copy *op into the client's queue. seq_out (optional) = the op's 0-based sequence
 * number within the client. ORION_E_AGAIN if the queue is full. */
int orion_submit(orion_t h, int client_id, const orion_op* op, uint64_t* seq_out);
/* Submit n ops as one batch (all or nothing: ORION_E_AGAIN if fewer than n slots are free). */
int orion_submit_n(orion_t h, int client_id, const orion_op* ops, uint32_t n, uint64_t* first_seq);
/* Block until every op the client submitted so far has completed on the GPU.
 * timeout_ns = 0 means no timeout. */
int orion_synchronize(orion_t h, int client_id, uint64_t timeout_ns);
/* Non-blocking progress: number of the client's ops completed so far. */
int orion_done_seq(orion_t h, int client_id, uint64_t* done);
/* Stop: let the scheduler drain every queue and outstanding op, then join it. */
int orion_stop(orion_t h);
/* Copy the binary log (header, op table, observation tape, decisions) into buf.
 * *written = bytes needed; ORION_E_NOMEM if cap is too small or the log overflowed. */
int orion_read_log(orion_t h, void* buf, size_t cap, size_t* written);
/* Scheduler counters: out[0]=iterations, [1]=HP launches, [2]=BE admits, [3]=BE defers,
 * [4]=memops, [5]=resets, [6]=launch errors, [7]=sum of launch-call ns. n = slots in out. */
int orion_stats(orion_t h, uint64_t* out, uint32_t n);
int orion_destroy(orion_t h);
const char* orion_strerror(int code);
/* After orion_stop: durations (ms) of the traced kernel's launches (trace_kernel_id_plus1), in
 * launch order. *n = number available (up to 8192); copies min(*n, cap) into ms_out. */
int orion_trace_read(orion_t h, float* ms_out, uint32_t cap, uint32_t* n);

/* ---------------------------------------------------------------------------------------------
 * Native client drivers (the bench's clients; C++ loops so no Python sits on the hot path).
 * ------------------------------------------------------------------------------------------- */

/* Open-loop request generator for an inference client. Request r is submitted at
 * start + arrivals_ns[r] (spin-wait); its ops are ops[0..n_ops) with per-request host pointers:
 * MEMCPY_H2D src += (r % in_cycle) * args[2], MEMCPY_D2H dst += (r % out_cycle) * args[2].
 * The first op of each request gets ORION_OPF_REQ_BEGIN and the last ORION_OPF_REQ_END.
 * On return t_arrival_ns[r] / t_done_ns[r] hold the scheduled arrival and the observed
 * completion (CLOCK_MONOTONIC ns, R19). */
int orion_run_requests(orion_t h, int client_id, const orion_op* ops, uint32_t n_ops,
                       const int64_t* arrivals_ns, uint32_t n_req, uint32_t in_cycle, uint32_t out_cycle,
                       int64_t* t_arrival_ns, int64_t* t_done_ns);

/* The "native" arm of R20 (P:1355-1360 reports Orion's overhead against direct execution): the
 * same open-loop request stream as orion_run_requests, but the calling thread launches every op
 * itself, in order, on the client's stream -- no ring, no scheduler, no policy. Only valid on an
 * instance that was never started (ORION_E_STATE otherwise) with a single registered client
 * in use; completion is observed through the same per-stream counters, so the latencies are
 * directly comparable with orion_run_requests. Arguments and outputs as orion_run_requests. */
int orion_run_requests_direct(orion_t h, int client_id, const orion_op* ops, uint32_t n_ops,
                              const int64_t* arrivals_ns, uint32_t n_req, uint32_t in_cycle, uint32_t out_cycle,
                              int64_t* t_arrival_ns, int64_t* t_done_ns);

/* Closed-loop training client: iteration i submits variant (i % n_variants) of
 * the op list (ops is n_variants x n_ops, row-major) and waits for it to complete before the
 * next. Runs until *stop != 0 (checked between iterations) or max_iters iterations (0 = no
 * limit). t_end_ns[i] (capacity cap_iters) = completion time of iteration i. *iters_out = count. */
int orion_run_iterations(orion_t h, int client_id, const orion_op* ops, uint32_t n_ops, uint32_t n_variants,
                         const volatile int32_t* stop, uint64_t max_iters, int64_t* t_end_ns,
                         uint64_t cap_iters, uint64_t* iters_out);

/* CLOCK_MONOTONIC now, ns (same clock as the drivers). */
int64_t orion_now_ns(void);

#ifdef __cplusplus
}
#endif
#endif /* ORION_H */
