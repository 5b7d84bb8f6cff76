/*
 * oracle/policy.c — CPU ORACLE (test infrastructure only) for Orion's scheduling policy.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg may load this.
 * It shares NO code with the product path (paper_conf_eurosys_stratimk24_b200/csrc): the
 * binary log format is re-implemented here from the format description in DESIGN.md §4.
 *
 * What it computes: Listing 1 of Strati et al., "Orion", EuroSys'24 (PAPER.md P:706-764,
 * §5.1.1), run as a replay over a recorded observation tape, with the readings
 * R1-R15, R27 of DESIGN.md §3 made explicit. Step numbers in comments
 * refer to SURVEY.md §8(c).1, listing line numbers (L5 ...) to Listing 1.
 *
 * Pins (tests/test_oracle_policy.py): worked examples WE1-WE6 (tests/golden/we*.txt, derived
 * by hand from Listing 1), brute-force invariants I1-I11 over every tape of tiny traces.
 * The faithfulness of the readings to the authors' code is "parity unpinned" (no code exists).
 *
 * Slow by design: plain loops, no cleverness beyond the quiescence jump (which is exact, see
 * DESIGN.md §4.3).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <stdio.h>

#define MAXC 16
#ifndef ORACLE_MUTANT
#define ORACLE_MUTANT 0   /* tests compile deliberate mistakes (1..10) to prove the pins catch them */
#endif
#define KIND_KERNEL 0
#define CLS_U 0
#define CLS_C 1
#define CLS_M 2
#define OPF_REQ_BEGIN 1
#define OPF_REQ_END 2

/* reading switches */
#define F_HP_BUSY_REQUEST 1u
#define F_HP_REF_ALL 2u
#define F_HP_UNKNOWN_STRICT 4u
#define F_THROTTLE_ONLY_HP_BUSY 8u
#define F_FREE_SMS 16u
#define F_NO_PRIORITY 32u        /* stream priorities only: no effect on decisions */
#define F_NO_PROFILE_TEST 64u    /* ablation (Fig. 14): skip L28 */
#define F_NO_SM_TEST 128u        /* ablation: skip L27 */
#define F_NO_THROTTLE 256u       /* ablation / Streams baselines: skip L12-L16 */

/* decision kinds */
enum { D_HP_LAUNCH = 1, D_PASS = 2, D_ADMIT_IDLE = 3, D_ADMIT_COLOC = 4, D_DEFER_SM = 5,
       D_DEFER_PROFILE = 6, D_DEFER_DUR = 7, D_RESET = 8 };
enum { R_NONE = 0, R_SM = 1, R_PROFILE = 2, R_DUR = 3 };
enum { T_VIS = 1, T_DONE = 2 };

typedef struct {
  uint32_t kernel_id; uint16_t kind; uint8_t opflags; uint8_t cls;
  uint32_t sm_needed; uint64_t dur_ns;
} o_op;

typedef struct { uint64_t k; uint32_t type; uint32_t client; uint64_t value; } o_tape;

typedef struct {
  uint64_t k; uint8_t kind; uint8_t client; uint32_t kernel_id; uint64_t seq; int64_t be_dur;
} o_dec;

typedef struct {
  uint32_t n_clients, num_sms, sm_thr, flags;
  uint64_t dur_thr;
  int32_t hp;                 /* client index of the HP client, -1 if none */
  uint32_t prio[MAXC];
  uint64_t k_end;
  uint64_t n_ops[MAXC];
  o_op *ops[MAXC];
  int n_be, be_idx[MAXC];     /* BE clients in registration order (R11) */
  uint64_t n_tape; o_tape *tape;
} o_cfg;

typedef struct {
  uint64_t vis[MAXC], done[MAXC], popped[MAXC];
  o_op hp_ref;
  int64_t be_dur;
  uint64_t ld_seq[MAXC]; uint8_t ld_reason[MAXC];
} o_state;

typedef struct { o_dec *d; uint64_t n, cap; } o_out;

static int out_push(o_out *o, uint64_t k, int kind, int client, uint32_t kid, uint64_t seq, int64_t be_dur) {
  if (o->n == o->cap) {
    uint64_t nc = o->cap ? o->cap * 2 : 1024;
    o_dec *nd = (o_dec *)realloc(o->d, nc * sizeof(o_dec));
    if (!nd) return -1;
    o->d = nd; o->cap = nc;
  }
  o_dec *r = &o->d[o->n++];
  r->k = k; r->kind = (uint8_t)kind; r->client = (uint8_t)client; r->kernel_id = kid; r->seq = seq; r->be_dur = be_dur;
  return 0;
}

/* ---------------- little-endian readers ---------------- */
static uint64_t rd64(const uint8_t *p) { uint64_t v = 0; for (int i = 7; i >= 0; i--) v = (v << 8) | p[i]; return v; }
static uint32_t rd32(const uint8_t *p) { return (uint32_t)p[0] | ((uint32_t)p[1] << 8) | ((uint32_t)p[2] << 16) | ((uint32_t)p[3] << 24); }
static uint16_t rd16(const uint8_t *p) { return (uint16_t)(p[0] | (p[1] << 8)); }
static void wr64(uint8_t *p, uint64_t v) { for (int i = 0; i < 8; i++) { p[i] = (uint8_t)(v & 0xff); v >>= 8; } }
static void wr32(uint8_t *p, uint32_t v) { for (int i = 0; i < 4; i++) { p[i] = (uint8_t)(v & 0xff); v >>= 8; } }

#define HDR_BYTES 240
#define OP_BYTES 24
#define TAPE_BYTES 24
#define DEC_BYTES 32

static void cfg_free(o_cfg *c) {
  for (int i = 0; i < MAXC; i++) free(c->ops[i]);
  free(c->tape);
  memset(c, 0, sizeof(*c));
}

/* Parse header + op tables (+ tape if present). Returns 0 or negative error. */
static int parse_log(const uint8_t *b, size_t len, o_cfg *c, int want_tape) {
  memset(c, 0, sizeof(*c));
  if (len < HDR_BYTES || memcmp(b, "ORIONLG1", 8) != 0) return -1;
  if (rd32(b + 8) != 1) return -2;
  c->n_clients = rd32(b + 12);
  c->num_sms = rd32(b + 16);
  c->sm_thr = rd32(b + 20);
  c->dur_thr = rd64(b + 24);
  c->flags = rd32(b + 32);
  c->hp = (int32_t)rd32(b + 36);
  if (c->n_clients > MAXC) return -3;
  for (int i = 0; i < MAXC; i++) c->prio[i] = rd32(b + 40 + 4 * i);
  c->k_end = rd64(b + 104);
  for (int i = 0; i < MAXC; i++) c->n_ops[i] = rd64(b + 112 + 8 * i);
  size_t off = HDR_BYTES;
  c->n_be = 0;
  for (uint32_t i = 0; i < c->n_clients; i++) {
    if (c->prio[i] == 1) c->be_idx[c->n_be++] = (int)i;
    uint64_t n = c->n_ops[i];
    if (off + n * OP_BYTES > len) { cfg_free(c); return -4; }
    c->ops[i] = (o_op *)calloc(n ? n : 1, sizeof(o_op));
    for (uint64_t j = 0; j < n; j++) {
      const uint8_t *p = b + off + j * OP_BYTES;
      o_op *o = &c->ops[i][j];
      o->kernel_id = rd32(p); o->kind = rd16(p + 4); o->opflags = p[6]; o->cls = p[7];
      o->sm_needed = rd32(p + 8); o->dur_ns = rd64(p + 16);
    }
    off += n * OP_BYTES;
  }
  if (!want_tape) return 0;
  if (off + 8 > len) { cfg_free(c); return -5; }
  c->n_tape = rd64(b + off); off += 8;
  if (off + c->n_tape * TAPE_BYTES > len) { cfg_free(c); return -6; }
  c->tape = (o_tape *)calloc(c->n_tape ? c->n_tape : 1, sizeof(o_tape));
  for (uint64_t j = 0; j < c->n_tape; j++) {
    const uint8_t *p = b + off + j * TAPE_BYTES;
    c->tape[j].k = rd64(p); c->tape[j].type = rd32(p + 8); c->tape[j].client = rd32(p + 12); c->tape[j].value = rd64(p + 16);
  }
  return 0;
}

/* ---------------- Listing 1 ---------------- */

/* differ(a, b): a = HP class, b = BE class. R4 (symmetric unknown optimism);
 * switch HP_UNKNOWN_STRICT keeps only BE-unknown optimism. */
static int differ(const o_cfg *c, int a, int b) {
  if (c->flags & F_NO_PROFILE_TEST) return 1;
  if (c->flags & F_HP_UNKNOWN_STRICT) return b == CLS_U || (a != CLS_U && a != b);
  if (ORACLE_MUTANT == 3) return a != b;   /* 'unknown' treated as a class of its own */
  return a == CLS_U || b == CLS_U || a != b;
}

/* thr(h): R5. STATIC = SM_THRESHOLD; FREE_SMS: be.sm + hp.sm <= num_sms. */
static int64_t thr(const o_cfg *c, const o_op *h) {
  if (c->flags & F_NO_SM_TEST) return INT64_MAX;
  if (c->flags & F_FREE_SMS) {
    int64_t t = (int64_t)c->num_sms - (int64_t)h->sm_needed + 1;
    return t < 0 ? 0 : t;
  }
  return (int64_t)c->sm_thr;
}

/* hp_busy (R2): default kernel-granular "some popped HP op not yet observed complete". */
static int hp_busy_now(const o_cfg *c, const o_state *s) {
  if (c->hp < 0) return 0;
  int h = c->hp;
  if (ORACLE_MUTANT == 7) return 0;
  if (!(c->flags & F_HP_BUSY_REQUEST)) return s->done[h] < s->popped[h];
  /* HP_BUSY_REQUEST: a popped REQ_BEGIN op whose request's REQ_END op is not done. */
  uint64_t begin = UINT64_MAX;
  for (uint64_t i = 0; i < c->n_ops[h]; i++) {
    const o_op *o = &c->ops[h][i];
    if (o->opflags & OPF_REQ_BEGIN) begin = i;
    if ((o->opflags & OPF_REQ_END) && begin != UINT64_MAX) {
      /* request spans [begin, i] */
      if ((ORACLE_MUTANT == 10 ? i < s->popped[h] : begin < s->popped[h]) && i >= s->done[h]) return 1;
      begin = UINT64_MAX;
    }
  }
  if (begin != UINT64_MAX && begin < s->popped[h]) return 1;  /* open request (REQ_END not in table) */
  return 0;
}

static const o_op U_PROF = {0xFFFFFFFFu, 0, 0, CLS_U, 0, 0};

/* schedule_be (L23-L30) with reason (R27: SM before PROFILE). Returns reason R_NONE if admissible. */
static int schedule_be(const o_cfg *c, const o_state *s, int hp_busy, const o_op *op) {
  if (!hp_busy) return R_NONE;                                    /* L25-L26 */
  if (!(c->flags & F_HP_REF_ALL) || c->hp < 0 || s->done[c->hp] >= s->popped[c->hp]) {
    const o_op *h = &s->hp_ref;                                   /* R3: sticky last popped HP op */
    if (ORACLE_MUTANT == 1 ? !((int64_t)op->sm_needed <= thr(c, h)) : !((int64_t)op->sm_needed < thr(c, h))) return R_SM; /* L27 */
    if (ORACLE_MUTANT == 2 ? differ(c, h->cls, op->cls) : !differ(c, h->cls, op->cls)) return R_PROFILE; /* L28 (R1: op_lp == op_be) */
    return R_NONE;
  }
  int h = c->hp, any_sm = 0, any_prof = 0;
  for (uint64_t i = (ORACLE_MUTANT == 9 ? s->popped[h] - 1 : s->done[h]); i < s->popped[h]; i++) {
    const o_op *ho = &c->ops[h][i];
    const o_op *hr = ho->kind == KIND_KERNEL ? ho : &U_PROF;
    if (!((int64_t)op->sm_needed < thr(c, hr))) any_sm = 1;
    else if (!differ(c, hr->cls, op->cls)) any_prof = 1;
  }
  if (any_sm) return R_SM;
  if (any_prof) return R_PROFILE;
  return R_NONE;
}

static int all_be_drained(const o_cfg *c, const o_state *s) {   /* R10: be_submitted.finished() */
  for (int t = 0; t < c->n_be; t++) { int j = c->be_idx[t]; if (s->done[j] != s->popped[j]) return 0; }
  return 1;
}

/* One scheduler iteration k. Returns 1 if any state changed. */
static int iterate(const o_cfg *c, o_state *s, uint64_t k, o_out *out, int *err) {
  int changed = 0;
  int hp_busy = hp_busy_now(c, s);                                          /* step 1 */
  if (c->hp >= 0 && s->popped[c->hp] < s->vis[c->hp]) {                     /* step 2: L5, L7 */
    int h = c->hp;
    const o_op *op = &c->ops[h][s->popped[h]];
    if (out_push(out, k, op->kind == KIND_KERNEL ? D_HP_LAUNCH : D_PASS, h, op->kernel_id, s->popped[h], s->be_dur)) *err = 1;
    s->popped[h]++;                                                         /* L8 launch */
    s->hp_ref = op->kind == KIND_KERNEL ? *op : U_PROF;                     /* R3 */
    hp_busy = 1;                                                            /* L9 */
    changed = 1;
  }
  for (int t = 0; t < c->n_be; t++) {                                       /* step 3, R11 */
    int j = c->be_idx[ORACLE_MUTANT == 8 ? (uint64_t)t : (k + (uint64_t)t) % (uint64_t)c->n_be];
    if (s->popped[j] == s->vis[j]) continue;                                /* L10 */
    uint64_t seq = s->popped[j];
    const o_op *op = &c->ops[j][seq];                                       /* L6 peek */
    if (op->kind != KIND_KERNEL) {                                          /* R14 memop pass-through */
      s->popped[j]++;
      if (out_push(out, k, D_PASS, j, op->kernel_id, seq, s->be_dur)) *err = 1;
      changed = 1;
      continue;
    }
    int reason = schedule_be(c, s, hp_busy, op);                            /* L11 */
    int sched = reason == R_NONE;
    int throttle = !(c->flags & F_NO_THROTTLE) && (!(c->flags & F_THROTTLE_ONLY_HP_BUSY) || hp_busy);   /* R7; ablation */
    if (throttle && (ORACLE_MUTANT == 4 ? s->be_dur >= (int64_t)c->dur_thr : s->be_dur > (int64_t)c->dur_thr)) { /* L12 (R6 strict >) */
      if (ORACLE_MUTANT == 5 ? 1 : all_be_drained(c, s)) {                  /* L13 */
        s->be_dur = 0;                                                      /* L14 */
        if (out_push(out, k, D_RESET, j, 0xFFFFFFFFu, UINT64_MAX, 0)) *err = 1;
        changed = 1;
      } else if (sched) {                                                   /* L15-L16 */
        sched = 0; reason = R_DUR;
      }
    }
    if (sched) {                                                            /* L17-L21 */
      s->popped[j]++;
      if (ORACLE_MUTANT != 6) s->be_dur += (int64_t)op->dur_ns;
      if (out_push(out, k, hp_busy ? D_ADMIT_COLOC : D_ADMIT_IDLE, j, op->kernel_id, seq, s->be_dur)) *err = 1;
      changed = 1;
    } else if (!(s->ld_seq[j] == seq && s->ld_reason[j] == reason)) {
      int kind = reason == R_SM ? D_DEFER_SM : reason == R_PROFILE ? D_DEFER_PROFILE : D_DEFER_DUR;
      if (out_push(out, k, kind, j, op->kernel_id, seq, s->be_dur)) *err = 1;
      s->ld_seq[j] = seq; s->ld_reason[j] = (uint8_t)reason;
      changed = 1;
    }
  }
  return changed;
}

static void state_init(o_state *s) {
  memset(s, 0, sizeof(*s));
  s->hp_ref = U_PROF;
  for (int i = 0; i < MAXC; i++) { s->ld_seq[i] = UINT64_MAX; s->ld_reason[i] = 0xff; }
}

static int apply_tape(o_state *s, const o_tape *t) {
  if (t->client >= MAXC) return -1;
  if (t->type == T_VIS) s->vis[t->client] = t->value;
  else if (t->type == T_DONE) s->done[t->client] = t->value;
  else return -1;
  return 0;
}

/* Replay: run iterations 0..k_end-1, jumping over quiescent stretches (exact: an iteration
 * that changes no state is a fixed point until the next tape stamp). */
static int replay(const o_cfg *c, o_out *out) {
  o_state s; state_init(&s);
  uint64_t ti = 0, k = 0;
  int err = 0;
  while (k < c->k_end) {
    while (ti < c->n_tape && c->tape[ti].k == k) { if (apply_tape(&s, &c->tape[ti])) return -10; ti++; }
    if (ti < c->n_tape && c->tape[ti].k < k) return -11;   /* tape not sorted */
    int changed = iterate(c, &s, k, out, &err);
    if (err) return -12;
    if (changed) k++;
    else if (ti < c->n_tape) k = c->tape[ti].k;
    else break;
  }
  return 0;
}

static size_t encode_decs(const o_out *o, uint8_t *buf, size_t cap) {
  size_t need = 8 + (size_t)o->n * DEC_BYTES;
  if (!buf || cap < need) return need;
  wr64(buf, o->n);
  for (uint64_t i = 0; i < o->n; i++) {
    uint8_t *p = buf + 8 + i * DEC_BYTES;
    memset(p, 0, DEC_BYTES);
    wr64(p, o->d[i].k); p[8] = o->d[i].kind; p[9] = o->d[i].client;
    wr32(p + 12, o->d[i].kernel_id); wr64(p + 16, o->d[i].seq); wr64(p + 24, (uint64_t)o->d[i].be_dur);
  }
  return need;
}

/* Public: replay a log (header + op table + tape; any decision section after it is ignored).
 * Writes u64 n + n decision records into out. Returns 0, or <0 on error; *written = bytes needed. */
int oracle_replay(const uint8_t *log, size_t len, uint8_t *out, size_t cap, size_t *written) {
  o_cfg c; int r = parse_log(log, len, &c, 1);
  if (r) return r;
  o_out o = {0};
  r = replay(&c, &o);
  if (r == 0) {
    size_t need = encode_decs(&o, out, cap);
    if (written) *written = need;
    if (cap < need) r = -20;
  }
  free(o.d); cfg_free(&c);
  return r;
}

/* ======================= brute force over tapes (invariants I1-I11) ======================= */

typedef struct {
  const o_cfg *c;
  uint64_t n_paths, n_nodes, max_nodes;
  int64_t max_dur;
  char *err; size_t errcap;
  int failed;
  /* current tape path for diagnostics and I9 */
  o_tape path[512]; int plen;
} o_brute;

static void bfail(o_brute *b, const char *what, uint64_t k) {
  if (b->failed) return;
  b->failed = 1;
  if (b->err && b->errcap) snprintf(b->err, b->errcap, "invariant %s violated at k=%llu (path len %d)", what, (unsigned long long)k, b->plen);
}

/* Check invariants on the records emitted by one iteration (pre = state before, post = after). */
static void check_iter(o_brute *b, const o_state *pre, const o_state *post, const o_dec *d, uint64_t nd, uint64_t k, int hp_busy_pre) {
  const o_cfg *c = b->c;
  int hp_launches = 0, reset_seen = 0;
  int64_t be_dur = pre->be_dur;
  for (uint64_t i = 0; i < nd; i++) {
    const o_dec *r = &d[i];
    if (r->client == (uint8_t)c->hp && (r->kind == D_HP_LAUNCH || r->kind == D_PASS)) {
      hp_launches++;
      if (i != 0) bfail(b, "I1 (HP launch not first in iteration)", k);       /* I1 */
      if (r->seq != pre->popped[c->hp]) bfail(b, "I2 (HP FIFO)", k);          /* I2 */
      continue;
    }
    if (r->kind == D_RESET) {
      if (!(be_dur > (int64_t)c->dur_thr)) bfail(b, "I10 (RESET below threshold)", k);
      if (!all_be_drained(c, pre)) bfail(b, "I10 (RESET not drained)", k);  /* popped unchanged since only RESETs/defers... */
      be_dur = 0; reset_seen = 1;
      continue;
    }
    const o_op *op = &c->ops[r->client][r->seq];
    if (r->seq >= pre->vis[r->client] && r->kind != D_DEFER_SM && r->kind != D_DEFER_PROFILE && r->kind != D_DEFER_DUR)
      bfail(b, "I7 (launch before visible)", k);
    if (r->kind == D_PASS) {
      if (op->kind == KIND_KERNEL) bfail(b, "I11 (kernel passed)", k);
      if (r->be_dur != be_dur) bfail(b, "I11 (memop counted)", k);
      continue;
    }
    if (r->kind == D_DEFER_SM || r->kind == D_DEFER_PROFILE || r->kind == D_DEFER_DUR) {
      if (op->kind != KIND_KERNEL) bfail(b, "I11 (memop deferred)", k);
      continue;
    }
    if (r->kind == D_ADMIT_COLOC || r->kind == D_ADMIT_IDLE) {
      if (op->kind != KIND_KERNEL) bfail(b, "I11 (memop admitted)", k);
      /* I3: co-location admission satisfies the SM and profile tests against the reference HP op */
      if (r->kind == D_ADMIT_COLOC && !(c->flags & F_HP_REF_ALL)) {
        const o_op *h = &post->hp_ref;
        if (!((int64_t)op->sm_needed < thr(c, h) && differ(c, h->cls, op->cls))) bfail(b, "I3 (coloc admit violates SM/profile)", k);
      }
      /* I3 under HP_REF_ALL (R3 switch): the tests hold against every HP op in flight at the
         admission, i.e. seq in [done sampled this iteration, popped after this iteration's HP
         launch); with none in flight (a busy request between ops) against the last popped one */
      if (r->kind == D_ADMIT_COLOC && (c->flags & F_HP_REF_ALL)) {
        const int hh = c->hp;
        if (pre->done[hh] >= post->popped[hh]) {
          const o_op *h = &post->hp_ref;
          if (!((int64_t)op->sm_needed < thr(c, h) && differ(c, h->cls, op->cls))) bfail(b, "I3 (coloc admit violates SM/profile, REF_ALL)", k);
        } else {
          for (uint64_t q = pre->done[hh]; q < post->popped[hh]; q++) {
            const o_op *hq = &c->ops[hh][q];
            o_op hu = {0u, 0, 0, CLS_U, 0, 0};
            const o_op *h = hq->kind == KIND_KERNEL ? hq : &hu;
            if (!((int64_t)op->sm_needed < thr(c, h) && differ(c, h->cls, op->cls))) bfail(b, "I3 (coloc admit violates SM/profile vs an in-flight HP op)", k);
          }
        }
      }
      /* I4: admission happens with be_dur <= thr, or after a RESET in this iteration */
      int throttle = !(c->flags & F_NO_THROTTLE) && (!(c->flags & F_THROTTLE_ONLY_HP_BUSY) || hp_busy_pre || hp_launches);
      if (throttle && !(be_dur <= (int64_t)c->dur_thr) && !reset_seen) bfail(b, "I4 (admit over threshold)", k);
      be_dur += (int64_t)op->dur_ns;
      if (r->be_dur != be_dur) bfail(b, "I4 (be_dur accounting)", k);
      continue;
    }
  }
  if (hp_launches > 1) bfail(b, "I2 (more than one HP launch per iteration)", k);
  /* I1: an HP op visible at k (earlier ones popped) is launched at k */
  if (c->hp >= 0 && pre->popped[c->hp] < pre->vis[c->hp] && hp_launches != 1) bfail(b, "I1 (visible HP op not launched)", k);
  /* I5: be_dur <= thr + max_dur always (overshoot bound) */
  const int throttled = !(c->flags & (F_THROTTLE_ONLY_HP_BUSY | F_NO_THROTTLE));
  if (throttled && post->be_dur > (int64_t)c->dur_thr + b->max_dur) bfail(b, "I5 (overshoot bound)", k);
  /* I6: outstanding profiled BE work <= thr + max_dur */
  if (throttled) {
    int64_t outst = 0;
    for (int t = 0; t < c->n_be; t++) {
      int j = c->be_idx[t];
      for (uint64_t q = post->done[j]; q < post->popped[j]; q++) if (c->ops[j][q].kind == KIND_KERNEL) outst += (int64_t)c->ops[j][q].dur_ns;
    }
    if (outst > (int64_t)c->dur_thr + b->max_dur) bfail(b, "I6 (outstanding BE work bound)", k);
  }
  /* I7: FIFO, each op at most once */
  for (uint32_t i = 0; i < c->n_clients; i++) if (post->popped[i] > post->vis[i] || post->popped[i] < pre->popped[i]) bfail(b, "I7 (FIFO/visibility)", k);
}

static int all_finished(const o_cfg *c, const o_state *s) {
  for (uint32_t i = 0; i < c->n_clients; i++) if (s->done[i] != c->n_ops[i] || s->popped[i] != c->n_ops[i]) return 0;
  return 1;
}

/* I8 liveness: from state s, with every op made visible and all completions delivered as soon as
 * launched, the policy launches everything within a bounded number of iterations. */
static void check_liveness(o_brute *b, const o_state *s0, uint64_t k0) {
  const o_cfg *c = b->c;
  o_state s = *s0;
  o_out o = {0}; int err = 0;
  uint64_t total = 0;
  for (uint32_t i = 0; i < c->n_clients; i++) { s.vis[i] = c->n_ops[i]; total += c->n_ops[i]; }
  for (uint64_t it = 0; it < 4 * total + 16; it++) {
    for (uint32_t i = 0; i < c->n_clients; i++) s.done[i] = s.popped[i];
    if (all_finished(c, &s)) { free(o.d); return; }
    iterate(c, &s, k0 + it, &o, &err);
  }
  free(o.d);
  bfail(b, "I8 (liveness)", k0);
}

/* I9 determinism: replaying the path's tape twice yields the same log. */

static void brute_rec(o_brute *b, o_state *s, uint64_t k, int last_changed);

static void brute_step(o_brute *b, const o_state *s_in, uint64_t k, const o_tape *ev, int nev) {
  if (b->failed) return;
  if (b->max_nodes && b->n_nodes >= b->max_nodes) return;
  b->n_nodes++;
  o_state s = *s_in;
  int save = b->plen;
  for (int i = 0; i < nev; i++) {
    apply_tape(&s, &ev[i]);
    if (b->plen < 512) { b->path[b->plen] = ev[i]; b->path[b->plen].k = k; b->plen++; }
  }
  o_state pre = s;
  o_out o = {0}; int err = 0;
  int hp_busy_pre = hp_busy_now(b->c, &pre);
  int changed = iterate(b->c, &s, k, &o, &err);
  check_iter(b, &pre, &s, o.d, o.n, k, hp_busy_pre);
  free(o.d);
  if (!b->failed) brute_rec(b, &s, k + 1, changed);
  b->plen = save;
}

static void brute_rec(o_brute *b, o_state *s, uint64_t k, int last_changed) {
  const o_cfg *c = b->c;
  if (b->failed) return;
  if (all_finished(c, s)) { b->n_paths++; return; }
  /* enabled observation changes: next VIS per client, DONE+1 per stream with popped > done */
  o_tape en[2 * MAXC]; int ne = 0;
  for (uint32_t i = 0; i < c->n_clients; i++) {
    if (s->vis[i] < c->n_ops[i]) { en[ne].type = T_VIS; en[ne].client = i; en[ne].value = s->vis[i] + 1; ne++; }
    if (s->done[i] < s->popped[i]) { en[ne].type = T_DONE; en[ne].client = i; en[ne].value = s->done[i] + 1; ne++; }
  }
  if (last_changed) check_liveness(b, s, k);
  uint32_t nsub = 1u << ne;
  /* after a quiescent iteration the next observation may land at any later iteration; only
   * its residue mod n_be matters (BE rotation R11), so branch over those stamps too. */
  int nk = (!last_changed && c->n_be > 1) ? c->n_be : 1;
  for (int dk = 0; dk < nk; dk++)
    for (uint32_t m = last_changed ? 0 : 1; m < nsub; m++) {
      o_tape ev[2 * MAXC]; int nev = 0;
      for (int i = 0; i < ne; i++) if (m & (1u << i)) ev[nev++] = en[i];
      brute_step(b, s, k + (uint64_t)dk, ev, nev);
      if (b->failed) return;
    }
  if (ne == 0 && !last_changed) {
    /* stuck: nothing observable can change and the policy is at a fixed point, yet not finished */
    bfail(b, "I8 (deadlock)", k);
  }
}

/* Public: exhaustive DFS over all observation tapes of the trace in `hdr` (header + op table;
 * k_end and tape ignored). Checks I1-I8, I10, I11 on every transition. Returns 0 if all hold,
 * 1 if an invariant failed (message in err), <0 on parse error. */
int oracle_brute(const uint8_t *hdr, size_t len, uint64_t max_nodes, uint64_t *n_paths, uint64_t *n_nodes, char *err, size_t errcap) {
  o_cfg c; int r = parse_log(hdr, len, &c, 0);
  if (r) return r;
  o_brute b; memset(&b, 0, sizeof(b));
  b.c = &c; b.err = err; b.errcap = errcap; b.max_nodes = max_nodes;
  if (err && errcap) err[0] = 0;
  for (uint32_t i = 0; i < c.n_clients; i++)
    for (uint64_t j = 0; j < c.n_ops[i]; j++)
      if (c.prio[i] == 1 && c.ops[i][j].kind == KIND_KERNEL && (int64_t)c.ops[i][j].dur_ns > b.max_dur) b.max_dur = (int64_t)c.ops[i][j].dur_ns;
  o_state s; state_init(&s);
  brute_rec(&b, &s, 0, 1);
  if (n_paths) *n_paths = b.n_paths;
  if (n_nodes) *n_nodes = b.n_nodes;
  cfg_free(&c);
  return b.failed ? 1 : 0;
}

/* Public: decisions per second of the replay (cpu_baseline of bench.py). */
int oracle_replay_count(const uint8_t *log, size_t len, uint64_t *n_decisions) {
  o_cfg c; int r = parse_log(log, len, &c, 1);
  if (r) return r;
  o_out o = {0};
  r = replay(&c, &o);
  if (n_decisions) *n_decisions = o.n;
  free(o.d); cfg_free(&c);
  return r;
}
