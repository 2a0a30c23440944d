/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously correct CPU implementation of what the Proteus hot
 * path computes (Ahmad et al., ASPLOS '24; citations "P:a-b" are lines of
 * PAPER.md).  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it.  It shares no code, header, table or
 * constant generator with paper_conf_asplos_ahmadgfwsw24_b200/csrc, and the
 * product path never calls it.
 *
 * Contents
 *   orc_capacity          capacity estimate P, readings C4-C7
 *   orc_family_lp         per-family assignment LP (Eqs. 2-6 with x fixed) by
 *                         exhaustive vertex enumeration; lexicographic
 *                         (served, accsum) objective (reading C1)
 *   orc_score_placement   Eq. 7 for one placement + canonical z (reading C10)
 *   orc_solve_enum        exhaustive search over every placement, flat
 *                         mixed-radix (mode 0) or per-type multiset (mode 1),
 *                         canonical lowest-index argmax (reading C9)
 *   orc_solve_factored    exhaustive per-family count-vector search + budget DP
 *                         + lexicographically-smallest reconstruction (mode 2)
 *   orc_route_swrr        literal smooth weighted round-robin router (R8)
 *   orc_replay_device     event-driven simulation of §5 adaptive batching on one
 *                         device, readings R1-R13
 *   orc_replay_device_nexus / _aimd
 *                         §8(f2) baseline batchers of §6.4:
 *                         Nexus early drop and Clipper AIMD, work-conserving,
 *                         event-driven; readings R14-R15
 *   orc_replay            route + simulate every (device, scenario) lane
 *   orc_replay_device_epochs / orc_replay_epochs
 *                         §8(f4) closed loop: one allocation per epoch (the
 *                         per-second re-solve), epoch-aware queues; F1-F4
 *   orc_pareto            system capacity vs capacity-weighted accuracy of
 *                         every placement of one family's variants, and its
 *                         Pareto frontier (Fig. 1b), readings P1-P4
 *
 * The oracle never uses the packed 64-bit score of the CUDA path: objective
 * values are (served, accsum) pairs of int64 compared lexicographically.
 *
 * Parity pins: tests/test_oracle_*.py (hand-worked H1/G1 fixtures, the literal
 * LP of Eqs. 2-6 in exact rationals, fractional brute force, closed forms of §5,
 * invariants).  Nothing here is "parity unpinned" except the readings listed as
 * such in DESIGN.md (C1's delta-loop, C11).
 */
#include <pthread.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <unistd.h>

#define ORC_MAXK 64     /* kinds in one family LP */
#define ORC_MAXD 64     /* devices */
#define ORC_MAXQ 32     /* families */
#define ORC_MAXT 8      /* device types */

typedef struct { int64_t served, accsum; } orc_val;

static int val_gt(orc_val a, orc_val b) {
  return a.served > b.served || (a.served == b.served && a.accsum > b.accsum);
}
static int val_eq(orc_val a, orc_val b) { return a.served == b.served && a.accsum == b.accsum; }
static orc_val val_add(orc_val a, orc_val b) { orc_val r = {a.served + b.served, a.accsum + b.accsum}; return r; }

static int ncores(int n) {
  if (n > 0) return n;
  long c = sysconf(_SC_NPROCESSORS_ONLN);
  return c > 0 ? (int)c : 1;
}

/* ------------------------------------------------------------------ a1 -- */
/* P:908-946 "Estimation of throughput capacity".  For each (type t, variant m):
 *   depth   = the largest b such that batches 1..b all fit in memory (lat != 0), C7
 *   b*      = the largest b <= depth with 2 * lat(b) <= SLO (C5: non-strict), C6
 *   P       = floor(b* * 10^6 / lat(b*)) QPS (C4), 0 when no such b.
 * lat is int32[T][M][bmax], entry [t][m][b-1]; slo_m is the SLO of m's family. */
int orc_capacity(int T, int M, int bmax, const int32_t *lat, const int32_t *slo_m,
                 int32_t *P, int32_t *bstar, int32_t *depth) {
  for (int t = 0; t < T; t++)
    for (int m = 0; m < M; m++) {
      const int32_t *row = lat + ((size_t)t * M + m) * bmax;
      int dep = 0;
      while (dep < bmax && row[dep] > 0) dep++;
      int bs = 0;
      for (int b = 1; b <= dep; b++)
        if (2LL * row[b - 1] <= (int64_t)slo_m[m]) bs = b;
      P[t * M + m] = bs ? (int32_t)(((int64_t)bs * 1000000LL) / row[bs - 1]) : 0;
      if (bstar) bstar[t * M + m] = bs;
      if (depth) depth[t * M + m] = dep;
    }
  return 0;
}

/* ---------------------------------------------------------- a3/a4 (LP) -- */
/* Eqs. 2-6 with the placement x fixed separate per family q (each device hosts
 * at most one variant, Eq. 1, and serves only its variant's family, Eq. 3).
 * Writing z_i for the QPS the i-th hosting device serves, Eq. 5 is
 * 0 <= z_i <= cap_i and Eqs. 2 + 4 give sum_i z_i <= s_q (y_i = z_i / s_q).
 * Reading C1 relaxes Eq. 6 (sum z = s) to: first maximise served = sum z, then
 * a_q = sum_i A_i z_i (Eq. 7 with reading C2).
 *
 * An LP optimum is attained at a vertex of the feasible polytope (and on the
 * optimal face of the first objective, at a vertex of that face, which is a
 * vertex of the polytope).  A vertex of {0 <= z <= cap, sum z <= s} has every
 * z_i at 0 or cap_i except at most one coordinate, which then makes sum z = s.
 * We enumerate all of them.  Devices with identical (A, cap) are grouped into
 * kinds of multiplicity mult; u_i = number of kind-i devices at z = cap_i. */
typedef struct {
  int nk;
  const int64_t *A, *cap;
  const int32_t *mult;
  int64_t s;
  int32_t u[ORC_MAXK];
  orc_val best;
} lp_ctx;

static void lp_consider(lp_ctx *c, int64_t served, int64_t acc) {
  orc_val v = {served, acc};
  if (val_gt(v, c->best)) c->best = v;
}

static void lp_rec(lp_ctx *c, int i, int64_t S, int64_t acc) {
  if (S > c->s) return; /* adding more only raises S: no feasible vertex below */
  if (i == c->nk) {
    lp_consider(c, S, acc); /* every coordinate at a bound */
    for (int j = 0; j < c->nk; j++) /* one coordinate strictly inside, budget tight */
      if (c->u[j] < c->mult[j]) {
        int64_t f = c->s - S;
        if (f >= 0 && f <= c->cap[j]) lp_consider(c, c->s, acc + f * c->A[j]);
      }
    return;
  }
  for (int u = 0; u <= c->mult[i]; u++) {
    c->u[i] = u;
    lp_rec(c, i + 1, S + (int64_t)u * c->cap[i], acc + (int64_t)u * c->cap[i] * c->A[i]);
  }
}

int orc_family_lp(int nk, const int64_t *A, const int64_t *cap, const int32_t *mult, int64_t s,
                  int64_t *served, int64_t *accsum) {
  if (nk < 0 || nk > ORC_MAXK || s < 0) return -1;
  lp_ctx c;
  memset(&c, 0, sizeof c);
  c.nk = nk; c.A = A; c.cap = cap; c.mult = mult; c.s = s;
  c.best.served = -1; c.best.accsum = -1;
  lp_rec(&c, 0, 0, 0);
  *served = c.best.served;
  *accsum = c.best.accsum;
  return 0;
}

/* ------------------------------------------------------------- problem -- */
typedef struct {
  int32_t T, Q, M, D;
  const int32_t *V;        /* [Q] */
  const int32_t *acc;      /* [M] accuracy, 1e-6 units */
  const int32_t *P;        /* [T][M] capacity, from orc_capacity */
  const int32_t *dev_type; /* [D] */
  const int32_t *s;        /* [Q] demand QPS */
} orc_problem;

typedef struct {
  int64_t served, accsum, unmet;
  uint64_t index;          /* canonical index (modes 0/1); UINT64_MAX for mode 2 */
  uint64_t n_candidates;
  int32_t eff;             /* floor(accsum / served), reading C3 */
  int32_t pad;
} orc_result;

static void fam_of(const orc_problem *p, int32_t *fam, int32_t *off) {
  int m = 0;
  for (int q = 0; q < p->Q; q++) {
    off[q] = m;
    for (int v = 0; v < p->V[q]; v++) fam[m++] = q;
  }
}

/* Eq. 7 for one placement (option[d] = 0 idle, else 1 + variant index m):
 * per family, group the hosting devices into (A, cap) kinds and solve the LP. */
static orc_val family_value(const orc_problem *p, const int32_t *fam, int q, const int32_t *option) {
  int64_t A[ORC_MAXK], cap[ORC_MAXK];
  int32_t mult[ORC_MAXK];
  int nk = 0;
  for (int d = 0; d < p->D; d++) {
    int o = option[d];
    if (o <= 0 || fam[o - 1] != q) continue;
    int64_t a = p->acc[o - 1], c = p->P[p->dev_type[d] * p->M + (o - 1)];
    int k;
    for (k = 0; k < nk; k++)
      if (A[k] == a && cap[k] == c) break;
    if (k == nk) { A[nk] = a; cap[nk] = c; mult[nk] = 0; nk++; }
    mult[k]++;
  }
  orc_val v;
  orc_family_lp(nk, A, cap, mult, p->s[q], &v.served, &v.accsum);
  return v;
}

/* Canonical z (reading C10): within each family, fill devices in the order
 * (A desc, option asc, device asc), each up to its capacity, until s_q.  The
 * caller checks the result against the LP optimum. */
static void canonical_z(const orc_problem *p, const int32_t *fam, const int32_t *option, int32_t *z) {
  int order[ORC_MAXD];
  for (int q = 0; q < p->Q; q++) {
    int n = 0;
    for (int d = 0; d < p->D; d++)
      if (option[d] > 0 && fam[option[d] - 1] == q) order[n++] = d;
    for (int i = 1; i < n; i++) /* insertion sort by the C10 key */
      for (int j = i; j > 0; j--) {
        int a = order[j - 1], b = order[j];
        int32_t Aa = p->acc[option[a] - 1], Ab = p->acc[option[b] - 1];
        int swap = (Ab > Aa) || (Ab == Aa && (option[b] < option[a] || (option[b] == option[a] && b < a)));
        if (!swap) break;
        order[j - 1] = b; order[j] = a;
      }
    int64_t rem = p->s[q];
    for (int i = 0; i < n; i++) {
      int d = order[i];
      int64_t c = p->P[p->dev_type[d] * p->M + option[d] - 1];
      int64_t take = rem < c ? rem : c;
      z[d] = (int32_t)take;
      rem -= take;
    }
  }
  for (int d = 0; d < p->D; d++)
    if (option[d] <= 0) z[d] = 0;
}

static void finish_result(const orc_problem *p, orc_val best, orc_result *r) {
  int64_t stot = 0;
  for (int q = 0; q < p->Q; q++) stot += p->s[q];
  r->served = best.served;
  r->accsum = best.accsum;
  r->unmet = stot - best.served;
  r->eff = best.served > 0 ? (int32_t)(best.accsum / best.served) : 0;
}

/* Score one placement; writes canonical z.  Returns 0, or -2 if the greedy z
 * does not reach the LP optimum (an internal consistency failure). */
int orc_score_placement(const orc_problem *p, const int32_t *option, orc_result *r, int32_t *z) {
  int32_t fam[4096], off[ORC_MAXQ];
  if (p->M > 4096 || p->Q > ORC_MAXQ || p->D > ORC_MAXD) return -1;
  fam_of(p, fam, off);
  orc_val tot = {0, 0};
  for (int q = 0; q < p->Q; q++) tot = val_add(tot, family_value(p, fam, q, option));
  memset(r, 0, sizeof *r);
  finish_result(p, tot, r);
  if (z) {
    canonical_z(p, fam, option, z);
    orc_val g = {0, 0};
    for (int d = 0; d < p->D; d++)
      if (option[d] > 0) { g.served += z[d]; g.accsum += (int64_t)z[d] * p->acc[option[d] - 1]; }
    if (!val_eq(g, tot)) return -2;
  }
  return 0;
}

/* ------------------------------------------------- modes 0/1 (a2-a6) ---- */
/* Candidate space (reading C9).  Devices are partitioned into groups; a group's
 * devices are interchangeable and take a non-decreasing tuple of option codes
 * in [0, K), K = 1 + M.  Mode 0 (flat mixed radix): every device is its own
 * group.  Mode 1 (multiset): group t = the devices of type t, ascending index.
 * Candidates are enumerated in lexicographic order of (tuple_0, tuple_1, ...);
 * the canonical index of a candidate is its position in that order (group 0 is
 * the most significant digit).  The argmax keeps the first maximum, i.e. the
 * lowest index among equal (served, accsum).
 *
 * Memoisation: a family's LP value depends only on how many devices of each
 * type host each of its variants, so values are cached per family keyed by
 * that count vector.  Each cached value is computed by orc_family_lp. */
typedef struct {
  const orc_problem *p;
  int32_t fam[4096], off[ORC_MAXQ];
  int K, npos;
  int32_t pos_dev[ORC_MAXD], pos_group[ORC_MAXD];
  int ngroups, group_start[ORC_MAXD + 1];
  int Nt[ORC_MAXT];
  /* memo: per family q, code[q][t] = sum_v n[t][v] * (N_t+1)^v; rank tables
   * map a code to a dense rank; key = sum_t rank * stride */
  int32_t *rank[ORC_MAXQ][ORC_MAXT], *code_of_rank[ORC_MAXQ][ORC_MAXT];
  int32_t pw[ORC_MAXQ][ORC_MAXT][16];
  int64_t stride[ORC_MAXQ][ORC_MAXT], nkeys[ORC_MAXQ];
  orc_val *memo[ORC_MAXQ];
  int split;                   /* positions enumerated as task prefixes */
  uint64_t completions;        /* candidates per task */
  int64_t ntasks;
  int32_t *task_opts;          /* [ntasks][split] */
  int64_t next_task;
  pthread_mutex_t mu;
  orc_val best;
  uint64_t best_idx;
  int32_t best_opt[ORC_MAXD];
  int have;
} enum_ctx;

static uint64_t binom(uint64_t n, uint64_t k) {
  if (k > n) return 0;
  unsigned __int128 r = 1;
  for (uint64_t i = 1; i <= k; i++) r = r * (n - k + i) / i;
  return (uint64_t)r;
}

/* number of non-decreasing tuples of length n over K symbols */
static uint64_t ntuples(int K, int n) { return binom((uint64_t)K + n - 1, (uint64_t)n); }

typedef struct {
  enum_ctx *c;
  int32_t opt[ORC_MAXD];
  int32_t code[ORC_MAXQ][ORC_MAXT];
  uint64_t idx;
  orc_val best;
  uint64_t best_idx;
  int32_t best_opt[ORC_MAXD];
  int have;
} enum_thr;

static void place(enum_thr *w, int p, int o, int sign) {
  enum_ctx *c = w->c;
  if (o == 0) return;
  int m = o - 1, q = c->fam[m], v = m - c->off[q];
  int t = c->p->dev_type[c->pos_dev[p]];
  w->code[q][t] += sign * c->pw[q][t][v];
}

static void leaf(enum_thr *w) {
  enum_ctx *c = w->c;
  orc_val tot = {0, 0};
  for (int q = 0; q < c->p->Q; q++) {
    int64_t key = 0;
    for (int t = 0; t < c->p->T; t++) key += (int64_t)c->rank[q][t][w->code[q][t]] * c->stride[q][t];
    tot = val_add(tot, c->memo[q][key]);
  }
  if (!w->have || val_gt(tot, w->best)) {
    w->have = 1; w->best = tot; w->best_idx = w->idx;
    for (int p = 0; p < c->npos; p++) w->best_opt[c->pos_dev[p]] = w->opt[p];
  }
  w->idx++;
}

static void enum_rec(enum_thr *w, int p) {
  enum_ctx *c = w->c;
  if (p == c->npos) { leaf(w); return; }
  int lo = (p > 0 && c->pos_group[p] == c->pos_group[p - 1]) ? w->opt[p - 1] : 0;
  for (int o = lo; o < c->K; o++) {
    w->opt[p] = o;
    place(w, p, o, +1);
    enum_rec(w, p + 1);
    place(w, p, o, -1);
  }
}

static void *enum_worker(void *arg) {
  enum_thr *w = (enum_thr *)arg;
  enum_ctx *c = w->c;
  for (;;) {
    int64_t task = __sync_fetch_and_add(&c->next_task, 1);
    if (task >= c->ntasks) break;
    memset(w->code, 0, sizeof w->code);
    for (int p = 0; p < c->split; p++) {
      w->opt[p] = c->task_opts[task * c->split + p];
      place(w, p, w->opt[p], +1);
    }
    w->idx = (uint64_t)task * c->completions;
    enum_rec(w, c->split);
  }
  pthread_mutex_lock(&c->mu);
  if (w->have && (!c->have || val_gt(w->best, c->best) ||
                  (val_eq(w->best, c->best) && w->best_idx < c->best_idx))) {
    c->have = 1; c->best = w->best; c->best_idx = w->best_idx;
    memcpy(c->best_opt, w->best_opt, sizeof c->best_opt);
  }
  pthread_mutex_unlock(&c->mu);
  return NULL;
}

/* prefix tuples of the first `split` positions, in lexicographic order */
static void collect_prefix(enum_ctx *c, int32_t *cur, int p, int64_t *n) {
  if (p == c->split) {
    if (c->task_opts) memcpy(c->task_opts + *n * c->split, cur, sizeof(int32_t) * c->split);
    (*n)++;
    return;
  }
  int lo = (p > 0 && c->pos_group[p] == c->pos_group[p - 1]) ? cur[p - 1] : 0;
  for (int o = lo; o < c->K; o++) { cur[p] = o; collect_prefix(c, cur, p + 1, n); }
}

typedef struct { enum_ctx *c; int q; int64_t k0, k1; } memo_job;

/* fill memo[q][key] for keys in [k0, k1): decode key -> count vector -> LP */
static void *memo_worker(void *arg) {
  memo_job *j = (memo_job *)arg;
  enum_ctx *c = j->c;
  const orc_problem *p = c->p;
  int q = j->q, Vq = p->V[q];
  /* inverse of the rank tables */
  for (int64_t key = j->k0; key < j->k1; key++) {
    int64_t A[ORC_MAXK], cap[ORC_MAXK];
    int32_t mult[ORC_MAXK];
    int nk = 0;
    /* decode: key = sum_t rank_t * stride_t with stride of type T-1 = 1 */
    int64_t rem = key;
    for (int t = 0; t < p->T; t++) {
      int64_t rk = rem / c->stride[q][t];
      rem -= rk * c->stride[q][t];
      int base = c->Nt[t] + 1;
      int code = c->code_of_rank[q][t][rk];
      for (int v = 0; v < Vq; v++) {
        int n = (code / c->pw[q][t][v]) % base;
        int m = c->off[q] + v;
        if (n == 0) continue;
        A[nk] = p->acc[m]; cap[nk] = p->P[t * p->M + m]; mult[nk] = n; nk++;
      }
    }
    orc_val v;
    orc_family_lp(nk, A, cap, mult, p->s[q], &v.served, &v.accsum);
    c->memo[q][key] = v;
  }
  return NULL;
}

int orc_enum_count(const orc_problem *p, int mode, uint64_t *count) {
  int K = 1 + p->M;
  if (mode == 0) {
    unsigned __int128 n = 1;
    for (int d = 0; d < p->D; d++) { n *= (unsigned)K; if (n > UINT64_MAX) return -5; }
    *count = (uint64_t)n;
    return 0;
  }
  unsigned __int128 n = 1;
  for (int t = 0; t < p->T; t++) {
    int nt = 0;
    for (int d = 0; d < p->D; d++) nt += p->dev_type[d] == t;
    n *= ntuples(K, nt);
    if (n > UINT64_MAX) return -5;
  }
  *count = (uint64_t)n;
  return 0;
}

int orc_solve_enum(const orc_problem *p, int mode, int nthreads, orc_result *r, int32_t *option, int32_t *z) {
  if (p->D > ORC_MAXD || p->Q > ORC_MAXQ || p->T > ORC_MAXT || p->M > 4095 || (mode != 0 && mode != 1))
    return -1;
  enum_ctx *c = (enum_ctx *)calloc(1, sizeof(enum_ctx));
  c->p = p;
  fam_of(p, c->fam, c->off);
  c->K = 1 + p->M;
  for (int t = 0; t < p->T; t++) c->Nt[t] = 0;
  for (int d = 0; d < p->D; d++) c->Nt[p->dev_type[d]]++;
  /* groups and positions */
  c->npos = 0;
  c->ngroups = 0;
  if (mode == 0) {
    for (int d = 0; d < p->D; d++) {
      c->group_start[c->ngroups] = c->npos;
      c->pos_dev[c->npos] = d; c->pos_group[c->npos] = c->ngroups; c->npos++; c->ngroups++;
    }
  } else {
    for (int t = 0; t < p->T; t++) {
      if (c->Nt[t] == 0) continue;
      c->group_start[c->ngroups] = c->npos;
      for (int d = 0; d < p->D; d++)
        if (p->dev_type[d] == t) { c->pos_dev[c->npos] = d; c->pos_group[c->npos] = c->ngroups; c->npos++; }
      c->ngroups++;
    }
  }
  c->group_start[c->ngroups] = c->npos;
  /* memo tables */
  for (int q = 0; q < p->Q; q++) {
    int64_t stride = 1;
    for (int t = p->T - 1; t >= 0; t--) {
      int base = c->Nt[t] + 1, ncode = 1;
      for (int v = 0; v < p->V[q]; v++) { c->pw[q][t][v] = ncode; ncode *= base; }
      c->rank[q][t] = (int32_t *)malloc(sizeof(int32_t) * ncode);
      c->code_of_rank[q][t] = (int32_t *)malloc(sizeof(int32_t) * ncode);
      int32_t cnt = 0;
      for (int cc = 0; cc < ncode; cc++) {
        int sum = 0;
        for (int v = 0; v < p->V[q]; v++) sum += (cc / c->pw[q][t][v]) % base;
        if (sum <= c->Nt[t]) { c->code_of_rank[q][t][cnt] = cc; c->rank[q][t][cc] = cnt++; }
        else c->rank[q][t][cc] = -1;
      }
      c->stride[q][t] = stride;
      stride *= cnt;
    }
    c->nkeys[q] = stride;
    c->memo[q] = (orc_val *)malloc(sizeof(orc_val) * stride);
  }
  int nth = ncores(nthreads);
  {
    int njobs = 0;
    memo_job *jobs = (memo_job *)malloc(sizeof(memo_job) * p->Q * nth);
    pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * p->Q * nth);
    for (int q = 0; q < p->Q; q++)
      for (int i = 0; i < nth; i++) {
        jobs[njobs].c = c; jobs[njobs].q = q;
        jobs[njobs].k0 = c->nkeys[q] * i / nth; jobs[njobs].k1 = c->nkeys[q] * (i + 1) / nth;
        njobs++;
      }
    for (int i = 0; i < njobs; i++) pthread_create(&th[i], NULL, memo_worker, &jobs[i]);
    for (int i = 0; i < njobs; i++) pthread_join(th[i], NULL);
    free(jobs); free(th);
  }
  /* task split at a group boundary: enough tasks to keep the threads busy */
  int g = 0;
  uint64_t ntask = 1;
  while (g < c->ngroups && ntask < (uint64_t)64 * nth) {
    ntask *= ntuples(c->K, c->group_start[g + 1] - c->group_start[g]);
    g++;
  }
  c->split = c->group_start[g];
  c->completions = 1;
  for (int h = g; h < c->ngroups; h++) c->completions *= ntuples(c->K, c->group_start[h + 1] - c->group_start[h]);
  c->ntasks = (int64_t)ntask;
  c->task_opts = (int32_t *)malloc(sizeof(int32_t) * (size_t)(c->split ? c->split : 1) * ntask);
  {
    int32_t cur[ORC_MAXD];
    int64_t n = 0;
    collect_prefix(c, cur, 0, &n);
  }
  pthread_mutex_init(&c->mu, NULL);
  enum_thr *w = (enum_thr *)calloc(nth, sizeof(enum_thr));
  pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * nth);
  for (int i = 0; i < nth; i++) { w[i].c = c; pthread_create(&th[i], NULL, enum_worker, &w[i]); }
  for (int i = 0; i < nth; i++) pthread_join(th[i], NULL);
  memset(r, 0, sizeof *r);
  finish_result(p, c->best, r);
  r->index = c->best_idx;
  r->n_candidates = (uint64_t)c->ntasks * c->completions;
  int rc = 0;
  if (option) memcpy(option, c->best_opt, sizeof(int32_t) * p->D);
  if (z) {
    orc_result chk;
    rc = orc_score_placement(p, c->best_opt, &chk, z);
    if (rc == 0 && (chk.served != r->served || chk.accsum != r->accsum)) rc = -2;
  }
  for (int q = 0; q < p->Q; q++) {
    for (int t = 0; t < p->T; t++) { free(c->rank[q][t]); free(c->code_of_rank[q][t]); }
    free(c->memo[q]);
  }
  free(c->task_opts); free(w); free(th); free(c);
  return rc;
}

/* --------------------------------------------------- mode 2 (a8, a10) -- */
/* Family-factored exact search.  Eqs. 1, 3 and 5 make a placement's value the
 * sum over families of the family's LP value, and that value depends only on
 * the count vector n[q][t][v] = number of type-t devices hosting variant v of
 * family q.  A count tensor is a placement iff sum_{q,v} n[q][t][v] <= N_t for
 * every type t.  So:
 *   g_q(u)  = best LP value of family q over its count vectors with usage u
 *             (u_t = sum_v n[q][t][v]),
 *   G_q(b)  = max_{u <= b} g_q(u) + G_{q+1}(b - u),   G_Q = 0,
 * and the optimum is G_0(N).  The canonical solution (reading C9) is the
 * lexicographically smallest tensor n (q-major, then t, then v) among optima,
 * found family by family.  Options with P = 0 are never used by that solution
 * (moving such a device to idle keeps the value and makes n smaller), so they
 * are left out of the enumeration (reading C16; pinned by a test that runs
 * with and without this pruning). */
typedef struct {
  orc_val val;
  int32_t ukey;
} fact_entry;  /* entries are stored in lexicographic order of n */

typedef struct {
  const orc_problem *p;
  int32_t off[ORC_MAXQ], fam[4096];
  int Nt[ORC_MAXT];
  int64_t ustride[ORC_MAXT], nu;
  int prune;
  /* per family */
  fact_entry *list[ORC_MAXQ];
  int64_t nlist[ORC_MAXQ], cap_list[ORC_MAXQ];
  orc_val *g[ORC_MAXQ];
  int8_t *gvalid[ORC_MAXQ];
} fact_ctx;

typedef struct { fact_ctx *c; int q; int32_t n[ORC_MAXT * 16]; } fact_thr;

static int64_t ukey_of(fact_ctx *c, const int32_t *u) {
  int64_t k = 0;
  for (int t = 0; t < c->p->T; t++) k += u[t] * c->ustride[t];
  return k;
}

static void fact_leaf(fact_thr *w) {
  fact_ctx *c = w->c;
  const orc_problem *p = c->p;
  int q = w->q, Vq = p->V[q];
  int64_t A[ORC_MAXK], cap[ORC_MAXK];
  int32_t mult[ORC_MAXK], u[ORC_MAXT];
  int nk = 0;
  for (int t = 0; t < p->T; t++) {
    u[t] = 0;
    for (int v = 0; v < Vq; v++) {
      int n = w->n[t * 16 + v];
      u[t] += n;
      if (!n) continue;
      int m = c->off[q] + v;
      A[nk] = p->acc[m]; cap[nk] = p->P[t * p->M + m]; mult[nk] = n; nk++;
    }
  }
  orc_val val;
  orc_family_lp(nk, A, cap, mult, p->s[q], &val.served, &val.accsum);
  if (c->nlist[q] == c->cap_list[q]) {
    c->cap_list[q] = c->cap_list[q] ? 2 * c->cap_list[q] : 1024;
    c->list[q] = (fact_entry *)realloc(c->list[q], sizeof(fact_entry) * c->cap_list[q]);
  }
  fact_entry *e = &c->list[q][c->nlist[q]++];
  e->ukey = (int32_t)ukey_of(c, u);
  e->val = val;
  if (!c->gvalid[q][e->ukey] || val_gt(val, c->g[q][e->ukey])) { /* first max in lex order */
    c->gvalid[q][e->ukey] = 1;
    c->g[q][e->ukey] = val;
  }
}

/* count vectors in lexicographic order: position (t, v) t-major, values ascending */
static void fact_rec(fact_thr *w, int t, int v, int left) {
  fact_ctx *c = w->c;
  const orc_problem *p = c->p;
  int q = w->q, Vq = p->V[q];
  if (t == p->T) { fact_leaf(w); return; }
  if (v == Vq) { fact_rec(w, t + 1, 0, t + 1 < p->T ? c->Nt[t + 1] : 0); return; }
  int m = c->off[q] + v;
  int hi = (c->prune && p->P[t * p->M + m] == 0) ? 0 : left;
  for (int n = 0; n <= hi; n++) {
    w->n[t * 16 + v] = n;
    fact_rec(w, t, v + 1, left - n);
  }
  w->n[t * 16 + v] = 0;
}

/* the same enumeration, stopping at the `target`-th count vector */
static int fact_find(fact_ctx *c, int q, int t, int v, int left, int64_t *k, int64_t target, int32_t *n) {
  const orc_problem *p = c->p;
  if (t == p->T) return (*k)++ == target;
  if (v == p->V[q]) return fact_find(c, q, t + 1, 0, t + 1 < p->T ? c->Nt[t + 1] : 0, k, target, n);
  int m = c->off[q] + v;
  int hi = (c->prune && p->P[t * p->M + m] == 0) ? 0 : left;
  for (int x = 0; x <= hi; x++) {
    n[t * 16 + v] = x;
    if (fact_find(c, q, t, v + 1, left - x, k, target, n)) return 1;
  }
  n[t * 16 + v] = 0;
  return 0;
}

static void *fact_worker(void *arg) {
  fact_thr *w = (fact_thr *)arg;
  memset(w->n, 0, sizeof w->n);
  fact_rec(w, 0, 0, w->c->Nt[0]);
  return NULL;
}

int orc_solve_factored(const orc_problem *p, int nthreads, int prune, orc_result *r, int32_t *option,
                       int32_t *z, int32_t *count_out /* [Q][T][16] or NULL */) {
  (void)nthreads;
  if (p->T > ORC_MAXT || p->Q > ORC_MAXQ || p->D > ORC_MAXD) return -1;
  for (int q = 0; q < p->Q; q++) if (p->V[q] > 16) return -1;
  fact_ctx *c = (fact_ctx *)calloc(1, sizeof(fact_ctx));
  c->p = p;
  c->prune = prune;
  fam_of(p, c->fam, c->off);
  for (int d = 0; d < p->D; d++) c->Nt[p->dev_type[d]]++;
  c->nu = 1;
  for (int t = p->T - 1; t >= 0; t--) { c->ustride[t] = c->nu; c->nu *= c->Nt[t] + 1; }
  for (int q = 0; q < p->Q; q++) {
    c->g[q] = (orc_val *)calloc(c->nu, sizeof(orc_val));
    c->gvalid[q] = (int8_t *)calloc(c->nu, 1);
  }
  /* one thread per family */
  fact_thr *w = (fact_thr *)calloc(p->Q, sizeof(fact_thr));
  pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * p->Q);
  for (int q = 0; q < p->Q; q++) { w[q].c = c; w[q].q = q; pthread_create(&th[q], NULL, fact_worker, &w[q]); }
  for (int q = 0; q < p->Q; q++) pthread_join(th[q], NULL);
  /* budget DP over the usage lattice */
  int T = p->T;
  orc_val *G = (orc_val *)calloc((size_t)(p->Q + 1) * c->nu, sizeof(orc_val));
  for (int q = p->Q - 1; q >= 0; q--)
    for (int64_t b = 0; b < c->nu; b++) {
      int32_t bv[ORC_MAXT];
      for (int t = 0; t < T; t++) bv[t] = (int32_t)((b / c->ustride[t]) % (c->Nt[t] + 1));
      orc_val best = {-1, -1};
      for (int64_t u = 0; u < c->nu; u++) {
        if (!c->gvalid[q][u]) continue;
        int ok = 1;
        int64_t rest = 0;
        for (int t = 0; t < T; t++) {
          int32_t ut = (int32_t)((u / c->ustride[t]) % (c->Nt[t] + 1));
          if (ut > bv[t]) { ok = 0; break; }
          rest += (bv[t] - ut) * c->ustride[t];
        }
        if (!ok) continue;
        orc_val cand = val_add(c->g[q][u], G[(size_t)(q + 1) * c->nu + rest]);
        if (val_gt(cand, best)) best = cand;
      }
      G[(size_t)q * c->nu + b] = best;
    }
  /* lexicographically smallest reconstruction */
  int32_t bvec[ORC_MAXT];
  for (int t = 0; t < T; t++) bvec[t] = c->Nt[t];
  int32_t cnt[ORC_MAXQ][ORC_MAXT * 16];
  memset(cnt, 0, sizeof cnt);
  for (int q = 0; q < p->Q; q++) {
    int64_t b = ukey_of(c, bvec);
    orc_val target = G[(size_t)q * c->nu + b];
    int64_t pick = -1;
    for (int64_t i = 0; i < c->nlist[q] && pick < 0; i++) {
      fact_entry *e = &c->list[q][i];
      int ok = 1;
      int64_t rest = 0;
      for (int t = 0; t < T; t++) {
        int32_t ut = (int32_t)((e->ukey / c->ustride[t]) % (c->Nt[t] + 1));
        if (ut > bvec[t]) { ok = 0; break; }
        rest += (bvec[t] - ut) * c->ustride[t];
      }
      if (ok && val_eq(val_add(e->val, G[(size_t)(q + 1) * c->nu + rest]), target)) pick = i;
    }
    if (pick < 0) return -3;
    fact_entry *e = &c->list[q][pick];
    int64_t k = 0;
    fact_find(c, q, 0, 0, c->Nt[0], &k, pick, cnt[q]);
    for (int t = 0; t < T; t++) bvec[t] -= (int32_t)((e->ukey / c->ustride[t]) % (c->Nt[t] + 1));
  }
  /* materialise: per type, devices ascending, options in (q, v) order */
  int32_t opt[ORC_MAXD];
  for (int d = 0; d < p->D; d++) opt[d] = 0;
  for (int t = 0; t < T; t++) {
    int d = 0;
    for (int q = 0; q < p->Q; q++)
      for (int v = 0; v < p->V[q]; v++)
        for (int k = 0; k < cnt[q][t * 16 + v]; k++) {
          while (p->dev_type[d] != t) d++;
          opt[d] = 1 + c->off[q] + v;
          d++;
        }
  }
  uint64_t ncand = 0;
  for (int q = 0; q < p->Q; q++) ncand += (uint64_t)c->nlist[q];
  memset(r, 0, sizeof *r);
  finish_result(p, G[c->nu - 1], r); /* G_0(N): b = N is the last lattice point */
  r->index = UINT64_MAX;
  r->n_candidates = ncand;
  if (option) memcpy(option, opt, sizeof(int32_t) * p->D);
  if (count_out) memcpy(count_out, cnt, sizeof(int32_t) * p->Q * ORC_MAXT * 16);
  int rc = 0;
  {
    orc_result chk;
    int32_t zz[ORC_MAXD];
    rc = orc_score_placement(p, opt, &chk, zz);
    if (rc == 0 && (chk.served != r->served || chk.accsum != r->accsum)) rc = -2;
    if (z) memcpy(z, zz, sizeof(int32_t) * p->D);
  }
  for (int q = 0; q < p->Q; q++) { free(c->list[q]); free(c->g[q]); free(c->gvalid[q]); }
  free(G); free(w); free(th); free(c);
  return rc;
}

/* ------------------------------------------------------------ replay -- */
/* R8: router.  Per family q, the members are the devices hosting q in
 * ascending index with weight w_d, then a drop sink with weight w_sink[q]
 * (members of weight 0 are left out).  For every query of family q, in
 * arrival order: add each member's weight to its current value, pick the member
 * with the largest current value (first on ties; the sink is last), subtract
 * the total weight W from it.  If W = 0 the query goes to the sink.
 * target[i] = device index, or D for the sink. */
int orc_route_swrr(int64_t N, const uint8_t *family, int Q, int D, const int32_t *dev_family,
                   const int32_t *w_dev, const int32_t *w_sink, int32_t *target) {
  int64_t *cur = (int64_t *)calloc((size_t)Q * (D + 1), sizeof(int64_t));
  for (int64_t i = 0; i < N; i++) {
    int q = family[i];
    if (q >= Q) { free(cur); return -1; }
    int64_t W = w_sink[q];
    for (int d = 0; d < D; d++) if (dev_family[d] == q) W += w_dev[d];
    if (W == 0) { target[i] = D; continue; }
    int64_t *cq = cur + (size_t)q * (D + 1);
    int best = -1;
    for (int d = 0; d <= D; d++) {
      int64_t w = d < D ? (dev_family[d] == q ? w_dev[d] : 0) : w_sink[q];
      if (w == 0) continue;
      cq[d] += w;
      if (best < 0 || cq[d] > cq[best]) best = d;
    }
    cq[best] -= W;
    target[i] = best;
  }
  free(cur);
  return 0;
}

/* §5 adaptive batching on one device, event-driven.
 * Events: query arrivals, batch completion, the wait timer.  At each event time
 * t: enqueue every arrival with a <= t (R3); if the device has finished (F <= t)
 * and the queue holds q >= 1 queries:
 *   q >= Bmax                   -> dispatch Bmax now (R4)
 *   t >= Tmax_wait(q+1)         -> dispatch q now (Case 1; R1)
 *   otherwise                   -> wait; timer at Tmax_wait(q+1) (Case 2 is the
 *                                  re-evaluation at the next arrival)
 * with Tmax_wait(q+1) = Texp(1) - Tprocess(q+1) = a_head + L - T(q+1).
 * A batch of b dispatched at t finishes at F = t + T(b); each of its queries
 * gets latency F - a (saturated at UINT32_MAX - 1).
 * Tproc[b] for b = 1..Bmax (index 0 unused). */
int orc_replay_device(int64_t n, const uint32_t *a, const int32_t *Tproc, int Bmax, int64_t L,
                      uint32_t *lat) {
  if (n == 0) return 0;
  if (Bmax < 1) return -1;
  const int64_t INF = INT64_MAX / 4;
  int64_t head = 0, tail = 0; /* queue = [head, tail) */
  int64_t F = 0;              /* device busy until F */
  int busy = 0, armed = 0;
  int64_t timer = 0;
  while (head < n) {
    int64_t te = INF;
    if (tail < n && (int64_t)a[tail] < te) te = a[tail];
    if (busy && F < te) te = F;
    if (armed && timer < te) te = timer;
    int64_t t = te;
    while (tail < n && (int64_t)a[tail] <= t) tail++;
    if (busy && F <= t) busy = 0;
    if (busy || tail == head) continue;
    int64_t q = tail - head;
    int64_t b = 0;
    if (q >= Bmax) b = Bmax;
    else {
      int64_t W = (int64_t)a[head] + L - Tproc[q + 1];
      if (t >= W) b = q;
      else { armed = 1; timer = W; }
    }
    if (b) {
      F = t + Tproc[b];
      for (int64_t j = head; j < head + b; j++) {
        int64_t l = F - (int64_t)a[j];
        lat[j] = l >= (int64_t)UINT32_MAX ? UINT32_MAX - 1 : (uint32_t)l;
      }
      head += b;
      busy = 1;
      armed = 0;
    }
  }
  return 0;
}

/* §8(f2) baseline batchers, P:1535-1630 (§6.4, Fig. 6): "we implement each of
 * these batching algorithms on top of Proteus".  Both are work-conserving
 * ("dispatches an inference batch to each device as soon as the previous
 * batch is finished"): whenever the device is free and the queue
 * is non-empty, a batch leaves at once.  Event-driven like orc_replay_device
 * (events: arrivals and batch completions; no timer).  DROPPED = UINT32_MAX.
 *
 * Nexus early drop (reading R14).  Batch size B (the
 * caller passes it: the largest b <= Bmax with 2 T(b) <= L, at least 1 -- the
 * capacity rule of P:923-928 that sizes Nexus's batches).  At a decision time t
 * the dispatcher slides a window of min(B, queued from i) queries from the
 * head: the first query i whose deadline a_i + L is met by the window's
 * completion t + T(w) starts the batch; every query before it is dropped. */
int orc_replay_device_nexus(int64_t n, const uint32_t *a, const int32_t *Tproc, int B, int64_t L,
                            uint32_t *lat) {
  if (n == 0) return 0;
  if (B < 1) return -1;
  const int64_t INF = INT64_MAX / 4;
  int64_t head = 0, tail = 0;
  int64_t F = 0;
  int busy = 0;
  while (head < n) {
    int64_t t = INF;
    if (tail < n) t = a[tail];
    if (busy && F < t) t = F;
    while (tail < n && (int64_t)a[tail] <= t) tail++;
    if (busy && F <= t) busy = 0;
    if (busy || tail == head) continue;
    /* sliding window over the queue [head, tail) */
    int64_t i = head, w = 0;
    for (; i < tail; i++) {
      w = tail - i < B ? tail - i : B;
      if (t + Tproc[w] <= (int64_t)a[i] + L) break;
      lat[i] = UINT32_MAX;          /* dropped early */
    }
    head = i;
    if (head == tail) continue;     /* everything queued was dropped */
    F = t + Tproc[w];
    for (int64_t j = head; j < head + w; j++) {
      int64_t l = F - (int64_t)a[j];
      lat[j] = l >= (int64_t)UINT32_MAX ? UINT32_MAX - 1 : (uint32_t)l;
    }
    head += w;
    busy = 1;
  }
  return 0;
}

/* Clipper AIMD (reading R15).  The batch-size limit
 * starts at 1; a batch takes min(queued, limit) queries.  When it completes,
 * the limit grows by 1 (additive increase, at most Bmax) if none of its
 * queries timed out (latency > L), else it shrinks to max(1, floor(9 limit /
 * 10)) (Clipper's 10 % multiplicative back-off).  No query is dropped. */
int orc_replay_device_aimd(int64_t n, const uint32_t *a, const int32_t *Tproc, int Bmax, int64_t L,
                           uint32_t *lat) {
  if (n == 0) return 0;
  if (Bmax < 1) return -1;
  const int64_t INF = INT64_MAX / 4;
  int64_t head = 0, tail = 0;
  int64_t F = 0;
  int busy = 0, limit = 1, pend = 0;  /* pend: the running batch's feedback is still to apply */
  int timed_out = 0;
  while (head < n) {
    int64_t t = INF;
    if (tail < n) t = a[tail];
    if (busy && F < t) t = F;
    while (tail < n && (int64_t)a[tail] <= t) tail++;
    if (busy && F <= t) {
      busy = 0;
      if (pend) {                   /* completion: AIMD update */
        if (timed_out) limit = limit * 9 / 10 < 1 ? 1 : limit * 9 / 10;
        else limit = limit + 1 > Bmax ? Bmax : limit + 1;
        pend = 0;
      }
    }
    if (busy || tail == head) continue;
    int64_t b = tail - head < limit ? tail - head : limit;
    F = t + Tproc[b];
    timed_out = 0;
    for (int64_t j = head; j < head + b; j++) {
      int64_t l = F - (int64_t)a[j];
      lat[j] = l >= (int64_t)UINT32_MAX ? UINT32_MAX - 1 : (uint32_t)l;
      if (l > L) timed_out = 1;
    }
    head += b;
    busy = 1;
    pend = 1;
  }
  return 0;
}

/* Full replay (a11-a13).  Scenario s: slo_mult_milli, batch_cap (0 = table
 * depth), routing (0 = SWRR over z with the unmet demand to the sink, 1 =
 * uniform over the hosting devices that fit batch 1, no sink), policy (0 = §5
 * adaptive batching, 1 = Nexus early drop, 2 = Clipper AIMD; §8(f2)).
 * SLO_q(s) = floor(mult * slo_base[q] / 1000) (R12).  Reading R4' (P:918-936:
 * "the maximum allowed batch size is the minimum of (i) the maximum batch size
 * that meets SLO, (ii) the maximum batch size that fits in the memory of d",
 * with (i) the half-SLO rule of P:920-926): the §5 policy batches at most
 * Bmax = the largest b <= min(cap, depth) with 2 T(b) <= SLO, at least 1 --
 * the same size as the Nexus baseline's (R14) and as the capacity estimate's
 * b*; Clipper AIMD grows its own limit up to min(cap, depth) (R15).
 * Outputs per scenario: violations (latency > SLO, R6, plus dropped), on_time,
 * acc_sum (sum of the serving variant's accuracy over on-time queries, R9);
 * latency[s][i] if non-NULL (UINT32_MAX = dropped). */
typedef struct {
  int64_t N; const uint32_t *arr; const uint8_t *fam;
  int Q, D, M, T, bmax;
  const int32_t *V, *acc, *lat_tab, *option, *dev_type, *slo_base, *sc;
  int S;
  int32_t *target[2];
  int64_t *idx_of_dev[2]; int64_t *dev_start[2];
  uint32_t *latency;
  uint64_t *viol, *ontime, *accsum;
  int64_t next; pthread_mutex_t mu;
} rep_ctx;

static void *rep_worker(void *arg) {
  rep_ctx *c = (rep_ctx *)arg;
  int32_t fam_m[4096];
  { int m = 0; for (int q = 0; q < c->Q; q++) for (int v = 0; v < c->V[q]; v++) fam_m[m++] = q; }
  for (;;) {
    int64_t lane = __sync_fetch_and_add(&c->next, 1);
    if (lane >= (int64_t)c->S * (c->D + 1)) break;
    int s = (int)(lane / (c->D + 1)), d = (int)(lane % (c->D + 1));
    int rt = c->sc[s * 4 + 2];
    int64_t st = c->dev_start[rt][d], en = c->dev_start[rt][d + 1];
    uint64_t viol = 0, ont = 0, accs = 0;
    if (d == c->D) { /* sink: dropped */
      viol = (uint64_t)(en - st);
      if (c->latency)
        for (int64_t k = st; k < en; k++) c->latency[(size_t)s * c->N + c->idx_of_dev[rt][k]] = UINT32_MAX;
    } else if (en > st) {
      int m = c->option[d] - 1, t = c->dev_type[d], q = fam_m[m];
      const int32_t *row = c->lat_tab + ((size_t)t * c->M + m) * c->bmax;
      int dep = 0;
      while (dep < c->bmax && row[dep] > 0) dep++;
      int cap = c->sc[s * 4 + 1];
      int Bmax = (cap > 0 && cap < dep) ? cap : dep;
      int64_t L = (int64_t)c->sc[s * 4 + 0] * c->slo_base[q] / 1000;
      int Bhalf = 1;  /* the maximum allowed batch size (R4', R14) */
      for (int b = 1; b <= Bmax && b <= 1024; b++) if (2LL * row[b - 1] <= L) Bhalf = b;
      int64_t n = en - st;
      uint32_t *a = (uint32_t *)malloc(sizeof(uint32_t) * n), *l = (uint32_t *)malloc(sizeof(uint32_t) * n);
      for (int64_t k = 0; k < n; k++) a[k] = c->arr[c->idx_of_dev[rt][st + k]];
      int32_t Tp[1025];
      Tp[0] = 0;
      for (int b = 1; b <= Bmax && b <= 1024; b++) Tp[b] = row[b - 1];
      const int policy = c->sc[s * 4 + 3];
      if (policy == 1) {          /* Nexus: batch size by the capacity rule (R14) */
        orc_replay_device_nexus(n, a, Tp, Bhalf, L, l);
      } else if (policy == 2) {
        orc_replay_device_aimd(n, a, Tp, Bmax, L, l);
      } else {                    /* §5 with the maximum allowed batch size (R4') */
        orc_replay_device(n, a, Tp, Bhalf, L, l);
      }
      for (int64_t k = 0; k < n; k++) {
        if ((int64_t)l[k] > L) viol++;
        else { ont++; accs += (uint64_t)c->acc[m]; }
        if (c->latency) c->latency[(size_t)s * c->N + c->idx_of_dev[rt][st + k]] = l[k];
      }
      free(a); free(l);
    }
    pthread_mutex_lock(&c->mu);
    c->viol[s] += viol; c->ontime[s] += ont; c->accsum[s] += accs;
    pthread_mutex_unlock(&c->mu);
  }
  return NULL;
}

int orc_replay(int64_t N, const uint32_t *arrival, const uint8_t *family,
               int T, int Q, const int32_t *V, const int32_t *acc, int bmax, const int32_t *lat_tab,
               int D, const int32_t *option, const int32_t *z, const int32_t *dev_type,
               const int32_t *demand, const int32_t *slo_base,
               int S, const int32_t *sc /* [S][4] */, int nthreads,
               uint32_t *latency, uint64_t *viol, uint64_t *ontime, uint64_t *accsum) {
  int M = 0;
  for (int q = 0; q < Q; q++) M += V[q];
  if (M > 4096 || D > ORC_MAXD) return -1;
  for (int64_t i = 1; i < N; i++) if (arrival[i] < arrival[i - 1]) return -5;
  int32_t fam_m[4096];
  { int m = 0; for (int q = 0; q < Q; q++) for (int v = 0; v < V[q]; v++) fam_m[m++] = q; }
  int32_t dev_family[ORC_MAXD];
  for (int d = 0; d < D; d++) dev_family[d] = option[d] > 0 ? fam_m[option[d] - 1] : -1;
  rep_ctx c;
  memset(&c, 0, sizeof c);
  c.N = N; c.arr = arrival; c.fam = family; c.Q = Q; c.D = D; c.M = M; c.T = T; c.bmax = bmax;
  c.V = V; c.acc = acc; c.lat_tab = lat_tab; c.option = option; c.dev_type = dev_type;
  c.slo_base = slo_base; c.sc = sc; c.S = S; c.latency = latency; c.viol = viol; c.ontime = ontime;
  c.accsum = accsum;
  for (int s = 0; s < S; s++) { viol[s] = 0; ontime[s] = 0; accsum[s] = 0; }
  for (int rt = 0; rt < 2; rt++) {
    int used = 0;
    for (int s = 0; s < S; s++) used |= sc[s * 4 + 2] == rt;
    if (!used) continue;
    int32_t wdev[ORC_MAXD], wsink[ORC_MAXQ];
    for (int q = 0; q < Q; q++) wsink[q] = 0;
    if (rt == 0) {
      for (int q = 0; q < Q; q++) wsink[q] = demand[q];
      for (int d = 0; d < D; d++) {
        wdev[d] = dev_family[d] >= 0 ? z[d] : 0;
        if (dev_family[d] >= 0) wsink[dev_family[d]] -= z[d];
      }
      for (int q = 0; q < Q; q++) if (wsink[q] < 0) return -1;
    } else {
      for (int d = 0; d < D; d++) {
        int fits = 0;
        if (dev_family[d] >= 0) fits = lat_tab[((size_t)dev_type[d] * M + option[d] - 1) * bmax] > 0;
        wdev[d] = fits ? 1 : 0;
      }
    }
    c.target[rt] = (int32_t *)malloc(sizeof(int32_t) * (N ? N : 1));
    orc_route_swrr(N, family, Q, D, dev_family, wdev, wsink, c.target[rt]);
    c.dev_start[rt] = (int64_t *)calloc(D + 2, sizeof(int64_t));
    for (int64_t i = 0; i < N; i++) c.dev_start[rt][c.target[rt][i] + 1]++;
    for (int d = 0; d <= D; d++) c.dev_start[rt][d + 1] += c.dev_start[rt][d];
    c.idx_of_dev[rt] = (int64_t *)malloc(sizeof(int64_t) * (N ? N : 1));
    int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (D + 1));
    for (int d = 0; d <= D; d++) fill[d] = c.dev_start[rt][d];
    for (int64_t i = 0; i < N; i++) c.idx_of_dev[rt][fill[c.target[rt][i]]++] = i;
    free(fill);
  }
  pthread_mutex_init(&c.mu, NULL);
  int nth = ncores(nthreads);
  pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * nth);
  for (int i = 0; i < nth; i++) pthread_create(&th[i], NULL, rep_worker, &c);
  for (int i = 0; i < nth; i++) pthread_join(th[i], NULL);
  free(th);
  for (int rt = 0; rt < 2; rt++) { free(c.target[rt]); free(c.dev_start[rt]); free(c.idx_of_dev[rt]); }
  return 0;
}

/* ------------------------------------------------------- §8(f4) loop -- */
/* Closed loop (P:707-723 re-allocation, P:1369-1370 period,
 * P:192-203 per-second demand changes).  Readings F1-F4:
 *   F1  time is cut into epochs of epoch_us; query i belongs to epoch
 *       floor(a_i / epoch_us), which must be < E;
 *   F2  epoch e runs allocation e (option[e][D], z[e][D]) solved by the
 *       caller for demand[e][Q] (the controller's estimate: the bench uses the
 *       previous epoch's observed counts); routing restarts each epoch: SWRR
 *       over z[e] with the sink weight demand[e][q] - sum z (R8), its state
 *       reset at the epoch start;
 *   F3  switching costs nothing (C14) but a device finishes the queue of one
 *       epoch with that epoch's variant before serving queries of the next:
 *       a batch holds queries of one epoch only, later-epoch queries wait;
 *   F4  the §5 rule (R1-R13) applies to the head's epoch: q counts the queued
 *       queries of the head's epoch, T, Bmax and L are that epoch's.
 *
 * One device, event-driven like orc_replay_device.  ep[j] = epoch of query j
 * (non-decreasing); Tp[e] = that epoch's T(b) row (index b), Bm[e], L[e]. */
int orc_replay_device_epochs(int64_t n, const uint32_t *a, const int32_t *ep, const int32_t *const *Tp,
                             const int32_t *Bm, const int64_t *L, uint32_t *lat) {
  if (n == 0) return 0;
  const int64_t INF = INT64_MAX / 4;
  int64_t head = 0, tail = 0;
  int64_t F = 0;
  int busy = 0, armed = 0;
  int64_t timer = 0;
  while (head < n) {
    int64_t te = INF;
    if (tail < n && (int64_t)a[tail] < te) te = a[tail];
    if (busy && F < te) te = F;
    if (armed && timer < te) te = timer;
    int64_t t = te;
    while (tail < n && (int64_t)a[tail] <= t) tail++;
    if (busy && F <= t) busy = 0;
    if (busy || tail == head) continue;
    const int e = ep[head];
    if (Bm[e] < 1) return -1;
    int64_t q = 0;                   /* queued queries of the head's epoch */
    while (head + q < tail && ep[head + q] == e) q++;
    int64_t b = 0;
    if (q >= Bm[e]) b = Bm[e];
    else {
      int64_t W = (int64_t)a[head] + L[e] - Tp[e][q + 1];
      if (t >= W) b = q;
      else { armed = 1; timer = W; }
    }
    if (b) {
      F = t + Tp[e][b];
      for (int64_t j = head; j < head + b; j++) {
        int64_t l = F - (int64_t)a[j];
        lat[j] = l >= (int64_t)UINT32_MAX ? UINT32_MAX - 1 : (uint32_t)l;
      }
      head += b;
      busy = 1;
      armed = 0;
    }
  }
  return 0;
}

/* Full closed-loop replay: route every epoch, simulate every (device,
 * scenario) lane across the epochs, count per scenario (violation: latency >
 * the query's epoch SLO, R6; accuracy of the serving epoch's variant, R9).
 * Scenarios as orc_replay ([S][4]); routing must be 0 and policy 0. */
int orc_replay_epochs(int64_t N, const uint32_t *arrival, const uint8_t *family, int E, int64_t epoch_us,
                      int T, int Q, const int32_t *V, const int32_t *acc, int bmax, const int32_t *lat_tab,
                      int D, const int32_t *option, const int32_t *z, const int32_t *dev_type,
                      const int32_t *demand, const int32_t *slo_base, int S, const int32_t *sc,
                      uint32_t *latency, uint64_t *viol, uint64_t *ontime, uint64_t *accsum) {
  (void)T;
  int M = 0;
  for (int q = 0; q < Q; q++) M += V[q];
  if (M > 4096 || D > ORC_MAXD || E < 1 || epoch_us < 1) return -1;
  for (int s = 0; s < S; s++) if (sc[s * 4 + 2] != 0 || sc[s * 4 + 3] != 0) return -1;
  for (int64_t i = 1; i < N; i++) if (arrival[i] < arrival[i - 1]) return -5;
  int32_t *fam_m = (int32_t *)malloc(sizeof(int32_t) * M);
  { int m = 0; for (int q = 0; q < Q; q++) for (int v = 0; v < V[q]; v++) fam_m[m++] = q; }
  int32_t *ep = (int32_t *)malloc(sizeof(int32_t) * (N ? N : 1));
  int32_t *target = (int32_t *)malloc(sizeof(int32_t) * (N ? N : 1));
  for (int64_t i = 0; i < N; i++) {
    int64_t e = (int64_t)arrival[i] / epoch_us;
    if (e >= E) { free(fam_m); free(ep); free(target); return -5; }
    ep[i] = (int32_t)e;
  }
  /* F2: route each epoch's queries with a fresh SWRR over that epoch's weights */
  for (int64_t i0 = 0; i0 < N;) {
    int64_t i1 = i0;
    while (i1 < N && ep[i1] == ep[i0]) i1++;
    const int e = ep[i0];
    int32_t dev_family[ORC_MAXD], wdev[ORC_MAXD], wsink[ORC_MAXQ];
    for (int q = 0; q < Q; q++) wsink[q] = demand[(size_t)e * Q + q];
    for (int d = 0; d < D; d++) {
      const int o = option[(size_t)e * D + d];
      dev_family[d] = o > 0 ? fam_m[o - 1] : -1;
      wdev[d] = o > 0 ? z[(size_t)e * D + d] : 0;
      if (o > 0) wsink[dev_family[d]] -= wdev[d];
    }
    for (int q = 0; q < Q; q++) if (wsink[q] < 0) { free(fam_m); free(ep); free(target); return -1; }
    orc_route_swrr(i1 - i0, family + i0, Q, D, dev_family, wdev, wsink, target + i0);
    i0 = i1;
  }
  for (int s = 0; s < S; s++) { viol[s] = 0; ontime[s] = 0; accsum[s] = 0; }
  uint32_t *a = (uint32_t *)malloc(sizeof(uint32_t) * (N ? N : 1));
  uint32_t *l = (uint32_t *)malloc(sizeof(uint32_t) * (N ? N : 1));
  int32_t *eq = (int32_t *)malloc(sizeof(int32_t) * (N ? N : 1));
  int64_t *idx = (int64_t *)malloc(sizeof(int64_t) * (N ? N : 1));
  const int32_t **Tp = (const int32_t **)malloc(sizeof(int32_t *) * E);
  int32_t *Tbuf = (int32_t *)malloc(sizeof(int32_t) * (size_t)E * (bmax + 1));
  int32_t *Bm = (int32_t *)malloc(sizeof(int32_t) * E);
  int64_t *Lv = (int64_t *)malloc(sizeof(int64_t) * E);
  for (int s = 0; s < S; s++) {
    for (int d = 0; d <= D; d++) {
      int64_t n = 0;
      for (int64_t i = 0; i < N; i++)
        if (target[i] == d) { a[n] = arrival[i]; eq[n] = ep[i]; idx[n] = i; n++; }
      if (d == D) {                  /* the sinks: dropped (R7) */
        viol[s] += (uint64_t)n;
        if (latency) for (int64_t k = 0; k < n; k++) latency[(size_t)s * N + idx[k]] = UINT32_MAX;
        continue;
      }
      if (n == 0) continue;
      for (int e = 0; e < E; e++) {  /* this device's variant in every epoch */
        const int o = option[(size_t)e * D + d];
        int32_t *row = Tbuf + (size_t)e * (bmax + 1);
        Tp[e] = row;
        Bm[e] = 0; Lv[e] = 0; row[0] = 0;
        if (o <= 0) continue;
        const int32_t *tr = lat_tab + ((size_t)dev_type[d] * M + o - 1) * bmax;
        int dep = 0;
        while (dep < bmax && tr[dep] > 0) dep++;
        for (int b = 1; b <= dep; b++) row[b] = tr[b - 1];
        const int cap = sc[s * 4 + 1];
        const int Bcap = (cap > 0 && cap < dep) ? cap : dep;
        Lv[e] = (int64_t)sc[s * 4 + 0] * slo_base[fam_m[o - 1]] / 1000;
        Bm[e] = 1;  /* the maximum allowed batch size of the epoch's variant (R4') */
        for (int b = 1; b <= Bcap && b <= 1024; b++) if (2LL * row[b] <= Lv[e]) Bm[e] = b;
      }
      if (orc_replay_device_epochs(n, a, eq, Tp, Bm, Lv, l) != 0) {
        free(fam_m); free(ep); free(target); free(a); free(l); free(eq); free(idx); free(Tp); free(Tbuf);
        free(Bm); free(Lv);
        return -1;
      }
      for (int64_t k = 0; k < n; k++) {
        const int e = eq[k], m = option[(size_t)e * D + d] - 1;
        if ((int64_t)l[k] > Lv[e]) viol[s]++;
        else { ontime[s]++; accsum[s] += (uint64_t)acc[m]; }
        if (latency) latency[(size_t)s * N + idx[k]] = l[k];
      }
    }
  }
  free(fam_m); free(ep); free(target); free(a); free(l); free(eq); free(idx); free(Tp); free(Tbuf); free(Bm);
  free(Lv);
  return 0;
}

/* --------------------------------------------------------------- Fig. 1b -- */
/* "all possible mappings between 5 EfficientNet variants and 5
 * devices ... all devices serve the maximum number of queries feasible without
 * SLO violations.  Out of all 3125 possible configurations, we are only
 * interested in those at the Pareto frontier".
 * Readings: P1 system throughput capacity = sum_d P(t_d, m_d) and
 * system accuracy = the capacity-weighted mean sum_d P A / sum_d P, kept as
 * the exact pair (cap, accsum); P2 a configuration of capacity 0 has accuracy
 * 0; P3 a configuration is on the frontier iff no configuration has capacity
 * >= and accuracy >= with one of them strict (accuracies compared exactly by
 * cross-multiplication); equal points are one frontier point, reported with
 * the lowest index; P4 configurations are digits o_d in [0, K), device 0 most
 * significant, K = V (every device hosts a variant, as in Fig. 1b) or V + 1
 * with o = 0 idle when allow_idle.
 * Enumerates every configuration; per distinct capacity keeps the largest
 * accsum (at equal capacity a larger accsum dominates) with the lowest index,
 * then tests every pair of those points for dominance.  P[t][m] is the a1
 * capacity table.  Writes up to max_out points sorted by capacity; returns the
 * number of configurations in *n_cfg and of frontier points in *n_out. */
static int acc_ge(int64_t a1, int64_t c1, int64_t a2, int64_t c2) {  /* a1/c1 >= a2/c2, 0/0 = 0 */
  const __int128 l = (__int128)a1 * (c2 > 0 ? c2 : 1), r = (__int128)a2 * (c1 > 0 ? c1 : 1);
  if (c1 == 0 && c2 == 0) return 1;
  if (c1 == 0) return a2 == 0;   /* accuracy 0 >= a2/c2 iff a2 == 0 */
  if (c2 == 0) return 1;         /* anything >= 0 */
  return l >= r;
}

int orc_pareto(int D, const int32_t *dev_type, int M, const int32_t *P, const int32_t *acc, int off, int V,
               int allow_idle, int64_t max_out, int64_t *cap_out, int64_t *accsum_out, uint64_t *idx_out,
               uint64_t *n_cfg, int64_t *n_out) {
  const int K = V + (allow_idle ? 1 : 0);
  uint64_t n = 1;
  for (int d = 0; d < D; d++) {
    if (n > (1ull << 40) / (uint64_t)K) return -1;
    n *= (uint64_t)K;
  }
  int64_t cmax = 0;
  for (int d = 0; d < D; d++) {
    int64_t b = 0;
    for (int v = 0; v < V; v++) b = P[dev_type[d] * M + off + v] > b ? P[dev_type[d] * M + off + v] : b;
    cmax += b;
  }
  int64_t *best_acc = malloc((cmax + 1) * sizeof(int64_t));
  uint64_t *best_idx = malloc((cmax + 1) * sizeof(uint64_t));
  for (int64_t c = 0; c <= cmax; c++) { best_acc[c] = -1; best_idx[c] = 0; }
  int32_t dig[ORC_MAXD];
  for (uint64_t i = 0; i < n; i++) {
    uint64_t x = i;
    for (int d = D - 1; d >= 0; d--) { dig[d] = (int32_t)(x % K); x /= K; }
    int64_t cap = 0, as = 0;
    for (int d = 0; d < D; d++) {
      const int o = dig[d];
      if (allow_idle && o == 0) continue;
      const int m = off + o - (allow_idle ? 1 : 0);
      const int64_t pc = P[dev_type[d] * M + m];
      cap += pc;
      as += pc * acc[m];
    }
    if (as > best_acc[cap]) { best_acc[cap] = as; best_idx[cap] = i; }  /* i ascends: first = lowest index */
  }
  int64_t nf = 0;
  for (int64_t c = 0; c <= cmax; c++) {
    if (best_acc[c] < 0) continue;
    int dominated = 0;
    for (int64_t c2 = 0; c2 <= cmax && !dominated; c2++) {
      if (c2 == c || best_acc[c2] < 0 || c2 < c) continue;
      /* c2 > c: dominated iff accuracy(c2) >= accuracy(c) */
      if (acc_ge(best_acc[c2], c2, best_acc[c], c)) dominated = 1;
    }
    if (dominated) continue;
    if (nf < max_out) { cap_out[nf] = c; accsum_out[nf] = best_acc[c]; idx_out[nf] = best_idx[c]; }
    nf++;
  }
  free(best_acc);
  free(best_idx);
  *n_cfg = n;
  *n_out = nf;
  return 0;
}
