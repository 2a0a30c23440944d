// internal.cuh -- shared declarations of libproteus (CUDA path).  Nothing in
// oracle/ is included or linked here.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <string>
#include <vector>

#include "proteus.h"

#define PX_MAXD 64
#define PX_MAXT 8
#define PX_MAXQ 32
#define PX_MAXV 16
#define PX_MAXM 255
#define PX_MAXB 1024
#define PX_PCLAMP (1 << 22)  // solve-path capacity clamp (prepare.cu): > any demand

// ------------------------------------------------------------ score ----
// Packed objective (reading C1): served in the high 22 bits, accuracy sum in
// the low 42.  With sum(s) < 2^22 and A <= 10^6 < 2^20, accsum < 2^42, so the
// integer order of the packed value is the lexicographic (served, accsum)
// order and per-family packed values add without carry.
#define PX_ACC_BITS 42
__host__ __device__ __forceinline__ uint64_t px_pack(uint64_t served, uint64_t accsum) {
  return (served << PX_ACC_BITS) + accsum;
}
__host__ __device__ __forceinline__ uint64_t px_served(uint64_t score) { return score >> PX_ACC_BITS; }
__host__ __device__ __forceinline__ uint64_t px_accsum(uint64_t score) {
  return score & ((1ull << PX_ACC_BITS) - 1);
}

// (score desc, index asc): the canonical argmax order (reading C9)
__host__ __device__ __forceinline__ bool px_better(uint64_t s1, uint64_t i1, uint64_t s2, uint64_t i2) {
  return s1 > s2 || (s1 == s2 && i1 < i2);
}

struct BestRec {
  uint64_t score, index;
};

// One solved demand vector, as written by the materialise kernels.
struct SolRec {
  uint64_t score, index;
  int64_t served, unmet, accsum;
  int32_t eff, status;  // status != 0: internal check failed
  uint64_t n_candidates;
  int32_t option[PX_MAXD];
  int32_t z[PX_MAXD];
};

// ------------------------------------------------------- device tables ----
// Built on the GPU by k_prepare from the profiles, SLOs and inventory (a1).
// Slot s = q * VM + j orders family q's variants by (accuracy desc, option
// code asc): j is the water-fill position (reading C10).  Pad slots (j >= V_q)
// have code 0, accuracy 0 and capacity 0.
struct Tables {
  int32_t *P;         // [T][M] capacity QPS
  int32_t *depth;     // [T][M] memory depth (leading non-zero run)
  int32_t *slot_of;   // [M]
  int32_t *slot_code; // [Q*VM]
  int32_t *slot_acc;  // [Q*VM]
  int32_t *code_slot; // [K] (code 0 -> -1)
  int32_t *Pdev;      // [D][K] capacity of option code on device d (code 0 -> 0)
};

// ------------------------------------------------------------ context ----
struct DevBuf {
  void *p = nullptr;
  size_t n = 0;
};

struct proteus_ctx {
  int device = 0;
  cudaStream_t stream = nullptr;
  std::string err;
  // profiles
  bool have_prof = false;
  int T = 0, Q = 0, M = 0, bmax = 0;
  std::vector<int32_t> V, acc, lat, fam, off;
  int32_t *d_lat = nullptr, *d_acc = nullptr, *d_fam = nullptr, *d_off = nullptr, *d_V = nullptr;
  DevBuf bufs[56];
  // instrumentation
  bool timing = false;
  uint64_t launches = 0;
  std::vector<const char *> tnames;
  std::vector<cudaEvent_t> tev;  // pairs
  std::vector<float> tms;
  std::vector<cudaEvent_t> ev_pool;
  // cached per-call solve tables (see solve_common)
  uint32_t prof_gen = 0;
  bool tab_valid = false;
  std::vector<int32_t> tab_key, tab_P, tab_slot_code;
  Tables tab;
  // cached DP budget orders of the factored search (solve_factored.cu)
  void *dp_order = nullptr;
  int32_t dp_order_U = -1;
  std::vector<int32_t> dp_order_key;
  int64_t dp_items_stride = 0;
  void *gv_order = nullptr;  // cells of the batched g kernel by decreasing size
  std::vector<int32_t> gv_order_key;
  std::vector<int32_t> dp_items_n;
  // cached count-vector lists of the factored search
  void *fact_lists_buf = nullptr;
  std::vector<int32_t> fact_lists_key;
  // flat kernel occupancy per (instantiation, shared-memory size) on this device
  std::vector<std::pair<std::pair<const void *, size_t>, int>> occ_cache;
  // NCCL communicator (comm.cu): calls shard over it while comm_on
  void *comm = nullptr;
  int comm_world = 1, comm_rank = 0;
  bool comm_on = false;
  // auxiliary stream for concurrent kernels of one call (replay.cu: k_stitch
  // alongside k_spec), joined back with events before the call continues
  cudaStream_t aux = nullptr, aux_hi = nullptr;  // lowest / highest stream priority
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr, ev_join2 = nullptr;
  // replay chain path: the ticket order last uploaded per routing mode (its key: lanes, chunks per lane)
  std::vector<int64_t> chain_ukey[3];  // [2]: the closed loop's
};

// scratch buffer ids
enum {
  B_TABLES = 0, B_BEST, B_SOL, B_IN0, B_IN1, B_IN2, B_IN3, B_FACT0, B_FACT1, B_FACT2, B_FACT3,
  B_R_PAT, B_R_TGT, B_R_HIST, B_R_BASE, B_R_DEVARR, B_R_DEVIDX, B_R_OFF, B_R_LAT, B_R_AGG, B_R_TGT1,
  B_R_DEVARR1, B_R_DEVIDX1, B_R_OFF1, B_R_MISC, B_R_LANE, B_R_DBASE0, B_R_DBASE1, B_R_LATD, B_R_VLAT, B_R_VEX, B_R_VOFF, B_FACT4, B_R_SCAN, B_R_BSCAN, B_PARETO, B_E_MISC, B_E_PAT, B_E_EXIT, B_R_WST, B_R_WEX, B_C_KEEP, B_C_GATHER, B_C_PTS, B_W_REC, B_W_ENT, B_W_AUX, B_R_READY, B_R_CHAIN, B_R_UNITS0, B_R_UNITS1, B_R_NX, B_R_CCNT, B_E_CHAIN, B_E_UNITS, B_NBUF
};
static_assert(B_NBUF <= 56, "proteus_ctx::bufs is too small");

// errors
int px_fail(proteus_ctx *ctx, int code, const char *fmt, ...);
#define PX_CUDA(ctx, call)                                                                 \
  do {                                                                                     \
    cudaError_t e_ = (call);                                                               \
    if (e_ != cudaSuccess) return px_fail(ctx, PROTEUS_ECUDA, "%s: %s", #call, cudaGetErrorString(e_)); \
  } while (0)

void *px_buf(proteus_ctx *ctx, int id, size_t bytes);  // grow-only; nullptr on failure
bool px_is_device_ptr(const void *p);

// launch bookkeeping (timing events when enabled)
void px_launch_begin(proteus_ctx *ctx, const char *name);
int px_launch_end(proteus_ctx *ctx);

#define PX_LAUNCH(ctx, name, kernel, grid, block, smem, ...)                    \
  do {                                                                          \
    px_launch_begin(ctx, name);                                                 \
    kernel<<<(grid), (block), (smem), (ctx)->stream>>>(__VA_ARGS__);            \
    int rc_ = px_launch_end(ctx);                                               \
    if (rc_) return rc_;                                                        \
  } while (0)

// ---------------------------------------------------------- sub-modules ----
int px_solve_enum(proteus_ctx *ctx, const proteus_solve_args *a, const int32_t *h_dev_type,
                  const int32_t *h_slo, const int32_t *h_demand, int VM, const Tables &tab,
                  const std::vector<int32_t> &h_P, const std::vector<int32_t> &h_slot_code,
                  SolRec *d_sol, int32_t vec_lo, int32_t vec_hi, bool materialize_only, uint64_t mat_index,
                  bool use_flat, const int32_t *d_demand /* [n_vec][Q] on the device */);
int px_solve_factored(proteus_ctx *ctx, const proteus_solve_args *a, const int32_t *h_dev_type,
                      const int32_t *d_dev, const int32_t *d_demand, int VM, const Tables &tab, const std::vector<int32_t> &h_P,
                      SolRec *d_sol);
int px_prepare_tables(proteus_ctx *ctx, int D, const int32_t *d_dev_type, const int32_t *d_slo, int VM,
                      Tables &tab, bool clamp);
uint64_t px_count_candidates(int mode, int D, const int32_t *dev_type, int T, int K, bool *overflow);

// comm.cu: the NCCL communicator and the combine kernels
enum { PX_RED_SUM = 0, PX_RED_MAX = 1 /* int64 */, PX_RED_MIN = 2 };
bool px_comm_active(const proteus_ctx *ctx);
int px_comm_allgather(proteus_ctx *ctx, const void *send, void *recv, size_t bytes);
int px_comm_allreduce_u64(proteus_ctx *ctx, void *buf, size_t count, int op);
int px_pick_solrec(proteus_ctx *ctx, const SolRec *d_gathered, int world, int n, SolRec *d_out);
int px_gather_vectors(proteus_ctx *ctx, const SolRec *d_gathered, int world, int n, int stride, SolRec *d_out);
int px_pareto_merge(proteus_ctx *ctx, const proteus_pareto_point *d_pts, int n, proteus_pareto_point *d_out,
                    int32_t *d_n);
void px_scenario_owner(const proteus_scenario *sc, int S, int world, int32_t *owner);
void px_comm_destroy(proteus_ctx *ctx);
int px_occupancy(proteus_ctx *ctx, const void *kern, int threads, size_t smem, int *occ);

int px_pareto(proteus_ctx *ctx, int D, const int32_t *h_dev_type, const int32_t *d_dev, const int32_t *d_slo,
              int family, int allow_idle, int rank, int world, proteus_pareto_point *out, int32_t max_points,
              int32_t *n_points, uint64_t *n_configs);
int px_replay(proteus_ctx *ctx, const uint32_t *d_arr, const uint8_t *d_fam, int64_t N, const int32_t *h_option,
              const int32_t *h_z, const int32_t *h_dev_type, int D, const int32_t *h_demand, const int32_t *h_slo,
              const proteus_scenario *h_sc, int S, uint32_t *d_lat_out, uint64_t *d_agg /* [3][S] */);
int px_replay_epochs(proteus_ctx *ctx, const uint32_t *d_arr, const uint8_t *d_fam, int64_t N, int E,
                     int64_t epoch_us, const int32_t *h_option, const int32_t *h_z, const int32_t *h_dev_type, int D,
                     const int32_t *h_demand, const int32_t *h_slo, const proteus_scenario *h_sc, int S,
                     uint32_t *d_lat_out, uint64_t *d_agg /* [3][S] */);
