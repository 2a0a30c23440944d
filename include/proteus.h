/*
 * proteus.h -- C ABI of libproteus.so, the B200-native hot path of Proteus's
 * accuracy-scaling method (Ahmad, Guan, Friedman, Williams, Sitaraman, Woo,
 * ASPLOS '24).  "P:a-b" cites lines a-b of the paper text; readings
 * C1-C17 / R1-R13 are listed in DESIGN.md §2.
 *
 * Three calls form the path:
 *   proteus_load_profiles  the profile store: accuracy and latency
 *                          per (device type, variant, batch size)
 *   proteus_solve          the joint allocation search: model selection +
 *                          placement + query assignment maximising effective
 *                          accuracy under the throughput constraint
 *                          (§4, Table 1, Eqs. 1-7)
 *   proteus_replay         trace replay of an allocation under the adaptive
 *                          batching policy of §5
 *
 * Conventions (all calls):
 *   - Every function returns an int status: PROTEUS_OK (0) or a negative
 *     PROTEUS_E* code; proteus_last_error() gives a one-line reason.  Input
 *     errors are detected before any output is touched; host output buffers
 *     are written only on success (outputs are staged and copied out last);
 *     a CUDA failure mid-call may leave device output buffers partly written.
 *   - Pointer arguments may point to host memory or to device memory of the
 *     context's GPU (detected with cudaPointerGetAttributes).  Host inputs are
 *     copied to the device inside the call; host outputs are copied back.
 *   - Inputs are borrowed for the duration of the call; the caller keeps
 *     ownership.  The library never frees caller memory.
 *   - Calls are synchronous: on return every output is valid.
 *   - A context is bound to one GPU and one CUDA stream and is not
 *     thread-safe; use one context per (process, GPU, host thread).
 *   - All arithmetic is integer: accuracy in 1e-6 units (0 < A <= 10^6),
 *     capacity and demand in integer QPS, latencies and timestamps in integer
 *     microseconds.  Results are deterministic and bit-identical across runs
 *     and shard counts.
 */
#ifndef PROTEUS_H
#define PROTEUS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PROTEUS_ABI_VERSION 3

enum {
  PROTEUS_OK = 0,
  PROTEUS_EINVAL = -1,  /* bad argument (null pointer, out-of-range value, no profiles loaded) */
  PROTEUS_ENOMEM = -2,  /* device or host allocation failed */
  PROTEUS_ECUDA = -3,   /* a CUDA call failed */
  PROTEUS_ENCCL = -4,   /* NCCL missing or an NCCL call failed (proteus_comm_*, distributed calls) */
  PROTEUS_ERANGE = -5,  /* overflow guard: sum of demand >= 2^22, N >= 2^32, unsorted
                           timestamps, or candidate space above max_candidates / 2^63 */
  PROTEUS_EINTERNAL = -6 /* an internal consistency check failed (a bug) */
};

typedef struct proteus_ctx proteus_ctx;

/* ABI version of the loaded library (== PROTEUS_ABI_VERSION). */
int proteus_abi_version(void);

/* Create a context on CUDA device `cuda_device`; kernels are issued on
 * `cuda_stream` (a cudaStream_t; NULL = the legacy default stream).
 * *out receives the context; free it with proteus_destroy. */
int proteus_create(proteus_ctx **out, int cuda_device, void *cuda_stream);
void proteus_destroy(proteus_ctx *ctx);
/* Change the stream later calls are issued on. */
int proteus_set_stream(proteus_ctx *ctx, void *cuda_stream);
/* Reason for the last failed call on this context ("" if none). */
const char *proteus_last_error(const proteus_ctx *ctx);

/* ------------------------------------------------------------ profiles --
 * P:675-680 (profile store keyed by variant, device type, batch size);
 * P:1137-1142 (accuracy normalised per family).  Variant m = 0..M-1 is
 * family-major in the caller's order; option code o = 1 + m, code 0 = idle
 * (reading C8).
 *   T          number of device types (1..8)
 *   Q          number of model families = query types (1..32)
 *   V[Q]       variants per family (1..16); M = sum V <= 255
 *   acc_micro  [M] normalised accuracy, 1..10^6
 *   bmax       batch sizes profiled (1..1024)
 *   lat_us     [T][M][bmax] average latency of a batch of b = 1..bmax at
 *              index [t][m][b-1], > 0; 0 = does not fit in memory (the table
 *              depth of (t, m) is the length of its leading non-zero run,
 *              reading C7).
 * Copied into the context (device memory); replaces earlier profiles. */
typedef struct {
  int32_t T, Q;
  const int32_t *V;
  const int32_t *acc_micro;
  int32_t bmax;
  const int32_t *lat_us;
} proteus_profiles;

int proteus_load_profiles(proteus_ctx *ctx, const proteus_profiles *prof);

/* --------------------------------------------------------------- solve --
 * §4.  For each demand vector s, find the placement x (each
 * device hosts at most one variant or idles, Eq. 1) and assignment z (Eqs.
 * 2-6) maximising, lexicographically, first the served QPS sum_q min(s_q,
 * capacity) (reading C1 of the infeasibility rule P:901-907), then the accuracy
 * sum sum_q a_q (Eq. 7, reading C2).  Capacity per (type, variant) is
 * P = floor(b* 10^6 / lat(b*)), b* = largest b <= depth with 2 lat(b) <= SLO
 * (readings C4-C6).  Within a family, demand is water-filled over
 * the hosting devices in (accuracy desc, option code asc, device asc) order,
 * which is an exact LP optimum (reading C10).
 *
 *   D, device_type[D]  inventory: device d has type device_type[d] in [0, T)
 *                      (D <= 64)
 *   mode   0  flat mixed radix: every assignment of K = 1 + M option codes
 *             to the D devices; canonical index = sum_d o_d K^(D-1-d)
 *          1  multiset: devices of one type are interchangeable; per type
 *             the sorted option tuple (lexicographic rank), types mixed
 *             radix with type 0 most significant
 *          2  family-factored: exact search over per-family count vectors
 *             n[q][t][v] combined by a budget DP; canonical solution = the
 *             lexicographically smallest n (q-major, then t, then v); devices
 *             of each type take options in (q, v) order, ascending device index
 *          Modes 0 and 1 return the lowest canonical index among optima
 *          (reading C9); all modes return the same optimal value.
 *   slo_us[Q]          latency SLO per family (used for capacity)
 *   n_vec, demand_qps  [n_vec][Q] demand vectors; each sum < 2^22
 *   max_candidates     modes 0/1: refuse (PROTEUS_ERANGE) if the candidate
 *                      space is larger; 0 = no limit besides 2^63
 *   shard_rank, shard_world
 *                      modes 0/1: scan only slice shard_rank of shard_world
 *                      contiguous slices of the index space; the returned
 *                      solution is the best of that slice (combine slices by
 *                      (score desc, index asc)).  world 1 = whole space.
 *                      Mode 2 ignores them (shard demand vectors instead).
 *   flags              bit 0 (PROTEUS_SOLVE_GENERIC): use the generic scoring
 *                      kernel even where a specialised one exists (testing).
 */
#define PROTEUS_SOLVE_GENERIC 1

typedef struct {
  int32_t D;
  const int32_t *device_type;
  int32_t mode;
  const int32_t *slo_us;
  int32_t n_vec;
  const int32_t *demand_qps;
  uint64_t max_candidates;
  int32_t shard_rank, shard_world;
  int32_t flags;
} proteus_solve_args;

/* One solution per demand vector.
 *   score         (served << 42) | accsum: integer order = lexicographic order
 *   index         canonical index (modes 0/1); UINT64_MAX in mode 2
 *   served, unmet, accsum   QPS served, QPS not served, sum of A * z
 *   eff_acc_micro floor(accsum / served), 0 if served = 0 (reading C3)
 *   n_candidates  placements (modes 0/1) or per-family count vectors (mode 2)
 *                 scored for this vector in this call
 *   option        caller buffer [D] or NULL: 0 idle or option code 1 + m
 *   z_qps         caller buffer [D] or NULL: assigned integer QPS per device
 */
typedef struct {
  uint64_t score, index;
  int64_t served, unmet, accsum;
  int32_t eff_acc_micro;
  int32_t reserved;
  uint64_t n_candidates;
  int32_t *option;
  int32_t *z_qps;
} proteus_solution;

int proteus_solve(proteus_ctx *ctx, const proteus_solve_args *args, proteus_solution *out /* [n_vec] */);

/* Batched form of proteus_solve for many demand vectors (the per-second
 * re-solve): the same search, outputs as arrays.
 * Every pointer may be NULL (not produced), host memory or device memory,
 * independently; device outputs are written by a kernel on the context's
 * stream without a host round trip of the solutions.
 *   score, index            [n_vec] as proteus_solution
 *   served, unmet, accsum   [n_vec]
 *   eff_acc_micro           [n_vec]
 *   option, z_qps           [n_vec][D] row-major
 * n_candidates (out) is the per-vector count of proteus_solve.  Host outputs
 * are written only on success; device outputs are written before the final
 * internal check, so a PROTEUS_EINTERNAL return may leave them written. */
typedef struct {
  uint64_t *score, *index;
  int64_t *served, *unmet, *accsum;
  int32_t *eff_acc_micro;
  int32_t *option;
  int32_t *z_qps;
  uint64_t n_candidates;  /* out: count vectors / placements scored per vector */
} proteus_batch;

int proteus_solve_batch(proteus_ctx *ctx, const proteus_solve_args *args, proteus_batch *out);

/* Modes 0/1: the full solution (placement, z, value) of canonical index
 * `index` for demand vector `vec` -- used after combining shard results. */
int proteus_materialize(proteus_ctx *ctx, const proteus_solve_args *args, int32_t vec, uint64_t index,
                        proteus_solution *out);

/* Size of the candidate space of args (modes 0/1), or PROTEUS_ERANGE. */
int proteus_candidate_count(proteus_ctx *ctx, const proteus_solve_args *args, uint64_t *count);

/* -------------------------------------------------------------- pareto --
 * Fig. 1b: every configuration of family `family`'s variants on
 * the D devices ("all possible mappings"), each device serving its capacity
 * P (the a1 estimate under slo_us, "the maximum number of queries feasible
 * without SLO violations"), and the Pareto frontier of system throughput
 * capacity C = sum_d P against system accuracy = the capacity-weighted mean
 * sum_d P A / C (readings P1-P4).
 *   D, device_type[D], slo_us[Q]   as proteus_solve (host or device)
 *   family        the family q whose variants are placed
 *   allow_idle    0: every device hosts one of the V_q variants (K = V_q, as
 *                 Fig. 1b's 5^5 = 3125); 1: a device may also idle (digit 0,
 *                 K = V_q + 1)
 *   shard_rank, shard_world   scan slice shard_rank of shard_world contiguous
 *                 slices of the index space; the union of the slices'
 *                 frontiers contains the whole space's, so the frontier of
 *                 that union (dist.py: pareto_merge) is the whole answer
 * A configuration is the mixed-radix number of its digits o_d in [0, K),
 * device 0 most significant.  A point is on the frontier iff no
 * configuration has capacity >= and accuracy >= with one of them strict
 * (accuracies compared exactly; capacity 0 has accuracy 0); each point is
 * reported once with the lowest index reaching it.
 * Output: up to max_points points sorted by increasing capacity (accuracy
 * strictly decreasing) in out[]; *n_points = the frontier size (may exceed
 * max_points: then only the first max_points are written); *n_configs = the
 * configurations scanned.  PROTEUS_ERANGE if the space exceeds 2^63 or the
 * capacity range 2^26. */
typedef struct {
  int32_t D;
  const int32_t *device_type;
  const int32_t *slo_us;
  int32_t family;
  int32_t allow_idle;
  int32_t shard_rank, shard_world;
} proteus_pareto_args;

typedef struct {
  int64_t capacity;  /* sum of P over the devices, QPS */
  int64_t accsum;    /* sum of P * A (accuracy = accsum / capacity, 1e-6 units) */
  uint64_t index;    /* lowest configuration index at this point */
} proteus_pareto_point;

int proteus_pareto(proteus_ctx *ctx, const proteus_pareto_args *args, proteus_pareto_point *out, int32_t max_points,
                   int32_t *n_points, uint64_t *n_configs);

/* -------------------------------------------------------------- replay --
 * §5 adaptive batching over an allocation, per scenario.
 *   arrival_us[N]   query arrival times, sorted non-decreasing, uint32 us
 *   family[N]       query type of each query, < Q
 *   option[D], z_qps[D], device_type[D]   the allocation (as from
 *                   proteus_solve) and the inventory
 *   demand_qps[Q]   the demand vector the allocation was solved for; unmet
 *                   demand s_q - sum z is routed to a drop sink
 *   slo_base_us[Q]  base SLO per family
 *   sc[S]           scenarios: slo_mult_milli (scenario SLO =
 *                   floor(mult * base / 1000), reading R12), batch_cap
 *                   (0 = table depth; Bmax = min(cap, depth), R4), routing
 *                   (0 = smooth weighted round-robin over z with the sink,
 *                   1 = uniform over hosting devices that fit batch 1, no
 *                   sink; reading R8), policy (the batching rule on every
 *                   device: 0 = §5 adaptive batching below; 1 = Nexus early
 *                   drop, 2 = Clipper AIMD -- the §6.4 baselines, P:1535-1630,
 *                   readings R14-R15 below)
 * Routing (R8): per family, query k goes to pattern_q[k mod W_q] of the SWRR
 * sequence over the members (hosting devices ascending, then the sink).
 * Batching per device (R1-R5): at decision time t with q queued, dispatch
 * Bmax if q >= Bmax, else q once t >= a_head + SLO - T(q+1), else wait for the
 * next arrival or that time; a batch of b dispatched at t finishes at t+T(b),
 * T(b) = lat_us of the device's variant (R10).
 * Baseline policies (§8(f2); work-conserving: a batch leaves at
 * t = max(F, a_head), the moment the device is free and a query waits):
 *   1 Nexus early drop (R14): batch size B = the
 *     largest b <= Bmax with 2 T(b) <= SLO (the capacity rule), at
 *     least 1; from the head, the first queued query i whose deadline
 *     a_i + SLO is met by t + T(min(B, queued from i)) starts the batch and
 *     the queries before it are dropped (latency UINT32_MAX).
 *   2 Clipper AIMD (R15): a batch takes
 *     min(queued, limit); limit starts at 1, grows by 1 (up to Bmax) after a
 *     batch with no query latency > SLO, else becomes max(1, floor(9 limit /
 *     10)).  Nothing is dropped.
 * Outputs (each may be NULL):
 *   latency_us[S][N]  per-query latency F - a (UINT32_MAX = dropped)
 *   violations[S]     latency > SLO (strict, R6) plus dropped
 *   on_time[S]        latency <= SLO
 *   acc_sum[S]        sum of the serving variant's accuracy over on-time queries
 */
typedef struct {
  int32_t slo_mult_milli;
  int32_t batch_cap;
  int32_t routing;
  int32_t policy;  /* 0 = §5 adaptive batching, 1 = Nexus early drop, 2 = Clipper AIMD (ABI 2) */
} proteus_scenario;

#define PROTEUS_POLICY_PROTEUS 0
#define PROTEUS_POLICY_NEXUS 1
#define PROTEUS_POLICY_AIMD 2

int proteus_replay(proteus_ctx *ctx, const uint32_t *arrival_us, const uint8_t *family, int64_t N,
                   const int32_t *option, const int32_t *z_qps, const int32_t *device_type, int32_t D,
                   const int32_t *demand_qps, const int32_t *slo_base_us,
                   const proteus_scenario *sc, int32_t S,
                   uint32_t *latency_us, uint64_t *violations, uint64_t *on_time, uint64_t *acc_sum);

/* ------------------------------------------------------ closed loop --
 * §8(f4): the per-second re-solve (the paper re-solves
 * every 30 s) feeding the replay.  Time is cut into E epochs of
 * epoch_us; epoch e runs allocation e (typically proteus_solve_batch's
 * outputs for the controller's demand estimates, left on the device).
 * Readings F1-F4:
 *   F1  query i belongs to epoch floor(arrival_us[i] / epoch_us) < E
 *       (PROTEUS_ERANGE otherwise);
 *   F2  routing restarts every epoch: SWRR over z[e] of the devices hosting
 *       the family with the sink weight demand[e][q] - sum z (R8);
 *   F3  switching is free (C14) but a device finishes the queue of one epoch
 *       with that epoch's variant before serving the next epoch's queries: a
 *       batch holds queries of one epoch;
 *   F4  the §5 rule (R1-R13) with the head's epoch's variant T(b), Bmax and
 *       SLO; violations and accuracy use the query's epoch's variant.
 *   arrival_us[N], family[N]   as proteus_replay
 *   option[E][D], z_qps[E][D]  allocation per epoch (row-major)
 *   demand_qps[E][Q]           the demand each allocation was solved for
 *   device_type[D], slo_base_us[Q], sc[S]   as proteus_replay; every scenario
 *                  must have routing 0 and policy 0 (PROTEUS_EINVAL otherwise)
 * Outputs as proteus_replay. */
int proteus_replay_epochs(proteus_ctx *ctx, const uint32_t *arrival_us, const uint8_t *family, int64_t N,
                          int32_t E, int64_t epoch_us, const int32_t *option, const int32_t *z_qps,
                          const int32_t *device_type, int32_t D, const int32_t *demand_qps,
                          const int32_t *slo_base_us, const proteus_scenario *sc, int32_t S, uint32_t *latency_us,
                          uint64_t *violations, uint64_t *on_time, uint64_t *acc_sum);

/* -------------------------------------------------------- multi-GPU --
 * one process per GPU, one context each, joined by an
 * NCCL communicator the context owns (NCCL is loaded at run time: the copy
 * already in the process, else libnccl.so.2; PROTEUS_NCCL_LIB overrides).
 * While the communicator is enabled, calls are DISTRIBUTED: every rank must
 * make the same call with the same arguments (collectives run on the
 * context's stream, in call order), and every rank returns the combined
 * result:
 *   proteus_solve / proteus_solve_batch, modes 0/1: rank r scans slice r of
 *     `world` contiguous slices of the index space (shard_rank / shard_world
 *     must be 0 / 0 or 1), its per-vector winners -- already materialised --
 *     are exchanged with one ncclAllGather and every rank keeps, per vector,
 *     the (score desc, index asc) maximum on the device; n_candidates is the
 *     whole space's.  Identical to the single-GPU answer.
 *   mode 2 (batched re-solve): demand vectors split by rank (slice r of
 *     n_vec), one ncclAllGather of the solutions; every rank returns all.
 *   proteus_pareto: index slices by rank, one ncclAllReduce(MAX) of the best
 *     accuracy sum per capacity and one ncclAllReduce(MIN) of the lowest
 *     index per frontier point; every rank returns the whole frontier.
 *   proteus_replay / proteus_replay_epochs: scenario s is replayed by rank
 *     owner[s] (proteus_scenario_owner); the per-scenario aggregates are
 *     combined with one ncclAllReduce(SUM) and are complete on every rank;
 *     latency_us holds only this rank's scenarios: row k = its k-th owned
 *     scenario in ascending scenario order ([S_own][N]).
 * Errors are detected before the first collective from the arguments alone,
 * so ranks given the same arguments fail together. */

/* 128-byte NCCL unique id (ncclGetUniqueId) into id_out; rank 0 calls it and
 * the caller broadcasts the bytes (any transport) to the other ranks. */
#define PROTEUS_COMM_ID_BYTES 128
int proteus_comm_unique_id(void *id_out);
/* Create the context's communicator (ncclCommInitRank on the context's GPU;
 * collective over the `world` ranks) and enable it. */
int proteus_comm_init(proteus_ctx *ctx, const void *nccl_unique_id, int world, int rank);
/* Disable (0) / re-enable (1) distributed calls; the communicator is kept. */
int proteus_comm_enable(proteus_ctx *ctx, int enable);
/* *world / *rank of the communicator (1 / 0 without one); returns 1 if calls
 * are distributed, else 0. */
int proteus_comm_info(const proteus_ctx *ctx, int32_t *world, int32_t *rank);
/* The rank that replays scenario s in a distributed replay (host only, no
 * GPU needed): longest-processing-time greedy over a per-scenario lane-cost
 * model, deterministic in (sc, world).  owner[S] out. */
int proteus_scenario_owner(const proteus_scenario *sc, int32_t S, int32_t world, int32_t *owner);

/* Combine per-slice results obtained by any transport (e.g. gloo, MPI):
 * parts[world] are proteus_solve_batch outputs of slices 0..world-1 of the
 * same search (modes 0/1; every part must have score, index, served, unmet,
 * accsum, eff_acc_micro, option, z_qps), combined per vector by (score desc,
 * index asc) on the device into out (as proteus_solve_batch; n_candidates
 * of out = the sum of the parts').  part_candidates[world]: the parts'
 * n_candidates.  Pointers may be host or device. */
int proteus_combine_solutions(proteus_ctx *ctx, int32_t world, int32_t n_vec, int32_t D, const proteus_batch *parts,
                              const uint64_t *part_candidates, proteus_batch *out);
/* Frontier of the union of shard frontiers (proteus_pareto with
 * shard_rank/shard_world, any transport): pts[n] concatenated; out as
 * proteus_pareto (sorted by capacity, lowest index per point). */
int proteus_pareto_merge(proteus_ctx *ctx, const proteus_pareto_point *pts, int32_t n, proteus_pareto_point *out,
                         int32_t max_points, int32_t *n_points);

/* ------------------------------------------------------- instrumentation --
 * proteus_set_timing(ctx, 1) makes later calls record CUDA events around
 * every kernel they launch (on the context's stream).  proteus_kernel_times
 * copies up to `cap` (name, milliseconds) pairs of the last call; names are
 * static strings.  proteus_launch_count returns the number of kernels the
 * context has launched since creation. */
int proteus_set_timing(proteus_ctx *ctx, int enable);
int proteus_kernel_times(const proteus_ctx *ctx, const char **names, float *ms, int cap);
uint64_t proteus_launch_count(const proteus_ctx *ctx);

#ifdef __cplusplus
}
#endif
#endif /* PROTEUS_H */
