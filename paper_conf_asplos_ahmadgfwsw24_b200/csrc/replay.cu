// replay.cu -- trace replay of an allocation under the adaptive batching
// policy of §5: a11 routing pre-pass, a12 lane kernel, a13
// per-scenario reductions.
//
// Routing (reading R8): per family q, the SWRR sequence over the members
// (hosting devices ascending with weight z_d, then a drop sink with weight
// s_q - sum z) has period W_q = sum of weights; query k of family q (k = its
// ordinal among family-q queries) goes to pattern_q[k mod W_q].  The pre-pass
// computes every query's family ordinal and target device with stable
// per-tile counting (warp match + per-tile offsets), then scatters the
// arrivals into per-device arrays (device-major, arrival order kept).
//
// Lanes: the §5 rule per (device, scenario) written as a window walk
// (readings R1-R5): at decision time t = max(F, a[h]) with q queued (capped at
// Bmax), dispatch Bmax when q >= Bmax; otherwise with W = a[h] + SLO - T(q+1)
// dispatch q once t >= W, else move t to the next arrival if it comes by W
// (Case 2), else to W (Case 1).  Three executions of that rule:
//   k_spec   (phase A) every (global window, device, scenario) piece replayed
//            from an idle device into a shared-memory tile of the window's
//            output rows, flushed with coalesced stores; exit states kept;
//   k_stitch (phase B) one warp per (device, scenario) carries the true state
//            across windows and replays only where the speculative start was
//            wrong, until the two runs meet (see below);
//   k_lanes  one thread per (device, scenario) walking everything (fallback,
//            and the reference formulation in the tests).
// a13: k_count reduces the final latency rows to per-scenario violations,
// on-time counts and accuracy sums.
#include <algorithm>
#include <array>
#include <utility>
#include <climits>
#include <cstdlib>
#include <cstring>

#include "internal.cuh"

#define TILE 512
#define TILE_WARPS 8
#define LANE_THREADS 128

// -------------------------------------------------------------- checks ----
__global__ void k_check_trace(const uint32_t *__restrict__ arr, const uint8_t *__restrict__ fam, int64_t N, int Q,
                              uint32_t *flags) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    if (i > 0 && arr[i] < arr[i - 1]) atomicOr(flags, 1u);
    if (fam[i] >= Q) atomicOr(flags, 2u);
  }
}

// ------------------------------------------------------------- routing ----
// Weights and the SWRR pattern of every family (R8); one warp per family.
//   routing 0: member weight z_d for hosting devices with z_d > 0, sink weight
//              s_q - sum z (unmet demand, reading R7)
//   routing 1: weight 1 per hosting device that fits batch 1 (depth >= 1); no sink
// Each step adds every member's weight to its current value, picks the
// largest current value (lowest member index on ties, the sink last) and
// subtracts the period W_q from it: lanes hold members d = lane, lane + 32,
// lane + 64 and the pick is a warp maximum of (current, -index).
__device__ __forceinline__ int32_t route_weight(int routing, int q, int d, int D, int M, int bmax,
                                                const int32_t *option, const int32_t *z, const int32_t *dev_type,
                                                const int32_t *demand, const int32_t *fam_of_m, const int32_t *lat) {
  if (d < D) {
    const int o = option[d];
    if (o <= 0 || fam_of_m[o - 1] != q) return 0;
    if (routing == 0) return z[d];
    return lat[((size_t)dev_type[d] * M + (o - 1)) * bmax] > 0 ? 1 : 0;
  }
  if (routing != 0) return 0;  // the sink: unmet demand
  int64_t zs = 0;
  for (int k = 0; k < D; k++) {
    const int o = option[k];
    if (o > 0 && fam_of_m[o - 1] == q) zs += z[k];
  }
  return (int32_t)(demand[q] - zs);
}

__global__ void k_route_prepare(int routing, int Q, int D, int M, int bmax, const int32_t *__restrict__ option,
                                const int32_t *__restrict__ z, const int32_t *__restrict__ dev_type,
                                const int32_t *__restrict__ demand, const int32_t *__restrict__ fam_of_m,
                                const int32_t *__restrict__ lat, uint8_t *pattern, int32_t *pat_off,
                                int32_t *pat_len) {
  __shared__ int32_t W[PX_MAXQ];
  const int q = blockIdx.x, lane = threadIdx.x;
  // periods of every family (for this family's pattern offset)
  for (int k = lane; k < Q; k += 32) {
    int64_t tot = 0;
    for (int d = 0; d <= D; d++) tot += route_weight(routing, k, d, D, M, bmax, option, z, dev_type, demand, fam_of_m, lat);
    W[k] = (int32_t)tot;
  }
  __syncwarp();
  int32_t off = 0;
  for (int k = 0; k < q; k++) off += W[k];
  const int32_t Wq = W[q];
  if (lane == 0) { pat_off[q] = off; pat_len[q] = Wq; }
  int32_t w[3], cur[3];
#pragma unroll
  for (int i = 0; i < 3; i++) {
    const int d = lane + 32 * i;
    w[i] = d <= D ? route_weight(routing, q, d, D, M, bmax, option, z, dev_type, demand, fam_of_m, lat) : 0;
    cur[i] = 0;
  }
  uint8_t *pat = pattern + off;
  for (int32_t k = 0; k < Wq; k++) {
    long long key = LLONG_MIN;
#pragma unroll
    for (int i = 0; i < 3; i++) {
      if (w[i] == 0) continue;
      cur[i] += w[i];
      const long long kk = ((long long)cur[i] << 32) | (0xFFFFFFFFu - (uint32_t)(lane + 32 * i));
      key = kk > key ? kk : key;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
      const long long v = __shfl_xor_sync(0xffffffffu, key, o);
      key = v > key ? v : key;
    }
    const int best = (int)(0xFFFFFFFFu - (uint32_t)(key & 0xFFFFFFFFll));
#pragma unroll
    for (int i = 0; i < 3; i++)
      if (best == lane + 32 * i) cur[i] -= Wq;
    if (lane == 0) pat[k] = (uint8_t)best;
  }
}

// per-tile key histogram: one warp per tile of TILE queries
__global__ void k_tile_count(const uint8_t *__restrict__ keys, int64_t N, int nkeys, int32_t *hist) {
  __shared__ int32_t cnt[TILE_WARPS][PX_MAXD + 2];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t tile = (int64_t)blockIdx.x * TILE_WARPS + w;
  for (int k = lane; k < nkeys; k += 32) cnt[w][k] = 0;
  __syncwarp();
  const int64_t t0 = tile * TILE;
  if (t0 < N) {
    for (int c = 0; c < TILE; c += 32) {
      const int64_t i = t0 + c + lane;
      const bool valid = i < N;
      const int key = valid ? keys[i] : 255;
      const unsigned peers = __match_any_sync(0xffffffffu, key);
      if (valid && lane == __ffs(peers) - 1) cnt[w][key] += __popc(peers);
      __syncwarp();
    }
    for (int k = lane; k < nkeys; k += 32) hist[tile * nkeys + k] = cnt[w][k];
  }
}

// exclusive scan over tiles, one block per key; totals[key]
__global__ void k_tile_scan(const int32_t *__restrict__ hist, int64_t ntiles, int nkeys, int32_t *base,
                            int64_t *totals) {
  const int key = blockIdx.x;
  __shared__ int64_t part[1024];
  const int64_t per = (ntiles + blockDim.x - 1) / blockDim.x;
  const int64_t lo = threadIdx.x * per, hi = lo + per < ntiles ? lo + per : ntiles;
  int64_t s = 0;
  for (int64_t t = lo; t < hi; t++) s += hist[t * nkeys + key];
  part[threadIdx.x] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    int64_t acc = 0;
    for (int i = 0; i < (int)blockDim.x; i++) { int64_t v = part[i]; part[i] = acc; acc += v; }
    totals[key] = acc;
    base[ntiles * nkeys + key] = (int32_t)acc;  // row ntiles: totals
  }
  __syncthreads();
  int64_t acc = part[threadIdx.x];
  for (int64_t t = lo; t < hi; t++) {
    base[t * nkeys + key] = (int32_t)acc;
    acc += hist[t * nkeys + key];
  }
}

// family ordinal -> target device (pattern lookup); per-tile target histogram
__global__ void k_route_target(const uint8_t *__restrict__ fam, int64_t N, int Q, const int32_t *__restrict__ famBase,
                               const uint8_t *__restrict__ pattern, const int32_t *__restrict__ pat_off,
                               const int32_t *__restrict__ pat_len, int D, uint8_t *target, int32_t *histDev) {
  __shared__ int32_t run[TILE_WARPS][PX_MAXQ];
  __shared__ int32_t cnt[TILE_WARPS][PX_MAXD + 2];
  __shared__ int32_t sOff[PX_MAXQ], sLen[PX_MAXQ];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x < Q) { sOff[threadIdx.x] = pat_off[threadIdx.x]; sLen[threadIdx.x] = pat_len[threadIdx.x]; }
  const int64_t tile = (int64_t)blockIdx.x * TILE_WARPS + w;
  const int64_t t0 = tile * TILE;
  if (t0 < N)
    for (int k = lane; k < Q; k += 32) run[w][k] = famBase[tile * Q + k];
  for (int k = lane; k <= D; k += 32) cnt[w][k] = 0;
  __syncthreads();
  if (t0 >= N) return;
  for (int c = 0; c < TILE; c += 32) {
    const int64_t i = t0 + c + lane;
    const bool valid = i < N;
    const int key = valid ? fam[i] : 255;
    const unsigned peers = __match_any_sync(0xffffffffu, key);
    const int rank = __popc(peers & ((1u << lane) - 1));
    int ord = 0;
    if (valid) ord = run[w][key] + rank;
    __syncwarp();
    if (valid && lane == __ffs(peers) - 1) run[w][key] += __popc(peers);
    int tgt = D;
    if (valid) {
      const int len = sLen[key];
      tgt = len > 0 ? pattern[sOff[key] + (ord % len)] : D;
      target[i] = (uint8_t)tgt;
    }
    const unsigned tp = __match_any_sync(0xffffffffu, valid ? tgt : 255);
    if (valid && lane == __ffs(tp) - 1) cnt[w][tgt] += __popc(tp);
    __syncwarp();
  }
  for (int k = lane; k <= D; k += 32) histDev[tile * (D + 1) + k] = cnt[w][k];
}

__global__ void k_dev_offsets(const int64_t *__restrict__ totals, int n, int64_t *off) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    int64_t acc = 0;
    for (int k = 0; k < n; k++) { off[k] = acc; acc += totals[k]; }
    off[n] = acc;
  }
}

// stable scatter into device-major arrays; inv[i] = device-major position of query i
__global__ void k_scatter(const uint8_t *__restrict__ target, const uint32_t *__restrict__ arr, int64_t N, int D,
                          const int32_t *__restrict__ devBase, const int64_t *__restrict__ devOff, uint32_t *devArr,
                          uint32_t *inv) {
  __shared__ int64_t run[TILE_WARPS][PX_MAXD + 2];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t tile = (int64_t)blockIdx.x * TILE_WARPS + w;
  const int64_t t0 = tile * TILE;
  if (t0 >= N) return;
  for (int k = lane; k <= D; k += 32) run[w][k] = devOff[k] + devBase[tile * (D + 1) + k];
  __syncwarp();
  for (int c = 0; c < TILE; c += 32) {
    const int64_t i = t0 + c + lane;
    const bool valid = i < N;
    const int key = valid ? target[i] : 255;
    const unsigned peers = __match_any_sync(0xffffffffu, key);
    const int rank = __popc(peers & ((1u << lane) - 1));
    int64_t pos = 0;
    if (valid) pos = run[w][key] + rank;
    __syncwarp();
    if (valid && lane == __ffs(peers) - 1) run[w][key] += __popc(peers);
    __syncwarp();
    if (valid) { devArr[pos] = arr[i]; inv[i] = (uint32_t)pos; }
  }
}

// --------------------------------------------------------------- lanes ----
// Latencies are produced in device-major order (latd[s][p], p = position in
// the per-device arrays), which every lane writes sequentially; k_unpermute
// turns them into per-query order at the end.
// Per (scenario, chunk): the run whose latencies a chunk's rows hold -- it
// entered the chunk at head st + edh with the device free at eF and left it
// at head en + xov with the device free at xF.  k_spec writes runs entered
// idle at the chunk start; k_fix and k_stitch replace them.
struct ChunkSt {
  int64_t xF;
  int64_t eF;
  int32_t xov;
  int32_t edh;
};

struct LaneParam {  // per (scenario, device)
  int32_t Bmax;     // §5: the maximum allowed batch size (R4'); AIMD: min(cap, depth); 0 for idle devices
  uint32_t A;       // accuracy of the hosted variant
  int64_t L;        // scenario SLO of the hosted family (R12)
  int32_t policy;   // 0 §5, 1 Nexus early drop, 2 Clipper AIMD (§8(f2))
  int32_t Bn;       // Nexus batch size: largest b <= Bmax with 2 T(b) <= L, at least 1 (R14)
  int32_t mono;     // T(b) non-decreasing over b = 1..Bmax (binary-search decisions)
};

__global__ void k_lane_params(int S, int D, int M, int bmax, const int32_t *__restrict__ option,
                              const int32_t *__restrict__ dev_type, const int32_t *__restrict__ fam_of_m,
                              const int32_t *__restrict__ acc, const int32_t *__restrict__ lat,
                              const int32_t *__restrict__ slo_base, const proteus_scenario *__restrict__ sc,
                              LaneParam *lp) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= S * D) return;
  const int s = i / D, d = i % D;
  LaneParam p = {0, 0, 0, sc[s].policy, 0, 0};
  const int o = option[d];
  if (o > 0) {
    const int32_t *T = lat + ((size_t)dev_type[d] * M + (o - 1)) * bmax;
    int depth = 0;
    while (depth < bmax && T[depth] > 0) depth++;
    const int cap = sc[s].batch_cap;
    p.Bmax = (cap > 0 && cap < depth) ? cap : depth;
    p.A = (uint32_t)acc[o - 1];
    p.L = (int64_t)sc[s].slo_mult_milli * slo_base[fam_of_m[o - 1]] / 1000;
    p.Bn = 1;  // the maximum allowed batch size: largest b <= min(cap, depth), 2 T(b) <= SLO
    for (int b = 1; b <= p.Bmax; b++)
      if (2 * (int64_t)T[b - 1] <= p.L) p.Bn = b;
    if (p.policy == 0) p.Bmax = p.Bn;  // §5 batches at most that (reading R4')
    p.mono = 1;
    for (int b = 1; b < p.Bmax; b++)
      if (T[b] < T[b - 1]) p.mono = 0;
  }
  lp[i] = p;
}

struct WinRec {     // chain of one entry offset o of one chunk (times relative to a_{c0})
  int64_t Fx;       // free time after the batch that crosses c1 (absolute; Bmax = 1: R of the max-plus form)
  int32_t tdisp;    // idle dispatch time at the entry head c0 + o, - a_{c0}
  int32_t R;        // backlog threshold of (iii) through the chunk, - a_{c0} (INT32_MAX: none)
  int32_t hx;       // first head >= c1 of the chain, - c0
  int32_t pad;
};
struct WinEntry {   // true state at a chunk start: first head >= c0 (device-relative), free time
  int64_t F;
  int32_t h, pad;
};

struct LaneArgs {
  int S, D, M, bmax, nsc, CH;
  int WU;                 // k_spec warm-up: queries replayed before each chunk (0 = start at the chunk)
  int64_t N, NCH;
  int64_t NS;             // row stride of latd (N rounded up to 32: 16-byte aligned rows for bulk copies)
  const int32_t *option, *dev_type, *lat, *sc_list;
  const LaneParam *lp;
  const int64_t *devOff;  // [D + 2]; segment D = the sink
  const int64_t *choff;   // [D + 1] chunk offsets
  const int32_t *goff;    // [D + 1] phase-A warp-group offsets
  const uint32_t *devArr;
  uint32_t *latd;         // [S][N] device-major
  ChunkSt *cs;            // [S][NCH] chunk runs (written by k_spec / k_fix, read by k_stitch)
  const ChunkSt *csp;     // k_fix: the previous round's
  uint64_t *agg;          // [3][S]
  int maxchk;             // convergence checks per chunk (free decisions only)
  int scan1;              // Bmax = 1 lanes are produced by k_scan1_* (the chunk kernels skip them)
  uint64_t dmask;         // devices whose lanes this launch of k_spec / k_fix / k_stitch takes
  int64_t *lstart;        // [S * D][2] (head, F) where k_stitch starts a lane the full-batch scan took (head -1: not taken);
                          // also the Nexus scan's start / end states (k_wc_lanes, nxmode)
  unsigned *lstat;        // [S * D][2] speculative decisions that were full batches sent when the device
                          // freed (backlog), and all speculative decisions; k_fix leaves backlogged lanes
                          // (a quarter or more) to the stitch's max-plus stretches
  long long debug;        // > 0: k_stitch prints lanes slower than this many cycles (diagnostic)
  uint8_t *wst;           // baseline chunk runs: [S][NS] 0, or 1 + the run's AIMD limit (Nexus: 1) at a
                          // decision whose head found the device free (NULL: no chunk runs)
  struct WcExit *wx;      // baseline chunk runs: [S][NCH] exit state
  // chunk tables of the idle-branch chains (k_win_tables over the CH chunks) for
  // lanes with large Bmax: the stitch hops a chunk entered on the idle branch
  // and k_rewrite replays it from the true entry (rw)
  const WinRec *trec;
  const int64_t *trecoff;  // [nsc * D] (list position * D + d)
  const int32_t *tE;       // [nsc * D] entry offsets per chunk (0: no table)
  WinEntry *rw;            // [nsc * D][NCH] true entry of a hopped chunk (pad = 1)
  // spec/stitch pipelining: k_spec sets cready[s][choff[d] + c] when chunk c's
  // latencies and exit state are written; k_stitch (running concurrently on
  // another stream) waits for the flags of the chunks it reads (null: no
  // wait); cready[-1]: the wait watchdog fired
  unsigned *cready;
  const int32_t *lane_order;  // k_stitch: lane (list position * D + d) of warp i (null: identity)
  int bsearch;                // k_stitch: binary-search decisions (fast_decide) on lanes with T non-decreasing
  const uint8_t *skip;        // [S * D] 1: the chunk / lane kernels leave the lane alone (a duplicate lane, or k_chain's)
  // Nexus overload scan (k_nx_*): nxsel[s * D + d] = 1 for the lanes it takes;
  // nxmode 1: k_wc_lanes walks those lanes only up to their first overload
  // stretch and records the state there (lstart), the others whole; nxmode 2:
  // only the selected lanes, from lstart (the state after the scan's batches)
  const uint8_t *nxsel;
  int nxmode;
};

struct WcExit {  // a baseline chunk run left its chunk at head h (>= chunk end), device free at F;
  int64_t h, F;    // its last decision dropped [.., first) and served [first, h) (Nexus drops can
  int64_t first;   // reach past the chunk end)
  int32_t limit, pad;
};

__device__ __forceinline__ uint32_t sat_lat(int64_t l) { return l >= 0xFFFFFFFFll ? 0xFFFFFFFEu : (uint32_t)l; }

// One decision of the §5 rule from head h (device free at F) over arr[0, n):
// returns the batch size b, *t_out = dispatch time.  T[b-1] = T(b).
template <class Arr>
__device__ __forceinline__ int decide(const Arr &arr, int64_t n, int64_t h, int64_t F, int Bmax, int64_t L,
                                      const int32_t *T, int64_t *t_out) {
  const int64_t ah = arr(h);
  int64_t t = F > ah ? F : ah;                                       // R5
  int q = 1;
  while (q < Bmax && h + q < n && (int64_t)arr(h + q) <= t) q++;      // R3
  int b;
  for (;;) {
    if (q >= Bmax) { b = Bmax; break; }                               // R4
    const int64_t W = ah + L - T[q];  // Tmax_wait(q+1) = Texp(1) - Tprocess(q+1)
    if (t >= W) { b = q; break; }                                     // R1
    if (h + q < n && (int64_t)arr(h + q) <= W) {                      // Case 2 (R2)
      t = arr(h + q);
      while (q < Bmax && h + q < n && (int64_t)arr(h + q) <= t) q++;
      continue;
    }
    t = W;                                                            // Case 1
    b = q;
    break;
  }
  *t_out = t;
  return b;
}

// idle decision at head h (fact (ii)); T[b-1] = T(b); n = the device's size
template <class Arr>
__device__ __forceinline__ int idle_decide(const Arr &A, int64_t n, int64_t h, int Bmax, int64_t L,
                                           const int32_t *T, bool mono, int64_t *t_out) {
  if (!mono) return decide(A, n, h, (int64_t)0, Bmax, L, T, t_out);
  const int64_t ah = A(h);
  int q0 = 1;
  while (q0 < Bmax && h + q0 < n && (int64_t)A(h + q0) <= ah) q0++;  // R3: simultaneous arrivals
  if (q0 >= Bmax) { *t_out = ah; return Bmax; }
  // first q in [q0, Bmax) whose stop test holds (monotone), Bmax if none
  int lo = q0, hi = Bmax;
  while (lo < hi) {
    const int q = (lo + hi) >> 1;
    const int64_t W = ah + L - T[q];
    const int64_t nxt = h + q < n ? (int64_t)A(h + q) : INT64_MAX;
    const bool stop = nxt > W || (int64_t)A(h + q - 1) >= W;
    if (stop) hi = q; else lo = q + 1;
  }
  int q = lo;
  while (q < Bmax && h + q < n && A(h + q) == A(h + q - 1)) q++;  // first stable count
  if (q >= Bmax) { *t_out = A(h + Bmax - 1); return Bmax; }      // R4: Bmax queued at that instant
  const int64_t W = ah + L - T[q];
  const int64_t tq = A(h + q - 1);
  *t_out = tq >= W ? tq : W;
  return q;
}

// #{j in [h, min(n, h + Bmax)) : A(j) <= F} by binary search (>= 1 when A(h) <= F)
template <class Arr>
__device__ __forceinline__ int count_upto(const Arr &A, int64_t n, int64_t h, int Bmax, int64_t F) {
  int lo = 0, hi = (int)(n - h < Bmax ? n - h : Bmax);
  while (lo < hi) {
    const int m = (lo + hi + 1) >> 1;
    if ((int64_t)A(h + m - 1) <= F) lo = m; else hi = m - 1;
  }
  return lo;
}

// one decision from head h with the device free at F (the rule R1-R5 in the
// form of facts (i)-(ii) of the window path, below): the idle decision by
// binary search, or, when the device frees after it would have dispatched,
// the greedy batch min(Bmax, queued at F) at F.  Same result as decide().
template <class Arr>
__device__ __forceinline__ int fast_decide(const Arr &A, int64_t n, int64_t h, int64_t F, int Bmax, int64_t L,
                                           const int32_t *T, bool mono, int64_t *t_out) {
  if (!mono) return decide(A, n, h, F, Bmax, L, T, t_out);
  int64_t t;
  const int b = idle_decide(A, n, h, Bmax, L, T, true, &t);
  if (F <= t) { *t_out = t; return b; }
  *t_out = F;
  return count_upto(A, n, h, Bmax, F);
}

struct GArr {
  const uint32_t *p;
  __device__ __forceinline__ uint32_t operator()(int64_t j) const { return __ldg(p + j); }
};

__device__ __forceinline__ void count_lat(uint32_t l, const LaneParam &p, unsigned long long &viol,
                                          unsigned long long &ont, unsigned long long &accs) {
  if ((int64_t)l > p.L) viol++;
  else { ont++; accs += p.A; }
}

__device__ __forceinline__ void warp_add_counts(unsigned long long v, unsigned long long o, unsigned long long ac,
                                                uint64_t *agg, int S, int s, int lane) {
  for (int k = 16; k; k >>= 1) {
    v += __shfl_xor_sync(0xffffffffu, v, k);
    o += __shfl_xor_sync(0xffffffffu, o, k);
    ac += __shfl_xor_sync(0xffffffffu, ac, k);
  }
  if (lane == 0) {
    if (v) atomicAdd((unsigned long long *)&agg[s], v);
    if (o) atomicAdd((unsigned long long *)&agg[S + s], o);
    if (ac) atomicAdd((unsigned long long *)&agg[2 * S + s], ac);
  }
}

// ---- fallback: one thread per (device, scenario) walks the whole array
__global__ void __launch_bounds__(LANE_THREADS) k_lanes(const __grid_constant__ LaneArgs a) {
  const int lane_id = blockIdx.x * blockDim.x + threadIdx.x;
  if (lane_id >= a.nsc * a.D) return;
  const int s = a.sc_list[lane_id / a.D], d = lane_id % a.D;
  const LaneParam p = a.lp[s * a.D + d];
  const int64_t st = a.devOff[d], n = a.devOff[d + 1] - st;
  if (n == 0) return;
  uint32_t *out = a.latd + (size_t)s * a.NS + st;
  if (p.Bmax < 1) {  // never routed to (z = 0 / depth 0); kept for safety
    for (int64_t j = 0; j < n; j++) out[j] = 0xFFFFFFFFu;
    return;
  }
  const int32_t *T = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
  GArr arr{a.devArr + st};
  int64_t h = 0, F = 0;  // R13
  while (h < n) {
    int64_t t;
    const int b = decide(arr, n, h, F, p.Bmax, p.L, T, &t);
    F = t + T[b - 1];
    for (int j = 0; j < b; j++) out[h + j] = sat_lat(F - (int64_t)arr(h + j));
    h += b;
  }
}

// ---- §8(f2) work-conserving baseline batchers, readings R14-R15
// Warp per (device, scenario).  Both rules decide at t = max(F, a_head) (the
// device is free and a query waits); the queue at t is
// [h, tail), tail advanced 32 arrivals per ballot (t never decreases, so tail
// only moves forward).  Nexus: the window test t + T(min(B, tail - i)) <=
// a_i + L for 32 candidate heads i per ballot, the first pass starts the batch
// and the lanes below it write the drops; AIMD: b = min(queued, limit) and the
// limit update at completion.  The lane's arrivals are staged in a per-warp
// shared-memory ring covering [b0, b0 + WC_RW) (refilled by halves with
// coalesced loads as the head advances; reads past it go to global memory),
// T(b) in shared memory; latencies are written 32 per store (coalesced).
#define WC_RW 1024
// Chunk runs of the baseline batchers (thread per (scenario, chunk of CH
// queries of a device)): the rule replayed from an idle device at the chunk's
// first query, latencies / drops written for the chunk's positions, and at
// every decision whose head finds the device free the mark 1 + limit (AIMD;
// Nexus: 1).  A decision from head h with the device free at a_h depends on h
// (and AIMD's limit) only, so the true run that reaches such a head in the
// same state continues exactly as this run: k_wc_lanes jumps to its exit.
__global__ void __launch_bounds__(128) k_wc_spec(const __grid_constant__ LaneArgs a) {
  const int64_t cg = (int64_t)blockIdx.y * blockDim.x + threadIdx.x;  // chunk over all devices
  if (cg >= a.choff[a.D]) return;
  int d = 0;
  while (cg >= a.choff[d + 1]) d++;
  const int s = a.sc_list[blockIdx.x];
  if (a.skip && a.skip[s * a.D + d]) return;
  const LaneParam p = a.lp[s * a.D + d];
  const int64_t off = a.devOff[d], n = a.devOff[d + 1] - off;
  const int64_t c = cg - a.choff[d];
  const int64_t st = c * a.CH, en = st + a.CH < n ? st + a.CH : n;
  uint32_t *out = a.latd + (size_t)s * a.NS + off;
  uint8_t *mk = a.wst + (size_t)s * a.NS + off;
  WcExit e = {en, 0, en, 1, 0};
  if (p.Bmax >= 1) {
    const int32_t *T = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
    const uint32_t *arr = a.devArr + off;
    const bool nexus = p.policy == 1;
    const int B = nexus ? p.Bn : p.Bmax;
    int64_t h = st, F = 0, last_first = st;
    int limit = 1;
    while (h < en) {
      const int64_t ah = __ldg(arr + h);
      const int64_t t = F > ah ? F : ah;
      if (F <= ah) mk[h] = (uint8_t)(nexus ? 1 : (limit < 254 ? limit + 1 : 255));
      int64_t first = h;
      int b;
      if (nexus) {
        int64_t i = h;
        int w = 0;
        for (;; i++) {  // sliding window from the head (R14)
          if (i >= n || (int64_t)__ldg(arr + i) > t) break;  // past the queue: all dropped
          w = 1;
          while (w < B && i + w < n && (int64_t)__ldg(arr + i + w) <= t) w++;
          if (t + T[w - 1] <= (int64_t)__ldg(arr + i) + p.L) break;
          if (i < en) out[i] = 0xFFFFFFFFu;
          w = 0;
        }
        if (w == 0) { h = i; last_first = i; continue; }  // everything queued was dropped
        first = i;
        b = w;
      } else {
        int q = 1;
        while (q < limit && h + q < n && (int64_t)__ldg(arr + h + q) <= t) q++;
        b = q;
      }
      const int64_t Fn = t + T[b - 1];
      for (int64_t j = first; j < first + b && j < en; j++) out[j] = sat_lat(Fn - (int64_t)__ldg(arr + j));
      if (!nexus) {
        if (Fn - ah > p.L) limit = limit * 9 / 10 < 1 ? 1 : limit * 9 / 10;
        else limit = limit + 1 > p.Bmax ? p.Bmax : limit + 1;
      }
      F = Fn;
      h = first + b;
      last_first = first;
    }
    e.h = h;
    e.F = F;
    e.first = last_first;
    e.limit = limit;
  }
  a.wx[(size_t)s * a.NCH + cg] = e;
}

template <bool CHUNKS>  // CHUNKS: meet the chunk runs of k_wc_spec (a.wst, a.wx)
__global__ void __launch_bounds__(128) k_wc_lanes(const __grid_constant__ LaneArgs a) {
  __shared__ uint32_t sA[4][WC_RW];
  __shared__ int32_t sT[4][PX_MAXB];
  const int wid = (int)((blockIdx.x * (unsigned)blockDim.x + threadIdx.x) >> 5), lane = threadIdx.x & 31;
  const int w = threadIdx.x >> 5;
  if (wid >= a.nsc * a.D) return;
  const int s = a.sc_list[wid / a.D], d = wid % a.D;
  if (a.skip && a.skip[s * a.D + d]) return;
  const bool nxs = a.nxsel && a.nxsel[s * a.D + d];
  if (a.nxmode == 2 && !nxs) return;
  const LaneParam p = a.lp[s * a.D + d];
  const int64_t st = a.devOff[d], n = a.devOff[d + 1] - st;
  if (n == 0) return;
  uint32_t *out = a.latd + (size_t)s * a.NS + st;
  if (p.Bmax < 1) {  // never routed to (z = 0 / depth 0); kept for safety
    for (int64_t j = lane; j < n; j += 32) out[j] = 0xFFFFFFFFu;
    return;
  }
  const int32_t *Tg = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
  int32_t *T = sT[w];
  for (int k = lane; k < p.Bmax; k += 32) T[k] = __ldg(Tg + k);
  const uint32_t *arr = a.devArr + st;
  uint32_t *ring = sA[w];
  int64_t b0 = 0;
  auto fill = [&](int64_t from, int cnt) {
    for (int k = lane; k < cnt; k += 32) {
      const int64_t j = from + k;
      ring[j & (WC_RW - 1)] = j < n ? __ldg(arr + j) : 0xFFFFFFFFu;
    }
  };
  fill(0, WC_RW);
  __syncwarp();
  // arrival j >= b0 (every index read is >= the head >= b0)
  auto A = [&](int64_t j) -> int64_t {
    return j - b0 < WC_RW ? (int64_t)ring[j & (WC_RW - 1)] : (int64_t)__ldg(arr + j);
  };
  const bool nexus = p.policy == 1;
  const int B = nexus ? p.Bn : p.Bmax;
  int64_t h = 0, tail = 0, F = 0;  // R13
  if (nxs && a.nxmode == 2) {      // after the overload scan's batches
    h = a.lstart[2 * ((size_t)s * a.D + d)];
    F = a.lstart[2 * ((size_t)s * a.D + d) + 1];
    tail = h;
  }
  int limit = 1;                   // AIMD batch-size limit
  const int64_t T1 = T[0];
  const bool fast = T1 <= p.L;     // isolated queries are on time
  bool try_stretch = true;         // Nexus: look for an overload stretch at the next busy decision
  int stretch_wait = 0;            // decisions to let pass before the next stretch test
  long long dbg_t0 = clock64(), dbg_steps = 0, dbg_st = 0, dbg_stb = 0;
  int64_t cc = 0, cend = a.CH < n ? a.CH : n;  // chunk of the head
  const uint8_t *wrow = CHUNKS ? a.wst + (size_t)s * a.NS + st : nullptr;
  while (h < n) {
    dbg_steps++;
    if (h - b0 >= WC_RW / 2) {     // slide the ring
      const int64_t nb = h & ~(int64_t)(WC_RW / 2 - 1);
      __syncwarp();
      if (nb == b0 + WC_RW / 2) fill(b0 + WC_RW, WC_RW / 2);
      else fill(nb, WC_RW);
      b0 = nb;
      __syncwarp();
    }
    if (CHUNKS) {  // chunk runs: meet one at a free head in the same state, jump to its exit
      while (h >= cend) { cc++; cend = (cc + 1) * a.CH < n ? (cc + 1) * a.CH : n; }
      const uint8_t mkh = F <= A(h) ? wrow[h] : 0;  // a global read only when the device is free
      if (mkh && (nexus || (int)mkh == limit + 1)) {
        const WcExit e = a.wx[(size_t)s * a.NCH + a.choff[d] + cc];
        // the run's last batch may reach into the next chunks: their rows hold
        // those chunks' own runs there, so this batch's latencies are rewritten
        for (int64_t j = cend + lane; j < e.h; j += 32) out[j] = j < e.first ? 0xFFFFFFFFu : sat_lat(e.F - A(j));
        h = e.h;
        F = e.F;
        limit = e.limit;
        if (tail < h) tail = h;
        continue;
      }
    }
    // Nexus with B = 1 takes the overload stretch below (when the device is
    // busy) before the batches of one
    const bool nx1 = nexus && B == 1 && try_stretch && F > A(h) && --stretch_wait <= 0;
    if (!nx1 && (nexus ? B == 1 : limit == 1)) {
      // Batches of one, 32 per step: query h + k leaves at max(F_{k-1}, a)
      // (work-conserving), F_k = max(F_{k-1}, a_{h+k}) + T(1), i.e. F_k - (k+1) T(1)
      // = max(F, max_{i<=k} a_{h+i} - i T(1)) -- a warp max-scan.  AIMD keeps
      // limit 1 while batches time out (and always when Bmax = 1): the step
      // ends after the first on-time batch (the limit becomes 2).  Nexus
      // (B = 1) serves a query iff it finishes on time; the first one that
      // would not is dropped (F unchanged) and ends the step.
      const int64_t j = h + lane;
      const bool valid = j < n;
      const int64_t aj = valid ? A(j) : 0;
      int64_t x = valid ? aj - (int64_t)lane * T1 : INT64_MIN / 4;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t v = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x = v > x ? v : x;
      }
      const int64_t Fk = (F > x ? F : x) + (int64_t)(lane + 1) * T1;
      const bool late = valid && Fk - aj > p.L;
      const int nval = n - h < 32 ? (int)(n - h) : 32;
      int r = nval;        // queries this step handles
      bool drop_last = false;
      if (nexus) {
        const unsigned m = __ballot_sync(0xffffffffu, late);
        if (m) { r = __ffs(m); drop_last = true; }
      } else if (p.Bmax > 1) {
        const unsigned m = __ballot_sync(0xffffffffu, valid && !late);
        if (m) { r = __ffs(m); limit = 2; }
      }
      const int served = drop_last ? r - 1 : r;
      if (nexus && drop_last) try_stretch = true;  // dropping: overload, a stretch may follow
      if (lane < served) out[j] = sat_lat(Fk - aj);
      if (drop_last && lane == r - 1) out[j] = 0xFFFFFFFFu;
      if (served > 0) F = __shfl_sync(0xffffffffu, Fk, served - 1);
      h += r;
      if (tail < h) tail = h;
      continue;
    }
    const int64_t ah = A(h);
    if (nexus && F > ah && try_stretch && (B == 1 ? nx1 : --stretch_wait <= 0)) {
      // Overload stretch (Nexus): the device is busy at every decision and the
      // queue holds a full window, so batch k of the stretch is decided at
      // t_k = F + k T(B): the window of B from the head passes iff a_i >=
      // t_k + T(B) - L, so its head is i_k = max(p_k, g_k), g_k = the first
      // arrival >= that threshold, p_k = i_{k-1} + B (p_0 = h): i_k = k B +
      // max(h, max_{j<=k} g_j - j B), a prefix maximum over the lanes.  The
      // queries in [p_k, i_k) are dropped.  Batch k is valid while the device
      // is busy (a_{p_k} <= t_k) and the window is full (a_{i_k + B - 1} <=
      // t_k); the stretch ends before the first invalid one (32 per step).
      const int64_t TB = T[B - 1];
      const int k = lane;
      const int64_t tk = F + (int64_t)k * TB;
      const int64_t thr = tk + TB - p.L;
      int64_t x = h + (int64_t)k * B;  // g_k clamped below by h + k B (only larger values matter)
      if (x < n && A(x) < thr) {       // gallop, then bisect: first index >= x with a >= thr
        int64_t lo = x, step = 1, hi = x + 1;
        while (hi < n && A(hi) < thr) { lo = hi; step <<= 1; hi = x + step; }
        if (hi > n) hi = n;
        while (hi - lo > 1) { const int64_t mid = (lo + hi) >> 1; if (A(mid) < thr) lo = mid; else hi = mid; }
        x = hi;
      }
      int64_t m = x - (int64_t)k * B;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t v = __shfl_up_sync(0xffffffffu, m, o);
        if (lane >= o) m = v > m ? v : m;
      }
      const int64_t ik = (int64_t)k * B + (m > h ? m : h);
      int64_t pk = __shfl_up_sync(0xffffffffu, ik + B, 1);
      if (lane == 0) pk = h;
      const bool ok = ik + B <= n && pk < n && A(pk) <= tk && A(ik + B - 1) <= tk;
      const unsigned vm = __ballot_sync(0xffffffffu, ok);
      const int r = vm == 0xffffffffu ? 32 : __ffs(~vm) - 1;
      if (r == 32 && nxs && a.nxmode == 1) {  // the state where the overload scan takes over
        if (lane == 0) {
          a.lstart[2 * ((size_t)s * a.D + d)] = h;
          a.lstart[2 * ((size_t)s * a.D + d) + 1] = F;
        }
        return;
      }
      if (r > 0) {
        dbg_st++; dbg_stb += r;
        stretch_wait = r < 4 ? 8 : 0;  // short stretches do not pay for the test: back off
        if (lane < r) {
          for (int64_t j = pk; j < ik; j++) out[j] = 0xFFFFFFFFu;  // dropped early
          const int64_t Fk = tk + TB;
          for (int q = 0; q < B; q++) out[ik + q] = sat_lat(Fk - A(ik + q));
        }
        F += (int64_t)r * TB;
        h = __shfl_sync(0xffffffffu, ik + B, r - 1);
        if (tail < h) tail = h;
        continue;
      }
      try_stretch = false;  // not in a stretch here: test again after a busy full-window batch
      stretch_wait = 8;
    }
    if (fast && ah >= F) {
      // Isolated queries, 32 per ballot: query j finds the device free (a_j >=
      // F, resp. a_j >= a_{j-1} + T(1) after its predecessor went alone) and no
      // other query queued (a_{j+1} > a_j), so it leaves alone at a_j: latency
      // T(1) <= L -- the Nexus window test passes and AIMD sees no timeout.
      const int64_t j = h + lane;
      const int64_t aj = j < n ? A(j) : 0;
      const int64_t ap = __shfl_up_sync(0xffffffffu, aj, 1);
      int64_t an = __shfl_down_sync(0xffffffffu, aj, 1);
      if (lane == 31) an = j + 1 < n ? A(j + 1) : INT64_MAX;
      if (j + 1 >= n) an = INT64_MAX;
      const bool iso = j < n && an > aj && (lane == 0 || aj >= ap + T1);
      const unsigned m = __ballot_sync(0xffffffffu, iso);
      const int r = __ffs(~m) - 1 < 0 ? 32 : __ffs(~m) - 1;
      if (r > 0) {
        if (lane < r) out[j] = (uint32_t)T1;
        F = __shfl_sync(0xffffffffu, aj, r - 1) + T1;
        if (!nexus) limit = limit + r > p.Bmax ? p.Bmax : limit + r;
        h += r;
        if (tail < h) tail = h;
        continue;
      }
    }
    const int64_t t = F > ah ? F : ah;
    if (tail <= h) tail = h + 1;
    for (;;) {  // queued at t: arrivals <= t (sorted: the ballot is a prefix)
      const int64_t j = tail + lane;
      const unsigned m = __ballot_sync(0xffffffffu, j < n && A(j) <= t);
      tail += __popc(m);
      if (m != 0xffffffffu) break;
    }
    int64_t first = h;
    if (nexus) {
      first = -1;
      for (int64_t i0 = h; i0 < tail; i0 += 32) {
        const int64_t i = i0 + lane;
        bool pass = false;
        if (i < tail) {
          const int64_t wl = tail - i < B ? tail - i : B;
          pass = t + T[wl - 1] <= A(i) + p.L;
        }
        const unsigned m = __ballot_sync(0xffffffffu, pass);
        const int nd = m ? __ffs(m) - 1 : 32;
        if (lane < nd && i < tail) out[i] = 0xFFFFFFFFu;  // dropped early
        if (m) { first = i0 + nd; break; }
      }
      if (first < 0) { h = tail; continue; }  // everything queued was dropped
    }
    const int cap = nexus ? B : limit;
    const int b = (int)(tail - first < cap ? tail - first : cap);
    if (nexus && b == B && t == F) try_stretch = true;  // busy, full window: a stretch may follow
    F = t + T[b - 1];
    for (int k = lane; k < b; k += 32) out[first + k] = sat_lat(F - A(first + k));
    if (!nexus) {  // completion feedback (the next decision is at >= F)
      if (F - ah > p.L) limit = limit * 9 / 10 < 1 ? 1 : limit * 9 / 10;
      else limit = limit + 1 > p.Bmax ? p.Bmax : limit + 1;
    }
    h = first + b;
  }
  if (nxs && a.nxmode == 1 && lane == 0) {  // walked to the end: nothing left for the scan / the second walk
    a.lstart[2 * ((size_t)s * a.D + d)] = n;
    a.lstart[2 * ((size_t)s * a.D + d) + 1] = F;
  }
  if (a.debug && lane == 0 && clock64() - dbg_t0 > a.debug)
    printf("wc s=%d d=%d n=%lld pol=%d B=%d cycles=%lld steps=%lld stretches=%lld stretch_batches=%lld\n", s, d,
           (long long)n, p.policy, B, clock64() - dbg_t0, dbg_steps, dbg_st, dbg_stb);
}

// ---- phase A: speculative chunks
// Each device array is cut into chunks of CH queries.  One warp per (device,
// scenario, 32 consecutive chunks); lane = chunk, replayed from an idle
// device at the chunk's first query (the true state at the start of the
// trace, R13).  All lanes follow the same rule parameters, so the warp stays
// close to converged.
__global__ void __launch_bounds__(128) k_spec(const __grid_constant__ LaneArgs a) {
  __shared__ int32_t sG[PX_MAXD + 1];
  for (int k = threadIdx.x; k <= a.D; k += blockDim.x) sG[k] = a.goff[k];
  __syncthreads();
  // blockIdx.x = scenario (fastest): consecutive blocks replay the same chunks
  // for different scenarios, so the device arrays are read from L2
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int g = blockIdx.y * 4 + w;
  if (g >= sG[a.D]) return;
  int d = 0;
  while (g >= sG[d + 1]) d++;
  if (!((a.dmask >> d) & 1ull)) return;
  const int s = a.sc_list[blockIdx.x];
  const LaneParam p = a.lp[s * a.D + d];
  const int64_t off = a.devOff[d], n = a.devOff[d + 1] - off;
  const int64_t nch = a.choff[d + 1] - a.choff[d];
  const int64_t c = (int64_t)(g - sG[d]) * 32 + lane;
  if (c >= nch || (a.scan1 && p.Bmax == 1) || (a.skip && a.skip[s * a.D + d])) return;
  const int64_t st = c * a.CH, en = st + a.CH < n ? st + a.CH : n;
  uint32_t *out = a.latd + (size_t)s * a.NS + off;
  int64_t h = st, F = 0, eF = 0, edh = 0;
  if (p.Bmax < 1) {
    for (int64_t j = st; j < en; j++) out[j] = 0xFFFFFFFFu;
    h = en;
  } else {
    const int32_t *T = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
    GArr arr{a.devArr + off};
    unsigned nfull = 0, ndec = 0;
    // warm-up: the run starts idle WU queries before the chunk, so that by the
    // chunk it has usually merged with the true run; the chunk's stored run is
    // the part from its first batch head >= st (entry st + edh, free time eF);
    // a batch straddling st writes the chunk's positions it covers
    h = c > 0 ? (st - a.WU > 0 ? st - a.WU : 0) : st;
    bool entered = h == st;
    while (h < en) {
      if (!entered && h >= st) { entered = true; edh = h - st; eF = F; }
      int64_t t;
      // linear scan (decide): the arrivals stream through L1; binary-search probes
      // (fast_decide) measured slower here (c5 k_spec 8.1 -> 10.0 ms)
      const int b = decide(arr, n, h, F, p.Bmax, p.L, T, &t);
      if (entered) { nfull += b == p.Bmax && t == F; ndec++; }
      const int64_t Fn = t + T[b - 1];
      const int64_t jlo = h > st ? h : st, jend = h + b < en ? h + b : en;
      for (int64_t j = jlo; j < jend; j++) out[j] = sat_lat(Fn - (int64_t)arr(j));
      F = Fn;
      h += b;
    }
    if (!entered) { edh = h - st; eF = F; }  // a warm-up batch covered the whole chunk
    unsigned *ls = a.lstat + 2 * ((size_t)s * a.D + d);
    if (nfull) atomicAdd(ls, nfull);
    atomicAdd(ls + 1, ndec);
  }
  ChunkSt e;
  e.xF = F;
  e.xov = (int32_t)(h - en);
  e.eF = eF;
  e.edh = (int32_t)edh;
  a.cs[(size_t)s * a.NCH + a.choff[d] + c] = e;
  if (a.cready) {  // publish: this chunk's latencies and exit state are written
    __threadfence();
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(a.cready + (size_t)s * a.NCH + a.choff[d] + c), "r"(1u)
                 : "memory");
  }
}

// k_stitch side of the pipelining: wait until chunk c of (s, d) is published.
// A watchdog bounds the wait (~8 s): on expiry it raises cready[-1] (the
// host turns it into PROTEUS_EINTERNAL) instead of hanging the device.
__device__ __forceinline__ void wait_chunk(unsigned *cready, int64_t idx) {
  unsigned v;
  for (uint32_t it = 0;; it++) {
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(cready + idx) : "memory");
    if (v) break;
    if (it > (1u << 25)) { atomicExch(cready - 1, 1u); break; }
    __nanosleep(256);
  }
}

// ---- one §5 decision by a whole warp (lane-parallel form of decide()):
// lane j (queue size q = j, 1 <= j < Bmax, rounds of 32) tests whether the
// rule stops at q -- q is a stable count (a_q > t_q = max(t0, a_{q-1}),
// t0 = max(F, a_h)) and either t_q >= Tmax_wait(q+1) = a_h + L - T(q+1)
// (dispatch now, Case 1) or the next arrival a_q comes after Tmax_wait(q+1)
// (dispatch then).  Case 2 walks through exactly the stable counts in
// increasing order, so the first stop is decide()'s batch; no stop below
// Bmax dispatches Bmax once the Bmax-th query is there (R4).  Arr(j) is the
// arrival of position j (< n); returns b, *t_out = dispatch time.
template <class Arr, class Tab>
__device__ __forceinline__ int decide_warp(const Arr &A, int64_t n, int64_t h, int64_t F, int Bmax, int64_t L,
                                           const Tab &T, int lane, int64_t *t_out) {
  const int64_t INF = INT64_MAX / 4;
  const int64_t a0 = A(h);
  const int64_t t0 = F > a0 ? F : a0;
  for (int r = 0; 1 + 32 * r < Bmax; r++) {
    const int j = 1 + 32 * r + lane;
    bool stop = false;
    int64_t tj = 0;
    if (j < Bmax) {
      const int64_t am = h + j - 1 < n ? A(h + j - 1) : INF;
      const int64_t aj = h + j < n ? A(h + j) : INF;
      const int64_t tq = t0 > am ? t0 : am;
      const int64_t W = a0 + L - T(j);
      stop = aj > tq && (tq >= W || aj > W);
      tj = tq >= W ? tq : W;
    }
    const unsigned m = __ballot_sync(0xffffffffu, stop);
    if (m) {
      const int f = __ffs(m) - 1;
      *t_out = __shfl_sync(0xffffffffu, tj, f);
      return 1 + 32 * r + f;
    }
  }
  const int64_t al = A(h + Bmax - 1);
  *t_out = t0 > al ? t0 : al;
  return Bmax;
}

// ---- phase B: exact stitch, one warp per (device, scenario)
// The true state (h, F) is carried from chunk to chunk.  A chunk whose
// speculative start (its first query, device idle) equals the true state is
// already right.  Otherwise the true run is replayed batch by batch until it
// meets the speculative run: after a batch [h, j2) finishing at Fn, if the
// speculative run also has a batch ending at j2 - 1 with finish Fn (its
// latency + arrival) and a new batch at j2, both runs are in the same state
// (j2, Fn) and agree from there on.  Only batches that the device waited for
// (t > F) are tested -- a batch dispatched the moment the previous one
// finished can only meet a run that had already met -- and at most a few per
// chunk.  Backlogged stretches (Bmax queued when the device frees) are full
// batches back to back -- batch k finishes at F + (k+1) T(Bmax) -- and are
// taken 32 batches per step with a ballot.  Rewritten latencies adjust the
// counts by their difference from the speculative ones.  Arrivals stream
// through a shared-memory ring; exit states are fetched 32 chunks at a time.
#define RSEG 1024                    // ring segment (queries), one bulk copy
#define RING (4 * RSEG)              // per-warp arrival ring
#define LEAN_C (1 << 30)
#define SUMAX 4
#ifdef PX_STITCH_DEBUG  // per-lane counters printed by k_stitch (PROTEUS_REPLAY_DEBUG=cycles)
#define PX_DBG(x) x
#else
#define PX_DBG(x)
#endif

// TMA bulk copies (cp.async.bulk, global -> shared, completion on an mbarrier)
__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *bar) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void bulk_load(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
  // the generic-proxy reads of dst are done (caller's __syncwarp): order them before the async write
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
// two bulk copies completing on one mbarrier (one arrival, both byte counts)
__device__ __forceinline__ void bulk_load2(void *dst0, const void *src0, void *dst1, const void *src1, uint32_t bytes,
                                           uint64_t *bar) {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(2 * bytes) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_u32(dst0)), "l"(src0), "r"(bytes), "r"(smem_u32(bar)) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_u32(dst1)), "l"(src1), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
  asm volatile("{\n\t.reg .pred P1;\n\tWAIT_%=:\n\t"
               "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
               "@!P1 bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)), "r"(parity) : "memory");
}

// number of j in [h + q, h + min(Bmax, n - h)) with arr(j) <= t, added to q
// (arrivals are sorted, so the ballot is a prefix)
template <class Arr>
__device__ __forceinline__ int count_le(const Arr &A, int64_t n, int64_t h, int q, int Bmax, int64_t t, int lane) {
  for (;;) {
    const int64_t j = h + q + lane;
    const bool le = q + lane < Bmax && j < n && (int64_t)A(j) <= t;
    const int c = __popc(__ballot_sync(0xffffffffu, le));
    q += c;
    if (c < 32) return q;
  }
}

// decide() with the serial Case-2 loop replaced by one ballot over up to 32
// queue states: state k holds k + 1 queries at tau_k = max(t0, a[h + k]); it
// is "complete" when the next arrival comes strictly later (or the queue is
// at Bmax), and the batch leaves at the first complete state that must
// dispatch now (k + 1 = Bmax, or tau_k >= Tmax_wait(k + 2)) or whose timer
// Tmax_wait(k + 2) fires before the next arrival.  Ts[b - 1] = T(b).
template <class Arr>
__device__ __forceinline__ int decide_par(const Arr &A, int64_t n, int64_t h, int64_t F, int Bmax, int64_t L,
                                          const int32_t *Ts, int lane, int64_t *t_out) {
  const int64_t ah = A(h);
  const int64_t t0 = F > ah ? F : ah;
  const int q0 = count_le(A, n, h, 1, Bmax, t0, lane);
  for (int kb = q0 - 1;; kb += 32) {
    const int k = kb + lane;
    const bool valid = k + 1 <= Bmax && h + k < n;
    bool stop = false, now = false;
    int64_t tau = 0, W = 0;
    if (valid) {
      const int64_t ak = A(h + k);
      tau = ak > t0 ? ak : t0;
      const bool capped = k + 1 == Bmax;
      const int64_t nxt = h + k + 1 < n ? (int64_t)A(h + k + 1) : INT64_MAX;
      W = capped ? 0 : ah + L - Ts[k + 1];
      now = capped || tau >= W;
      stop = (capped || nxt > tau) && (now || nxt > W);
    }
    const unsigned bal = __ballot_sync(0xffffffffu, stop);
    if (bal) {
      const int src = __ffs(bal) - 1;
      *t_out = __shfl_sync(0xffffffffu, now ? tau : W, src);
      return kb + src + 1;
    }
  }
}

__host__ __device__ __forceinline__ size_t stitch_wstride(int bmax) {
  return ((size_t)2 * RING + 8 + 64 * SUMAX + bmax + 3) & ~(size_t)3;
}
static size_t stitch_smem(int bmax) { return 4 * stitch_wstride(bmax) * 4; }

__global__ void __launch_bounds__(128) k_stitch(const __grid_constant__ LaneArgs a) {
  // shared memory per warp: arrival ring [RING], stored-latency ring [RING]
  // (the chunk runs' rows, same segments), mbarriers [4 ring slots], stretch
  // finishes [32 SUMAX], T [bmax]
  extern __shared__ __align__(16) uint32_t ssm[];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int64_t gw0 = (int64_t)blockIdx.x * 4 + w;
  if (gw0 >= (int64_t)a.nsc * a.D) return;
  const int64_t gw = a.lane_order ? a.lane_order[gw0] : gw0;  // pipelined: the longest lanes first
  const int s = a.sc_list[gw / a.D], d = (int)(gw % a.D);
  if (!((a.dmask >> d) & 1ull)) return;
  const LaneParam p = a.lp[s * a.D + d];
  const int64_t off = a.devOff[d], n = a.devOff[d + 1] - off;
  const int64_t nch = a.choff[d + 1] - a.choff[d];
  if (p.Bmax < 1 || nch < 2 || (a.scan1 && p.Bmax == 1) || (a.skip && a.skip[s * a.D + d])) return;
  uint32_t *wsm = ssm + (size_t)w * stitch_wstride(a.bmax);
  uint32_t *ring = wsm;
  uint32_t *lring = wsm + RING;
  uint64_t *bars = (uint64_t *)(wsm + 2 * RING);  // ring slots
  int64_t *FeS = (int64_t *)(wsm + 2 * RING + 8);  // [32 SUMAX] stretch batch finishes
  int32_t *T = (int32_t *)(wsm + 2 * RING + 8 + 64 * SUMAX);
  const int32_t *Tg = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
  for (int k = lane; k < a.bmax; k += 32) T[k] = Tg[k];
  if (lane < 4) mbar_init(bars + lane);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  uint32_t *out = a.latd + (size_t)s * a.NS + off;
  const ChunkSt *cst = a.cs + (size_t)s * a.NCH + a.choff[d];
  const int64_t CH = a.CH;
  if (a.cready) wait_chunk(a.cready, (size_t)s * a.NCH + a.choff[d]);  // chunk 0's exit (pipelined k_spec)
  int64_t h = (CH < n ? CH : n) + cst[0].xov, F = cst[0].xF;
  int64_t cstart = 1;  // first chunk to stitch; a lane the full-batch scan took starts where it stopped
  bool fresh = false;  // ... with the positions below h of that chunk already written
  if (a.lstart && a.lstart[2 * ((size_t)s * a.D + d)] >= 0) {
    h = a.lstart[2 * ((size_t)s * a.D + d)];
    F = a.lstart[2 * ((size_t)s * a.D + d) + 1];
    cstart = h / CH;
    fresh = true;
  }
  // Arrivals stream through a 4-segment ring by TMA bulk copies of whole
  // 1024-query segments of the routed array (segment g >> 10 of the absolute
  // index g = off + j sits in slot (g >> 10) & 3, so ring[g & (RING - 1)] is
  // query g).  Segments up to the one 2 past h's are in flight; a slot is
  // refilled only after its previous segment has been waited for and lies
  // 2 segments behind h (the stitch reads back at most Bmax - 1 <= 1023).
  const int64_t sg0 = (off + (fresh ? h : CH)) >> 10;  // first segment ever read (chunk 1 starts at CH)
  int64_t sg_iss = sg0, sg_wait = sg0;
  auto seg_wait_one = [&]() {
    mbar_wait(bars + (sg_wait & 3), (uint32_t)(((sg_wait - sg0) >> 2) & 1));
    sg_wait++;
  };
  auto seg_issue = [&](int64_t hcur) {
    const int64_t lim = ((off + hcur) >> 10) + 3;
    while (sg_iss < lim) {
      while (sg_wait <= sg_iss - 4) seg_wait_one();
      __syncwarp();
      // arrivals and the stored latencies of the same positions (the row holds
      // the chunk runs' values at every position >= h: rewritten ones lie below)
      if (lane == 0) {
        if (a.cready) {  // the segment's chunks of this device are published (pipelined k_spec)
          const int64_t j0 = sg_iss * RSEG - off, j1 = j0 + RSEG - 1;
          const int64_t ca = (j0 > 0 ? j0 : 0) / CH, cb = (j1 < n - 1 ? j1 : n - 1) / CH;
          for (int64_t cc = ca; cc <= cb && cc < nch; cc++) wait_chunk(a.cready, (size_t)s * a.NCH + a.choff[d] + cc);
          asm volatile("fence.proxy.async.global;" ::: "memory");  // generic-proxy writes -> the bulk copy
        }
        bulk_load2(ring + (sg_iss & 3) * RSEG, a.devArr + sg_iss * RSEG, lring + (sg_iss & 3) * RSEG,
                   a.latd + (size_t)s * a.NS + sg_iss * RSEG, RSEG * 4, bars + (sg_iss & 3));
      }
      sg_iss++;
    }
  };
  // make queries [.., jend) of the device readable (jend <= the segment 3 past h's);
  // h_safe: below it a decision at h needs no ring work (issue or wait)
  int64_t h_safe = 0;
  const int64_t look = p.Bmax <= 512 ? 2 * p.Bmax : p.Bmax;  // read-ahead of a decision (+ stretch test)
  auto need = [&](int64_t hcur, int64_t jend) {
    seg_issue(hcur);
    const int64_t gend = off + jend;
    while (sg_wait * RSEG < gend) seg_wait_one();
    const int64_t s1 = (sg_iss - 2) * RSEG - off, s2 = sg_wait * RSEG - off - look;
    h_safe = s1 < s2 ? s1 : s2;
  };
  const uint32_t ro = (uint32_t)(off & (RING - 1));
  auto AR = [&](int64_t j) -> int64_t { return ring[(ro + (uint32_t)j) & (RING - 1)]; };
  auto LR = [&](int64_t j) -> uint32_t { return lring[(ro + (uint32_t)j) & (RING - 1)]; };
  auto put = [&](int64_t j, int64_t Fb) { out[j] = sat_lat(Fb - AR(j)); };
  // the stored run's finish time of the batch holding query j (its latency
  // row is rewritten only below the current head)
  auto spec_F = [&](int64_t j) -> int64_t { return AR(j) + LR(j); };
  const int64_t TB = T[p.Bmax - 1];
  // the 32-bit decision needs L < C / 2 and every T(b) < C (so W_k < C and
  // t + T(b) < 2^31); per-lane W_k = L - T(k + 2) and T(k + 1) for the
  // first two ballot rounds stay in registers
  int32_t tmax = 0;
  for (int k = lane; k < p.Bmax; k += 32) tmax = T[k] > tmax ? T[k] : tmax;
  tmax = __reduce_max_sync(0xffffffffu, tmax);
  const bool lean = !(a.bsearch && p.mono) && p.L < LEAN_C / 2 && tmax < LEAN_C;
  const int32_t W0 = lane + 1 < p.Bmax ? (int32_t)p.L - T[lane + 1] : 0;
  const int32_t W1 = lane + 33 < p.Bmax ? (int32_t)p.L - T[lane + 33] : 0;
  const int32_t T0 = lane < p.Bmax ? T[lane] : 0;
  const int32_t T1 = lane + 32 < p.Bmax ? T[lane + 32] : 0;
  const int SU = p.Bmax >= 16 ? 1 : p.Bmax >= 8 ? 2 : SUMAX;  // batches per lane in a full-batch stretch
  const uint32_t bmagic = (uint32_t)((1ull << 32) / (uint64_t)p.Bmax + 1);  // q / Bmax = umulhi(q, bmagic), q < 2^16
  // SW: a full batch needs its last arrival <= max(F_i, a[h_i] + SW) (see the stretch)
  int32_t tbig = 0;
  for (int k = lane; k + 1 < p.Bmax; k += 32) tbig = T[k] > tbig ? T[k] : tbig;
  tbig = __reduce_max_sync(0xffffffffu, tbig);
  const int64_t SW = tbig <= TB ? (p.L - TB > 0 ? p.L - TB : 0) : INT64_MIN / 4;
  bool lastfull = true;
  const int64_t li_t = (gw / a.D) * a.D + d;  // lane index of the chunk tables
  const int tEl = a.tE ? a.tE[li_t] : 0;
  const WinRec *trow = tEl ? a.trec + a.trecoff[li_t] : nullptr;
  WinEntry *rwrow = tEl ? a.rw + li_t * a.NCH : nullptr;
  long long dbg_t0 = clock64(), dbg_dec = 0, dbg_jump = 0, dbg_match = 0, dbg_chk = 0;
  long long dbg_sec[5] = {0, 0, 0, 0, 0}, dbg_tk = 0;
  for (int64_t c0 = cstart; c0 < nch; c0 += 32) {
    ChunkSt cr = {0, 0, 0, 0};
    if (a.cready && c0 + lane < nch) wait_chunk(a.cready, (size_t)s * a.NCH + a.choff[d] + c0 + lane);
    if (c0 + lane < nch) cr = cst[c0 + lane];
    const int cnt = nch - c0 < 32 ? (int)(nch - c0) : 32;
    for (int k = 0; k < cnt; k++) {
      const int64_t c = c0 + k;
      const int64_t st = c * CH, en = st + CH < n ? st + CH : n;
      const int64_t xF = __shfl_sync(0xffffffffu, cr.xF, k);
      const int xov = __shfl_sync(0xffffffffu, cr.xov, k);
      const int64_t eF = __shfl_sync(0xffffffffu, cr.eF, k);
      const int edh = __shfl_sync(0xffffffffu, cr.edh, k);
      need(h, (h < en ? h : en) + p.Bmax + 1);
      if (h > st && !(fresh && c == cstart)) {  // queries of this chunk in the last batch of the previous one
        const int64_t hi = h < en ? h : en;
        for (int64_t j = st + lane; j < hi; j += 32) put(j, F);
      }
      if (h >= en) continue;
      // the stored run of the chunk entered at (st + edh, eF): the true run
      // takes the same decisions from the same head when its device is free
      // at the same time, or when both are free by the head's arrival
      if (h - st == edh && (F == eF || (F <= AR(h) && eF <= AR(h)))) {
        h = en + xov;
        F = xF;
        PX_DBG(dbg_match++);
        continue;
      }
      if (tEl > h - st) {  // the chain table: an entry on the idle branch is a function of its head
        const WinRec r = trow[c * tEl + (h - st)];
        if (F <= AR(st) + r.tdisp) {
          if (lane == 0) { WinEntry e; e.F = F; e.h = (int32_t)h; e.pad = 1; rwrow[c] = e; }
          h = st + r.hx;
          F = r.Fx;
          continue;
        }
      }
      int checks = a.maxchk;
      const bool spec_ready = true;  // stored latencies stream through lring (positions >= h)
      while (h < en) {
        PX_DBG(if (dbg_tk) dbg_sec[3] += clock64() - dbg_tk; dbg_tk = clock64());
        if (h >= h_safe) need(h, h + look + 1);  // decision + the stretch test's two batches
        const int64_t ah = AR(h);
        PX_DBG(__syncwarp(); dbg_sec[4] += clock64() - dbg_tk; dbg_tk = clock64());
        bool stretch = false;
        if ((lastfull || F > ah) && p.Bmax <= 512 && h + 2 * p.Bmax - 1 < n) {  // are the next two batches full?
          const int64_t A0 = AR(h + p.Bmax - 1), A1 = AR(h + 2 * p.Bmax - 1), a1 = AR(h + p.Bmax);
          const int64_t F1 = (F > A0 ? F : A0) + TB;
          stretch = A0 <= (F > ah + SW ? F : ah + SW) && A1 <= (F1 > a1 + SW ? F1 : a1 + SW);
        }
        if (stretch) {
          // full-batch stretch: while every batch is full (Bmax queries), batch i
          // dispatches when the device is free and its last query has arrived,
          // F_{i+1} = max(F_i, A_i) + T(Bmax), A_i = a[h_i + Bmax - 1], so
          // F_i = i T(Bmax) + max(F_0, max_{j<i} (A_j - j T(Bmax))): a max-plus
          // scan.  Batch i is full if A_i <= max(F_i, a[h_i] + SW): every queue
          // state k < Bmax - 1 then has its next arrival <= max(tau_k, W_k)
          // because W_k = a[h_i] + L - T(k+2) >= a[h_i] + L - T(Bmax) when
          // T(Bmax) is the largest of T(1..Bmax) (else SW = -inf: A_i <= F_i,
          // the queue already holds Bmax queries).  Rounds of 32 SU batches,
          // lane l taking [l SU, l SU + SU) of the round.
          auto divB = [&](int64_t x) -> int64_t {  // x / Bmax for 0 <= x (capped at 2^15)
            const uint32_t u = (uint32_t)(x < 32768 ? x : 32768);
            return p.Bmax == 1 ? u : __umulhi(u, bmagic);
          };
          int64_t kmax = divB(en - h + p.Bmax - 1);  // batches starting in this chunk
          const int64_t room = divB((((off + h) >> 10) + 3) * RSEG - (off + h));
          const int64_t avail = divB(n - h);
          if (kmax > room) kmax = room;
          if (kmax > avail) kmax = avail;
          need(h, h + kmax * p.Bmax);
          int64_t Mc = F;  // max(F_0, G_j for the batches taken so far)
          int64_t done = 0;
          while (done < kmax) {
            const int64_t ib = done + lane * SU;
            int64_t G[SUMAX];
            int64_t gl = INT64_MIN;
#pragma unroll
            for (int u = 0; u < SUMAX; u++) {
              G[u] = INT64_MIN;
              if (u < SU && ib + u < kmax) {
                G[u] = AR(h + (ib + u + 1) * p.Bmax - 1) - (ib + u) * TB;
                gl = G[u] > gl ? G[u] : gl;
              }
            }
            int64_t inc = gl;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
              const int64_t v = __shfl_up_sync(0xffffffffu, inc, o);
              if (lane >= o && v > inc) inc = v;
            }
            int64_t exc = __shfl_up_sync(0xffffffffu, inc, 1);
            if (lane == 0) exc = INT64_MIN;
            int64_t M = Mc > exc ? Mc : exc;
            int fl = SU;
#pragma unroll
            for (int u = 0; u < SUMAX; u++) {
              if (u < SU && fl == SU) {
                const int64_t i = ib + u;
                if (i >= kmax) {
                  fl = u;
                } else {
                  const int64_t Fi = i * TB + M;
                  const int64_t lim = AR(h + i * p.Bmax) + SW;
                  if (G[u] + i * TB > (Fi > lim ? Fi : lim)) fl = u;
                  else M = G[u] > M ? G[u] : M;
                }
              }
            }
            const unsigned bal = __ballot_sync(0xffffffffu, fl < SU);
            const int fs = bal ? __ffs(bal) - 1 : 31;
            const int64_t r = bal ? (int64_t)fs * SU + __shfl_sync(0xffffffffu, fl, fs) : 32 * SU;
            // latencies of the accepted batches: finishes through shared
            // memory, then the round's queries in coalesced lane strides
            M = Mc > exc ? Mc : exc;
#pragma unroll
            for (int u = 0; u < SUMAX; u++) {
              const int64_t i = ib + u;
              if (u < SU && i < done + r) {
                M = G[u] > M ? G[u] : M;
                FeS[lane * SU + u] = (i + 1) * TB + M;
              }
            }
            __syncwarp();
            const int64_t hb = h + done * p.Bmax;
            const uint32_t np = (uint32_t)(r * p.Bmax);
            for (uint32_t q = lane; q < np; q += 32)
              out[hb + q] = sat_lat(FeS[p.Bmax == 1 ? q : __umulhi(q, bmagic)] - AR(hb + q));
            __syncwarp();
            if (r > 0) {
              Mc = __shfl_sync(0xffffffffu, M, (int)((r - 1) / SU));
              done += r;
            }
            if (r < 32 * SU) break;
          }
          if (done > 0) {
            F = done * TB + Mc;
            h += done * p.Bmax;
            lastfull = true;
            PX_DBG(dbg_jump++);
            // no meeting test here: the latency cache is filled lazily and
            // position h - 1 was just rewritten; the next decision tests
            continue;
          }
        }
        PX_DBG(dbg_dec++; dbg_tk = clock64());
        // one decision (see decide_par): queue states k = 0.. in rounds of 32;
        // states inside the initial queue are incomplete and never stop
        int b;
        int64_t Fn;
        const int64_t fr = F - ah;
        if (lean && fr < LEAN_C) {
          // 32-bit form relative to a_h: d_k = min(a_{h+k} - a_h, C), t0 = max(F - a_h, 0),
          // W_k = L - T(k + 2).  Exact: C > max W_k and t0 < C, and the first
          // state whose next arrival clamps (d >= C) is preceded by a state
          // that stops (its next arrival exceeds both tau and W), so no clamped
          // value ever reaches the chosen state.  Lane k holds state k; it
          // then writes query h + k's latency from its own d_k, and tests
          // whether the speculative run's batch holding h + k finishes at Fn:
          // the runs meet at j2 = h + b when lane b - 1 says yes and lane b no.
          const int32_t t0 = fr > 0 ? (int32_t)fr : 0;
          const int64_t rem = n - h;
          const int lim = rem < p.Bmax ? (int)rem : p.Bmax;
          const uint32_t uah = (uint32_t)ah;
          const bool test = spec_ready && checks > 0;
          // lane holds states k = lane and (Bmax > 32) k = lane + 32
          struct St {
            uint32_t du, sp;
            int32_t dk, cand;
            bool stop, fre;
          };
          auto st = [&](int k, int32_t Wk, int32_t Tk) {
            St r;
            // only queries the ring holds for this decision are read (k <= lim: the meeting test's lane b)
            r.du = k <= lim && h + k < n ? (uint32_t)AR(h + k) - uah : 0u;
            const uint32_t dn = k + 1 < lim ? (uint32_t)AR(h + k + 1) - uah : 0u;
            r.sp = test && h + k < en ? LR(h + k) : 0u;
            r.dk = r.du < (uint32_t)LEAN_C ? (int32_t)r.du : LEAN_C;
            const int32_t tau = r.dk > t0 ? r.dk : t0;
            const bool capped = k + 1 == p.Bmax;
            const int32_t nx = k + 1 < lim ? (dn < (uint32_t)LEAN_C ? (int32_t)dn : LEAN_C) : LEAN_C;
            const bool now = capped || tau >= Wk;
            const int32_t tr = now ? tau : Wk;
            r.stop = k < lim && (capped || nx > tau) && (now || nx > Wk);
            r.fre = tr > t0;
            r.cand = tr + Tk;
            return r;
          };
          const St s0 = st(lane, W0, T0);
          const unsigned bal0 = __ballot_sync(0xffffffffu, s0.stop);
          const unsigned fb0 = __ballot_sync(0xffffffffu, s0.fre);
          int32_t c;
          unsigned fbs, bals;
          St s1{};
          if (bal0) {
            bals = bal0;
            fbs = fb0;
            b = 0;
          } else {  // no stop among the first 32 states (Bmax > 32)
            if (p.Bmax > 64) goto long_queue;
            s1 = st(lane + 32, W1, T1);
            bals = __ballot_sync(0xffffffffu, s1.stop);
            fbs = __ballot_sync(0xffffffffu, s1.fre);
            b = 32;
          }
          const int sl = __ffs(bals) - 1;
          c = __shfl_sync(0xffffffffu, b ? s1.cand : s0.cand, sl);  // Fn - a_h
          Fn = ah + c;
          b += sl + 1;
          const bool isfree = fr < 0 || ((fbs >> sl) & 1u);  // dispatched after the device freed (t > F)
          const int64_t j2 = h + b;
          bool conv = false;
          if (isfree && j2 < en && checks > 0) {
            checks--;
            PX_DBG(dbg_chk++);
            if (test && b < 32) {
              // bit k: the speculative batch holding h + k finishes at Fn
              const unsigned e = __ballot_sync(0xffffffffu, (uint64_t)s0.sp + s0.du == (uint64_t)(uint32_t)c);
              conv = ((e >> (b - 1)) & 1u) && !((e >> b) & 1u);
            } else {
              conv = spec_F(j2 - 1) == Fn && spec_F(j2) != Fn;
            }
          }
          // latencies of queries h + k (< 2^31); after the test: a phase run's cache reads out[] at its first fill
          if (lane < b && h + lane < en) out[h + lane] = (uint32_t)(c - s0.dk);
          if (lane + 32 < b && h + lane + 32 < en) out[h + lane + 32] = (uint32_t)(c - s1.dk);
          PX_DBG(__syncwarp(); dbg_sec[0] += clock64() - dbg_tk; dbg_tk = clock64());
          h = j2;
          F = Fn;
          lastfull = b == p.Bmax;
          if (conv) {
            // the rest of the chunk is the stored run's
            h = en + xov;
            F = xF;
            break;
          }
          continue;
        }
      long_queue:
        bool isfree;
        if (lean && fr < LEAN_C) {
          const int32_t t0 = fr > 0 ? (int32_t)fr : 0;
          const int64_t rem = n - h;
          const int lim = rem < p.Bmax ? (int)rem : p.Bmax;
          const uint32_t uah = (uint32_t)ah;
          auto state = [&](int k, int32_t Wk, int32_t Tk, int32_t &cand, bool &fre) -> bool {
            if (k >= lim) return false;
            const uint32_t du = (uint32_t)AR(h + k) - uah;
            const int32_t dk = du < (uint32_t)LEAN_C ? (int32_t)du : LEAN_C;
            const int32_t tau = dk > t0 ? dk : t0;
            const bool capped = k + 1 == p.Bmax;
            const uint32_t dn = k + 1 < lim ? (uint32_t)AR(h + k + 1) - uah : 0u;
            const int32_t nx = k + 1 < lim ? (dn < (uint32_t)LEAN_C ? (int32_t)dn : LEAN_C) : LEAN_C;
            const bool now = capped || tau >= Wk;
            const int32_t tr = now ? tau : Wk;
            fre = tr > t0;
            cand = tr + Tk;
            return (capped || nx > tau) && (now || nx > Wk);
          };
          int32_t cand = 0;
          bool fre = false;
          unsigned bal = __ballot_sync(0xffffffffu, state(lane, W0, T0, cand, fre));
          unsigned fb = __ballot_sync(0xffffffffu, fre);
          int kb = 0;
          while (!bal) {  // queues longer than 32 (Bmax > 32)
            kb += 32;
            const int k = kb + lane;
            const int32_t Wk = kb == 32 ? W1 : (k + 1 < p.Bmax ? (int32_t)p.L - T[k + 1] : 0);
            const int32_t Tk = kb == 32 ? T1 : (k < p.Bmax ? T[k] : 0);
            bal = __ballot_sync(0xffffffffu, state(k, Wk, Tk, cand, fre));
            fb = __ballot_sync(0xffffffffu, fre);
          }
          const int sl = __ffs(bal) - 1;
          Fn = ah + __shfl_sync(0xffffffffu, cand, sl);
          b = kb + sl + 1;
          isfree = fr < 0 || ((fb >> sl) & 1u);  // dispatched after the device freed (t > F)
        } else if (a.bsearch && p.mono) {
          // facts (i)-(ii) of the window path: the idle decision by binary search
          // over the ring, or the greedy batch when the device frees after it
          // (every lane the same probes: shared-memory broadcasts, no ballots)
          int64_t t;
          b = fast_decide(AR, n, h, F, p.Bmax, p.L, T, true, &t);
          Fn = t + T[b - 1];
          isfree = t > F;
        } else {
          const int64_t t0 = F > ah ? F : ah;
          int64_t t;
          for (int kb = 0;; kb += 32) {
            const int k = kb + lane;
            bool stop = false, now = false;
            int64_t tau = 0, W = 0;
            if (k < p.Bmax && h + k < n) {
              const int64_t ak = AR(h + k);
              tau = ak > t0 ? ak : t0;
              const bool capped = k + 1 == p.Bmax;
              const int64_t nxt = h + k + 1 < n ? AR(h + k + 1) : INT64_MAX;
              W = capped ? 0 : ah + p.L - T[k + 1];
              now = capped || tau >= W;
              stop = (capped || nxt > tau) && (now || nxt > W);
            }
            const unsigned bal = __ballot_sync(0xffffffffu, stop);
            if (bal) {
              const int sl = __ffs(bal) - 1;
              t = __shfl_sync(0xffffffffu, now ? tau : W, sl);
              b = kb + sl + 1;
              break;
            }
          }
          Fn = t + T[b - 1];
          isfree = t > F;
        }
        PX_DBG(__syncwarp(); dbg_sec[0] += clock64() - dbg_tk; dbg_tk = clock64());
        const int64_t j2 = h + b;
        bool conv = false;
        if (isfree && j2 < en && checks > 0) {
          checks--;
          PX_DBG(dbg_chk++);
          conv = spec_F(j2 - 1) == Fn && spec_F(j2) != Fn;
        }
        PX_DBG(__syncwarp(); dbg_sec[1] += clock64() - dbg_tk; dbg_tk = clock64());
        const int64_t hi = j2 < en ? j2 : en;
        for (int64_t jj = h + lane; jj < hi; jj += 32) out[jj] = sat_lat(Fn - AR(jj));
        PX_DBG(__syncwarp(); dbg_sec[2] += clock64() - dbg_tk; dbg_tk = clock64());
        h = j2;
        F = Fn;
        lastfull = b == p.Bmax;
        if (conv) {
          // the rest of the chunk is the stored run's
          h = en + xov;
          F = xF;
          break;
        }
      }
    }
  }
  if (a.debug && lane == 0) {
    const long long cyc = clock64() - dbg_t0;
    if (cyc > a.debug) printf("stitch s=%d d=%d n=%lld Bmax=%d L=%lld nch=%lld start=%lld full=%u dec_spec=%u cycles=%lld dec=%lld jump=%lld match=%lld chk=%lld "
                              "sdec=%lld schk=%lld swr=%lld sloop=%lld sring=%lld\n", s, d,
                              (long long)n, p.Bmax, (long long)p.L, (long long)nch, (long long)(fresh ? cstart * CH : -1),
                              a.lstat[2 * ((size_t)s * a.D + d)], a.lstat[2 * ((size_t)s * a.D + d) + 1], cyc, dbg_dec, dbg_jump, dbg_match, dbg_chk,
                              dbg_sec[0], dbg_sec[1], dbg_sec[2], dbg_sec[3], dbg_sec[4]);
  }
}

// ---- phase B, parallel form: fix-up rounds, one warp per (chunk, scenario)
// Round k re-walks every chunk c >= 1 whose entry state -- the exit of chunk
// c - 1 in round k - 1 -- differs from the entry of the run its rows hold,
// from that entry until the new run meets the stored one (same head and the
// same finish time after a batch the device waited for: from there on the
// two runs take the same decisions) or the chunk ends.  Entries that differ
// only in a device-free time that is <= the head's arrival give the same
// decisions and need only the overhang rewritten.  Chunk c's exit changes
// only if it did not meet; *changed counts those, and a round with no
// change leaves every chunk exact (chunk 0 starts at the true initial state,
// R13, and by induction each chunk entry is the true one).  Reads of the
// stored row happen before the round rewrites them (positions >= the head).
// chunks the stitch hopped with a chain table: replay from the true entry
// (head h >= chunk start, free time F) to the chunk end (the positions before
// h were written by the stitch; those past the end belong to the next chunk,
// whose entry F the stitch carried).  Thread per (lane, chunk).
__global__ void __launch_bounds__(128) k_rewrite(const __grid_constant__ LaneArgs a) {
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g >= (int64_t)a.nsc * a.D * a.NCH) return;
  const int64_t li = g / a.NCH, c = g % a.NCH;
  if (!a.tE || a.tE[li] == 0) return;
  const WinEntry e = a.rw[li * a.NCH + c];
  if (e.pad != 1) return;
  const int d = (int)(li % a.D), s = a.sc_list[li / a.D];
  const LaneParam p = a.lp[s * a.D + d];
  const int64_t off = a.devOff[d], n = a.devOff[d + 1] - off;
  const int64_t st = c * a.CH, en = st + a.CH < n ? st + a.CH : n;
  const int32_t *T = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
  GArr arr{a.devArr + off};
  uint32_t *out = a.latd + (size_t)s * a.NS + off;
  int64_t h = e.h, F = e.F;
  while (h < en) {
    int64_t t;
    const int b = decide(arr, n, h, F, p.Bmax, p.L, T, &t);
    F = t + T[b - 1];
    const int64_t jend = h + b < en ? h + b : en;
    for (int64_t j = h; j < jend; j++) out[j] = sat_lat(F - (int64_t)arr(j));
    h += b;
  }
}

__global__ void __launch_bounds__(128) k_fix(const __grid_constant__ LaneArgs a, unsigned *changed) {
  __shared__ int64_t sC[PX_MAXD + 1];
  for (int k = threadIdx.x; k <= a.D; k += blockDim.x) sC[k] = a.choff[k];
  __syncthreads();
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t g = (int64_t)blockIdx.y * 4 + w;  // chunk index over all devices of the routing mode
  if (g >= sC[a.D]) return;
  int d = 0;
  while (g >= sC[d + 1]) d++;
  if (!((a.dmask >> d) & 1ull)) return;
  const int s = a.sc_list[blockIdx.x];
  const int64_t c = g - sC[d];
  const size_t row = (size_t)s * a.NCH + sC[d];
  const ChunkSt old = a.csp[row + c];
  const LaneParam p = a.lp[s * a.D + d];
  if (a.scan1 && p.Bmax == 1) return;  // produced by k_scan1_*
  const unsigned *ls = a.lstat + 2 * ((size_t)s * a.D + d);
  if (c == 0 || p.Bmax < 1 || 4ull * ls[0] >= ls[1]) {
    // chunk 0 is exact from the start; unrouted devices have no runs;
    // backlogged lanes are left to the stitch (changed[1] says one exists)
    if (c == 1 && p.Bmax >= 1 && 4ull * ls[0] >= ls[1] && lane == 0) atomicOr(changed + 1, 1u);
    if (lane == 0) a.cs[row + c] = old;
    return;
  }
  const int64_t off = a.devOff[d], n = a.devOff[d + 1] - off;
  const int64_t st = c * a.CH, en = st + a.CH < n ? st + a.CH : n;
  const ChunkSt prev = a.csp[row + c - 1];
  int64_t h = st + prev.xov, F = prev.xF;
  const uint32_t *A = a.devArr + off;
  uint32_t *out = a.latd + (size_t)s * a.NS + off;
  const int32_t *T = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
  ChunkSt nw = old;
  nw.edh = (int32_t)(h - st);
  nw.eF = F;
  const int64_t ah0 = h < n ? (int64_t)__ldg(A + h) : INT64_MAX;
  const bool same_head = h - st == old.edh;
  if (same_head && (F == old.eF || (F <= ah0 && old.eF <= ah0))) {
    if (F != old.eF) {  // same decisions; the overhang belongs to the new finish time
      const int64_t hi = h < en ? h : en;
      for (int64_t j = st + lane; j < hi; j += 32) out[j] = sat_lat(F - (int64_t)__ldg(A + j));
    }
    if (lane == 0) a.cs[row + c] = nw;
    return;
  }
  {
    const int64_t hi = h < en ? h : en;  // queries of this chunk in the last batch of the previous one
    for (int64_t j = st + lane; j < hi; j += 32) out[j] = sat_lat(F - (int64_t)__ldg(A + j));
  }
  bool met = false;
  while (h < en) {
    // decision (R1-R5) as a ballot over queue states k = 0, 1, ... (decide_par),
    // with the stored run's finish times of the same positions for the
    // meeting test, all read before this batch's latencies are written
    const int64_t ah = __ldg(A + h);
    const int64_t t0 = F > ah ? F : ah;
    int q0 = 1;
    for (;;) {  // queries queued at t0 (arrivals are sorted: a prefix)
      const int64_t j = h + q0 + lane;
      const bool le = q0 + lane < p.Bmax && j < n && (int64_t)__ldg(A + j) <= t0;
      const int cnt = __popc(__ballot_sync(0xffffffffu, le));
      q0 += cnt;
      if (cnt < 32) break;
    }
    int b = 0;
    int64_t t = 0;
    for (int kb = q0 - 1;; kb += 32) {
      const int k = kb + lane;
      bool stop = false, now = false;
      int64_t tau = 0, W = 0;
      if (k + 1 <= p.Bmax && h + k < n) {
        const int64_t ak = __ldg(A + h + k);
        tau = ak > t0 ? ak : t0;
        const bool capped = k + 1 == p.Bmax;
        const int64_t nxt = h + k + 1 < n ? (int64_t)__ldg(A + h + k + 1) : INT64_MAX;
        W = capped ? 0 : ah + p.L - T[k + 1];
        now = capped || tau >= W;
        stop = (capped || nxt > tau) && (now || nxt > W);
      }
      const unsigned bal = __ballot_sync(0xffffffffu, stop);
      if (bal) {
        const int sl = __ffs(bal) - 1;
        t = __shfl_sync(0xffffffffu, now ? tau : W, sl);
        b = kb + sl + 1;
        break;
      }
    }
    const int64_t Fn = t + T[b - 1];
    const int64_t j2 = h + b;
    if (t > F && j2 < en) {  // met: the stored run also ends a batch at j2 - 1 finishing at Fn
      const int64_t f1 = (int64_t)__ldg(A + j2 - 1) + out[j2 - 1];
      const int64_t f2 = (int64_t)__ldg(A + j2) + out[j2];
      met = f1 == Fn && f2 != Fn;
    }
    __syncwarp();
    const int64_t hi = j2 < en ? j2 : en;
    for (int64_t j = h + lane; j < hi; j += 32) out[j] = sat_lat(Fn - (int64_t)__ldg(A + j));
    h = j2;
    F = Fn;
    if (met) break;
  }
  if (!met) {
    nw.xF = F;
    nw.xov = (int32_t)(h - en);
    if (lane == 0 && (nw.xF != old.xF || nw.xov != old.xov)) atomicAdd(changed, 1u);
  }
  if (lane == 0) a.cs[row + c] = nw;
}

// ---- lanes with Bmax = 1 (no batching, "w/o AB"): every
// decision dispatches the head at t = max(F, a_h) (R4: a queue of one is
// full), so F_i = max(F_{i-1}, a_i) + T(1) with F_{-1} = 0 (R13).  With
// G_i = F_i - (i + 1) T(1) this is G_i = max(G_{i-1}, a_i - i T(1)), G_{-1} = 0:
// a prefix maximum, computed exactly in parallel (block maxima, per-device
// prefix over blocks, then per-warp scans).  The SLO does not enter the rule,
// so every Bmax = 1 scenario of a device gets the same latency row.
#define SCAN_BLK 4096
struct Scan1Args {
  int D, nsc;
  int64_t N, NS;
  int64_t boff[PX_MAXD + 1];  // block offsets per device (SCAN_BLK queries per block)
  const int64_t *devOff;
  const uint32_t *devArr;
  const int32_t *T1;          // [D] T(1) of the device's variant (0: device has no Bmax = 1 lane)
  const int32_t *sc_list;
  const LaneParam *lp;
  uint32_t *latd;
  int64_t *bmx, *bpre;        // [blocks] block maxima, exclusive prefix maxima
};

__device__ __forceinline__ int scan1_dev(const Scan1Args &a, int64_t b) {
  int d = 0;
  while (b >= a.boff[d + 1]) d++;
  return d;
}

__global__ void __launch_bounds__(256) k_scan1_reduce(const __grid_constant__ Scan1Args a) {
  const int64_t b = blockIdx.x;
  const int d = scan1_dev(a, b);
  const int64_t T1 = a.T1[d];
  int64_t m = INT64_MIN;
  if (T1 > 0) {
    const int64_t off = a.devOff[d], n = a.devOff[d + 1] - off;
    const int64_t i0 = (b - a.boff[d]) * SCAN_BLK;
    for (int64_t i = i0 + threadIdx.x; i < i0 + SCAN_BLK && i < n; i += blockDim.x) {
      const int64_t x = (int64_t)__ldg(a.devArr + off + i) - i * T1;
      m = x > m ? x : m;
    }
  }
  __shared__ int64_t red[8];
  for (int o = 16; o; o >>= 1) {
    const int64_t v = __shfl_xor_sync(0xffffffffu, m, o);
    m = v > m ? v : m;
  }
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = m;
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int k = 1; k < 8; k++) m = red[k] > m ? red[k] : m;
    a.bmx[b] = m;
  }
}

// one warp per device: exclusive prefix maximum over its blocks, seeded with G_{-1} = 0
__global__ void k_scan1_prefix(const __grid_constant__ Scan1Args a) {
  const int d = blockIdx.x, lane = threadIdx.x;
  int64_t carry = 0;
  for (int64_t b0 = a.boff[d]; b0 < a.boff[d + 1]; b0 += 32) {
    const int64_t b = b0 + lane;
    int64_t v = b < a.boff[d + 1] ? a.bmx[b] : INT64_MIN;
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t u = __shfl_up_sync(0xffffffffu, v, o);
      if (lane >= o && u > v) v = u;
    }
    int64_t ex = __shfl_up_sync(0xffffffffu, v, 1);
    if (lane == 0) ex = INT64_MIN;
    if (b < a.boff[d + 1]) a.bpre[b] = ex > carry ? ex : carry;
    const int64_t tot = __shfl_sync(0xffffffffu, v, 31);
    carry = tot > carry ? tot : carry;
  }
}

__global__ void __launch_bounds__(256) k_scan1_apply(const __grid_constant__ Scan1Args a) {
  __shared__ int64_t wmax[8];
  __shared__ int32_t rows[4096];
  __shared__ int nrows;
  const int64_t b = blockIdx.x;
  const int d = scan1_dev(a, b);
  const int64_t T1 = a.T1[d];
  if (T1 <= 0) return;
  if (threadIdx.x == 0) {
    int k = 0;
    for (int i = 0; i < a.nsc && k < 4096; i++) {
      const int s = a.sc_list[i];
      if (a.lp[s * a.D + d].Bmax == 1) rows[k++] = s;
    }
    nrows = k;
  }
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t off = a.devOff[d], n = a.devOff[d + 1] - off;
  const int64_t i0 = (b - a.boff[d]) * SCAN_BLK + (int64_t)w * (SCAN_BLK / 8);
  const int64_t i1 = i0 + SCAN_BLK / 8 < n ? i0 + SCAN_BLK / 8 : n;
  int64_t m = INT64_MIN;  // this warp's segment maximum
  for (int64_t i = i0 + lane; i < i1; i += 32) {
    const int64_t x = (int64_t)__ldg(a.devArr + off + i) - i * T1;
    m = x > m ? x : m;
  }
  for (int o = 16; o; o >>= 1) {
    const int64_t v = __shfl_xor_sync(0xffffffffu, m, o);
    m = v > m ? v : m;
  }
  if (lane == 0) wmax[w] = m;
  __syncthreads();
  int64_t carry = a.bpre[b];
  for (int k = 0; k < w; k++) carry = wmax[k] > carry ? wmax[k] : carry;
  const int nr = nrows;
  for (int64_t c0 = i0; c0 < i1; c0 += 32) {
    const int64_t i = c0 + lane;
    const int64_t ai = i < i1 ? (int64_t)__ldg(a.devArr + off + i) : 0;
    int64_t v = i < i1 ? ai - i * T1 : INT64_MIN;
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t u = __shfl_up_sync(0xffffffffu, v, o);
      if (lane >= o && u > v) v = u;
    }
    const int64_t G = v > carry ? v : carry;
    carry = __shfl_sync(0xffffffffu, G, 31);
    if (i < i1) {
      const uint32_t l = sat_lat(G + (i + 1) * T1 - ai);
      for (int r = 0; r < nr; r++) a.latd[(size_t)rows[r] * a.NS + off + i] = l;
    }
  }
}

// ---- backlogged lanes (Bmax = B >= 2): while the device is backlogged
// every batch is full, batch k = queries [kB, kB + B) from the trace start,
// dispatched when the device frees and its last query A_k has arrived:
// F_k = max(F_{k-1}, A_k) + T(B), F_{-1} = 0 -- the same prefix maximum as
// above, G_k = max(G_{k-1}, A_k - k T(B)).  Batch k is full under the rule
// (R1-R4) if A_k <= max(F_{k-1}, a_{kB} + SW), SW = L - T(B) when T(B) is the
// largest of T(1..B) (else SW = -inf: the queue must hold B when the device
// frees) -- the stretch condition of k_stitch.  The scan is exact up to the
// first batch k* that fails it; k_stitch continues from (k* B, F_{k*-1}).
// Lanes are taken when a quarter or more of their speculative decisions were
// full batches sent the moment the device freed (k_spec's statistics).
#define BSCAN_BLK 1024  // batches per block
struct BScanArgs {
  int D, nl;
  int64_t NS;
  const int64_t *loff;       // [nl + 1] block offsets per lane
  const int32_t *lid;        // [nl] lane = s * D + d
  const int64_t *devOff;
  const uint32_t *devArr;
  const int32_t *lat, *option, *dev_type;
  int M, bmax;
  const LaneParam *lp;
  const unsigned *lstat;
  uint32_t *latd;
  int64_t *bmx, *bpre;       // [blocks]
  unsigned long long *vio;   // [nl] first batch that fails the fullness test (init ~0)
  int64_t *lstart;           // [S * D][2] stitch start (head, F); head -1 = lane not scanned
};

struct BScanLane {
  int64_t off, n, nb, TB, SW;  // nb = full batches of the lane
  int B, lane, blk;            // blk = block index within the lane
  bool on;
};

__device__ __forceinline__ int bscan_find(const BScanArgs &a, int64_t b) {  // lane l: loff[l] <= b < loff[l + 1]
  int lo = 0, hi = a.nl;
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    if (__ldg(a.loff + mid) <= b) lo = mid; else hi = mid;
  }
  return lo;
}

__device__ __forceinline__ BScanLane bscan_lane(const BScanArgs &a, int64_t b) {
  BScanLane r;
  const int l = bscan_find(a, b);
  r.lane = a.lid[l];
  r.blk = (int)(b - a.loff[l]);
  const int d = r.lane % a.D;
  const LaneParam p = a.lp[r.lane];
  const unsigned *ls = a.lstat + 2 * (size_t)r.lane;
  r.B = p.Bmax;
  r.on = p.Bmax >= 2 && ls[1] > 0 && 4ull * ls[0] >= ls[1];
  if (!r.on) return r;
  r.off = a.devOff[d];
  r.n = a.devOff[d + 1] - r.off;
  r.nb = r.n / (r.B > 0 ? r.B : 1);
  const int32_t *T = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
  r.TB = r.B > 0 ? T[r.B - 1] : 0;
  int32_t tbig = 0;
  for (int k = 0; k + 1 < r.B; k++) tbig = T[k] > tbig ? T[k] : tbig;
  r.SW = tbig <= r.TB ? (p.L - r.TB > 0 ? p.L - r.TB : 0) : INT64_MIN / 4;
  return r;
}

__global__ void __launch_bounds__(256) k_bscan_reduce(const __grid_constant__ BScanArgs a) {
  const BScanLane L = bscan_lane(a, blockIdx.x);
  int64_t m = INT64_MIN;
  if (L.on) {
    const int64_t k0 = (int64_t)L.blk * BSCAN_BLK;
    for (int64_t k = k0 + threadIdx.x; k < k0 + BSCAN_BLK && k < L.nb; k += blockDim.x) {
      const int64_t x = (int64_t)__ldg(a.devArr + L.off + k * L.B + L.B - 1) - k * L.TB;
      m = x > m ? x : m;
    }
  }
  __shared__ int64_t red[8];
  for (int o = 16; o; o >>= 1) {
    const int64_t v = __shfl_xor_sync(0xffffffffu, m, o);
    m = v > m ? v : m;
  }
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = m;
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int k = 1; k < 8; k++) m = red[k] > m ? red[k] : m;
    a.bmx[blockIdx.x] = m;
  }
}

__global__ void k_bscan_prefix(const __grid_constant__ BScanArgs a) {
  const int l = blockIdx.x, lane = threadIdx.x;
  int64_t carry = 0;  // G_{-1} = 0
  for (int64_t b0 = a.loff[l]; b0 < a.loff[l + 1]; b0 += 32) {
    const int64_t b = b0 + lane;
    int64_t v = b < a.loff[l + 1] ? a.bmx[b] : INT64_MIN;
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t u = __shfl_up_sync(0xffffffffu, v, o);
      if (lane >= o && u > v) v = u;
    }
    int64_t ex = __shfl_up_sync(0xffffffffu, v, 1);
    if (lane == 0) ex = INT64_MIN;
    if (b < a.loff[l + 1]) a.bpre[b] = ex > carry ? ex : carry;
    const int64_t tot = __shfl_sync(0xffffffffu, v, 31);
    carry = tot > carry ? tot : carry;
  }
}

// F_k of the block's batches into Fs (block-wide scan: per-warp segments of
// BSCAN_BLK / 8 batches); returns false if the lane is not scanned
__device__ __forceinline__ bool bscan_block_F(const BScanArgs &a, const BScanLane &L, int64_t *Fs, int64_t *wmax) {
  if (!L.on) return false;
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t k0 = (int64_t)L.blk * BSCAN_BLK + (int64_t)w * (BSCAN_BLK / 8);
  const int64_t k1 = k0 + BSCAN_BLK / 8 < L.nb ? k0 + BSCAN_BLK / 8 : L.nb;
  int64_t m = INT64_MIN;
  for (int64_t k = k0 + lane; k < k1; k += 32) {
    const int64_t x = (int64_t)__ldg(a.devArr + L.off + k * L.B + L.B - 1) - k * L.TB;
    m = x > m ? x : m;
  }
  for (int o = 16; o; o >>= 1) {
    const int64_t v = __shfl_xor_sync(0xffffffffu, m, o);
    m = v > m ? v : m;
  }
  if (lane == 0) wmax[w] = m;
  __syncthreads();
  int64_t carry = a.bpre[blockIdx.x];
  for (int k = 0; k < w; k++) carry = wmax[k] > carry ? wmax[k] : carry;
  for (int64_t c0 = k0; c0 < k1; c0 += 32) {
    const int64_t k = c0 + lane;
    int64_t v = k < k1 ? (int64_t)__ldg(a.devArr + L.off + k * L.B + L.B - 1) - k * L.TB : INT64_MIN;
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t u = __shfl_up_sync(0xffffffffu, v, o);
      if (lane >= o && u > v) v = u;
    }
    const int64_t G = v > carry ? v : carry;
    carry = __shfl_sync(0xffffffffu, G, 31);
    if (k < k1) Fs[k - (int64_t)L.blk * BSCAN_BLK] = G + (k + 1) * L.TB;
  }
  __syncthreads();
  return true;
}

__global__ void __launch_bounds__(256) k_bscan_verify(const __grid_constant__ BScanArgs a) {
  __shared__ int64_t Fs[BSCAN_BLK], wmax[8];
  const BScanLane L = bscan_lane(a, blockIdx.x);
  if (!bscan_block_F(a, L, Fs, wmax)) return;
  const int64_t kb = (int64_t)L.blk * BSCAN_BLK;
  const int l = bscan_find(a, blockIdx.x);
  for (int i = threadIdx.x; i < BSCAN_BLK && kb + i < L.nb; i += blockDim.x) {
    const int64_t k = kb + i;
    // F_{k-1} (F_{-1} = 0; at a block start G_{k-1} is the block's exclusive prefix)
    const int64_t Fp = i > 0 ? Fs[i - 1] : k == 0 ? 0 : a.bpre[blockIdx.x] + k * L.TB;
    const int64_t Ak = __ldg(a.devArr + L.off + k * L.B + L.B - 1);
    const int64_t ah = __ldg(a.devArr + L.off + k * L.B);
    const int64_t lim = Fp > ah + L.SW ? Fp : ah + L.SW;
    if (Ak > lim) atomicMin(a.vio + l, (unsigned long long)k);
  }
}

__global__ void __launch_bounds__(256) k_bscan_apply(const __grid_constant__ BScanArgs a) {
  __shared__ int64_t Fs[BSCAN_BLK], wmax[8];
  const BScanLane L = bscan_lane(a, blockIdx.x);
  if (!bscan_block_F(a, L, Fs, wmax)) return;
  const int l = bscan_find(a, blockIdx.x);
  const unsigned long long v = a.vio[l];
  const int64_t kstar = v < (unsigned long long)L.nb ? (int64_t)v : L.nb;  // batches taken
  const int64_t kb = (int64_t)L.blk * BSCAN_BLK;
  const int64_t ke = kb + BSCAN_BLK < kstar ? kb + BSCAN_BLK : kstar;
  uint32_t *out = a.latd + (size_t)(L.lane / a.D) * a.NS + L.off;
  for (int64_t j = kb * L.B + threadIdx.x; j < ke * L.B; j += blockDim.x)
    out[j] = sat_lat(Fs[j / L.B - kb] - (int64_t)__ldg(a.devArr + L.off + j));
  // the stitch starts at batch k* with the device free at F_{k*-1}
  if (threadIdx.x == 0 && ((kstar == 0 && L.blk == 0) || (kstar > kb && kstar <= kb + BSCAN_BLK))) {
    a.lstart[2 * (size_t)L.lane] = kstar * L.B;
    a.lstart[2 * (size_t)L.lane + 1] = kstar == 0 ? 0 : Fs[kstar - 1 - kb];
  }
}

// ---- §8(f2) Nexus overload scan (reading R14)
// In an overload stretch of a Nexus lane (the device busy at every decision,
// a full window queued) batch k is decided at t_k = F + k T(B) from the state
// (h, F) where the stretch starts; its window starts at i_k = max(p_k, g_k),
// g_k = the first arrival >= t_k + T(B) - L, p_k = i_{k-1} + B (p_0 = h), and
// [p_k, i_k) are dropped: i_k = k B + max(h, max_{j<=k} (g_j - j B)), a prefix
// maximum (k_wc_lanes's stretch, 32 batches per warp step).  The scan takes the
// whole lane at once from the state k_wc_lanes recorded at its first stretch
// (nxmode 1): the g_k are independent searches, the prefix maximum a
// two-level scan, and the stretch is exact up to the first batch that is not
// valid (a_{p_k} <= t_k: busy; a_{i_k + B - 1} <= t_k: full window), where
// the second walk of k_wc_lanes takes over.  Block = NX_BLK batches of a lane.
#define NX_BLK 1024
struct NxArgs {
  int D, nl;
  int64_t NS;
  const int64_t *loff;       // [nl + 1] block offsets per lane
  const int32_t *lid;        // [nl] lane = s * D + d
  const int64_t *devOff;
  const uint32_t *devArr;
  const int32_t *lat, *option, *dev_type;
  int M, bmax;
  const LaneParam *lp;
  int64_t *lstart;           // [S * D][2] (h, F): the scan's start, then the second walk's
  uint32_t *latd;
  int64_t *bmx, *bpre;       // [blocks]
  int32_t *ik;               // [blocks * NX_BLK] window heads i_k (device-relative)
  unsigned long long *vio;   // [nl] first invalid batch (init ~0)
  int64_t *nxst;             // [nl][2] the second walk's start (k_nx_apply), copied to lstart by k_nx_commit
};

struct NxLane {
  int64_t off, n, h0, F0, TB, L, nb;
  int B, lane, blk;
  bool on;
};

__device__ __forceinline__ NxLane nx_lane(const NxArgs &a, int64_t b) {
  NxLane r;
  int lo = 0, hi = a.nl;
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    if (__ldg(a.loff + mid) <= b) lo = mid; else hi = mid;
  }
  r.lane = a.lid[lo];
  r.blk = (int)(b - a.loff[lo]);
  const int d = r.lane % a.D;
  const LaneParam p = a.lp[r.lane];
  r.B = p.Bn;
  r.L = p.L;
  r.off = a.devOff[d];
  r.n = a.devOff[d + 1] - r.off;
  r.h0 = a.lstart[2 * (size_t)r.lane];
  r.F0 = a.lstart[2 * (size_t)r.lane + 1];
  r.on = r.h0 >= 0 && r.h0 < r.n && r.B >= 1;
  const int32_t *T = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
  r.TB = T[r.B - 1];
  r.nb = r.on ? (r.n - r.h0) / r.B : 0;  // at most this many batches (i_k >= h0 + k B)
  return r;
}

// g_k - k B with g_k clamped below by h0 + k B (only larger values matter)
__device__ __forceinline__ int64_t nx_m(const NxArgs &a, const NxLane &L, int64_t k) {
  const uint32_t *arr = a.devArr + L.off;
  const int64_t thr = L.F0 + (k + 1) * L.TB - L.L;
  int64_t x = L.h0 + k * L.B;
  if (x < L.n && (int64_t)__ldg(arr + x) < thr) {  // gallop, then bisect
    int64_t lo = x, step = 1, hi = x + 1;
    while (hi < L.n && (int64_t)__ldg(arr + hi) < thr) { lo = hi; step <<= 1; hi = x + step; }
    if (hi > L.n) hi = L.n;
    while (hi - lo > 1) {
      const int64_t mid = (lo + hi) >> 1;
      if ((int64_t)__ldg(arr + mid) < thr) lo = mid; else hi = mid;
    }
    x = hi;
  }
  return x - k * L.B;
}

__global__ void __launch_bounds__(256) k_nx_reduce(const __grid_constant__ NxArgs a) {
  const NxLane L = nx_lane(a, blockIdx.x);
  int64_t m = INT64_MIN;
  if (L.on) {
    const int64_t k0 = (int64_t)L.blk * NX_BLK;
    for (int64_t k = k0 + threadIdx.x; k < k0 + NX_BLK && k < L.nb; k += blockDim.x) {
      const int64_t v = nx_m(a, L, k);
      m = v > m ? v : m;
    }
  }
  __shared__ int64_t red[8];
  for (int o = 16; o; o >>= 1) {
    const int64_t v = __shfl_xor_sync(0xffffffffu, m, o);
    m = v > m ? v : m;
  }
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = m;
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int k = 1; k < 8; k++) m = red[k] > m ? red[k] : m;
    a.bmx[blockIdx.x] = m;
  }
}

__global__ void k_nx_prefix(const __grid_constant__ NxArgs a) {  // warp per lane: exclusive block prefix
  const int l = blockIdx.x, lane = threadIdx.x;
  int64_t carry = INT64_MIN;
  for (int64_t b0 = a.loff[l]; b0 < a.loff[l + 1]; b0 += 32) {
    const int64_t b = b0 + lane;
    int64_t v = b < a.loff[l + 1] ? a.bmx[b] : INT64_MIN;
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t u = __shfl_up_sync(0xffffffffu, v, o);
      if (lane >= o && u > v) v = u;
    }
    int64_t ex = __shfl_up_sync(0xffffffffu, v, 1);
    if (lane == 0) ex = INT64_MIN;
    if (b < a.loff[l + 1]) a.bpre[b] = ex > carry ? ex : carry;
    const int64_t tot = __shfl_sync(0xffffffffu, v, 31);
    carry = tot > carry ? tot : carry;
  }
}

// window heads of the block's batches (block-wide inclusive max-scan with the
// lane's prefix), then the validity test; the first invalid batch -> vio
__global__ void __launch_bounds__(256) k_nx_verify(const __grid_constant__ NxArgs a) {
  const NxLane L = nx_lane(a, blockIdx.x);
  if (!L.on) return;
  const int64_t k0 = (int64_t)L.blk * NX_BLK;
  if (k0 >= L.nb) return;
  constexpr int PER = NX_BLK / 256;
  int64_t v[PER];
  int64_t tm = INT64_MIN;
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int64_t k = k0 + threadIdx.x * PER + q;
    v[q] = k < L.nb ? nx_m(a, L, k) : INT64_MIN;
    tm = v[q] > tm ? v[q] : tm;
  }
  // exclusive scan of the thread maxima across the block
  __shared__ int64_t wsum[8];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int64_t x = tm;
  for (int o = 1; o < 32; o <<= 1) {
    const int64_t u = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o && u > x) x = u;
  }
  if (lane == 31) wsum[w] = x;
  int64_t ex = __shfl_up_sync(0xffffffffu, x, 1);
  if (lane == 0) ex = INT64_MIN;
  __syncthreads();
  int64_t carry = a.bpre[blockIdx.x];
  carry = carry > L.h0 ? carry : L.h0;
  for (int k = 0; k < w; k++) carry = wsum[k] > carry ? wsum[k] : carry;
  carry = ex > carry ? ex : carry;
  const uint32_t *arr = a.devArr + L.off;
  int32_t *ik = a.ik + (size_t)blockIdx.x * NX_BLK;
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int64_t k = k0 + threadIdx.x * PER + q;
    carry = v[q] > carry ? v[q] : carry;
    if (k >= L.nb) break;
    ik[threadIdx.x * PER + q] = (int32_t)(k * L.B + carry);  // i_k
  }
  __syncthreads();
  // validity: p_k = i_{k-1} + B (p_0 = h0); a[p_k] <= t_k and a[i_k + B - 1] <= t_k
  for (int j = threadIdx.x; j < NX_BLK; j += blockDim.x) {
    const int64_t k = k0 + j;
    if (k >= L.nb) break;
    const int64_t i = ik[j];
    // i_{k0 - 1} from the lane's exclusive block prefix (another block's)
    const int64_t pb = a.bpre[blockIdx.x] > L.h0 ? a.bpre[blockIdx.x] : L.h0;
    const int64_t pk = k == 0 ? L.h0 : (j > 0 ? (int64_t)ik[j - 1] : (k0 - 1) * L.B + pb) + L.B;
    const int64_t tk = L.F0 + k * L.TB;
    const bool ok = i + L.B <= L.n && pk < L.n && (int64_t)__ldg(arr + pk) <= tk &&
                    (int64_t)__ldg(arr + i + L.B - 1) <= tk;
    if (!ok) {
      int l = 0, hi = a.nl;
      while (hi - l > 1) { const int mid = (l + hi) >> 1; if (__ldg(a.loff + mid) <= (int64_t)blockIdx.x) l = mid; else hi = mid; }
      atomicMin(a.vio + l, (unsigned long long)k);
    }
  }
}

__global__ void __launch_bounds__(256) k_nx_apply(const __grid_constant__ NxArgs a) {
  const NxLane L = nx_lane(a, blockIdx.x);
  if (!L.on) return;
  int l = 0, hi = a.nl;
  while (hi - l > 1) { const int mid = (l + hi) >> 1; if (__ldg(a.loff + mid) <= (int64_t)blockIdx.x) l = mid; else hi = mid; }
  const unsigned long long v = a.vio[l];
  const int64_t kstar = v < (unsigned long long)L.nb ? (int64_t)v : L.nb;  // batches taken
  const int64_t k0 = (int64_t)L.blk * NX_BLK;
  const uint32_t *arr = a.devArr + L.off;
  uint32_t *out = a.latd + (size_t)(L.lane / a.D) * a.NS + L.off;
  const int32_t *ik = a.ik + (size_t)blockIdx.x * NX_BLK;
  for (int j = threadIdx.x; j < NX_BLK; j += blockDim.x) {
    const int64_t k = k0 + j;
    if (k >= kstar) break;
    const int64_t i = ik[j];
    const int64_t pb = a.bpre[blockIdx.x] > L.h0 ? a.bpre[blockIdx.x] : L.h0;
    const int64_t pk = k == 0 ? L.h0 : (j > 0 ? (int64_t)ik[j - 1] : (k0 - 1) * L.B + pb) + L.B;
    for (int64_t q = pk; q < i; q++) out[q] = 0xFFFFFFFFu;  // dropped early
    const int64_t Fk = L.F0 + (k + 1) * L.TB;
    for (int q = 0; q < L.B; q++) out[i + q] = sat_lat(Fk - (int64_t)__ldg(arr + i + q));
  }
  // the second walk starts at batch k* with the device free at F0 + k* T(B)
  const bool mine = (kstar == 0 && L.blk == 0) || (kstar > k0 && kstar <= k0 + NX_BLK);
  if (threadIdx.x == 0 && mine) {  // (lstart itself is the start every block of the lane reads)
    a.nxst[2 * (size_t)l] = kstar == 0 ? L.h0 : (int64_t)ik[kstar - 1 - k0] + L.B;
    a.nxst[2 * (size_t)l + 1] = L.F0 + kstar * L.TB;
  }
}

__global__ void k_nx_commit(const __grid_constant__ NxArgs a) {
  for (int l = blockIdx.x * blockDim.x + threadIdx.x; l < a.nl; l += gridDim.x * blockDim.x)
    if (a.nxst[2 * (size_t)l] >= 0) {
      a.lstart[2 * (size_t)a.lid[l]] = a.nxst[2 * (size_t)l];
      a.lstart[2 * (size_t)a.lid[l] + 1] = a.nxst[2 * (size_t)l + 1];
    }
}

// dropped queries (the sink segment, device index D): latency UINT32_MAX (R7)
__global__ void k_sink(int64_t NS, int S, int D, const int32_t *__restrict__ sc_list, int nsc, const int64_t *devOff,
                       uint32_t *latd, uint64_t *agg) {
  for (int k = blockIdx.y; k < nsc; k += gridDim.y) {
    const int64_t st = devOff[D], n = devOff[D + 1] - st;
    const int s = sc_list[k];
    uint32_t *row = latd + (size_t)s * NS + st;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
      row[j] = 0xFFFFFFFFu;
  }
}

// a13: per scenario, violations (latency > the SLO of the device's family, R6;
// dropped queries included), on-time count and the serving variant's accuracy
// summed over on-time queries (R9), over the device-major rows.  A block takes
// CNT_PER positions of one row and walks the device segments inside them:
// per segment only the on-time count is accumulated (16-byte loads, one
// compare per latency), then violations = length - on-time and the accuracy
// sum = on-time x A.  The sink segment is all violations (nothing to read).
// the counts of the lanes k_chain wrote (and of their duplicates): ccov[s * D
// + d] = the chain lane index holding lane (s, d)'s latencies, -1 otherwise
__global__ void k_chain_agg(int S, int D, int nsc, const int32_t *__restrict__ sc_list, const int32_t *__restrict__ ccov,
                            const unsigned long long *__restrict__ lcnt, const int64_t *__restrict__ devOff,
                            const LaneParam *__restrict__ lp, uint64_t *agg) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nsc * D) return;
  const int s = sc_list[i / D], d = i % D;
  const int li = ccov[(size_t)s * D + d];
  if (li < 0) return;
  const unsigned long long on = lcnt[li], n = (unsigned long long)(devOff[d + 1] - devOff[d]);
  if (n > on) atomicAdd((unsigned long long *)&agg[s], n - on);
  if (on) {
    atomicAdd((unsigned long long *)&agg[S + s], on);
    atomicAdd((unsigned long long *)&agg[2 * S + s], on * lp[(size_t)s * D + d].A);
  }
}

#define CNT_PER 16384
__global__ void __launch_bounds__(256) k_count(int64_t N, int64_t NS, int S, int D, const int32_t *__restrict__ sc_list,
                                               const int64_t *__restrict__ devOff, const LaneParam *__restrict__ lp,
                                               const int32_t *__restrict__ rep, const uint32_t *__restrict__ latd,
                                               uint64_t *agg, const int32_t *__restrict__ ccov) {
  __shared__ unsigned long long red[3][8];
  const int s = sc_list[blockIdx.y];
  const int64_t lo = (int64_t)blockIdx.x * CNT_PER, hi = lo + CNT_PER < N ? lo + CNT_PER : N;
  unsigned long long viol = 0, accs = 0, ont_all = 0;
  for (int d = 0; d <= D; d++) {
    const int64_t a0 = devOff[d] > lo ? devOff[d] : lo, a1 = devOff[d + 1] < hi ? devOff[d + 1] : hi;
    if (a0 >= a1) continue;
    if (d == D) {  // the sink: dropped (R7)
      if (threadIdx.x == 0) viol += (unsigned long long)(a1 - a0);
      continue;
    }
    if (ccov && ccov[(size_t)s * D + d] >= 0) continue;  // counted by k_chain (k_chain_agg)
    const LaneParam q = lp[(size_t)s * D + d];
    const uint32_t *row = latd + (size_t)(rep ? rep[(size_t)s * (D + 1) + d] : s) * NS;  // a duplicate lane: its row's
    const uint32_t L = q.L < 0 ? 0u : q.L > 0xFFFFFFFEll ? 0xFFFFFFFFu : (uint32_t)q.L;
    const bool all_on = q.L >= 0xFFFFFFFFll;  // every latency (<= UINT32_MAX) is on time
    unsigned ont = 0;
    // scalar head up to a 16-byte boundary, uint4 body, scalar tail
    const int64_t a0r = (a0 + 3) & ~(int64_t)3;  // row starts are 16-byte aligned (NS % 32 == 0)
    const int64_t b0 = a0r < a1 ? a0r : a1;
    const int64_t b1 = b0 + ((a1 - b0) & ~(int64_t)3);
    for (int64_t p = a0 + threadIdx.x; p < b0; p += blockDim.x) ont += all_on || row[p] <= L;
    for (int64_t p = b0 + 4 * (int64_t)threadIdx.x; p < b1; p += 4 * (int64_t)blockDim.x) {
      const uint4 v = *(const uint4 *)(row + p);
      ont += all_on ? 4u : (unsigned)(v.x <= L) + (v.y <= L) + (v.z <= L) + (v.w <= L);
    }
    for (int64_t p = b1 + threadIdx.x; p < a1; p += blockDim.x) ont += all_on || row[p] <= L;
    // q.L < 0 cannot happen for a routed device (L = mult * base / 1000 >= 0)
    ont_all += ont;
    accs += (unsigned long long)ont * q.A;
    if (threadIdx.x == 0) viol += (unsigned long long)(a1 - a0);  // minus the on-time ones below
  }
  for (int o = 16; o; o >>= 1) {
    viol += __shfl_xor_sync(0xffffffffu, viol, o);
    ont_all += __shfl_xor_sync(0xffffffffu, ont_all, o);
    accs += __shfl_xor_sync(0xffffffffu, accs, o);
  }
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) { red[0][w] = viol; red[1][w] = ont_all; red[2][w] = accs; }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long v = 0, o2 = 0, a2 = 0;
    for (int k = 0; k < (int)(blockDim.x >> 5); k++) { v += red[0][k]; o2 += red[1][k]; a2 += red[2][k]; }
    v -= o2;
    if (v) atomicAdd((unsigned long long *)&agg[s], v);
    if (o2) atomicAdd((unsigned long long *)&agg[S + s], o2);
    if (a2) atomicAdd((unsigned long long *)&agg[2 * S + s], a2);
  }
}

// duplicate lanes (same policy, Bmax and SLO on a device as an earlier
// scenario): the representative's row segment copied into the duplicate's
// row; blockIdx.y = pair k (dup[k], src[k], device dev[k]).  Both rows share
// the segment's offset, so the body moves in 16-byte words.
__global__ void __launch_bounds__(256) k_dupcopy(int64_t NS, const int32_t *__restrict__ pairs,
                                                 const int64_t *__restrict__ devOff, uint32_t *latd) {
  const int32_t dst = pairs[3 * blockIdx.y], src = pairs[3 * blockIdx.y + 1], d = pairs[3 * blockIdx.y + 2];
  const int64_t a0 = devOff[d], a1 = devOff[d + 1];
  const uint32_t *in = latd + (size_t)src * NS;
  uint32_t *o = latd + (size_t)dst * NS;
  const int64_t b0 = ((a0 + 3) & ~(int64_t)3) < a1 ? ((a0 + 3) & ~(int64_t)3) : a1;
  const int64_t b1 = b0 + ((a1 - b0) & ~(int64_t)3);
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, nt = (int64_t)gridDim.x * blockDim.x;
  if (t < b0 - a0) o[a0 + t] = in[a0 + t];
  if (t < a1 - b1) o[b1 + t] = in[b1 + t];
  for (int64_t p = b0 + 4 * t; p < b1; p += 4 * nt) *(uint4 *)(o + p) = *(const uint4 *)(in + p);
}

// per-query order: out[s][i] = latd[s][inv(i)] (coalesced stores, gathered loads
// that walk ~D sequential streams)
#define UNP_PER 16
__global__ void __launch_bounds__(256) k_unpermute(int64_t N, int64_t NS, int S, const proteus_scenario *__restrict__ sc,
                                                   const uint32_t *__restrict__ inv0, const uint32_t *__restrict__ inv1,
                                                   const uint32_t *__restrict__ latd, uint32_t *out) {
  // one block per chunk of 256 * UNP_PER queries, all scenario rows: every
  // 32-byte sector of a device stream read for a row is used by this block,
  // and the positions stay in registers across the rows
  __shared__ int8_t rt[4096];
  for (int k = threadIdx.x; k < S; k += blockDim.x) rt[k] = (int8_t)sc[k].routing;
  __syncthreads();
  const int64_t i0 = (int64_t)blockIdx.x * (256 * UNP_PER) + threadIdx.x;
  uint32_t p0[UNP_PER], p1[UNP_PER];
#pragma unroll
  for (int k = 0; k < UNP_PER; k++) {
    const int64_t i = i0 + 256 * k;
    p0[k] = (inv0 && i < N) ? inv0[i] : 0;
    p1[k] = (inv1 && i < N) ? inv1[i] : 0;
  }
  for (int s = 0; s < S; s++) {
    const size_t r = (size_t)s * N, rs = (size_t)s * NS;
    if (rt[s] < 0) continue;  // written by the window path
    const bool m1 = rt[s] != 0;
    uint32_t v[UNP_PER];
#pragma unroll
    for (int k = 0; k < UNP_PER; k++)
      if (i0 + 256 * k < N) v[k] = latd[rs + (m1 ? p1[k] : p0[k])];
#pragma unroll
    for (int k = 0; k < UNP_PER; k++)
      if (i0 + 256 * k < N) out[r + i0 + 256 * k] = v[k];
  }
}

// ======================================================= window path ======
// The §5 lanes as three data-parallel passes over GLOBAL WINDOWS of WT tiles
// (TQ = WT * TILE queries; chunk (d, k) = device d's positions of window k,
// [cb[k][d], cb[k+1][d]) from the routing's per-tile bases).  It rests on
// three facts about the rule (readings R1-R5, R4'):
//  (i)   from head h with the device free at F, the decision is the one from
//        an idle device (F <= a_h) iff F <= t_idle(h), the idle decision's
//        dispatch time (the busy run sees the same queue states once t passes
//        F); otherwise the queue is already past the idle decision when the
//        device frees, so the batch leaves at F with min(Bmax, #{j >= h :
//        a_j <= F}) queries ("greedy");
//  (ii)  the idle decision is a binary search: with T non-decreasing, the stop
//        test of queue size q -- the next arrival a_{h+q} comes after
//        W(q) = a_h + L - T(q+1), or the queue's last arrival a_{h+q-1} is at
//        or past it -- is monotone in q; the batch is the first stable count
//        (next arrival strictly later) at or after the first q that stops,
//        leaving at max(a_{h+q-1}, W(q));
//  (iii) whenever a_{h+Bmax-1} <= F, Bmax queries are queued when the device
//        frees and a full batch leaves at F (R4), whatever the branch: a
//        backlogged stretch from (h, F) is m full batches, F + m T(Bmax), iff
//        F >= max_k a_{h+(k+1)Bmax-1} - k T(Bmax) (max-plus).
// A chain entered on the idle branch at head e is a function of e alone, and
// the first head of the true run in chunk k lies in [c0, c0 + Bmax).  So:
//   k_win_tables   block per chunk (d, k), arrivals staged in shared memory,
//                  a warp per scenario lane: per entry offset o < min(Bmax,
//                  chunk) the idle-branch chain to its first head >= c1
//                  (chains reaching a head another chain took on the idle
//                  branch merge into it) and the backlog threshold of (iii);
//                  Bmax = 1: the max-plus form F_out = max(F_in + m T(1),
//                  max_i a_i + (c1 - i) T(1));
//   k_win_compose  warp per lane: the true state across the chunks -- one hop
//                  per chunk when the entry is on the idle branch or the whole
//                  chunk is backlogged, else the rule walked to the chunk end
//                  (32 idle decisions per step, in parallel);
//   k_win_write    block per (scenario, window), arrivals staged in shared
//                  memory: every device's chunk replayed from its true entry
//                  state, latencies into a shared-memory tile in device order,
//                  written ONCE in query order with the per-scenario counts
//                  folded in (a13) -- no device-major latency rows, no
//                  un-permute pass.
// Lanes with Bmax <= WIN_EMAX take this path; a lane whose T is not
// non-decreasing in b (the table need not be, reading C6) makes its idle
// decisions linear (decide()).
#define WIN_EMAX 64
#define WIN_EXT (2 * WIN_EMAX + 64)  // arrivals staged past a chunk's end (look-ahead of its decisions)
#define WIN_WARPS 8

struct WinArgs {
  int S, D, M, bmax, nsc, WT, D1;
  int64_t CHF;                 // > 0: chunks of CHF positions per device (the stitch's), not windows
  int64_t N, nw, ntiles;
  const int32_t *option, *dev_type, *lat, *sc_list;
  const LaneParam *lp;
  const uint8_t *mono;         // [S * D] T non-decreasing over 1..Bmax
  const int64_t *devOff;       // [D + 2]
  const int32_t *dbase;        // [(ntiles + 1)][D + 1] per-tile bases (device-relative)
  const uint32_t *devArr, *inv;
  const uint8_t *tgt;
  const int64_t *recoff;       // [nsc * D] offset of the lane's WinRec rows (E per chunk)
  const int32_t *E;            // [nsc * D] entry offsets per chunk of the lane (min(Bmax, 64); 0 = no lane)
  WinRec *rec;
  WinEntry *ent;               // [nsc * D][nw]
  uint32_t *out;               // [S][N] or null
  uint64_t *agg;               // [3][S]
  unsigned long long *dbg;     // [nsc * D][4] (PROTEUS_REPLAY_DEBUG): idle hops, backlog hops, walks, walked batches
};

__device__ __forceinline__ int64_t win_cb(const WinArgs &a, int64_t k, int d) {
  if (a.CHF > 0) {
    const int64_t n = a.devOff[d + 1] - a.devOff[d];
    return k * a.CHF < n ? k * a.CHF : n;
  }
  const int64_t t = k * a.WT < a.ntiles ? k * a.WT : a.ntiles;
  return a.dbase[t * a.D1 + d];
}

// arrivals of one device: positions [lo, lo + len) from shared memory, the rest from global
struct SArr {
  const uint32_t *s, *g;
  int64_t lo, len;
  __device__ __forceinline__ uint32_t operator()(int64_t j) const {
    const int64_t r = j - lo;
    return (r >= 0 && r < len) ? s[r] : __ldg(g + j);
  }
};

__device__ __forceinline__ int32_t clamp_rel(int64_t v) {  // upward clamp keeps "F <= tdisp" / "F >= R" tests safe
  return v > (int64_t)INT32_MAX ? INT32_MAX : (v < -(int64_t)(1 << 30) ? -(1 << 30) : (int32_t)v);
}

// ---- pass 1: chunk tables, block per chunk (d, k), warp per scenario lane
__global__ void __launch_bounds__(WIN_WARPS * 32) k_win_tables(const __grid_constant__ WinArgs a) {
  extern __shared__ __align__(16) uint8_t win_sm[];  // [TQ + WIN_EXT] arrivals, then [WIN_WARPS][TQ] marks
  __shared__ int32_t sT[WIN_WARPS][WIN_EMAX];
  __shared__ int64_t exF[WIN_WARPS][WIN_EMAX];
  __shared__ int32_t exH[WIN_WARPS][WIN_EMAX], mg[WIN_WARPS][WIN_EMAX];
  __shared__ int64_t tdE[WIN_WARPS][WIN_EMAX];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int d = blockIdx.x % a.D;
  const int64_t k = blockIdx.x / a.D;
  const int64_t c0 = win_cb(a, k, d), c1 = win_cb(a, k + 1, d);
  if (c1 <= c0) return;
  const int64_t TQ = a.CHF > 0 ? a.CHF : (int64_t)a.WT * TILE;
  const int64_t off = a.devOff[d], n = a.devOff[d + 1] - off;
  uint32_t *sarr = (uint32_t *)win_sm;
  const int64_t slen = (c1 + WIN_EXT < n ? c1 + WIN_EXT : n) - c0;
  for (int64_t i = threadIdx.x; i < slen; i += blockDim.x) sarr[i] = __ldg(a.devArr + off + c0 + i);
  __syncthreads();
  SArr A{sarr, a.devArr + off, c0, slen};
  volatile uint8_t *vis = win_sm + (TQ + WIN_EXT) * 4 + (size_t)w * TQ;
  const int32_t *Tg = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
  const int64_t len = c1 - c0;  // <= TQ
  const int64_t a0 = A(c0);
  for (int si = w; si < a.nsc; si += WIN_WARPS) {
    const int li = si * a.D + d;
    const int E = a.E[li];
    if (E <= 0) continue;
    const int s = a.sc_list[si];
    const LaneParam p = a.lp[(size_t)s * a.D + d];
    WinRec *R = a.rec + a.recoff[li] + k * (int64_t)E;
    if (p.Bmax == 1) {  // max-plus form: R = max_i a_i + (c1 - i) T(1)
      const int64_t T1 = Tg[0];
      int64_t m = INT64_MIN;
      for (int64_t i = c0 + lane; i < c1; i += 32) {
        const int64_t v = (int64_t)A(i) + (c1 - i) * T1;
        m = v > m ? v : m;
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        const int64_t v = __shfl_xor_sync(0xffffffffu, m, o);
        m = v > m ? v : m;
      }
      if (lane == 0) { WinRec r; r.Fx = m; r.tdisp = 0; r.R = 0; r.hx = (int32_t)len; r.pad = 0; R[0] = r; }
      continue;
    }
    const int Bm = p.Bmax;
    const bool mono = a.mono[(size_t)s * a.D + d] != 0;
    __syncwarp();  // the previous lane's reads of sT / vis are done
    for (int b = lane; b < Bm; b += 32) sT[w][b] = Tg[b];
    for (int64_t i = lane; i < len; i += 32) vis[i] = 0xFF;
    __syncwarp();
    const int32_t *T = sT[w];
    const int Ee = (int)(E < len ? E : len);
    const int64_t TB = T[Bm - 1];
    for (int r0 = 0; r0 < Ee; r0 += 32) {
      const int o = r0 + lane;
      bool live = o < Ee;
      int64_t h = c0 + o, F = 0;
      int merged = -1;
      bool first = true;
      while (__any_sync(0xffffffffu, live)) {
        // lockstep over the warp: decide, read the marks, __syncwarp, mark (one
        // lane per head), __syncwarp -- no unordered shared-memory access
        bool idle = false;
        int b = 0;
        int64_t t = 0;
        if (live && h >= c1) live = false;
        if (live) {
          b = idle_decide(A, n, h, Bm, p.L, T, mono, &t);
          if (first) { tdE[w][o] = t; first = false; F = t; }  // the entry: idle branch by construction
          idle = F <= t;  // idle branch (fact (i)): a function of h alone
        }
        const uint8_t mk = idle ? vis[h - c0] : (uint8_t)0xFF;
        __syncwarp();
        // another chain took h on the idle branch: the same future from here
        if (idle && mk != 0xFF) { merged = mk; live = false; idle = false; }
        const unsigned same = __match_any_sync(0xffffffffu, idle ? h : -1 - (int64_t)lane);
        if (idle && lane == __ffs(same) - 1) vis[h - c0] = (uint8_t)o;
        __syncwarp();
        if (live) {
          if (idle) {
            F = t + T[b - 1];
          } else {  // greedy
            b = count_upto(A, n, h, Bm, F);
            F = F + T[b - 1];
          }
          h += b;
        }
      }
      if (o < Ee) {
        exH[w][o] = (int32_t)h; exF[w][o] = F; mg[w][o] = merged;
        // backlog threshold (fact (iii)) from the entry head: full batches to the first head >= c1
        int64_t Rb = INT64_MIN;
        bool ok = true;
        int64_t kk = 0;
        for (int64_t hh = c0 + o; hh < c1; hh += Bm, kk++) {
          if (hh + Bm - 1 >= n) { ok = false; break; }  // the trace ends: no full batch
          const int64_t v = (int64_t)A(hh + Bm - 1) - kk * TB;
          Rb = v > Rb ? v : Rb;
        }
        tdE[w][o] = tdE[w][o] - a0;
        exF[w][o] = F;
        R[o].R = ok ? clamp_rel(Rb - a0) : INT32_MAX;  // rest of the record below
      }
      __syncwarp();
    }
    // resolve merges (pointers strictly increase the stopping position: no cycles)
    for (int o = lane; o < Ee; o += 32) {
      int r = o;
      while (mg[w][r] >= 0) r = mg[w][r];
      R[o].Fx = exF[w][r];
      R[o].hx = (int32_t)(exH[w][r] - c0);
      R[o].tdisp = clamp_rel(tdE[w][o]);
      R[o].pad = 0;
    }
    __syncwarp();
  }
}

// ---- pass 2: the true state across the chunks, one warp per lane
__global__ void __launch_bounds__(128) k_win_compose(const __grid_constant__ WinArgs a) {
  __shared__ int32_t sT[4][WIN_EMAX];
  __shared__ uint32_t sW[4][32 + WIN_EXT];  // a walk's arrivals
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int li = blockIdx.x * 4 + w;
  if (li >= a.nsc * a.D) return;
  const int d = li % a.D, s = a.sc_list[li / a.D];
  const int E = a.E[li];
  if (E <= 0) return;
  const LaneParam p = a.lp[(size_t)s * a.D + d];
  const int Bm = p.Bmax;
  const int64_t off = a.devOff[d], n = a.devOff[d + 1] - off;
  const uint32_t *G = a.devArr + off;
  const bool mono = a.mono[(size_t)s * a.D + d] != 0;
  const int32_t *Tg = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
  for (int b = lane; b < Bm; b += 32) sT[w][b] = Tg[b];
  __syncwarp();
  const int32_t *T = sT[w];
  const int64_t TB = T[Bm - 1];
  const WinRec *R = a.rec + a.recoff[li];
  WinEntry *ent = a.ent + (int64_t)li * a.nw;
  unsigned long long n_idle = 0, n_back = 0, n_walk = 0, n_wb = 0;
  int64_t h = 0, F = 0;  // R13: idle at t = 0
  // chunk bounds and first arrivals 32 chunks at a time; the next chunk's records prefetched
  int64_t cb0 = 0, cb1 = 0, ca0 = 0;
  WinRec r0 = {}, r1 = {}, q0 = {}, q1 = {};
  auto load_row = [&](int64_t k, WinRec &x0, WinRec &x1) {
    if (k < a.nw) {
      if (lane < E) x0 = R[k * E + lane];
      if (lane + 32 < E) x1 = R[k * E + lane + 32];
    }
  };
  load_row(0, r0, r1);
  for (int64_t k = 0; k < a.nw; k++) {
    const int kk = (int)(k & 31);
    if (kk == 0) {
      cb0 = k + lane < a.nw ? win_cb(a, k + lane, d) : 0;
      cb1 = k + lane < a.nw ? win_cb(a, k + lane + 1, d) : 0;
      ca0 = (k + lane < a.nw && cb0 < cb1) ? (int64_t)__ldg(G + cb0) : 0;
    }
    load_row(k + 1, q0, q1);
    const int64_t c0 = __shfl_sync(0xffffffffu, cb0, kk), c1 = __shfl_sync(0xffffffffu, cb1, kk);
    const int64_t a0 = __shfl_sync(0xffffffffu, ca0, kk);
    if (lane == 0) { WinEntry e; e.F = F; e.h = (int32_t)h; e.pad = 0; ent[k] = e; }
    if (c1 > c0 && h < c1) {
      if (Bm == 1) {
        const int64_t Rk = __shfl_sync(0xffffffffu, r0.Fx, 0);
        const int64_t v = F + (c1 - h) * (int64_t)T[0];
        F = v > Rk ? v : Rk;
        h = c1;
      } else {
        const int o = (int)(h - c0);  // < min(Bmax, chunk): the first head >= c0
        const int src = o & 31;
        const int64_t tdisp = a0 + __shfl_sync(0xffffffffu, o < 32 ? r0.tdisp : r1.tdisp, src);
        const int32_t Rr = __shfl_sync(0xffffffffu, o < 32 ? r0.R : r1.R, src);
        const int64_t Fx = __shfl_sync(0xffffffffu, o < 32 ? r0.Fx : r1.Fx, src);
        const int32_t hx = __shfl_sync(0xffffffffu, o < 32 ? r0.hx : r1.hx, src);
        if (F <= tdisp) {  // idle branch at the entry: the chain of the table
          h = c0 + hx;
          F = Fx;
          n_idle++;
        } else if (Rr != INT32_MAX && F >= a0 + Rr) {  // backlogged through the chunk (iii)
          const int64_t m = (c1 - h + Bm - 1) / Bm;
          h += m * Bm;
          F += m * TB;
          n_back++;
        } else {  // the rule itself to the chunk end: 32 idle decisions per step, in parallel
          n_walk++;
          uint32_t *sw = sW[w];
          while (h < c1) {
            const int64_t base = h;
            const int64_t wl = (n - base < 32 + WIN_EXT) ? n - base : 32 + WIN_EXT;
            for (int i = lane; i < wl; i += 32) sw[i] = __ldg(G + base + i);
            __syncwarp();
            SArr A{sw, G, base, wl};
            int64_t tl = 0;
            int bl = 0;
            if (base + lane < c1) bl = idle_decide(A, n, base + lane, Bm, p.L, T, mono, &tl);
            while (h < c1 && h < base + 32) {
              const int i = (int)(h - base);
              int b = __shfl_sync(0xffffffffu, bl, i);
              int64_t t = __shfl_sync(0xffffffffu, tl, i);
              if (F > t) {  // greedy (fact (i))
                b = count_upto(A, n, h, Bm, F);
                t = F;
              }
              F = t + T[b - 1];
              h += b;
              n_wb++;
            }
            __syncwarp();
          }
        }
      }
    }
    r0 = q0;
    r1 = q1;
  }
  if (a.dbg && lane == 0) {
    atomicAdd(a.dbg + 4 * li, n_idle);
    atomicAdd(a.dbg + 4 * li + 1, n_back);
    atomicAdd(a.dbg + 4 * li + 2, n_walk);
    atomicAdd(a.dbg + 4 * li + 3, n_wb);
  }
}

// ---- pass 3: latencies in query order, block per (scenario, window)
#define WIN_THREADS 256
__global__ void __launch_bounds__(WIN_THREADS) k_win_write(const __grid_constant__ WinArgs a) {
  // dynamic: [TQ] latencies (device-major: wbase[d] + position - c0), then the
  // arrivals of every device's chunk plus WIN_EXT look-ahead (abase[d] + position - c0)
  extern __shared__ __align__(16) uint32_t wsm[];
  __shared__ int32_t wbase[PX_MAXD + 2], abase[PX_MAXD + 2], wc0[PX_MAXD + 1], wlen[PX_MAXD + 1],
      walen[PX_MAXD + 1], wown[PX_MAXD + 1];
  __shared__ int64_t wL[PX_MAXD + 1];
  __shared__ uint32_t wA[PX_MAXD + 1];
  __shared__ int32_t sT[WIN_THREADS / 32][WIN_EMAX];
  __shared__ unsigned long long red[3][WIN_THREADS / 32];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31, nwarps = WIN_THREADS / 32;
  const int si = blockIdx.x;  // scenario list position (fastest: the window's inputs are shared in L2)
  const int64_t k = blockIdx.y;
  const int s = a.sc_list[si];
  const int D = a.D;
  const int64_t TQ = (int64_t)a.WT * TILE;
  uint32_t *slat = wsm, *sarr = wsm + TQ;
  if (threadIdx.x < D) {
    const int d = threadIdx.x;
    const int64_t c0 = win_cb(a, k, d), c1 = win_cb(a, k + 1, d);
    const int64_t n = a.devOff[d + 1] - a.devOff[d];
    wc0[d] = (int32_t)c0;
    wlen[d] = (int32_t)(c1 - c0);
    walen[d] = (int32_t)((c1 + WIN_EXT < n ? c1 + WIN_EXT : n) - c0);
    const LaneParam q = a.lp[(size_t)s * D + d];
    wL[d] = q.L;
    wA[d] = q.A;
  }
  __syncthreads();
  if (threadIdx.x == 0) {  // tile layouts; devices to warps, largest chunk first (LPT)
    int acc = 0, acc2 = 0;
    for (int d = 0; d < D; d++) { wbase[d] = acc; acc += wlen[d]; abase[d] = acc2; acc2 += walen[d]; }
    wbase[D] = acc;
    abase[D] = acc2;
    unsigned long long load[WIN_THREADS / 32];
    for (int x = 0; x < nwarps; x++) load[x] = 0;
    unsigned long long used = 0;
    for (int it = 0; it < D; it++) {
      int bd = -1;
      for (int d = 0; d < D; d++)
        if (!((used >> d) & 1ull) && (bd < 0 || wlen[d] > wlen[bd])) bd = d;
      used |= 1ull << bd;
      int bw = 0;
      for (int x = 1; x < nwarps; x++) if (load[x] < load[bw]) bw = x;
      wown[bd] = bw;
      load[bw] += (unsigned long long)wlen[bd] + 64;
    }
  }
  __syncthreads();
  for (int d = 0; d < D; d++) {  // stage the arrivals (block-wide, coalesced)
    const uint32_t *g = a.devArr + a.devOff[d] + wc0[d];
    for (int i = threadIdx.x; i < walen[d]; i += WIN_THREADS) sarr[abase[d] + i] = __ldg(g + i);
  }
  __syncthreads();
  for (int d = 0; d < D; d++) {
    if (wown[d] != w || wlen[d] == 0) continue;
    const int li = si * D + d;
    const LaneParam p = a.lp[(size_t)s * D + d];
    const int64_t off = a.devOff[d], n = a.devOff[d + 1] - off;
    const int64_t c0 = wc0[d], c1 = c0 + wlen[d];
    uint32_t *lt = slat + wbase[d];  // lt[position - c0]
    SArr A{sarr + abase[d], a.devArr + off, c0, walen[d]};
    if (p.Bmax < 1) {  // never routed to (kept for safety): dropped
      for (int64_t j = c0 + lane; j < c1; j += 32) lt[j - c0] = 0xFFFFFFFFu;
      continue;
    }
    const int Bm = p.Bmax;
    const int32_t *Tg = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
    __syncwarp();  // the previous device's reads of sT are done
    for (int b = lane; b < Bm; b += 32) sT[w][b] = Tg[b];
    __syncwarp();
    const int32_t *T = sT[w];
    const bool mono = a.mono[(size_t)s * D + d] != 0;
    const WinEntry e = a.ent[(int64_t)li * a.nw + k];
    int64_t h = e.h, F = e.F;
    // positions before the first head: the batch that crossed c0 (finish F)
    const int64_t hs = h < c1 ? h : c1;
    for (int64_t j = c0 + lane; j < hs; j += 32) lt[j - c0] = sat_lat(F - (int64_t)A(j));
    if (Bm == 1) {  // F_i = max(F_{i-1}, a_i) + T(1): a prefix maximum, 32 positions per step
      const int64_t T1 = T[0];
      for (int64_t b0 = h; b0 < c1; b0 += 32) {
        const int64_t j = b0 + lane;
        int64_t x = j < c1 ? (int64_t)A(j) - (j - b0) * T1 : INT64_MIN;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int64_t y = __shfl_up_sync(0xffffffffu, x, o);
          if (lane >= o) x = y > x ? y : x;
        }
        const int64_t g = F > x ? F : x;
        const int64_t Fj = g + (j - b0 + 1) * T1;
        if (j < c1) lt[j - c0] = sat_lat(Fj - (int64_t)A(j));
        F = __shfl_sync(0xffffffffu, Fj, (int)((c1 - b0 < 32 ? c1 - b0 : 32) - 1));
      }
      continue;
    }
    while (h < c1) {
      // the idle decisions of the 32 positions from h, in parallel
      const int64_t base = h;
      int64_t tl = 0;
      int bl = 0;
      if (base + lane < c1) bl = idle_decide(A, n, base + lane, Bm, p.L, T, mono, &tl);
      while (h < c1 && h < base + 32) {
        const int i = (int)(h - base);
        int b = __shfl_sync(0xffffffffu, bl, i);
        int64_t t = __shfl_sync(0xffffffffu, tl, i);
        if (F > t) {  // greedy (fact (i)): leave at F with what has arrived by then
          int c = 0;
          for (int r = 0; r < Bm; r += 32) {
            const int64_t j = h + r + lane;
            const bool le = r + lane < Bm && j < n && (int64_t)A(j) <= F;
            c += __popc(__ballot_sync(0xffffffffu, le));
          }
          b = c;
          t = F;
        }
        const int64_t Fn = t + T[b - 1];
        for (int r = lane; r < b; r += 32)
          if (h + r < c1) lt[h + r - c0] = sat_lat(Fn - (int64_t)A(h + r));
        F = Fn;
        h += b;
      }
    }
  }
  __syncthreads();
  // query order: out[s][i] for the window's queries; counts (a13)
  const int64_t i0 = k * TQ;
  const int64_t i1 = i0 + TQ < a.N ? i0 + TQ : a.N;
  unsigned long long viol = 0, ont = 0, accs = 0;
  uint32_t *orow = a.out ? a.out + (size_t)s * a.N : nullptr;
  for (int64_t i = i0 + threadIdx.x; i < i1; i += WIN_THREADS) {
    const int d = a.tgt[i];
    uint32_t l;
    if (d >= D) {
      l = 0xFFFFFFFFu;  // the sink: dropped (R7)
      viol++;
    } else {
      const int64_t pos = (int64_t)a.inv[i] - a.devOff[d];
      l = slat[wbase[d] + (pos - wc0[d])];
      if ((int64_t)l > wL[d]) viol++;  // R6
      else { ont++; accs += wA[d]; }   // R9
    }
    if (orow) orow[i] = l;
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    viol += __shfl_xor_sync(0xffffffffu, viol, o);
    ont += __shfl_xor_sync(0xffffffffu, ont, o);
    accs += __shfl_xor_sync(0xffffffffu, accs, o);
  }
  if (lane == 0) { red[0][w] = viol; red[1][w] = ont; red[2][w] = accs; }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long v = 0, o2 = 0, a2 = 0;
    for (int x = 0; x < nwarps; x++) { v += red[0][x]; o2 += red[1][x]; a2 += red[2][x]; }
    if (v) atomicAdd((unsigned long long *)&a.agg[s], v);
    if (o2) atomicAdd((unsigned long long *)&a.agg[a.S + s], o2);
    if (a2) atomicAdd((unsigned long long *)&a.agg[2 * a.S + s], a2);
  }
}

// a13 + un-permute in one pass (the chunk-run / stitch path): per query i and
// scenario s, the latency from the device-major rows (gathered through inv;
// the sink: dropped, R7) written once in query order, and the per-scenario
// violations (R6), on-time count and accuracy sum (R9) of the same values --
// each latency read once (k_count + k_unpermute read every row twice).
#define FIN_PER 16
__global__ void __launch_bounds__(256) k_finish(int64_t N, int64_t NS, int S, int D,
                                                const proteus_scenario *__restrict__ sc,
                                                const uint32_t *__restrict__ inv0, const uint32_t *__restrict__ inv1,
                                                const uint8_t *__restrict__ tgt0, const uint8_t *__restrict__ tgt1,
                                                const LaneParam *__restrict__ lp, const uint32_t *__restrict__ latd,
                                                uint32_t *out, uint64_t *agg) {
  __shared__ unsigned long long red[3][8];
  const int64_t i0 = (int64_t)blockIdx.x * (256 * FIN_PER) + threadIdx.x;
  uint32_t p0[FIN_PER], p1[FIN_PER];
  uint8_t g0[FIN_PER], g1[FIN_PER];
#pragma unroll
  for (int k = 0; k < FIN_PER; k++) {
    const int64_t i = i0 + 256 * k;
    const bool v = i < N;
    p0[k] = (inv0 && v) ? inv0[i] : 0;
    p1[k] = (inv1 && v) ? inv1[i] : 0;
    g0[k] = (tgt0 && v) ? tgt0[i] : 0;
    g1[k] = (tgt1 && v) ? tgt1[i] : 0;
  }
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int s = 0; s < S; s++) {
    const int rt = sc[s].routing;
    if (rt < 0) continue;  // written by the window path
    const size_t rs = (size_t)s * NS;
    const LaneParam *lps = lp + (size_t)s * D;
    unsigned long long viol = 0, ont = 0, accs = 0;
    uint32_t v[FIN_PER];
#pragma unroll
    for (int k = 0; k < FIN_PER; k++) {
      const int d = rt ? g1[k] : g0[k];
      v[k] = 0xFFFFFFFFu;
      if (i0 + 256 * k < N && d < D) v[k] = latd[rs + (rt ? p1[k] : p0[k])];
    }
#pragma unroll
    for (int k = 0; k < FIN_PER; k++) {
      if (i0 + 256 * k >= N) continue;
      const int d = rt ? g1[k] : g0[k];
      if (d >= D) { viol++; }
      else {
        const LaneParam q = lps[d];
        if ((int64_t)v[k] > q.L) viol++;
        else { ont++; accs += q.A; }
      }
      if (out) out[(size_t)s * N + i0 + 256 * k] = v[k];
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
      viol += __shfl_xor_sync(0xffffffffu, viol, o);
      ont += __shfl_xor_sync(0xffffffffu, ont, o);
      accs += __shfl_xor_sync(0xffffffffu, accs, o);
    }
    if (lane == 0) { red[0][w] = viol; red[1][w] = ont; red[2][w] = accs; }
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned long long a0 = 0, a1 = 0, a2 = 0;
      for (int x = 0; x < 8; x++) { a0 += red[0][x]; a1 += red[1][x]; a2 += red[2][x]; }
      if (a0) atomicAdd((unsigned long long *)&agg[s], a0);
      if (a1) atomicAdd((unsigned long long *)&agg[S + s], a1);
      if (a2) atomicAdd((unsigned long long *)&agg[2 * S + s], a2);
    }
    __syncthreads();
  }
}

// ---- chain path: the §5 lanes as a chained scan over chunk maps
// For a lane with T(b) non-decreasing (facts (i)-(ii) of the window path), the
// decision at head h with the device free at F is the idle decision
// (b_i(h), t_i(h)) when F <= t_i(h), else the greedy batch min(Bmax, queued at
// F) at F.  The idle decision depends on h only, so a chunk of C heads is
// tabulated in parallel (one binary search per head), and so is, for every
// head i, the rest of the run after an idle-branch decision at i, up to the end
// of i's segment (SEG heads): the next head at which the run decides on the
// idle branch again (the greedy batches between are a function of i too), or
// the state (first head past the segment, free time) in which it leaves the
// segment.  Every head's last idle-branch head inside its segment follows by a
// backward scan of the segment (thread per segment).  Units (lane, chunk) are
// taken in chunk-major ticket order by persistent blocks; each builds its
// tables, then warp 0 waits for the previous chunk's exit (a single 64-bit
// word: ((F + 1) << 8) | (head - chunk start)), walks the chunk from the true
// entry one segment per hop (greedy stretches in between, full batches 32 per
// ballot), recording the true state at the first batch head of every segment,
// and publishes the chunk's exit; then one thread per segment writes the
// segment's latencies from its true state (device-major rows, like the chunk
// runs).  The serial dependency per lane is one hop per segment.
#ifndef CHAIN_THREADS
#define CHAIN_THREADS 256
#endif
#define CHAIN_WARPS (CHAIN_THREADS / 32)
#define CHAIN_CMAX 8192   // largest chunk (heads are int16 in the tables)
#define CHAIN_SEGMIN 16   // smallest segment
#ifndef CHAIN_MINB
#define CHAIN_MINB 6      // blocks per SM (40 registers; 8 blocks at 32 registers measured slower)
#endif
#ifdef PX_CHAIN_DEBUG  // per-phase cycle totals of k_chain (thread 0), printed by the host
#define CX_T(k) do { if (threadIdx.x == 0) { const long long t_ = clock64(); atomicAdd(a.dbg + (k), (unsigned long long)(t_ - cx_t)); cx_t = t_; } } while (0)
#else
#define CX_T(k) do { } while (0)
#endif
struct ChainArgs {
  int D, M, bmax, nl, C;
  int K;                       // greedy batches a head's chain follows in the tables
  int SEG;                     // heads per segment (writer thread, link hop)
  int64_t NS, maxch, nunits;   // tickets
  const unsigned long long *units;  // [nunits] (lane index << 32) | chunk, in ticket order (host-built)
  const int32_t *lid;          // [nl] lane = s * D + d (device-major: consecutive tickets share arrivals)
  const int32_t *nch;          // [nl] chunks of the lane
  const uint8_t *cmode;        // [nl] 0: chunk tables, 1: near overload (full-batch walks, no tables)
  const LaneParam *lp;
  const int32_t *option, *dev_type, *lat;
  const int64_t *devOff;
  const uint32_t *devArr;
  uint32_t *latd;
  unsigned long long *ex;      // [nl][maxch] packed chunk exits, 0 = not yet published
  unsigned long long *counter; // ticket counter
  unsigned *watchdog;          // set when a wait for a previous chunk's exit times out
  unsigned long long *dbg;     // PX_CHAIN_DEBUG: [16] phase cycles, units, batches, hops
  unsigned long long *lcnt;    // [nl] on-time latencies per lane (the counts folded into the writers), or null
  // EP (k_chain<true>, the closed loop): epochs of epoch_us, per (scenario, epoch, device) {Bmax, L, T row offset}
  int E;
  int64_t epoch_us;
  const int32_t *epP;             // [S][E][D][4] {Bmax, L, T row offset, accuracy of the epoch's variant}
  uint64_t *agg;                  // EP: [3][S] the counts, folded into the writers (the sink: k_ep_count)
  int S;
  const int32_t *segBase, *cntED; // [E][D] segment of (epoch, device) in the device's array
};

struct ShArr {  // arrivals of a chunk in shared memory, from its first head
  const uint32_t *p;
  __device__ __forceinline__ uint32_t operator()(int64_t j) const { return p[j]; }
};

// per routing mode: lid [nl] i32, nch [nl] i32, cmode [nl] u8, ticket + watchdog, exits [nl][maxch] u64
static size_t chain_ctroff(size_t nl) { return (nl * 9 + 15) & ~(size_t)15; }
static size_t chain_exoff(size_t nl) { return chain_ctroff(nl) + 16; }
static size_t chain_smem(int C, int bmax, int SEG, bool ep = false) {
  const size_t E = (size_t)C + bmax + 2;
  const size_t nseg = ((size_t)C + SEG - 1) / SEG;
  return nseg * 8 /* sSegF */ + (size_t)bmax * 4 /* sT */ + E * 4 /* sA */ +
         (size_t)C * 4 /* sTi */ + nseg * 4 /* sSegH */ + (size_t)C * 8 /* sNx, sNc, sJ, sJc */ +
         (size_t)C /* sB */ + 64 + (ep ? (size_t)C * 4 + 16 : 0) /* sEp, sEnd */;
}

template <bool EP>  // EP: the closed loop's lanes (§8(f4)): rule parameters and queue ends per epoch segment
__global__ void __launch_bounds__(CHAIN_THREADS, CHAIN_MINB) k_chain(const __grid_constant__ ChainArgs a) {
  extern __shared__ __align__(16) unsigned char csm[];
  const int C = a.C, SEG = a.SEG;
  const int NSEG = (C + SEG - 1) / SEG;
  int64_t *sSegF = (int64_t *)csm;                  // [NSEG] true free time at the first batch head of a segment
  int32_t *sT = (int32_t *)(sSegF + NSEG);          // [bmax] T(b) at b - 1
  uint32_t *sA = (uint32_t *)(sT + a.bmax);         // [C + bmax + 2] arrivals from the chunk start
  int32_t *sTi = (int32_t *)(sA + C + a.bmax + 2);  // [C] t_i(h) - a_h
  int *sSegH = (int *)(sTi + C);                    // [NSEG] ... and that head (-1: not recorded yet)
  int16_t *sNx = (int16_t *)(sSegH + NSEG);              // [C] next idle-branch head in the segment, -1: leaves, -2: left to
                                                    // the walk, -3: leaves onto an idle-branch head in the chunk
  int16_t *sNc = sNx + C;                           // [C] next idle-branch head in the chunk, -1: leaves, -2: left to the walk
  int16_t *sJ = sNc + C;                            // [C] last idle-branch head of h's run in its segment
  int16_t *sJc = sJ + C;                            // [C] last idle-branch head of h's run in the chunk
  uint8_t *sB = (uint8_t *)(sJc + C);               // [C] b_i(h)
  uint16_t *sEp = (uint16_t *)(sB + ((C + 15) & ~15));  // EP: [C] epoch of head h
  int16_t *sEnd = (int16_t *)(sEp + C);             // EP: [C] end of h's epoch segment (chunk-relative, capped)
  __shared__ unsigned long long sTicket;
  const int tid = threadIdx.x;
  for (;;) {
    if (tid == 0) sTicket = atomicAdd(a.counter, 1ull);
    __syncthreads();
    const unsigned long long tk = sTicket;
    if (tk >= (unsigned long long)a.nunits) return;
    const unsigned long long u = a.units[tk];
    const int li = (int)(u >> 32);
    const int64_t c = (int64_t)(u & 0xffffffffull);
    if (c < a.nch[li]) {
#ifdef PX_CHAIN_DEBUG
      long long cx_t = clock64();
#endif
      const int lane_id = a.lid[li];
      const int s = lane_id / a.D, d = lane_id % a.D;
      LaneParam p = {0, 0, 0, 0, 0, 0};
      if (!EP) p = a.lp[lane_id];
      const int Bm = p.Bmax;
      const int64_t off = a.devOff[d], nloc0 = a.devOff[d + 1] - off;
      const int64_t c0 = c * C;
      const int64_t nloc = nloc0 - c0;  // heads from the chunk start to the device's end
      const int Cn = (int)(nloc < C ? nloc : C);
      const int Bst = EP ? a.bmax : Bm;  // look-ahead of a decision
      const int na = (int)(nloc < (int64_t)Cn + Bst + 1 ? nloc : (int64_t)Cn + Bst + 1);
      const int nseg = (Cn + SEG - 1) / SEG;
      if (!EP) {
        const int32_t *Tg = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
        for (int k = tid; k < Bm; k += CHAIN_THREADS) sT[k] = Tg[k];
      }
      const uint32_t *src = a.devArr + off + c0;
      for (int j = tid; j < na; j += CHAIN_THREADS) sA[j] = src[j];
      for (int sg = tid; sg < nseg; sg += CHAIN_THREADS) sSegH[sg] = -1;  // not recorded yet
      if (EP) {  // F1: query j belongs to epoch a_j / epoch_us; its segment ends where the epoch's queries end
        __syncthreads();
        for (int i = tid; i < Cn; i += CHAIN_THREADS) {
          const int e = (int)((int64_t)sA[i] / a.epoch_us);
          sEp[i] = (uint16_t)e;
          const int64_t end = (int64_t)a.segBase[(size_t)e * a.D + d] + a.cntED[(size_t)e * a.D + d] - c0;
          sEnd[i] = (int16_t)(end < (int64_t)Cn + Bst + 1 ? end : (int64_t)Cn + Bst + 1);
        }
      }
      __syncthreads();
      CX_T(0);
      const ShArr A{sA};
      const int w = tid >> 5, lane = tid & 31;
      const int64_t TB = EP ? 0 : sT[Bm - 1];
      // the rule's parameters for a decision at head h: Bmax, SLO, T(b) row, queue end
      auto epp = [&](int h) -> const int32_t * { return a.epP + ((size_t)(s * a.E + sEp[h]) * a.D + d) * 4; };
      auto HB = [&](int h) -> int { if constexpr (EP) return epp(h)[0]; else return Bm; };
      auto HL = [&](int h) -> int64_t { if constexpr (EP) return epp(h)[1]; else return p.L; };
      auto HT = [&](int h) -> const int32_t * { if constexpr (EP) return a.lat + epp(h)[2]; else return sT; };
      auto HN = [&](int h) -> int64_t { if constexpr (EP) return sEnd[h]; else return nloc; };
      uint32_t *out = a.latd + (size_t)s * a.NS + off + c0;
      // full-batch stretch at (hh, FF): batch i (head hh + i Bm) leaves full at
      // FF + i T(Bmax) while its last query has arrived by then -- with Bmax
      // queued when the device frees, the decision is Bmax at that instant
      // whether or not the idle run would have dispatched earlier.  Returns
      // the number of such batches whose heads lie below lim (32 per ballot).
      auto stretch = [&](int hh, int64_t FF, int lim) -> int {
        const int B_ = HB(hh);
        const int64_t TB_ = HT(hh)[B_ - 1], N_ = HN(hh);
        if (N_ < lim) lim = (int)N_;  // EP: a batch holds one epoch's queries (F3)
        int k = 0;
        for (;;) {
          const int i = k + lane;
          const int64_t last = (int64_t)hh + (int64_t)(i + 1) * B_ - 1;
          const bool full = (int64_t)hh + (int64_t)i * B_ < lim && last < N_ &&
                            (int64_t)sA[last] <= FF + (int64_t)i * TB_;
          const unsigned bal = __ballot_sync(0xffffffffu, !full);
          if (bal) return k + __ffs(bal) - 1;
          k += 32;
        }
      };
      // latencies of the batch [hh, hh + b) finishing at fin, positions < lim
      unsigned long long ont = 0;  // on-time latencies this thread wrote (R6: latency <= SLO)
      unsigned long long nwr = 0, accs = 0;  // EP: latencies written, accuracy sum of the on-time ones (R9)
      auto put = [&](int hh, int b, int64_t fin, int lim) {
        const int e = hh + b < lim ? hh + b : lim;
        for (int j = hh + lane; j < e; j += 32) {
          const uint32_t l = sat_lat(fin - (int64_t)sA[j]);
          out[j] = l;
          ont += (int64_t)l <= p.L;
        }
      };
      // the chunk's entry (warp 0): R13 for the first chunk, else the previous
      // chunk's exit, a single 64-bit word ((F + 1) << 8 | head - chunk start)
      auto entry = [&](int &h, int64_t &F) {
        if (c == 0) {
          h = 0;
          F = 0;  // R13: the device starts idle
          return;
        }
        unsigned long long v = 0;
        if (lane == 0) {
          const unsigned long long *pe = a.ex + (size_t)li * a.maxch + (c - 1);
          for (uint32_t it = 0;; it++) {
            asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(pe) : "memory");
            if (v) break;
            if (it > (1u << 24)) { atomicExch(a.watchdog, 1u); v = 1ull << 8; break; }
            __nanosleep(32);
          }
        }
        v = __shfl_sync(0xffffffffu, v, 0);
        h = (int)(v & 255u);
        F = (int64_t)(v >> 8) - 1;
      };
      auto publish = [&](int hx, int64_t Fx) {
        if (lane == 0) {
          const unsigned long long v = ((unsigned long long)(Fx + 1) << 8) | (unsigned long long)hx;
          asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(a.ex + (size_t)li * a.maxch + c), "l"(v) : "memory");
        }
      };
      if (!EP && a.cmode[li]) {
        // a lane near overload: mostly full batches back to back, taken 32 per
        // ballot; the other decisions directly (idle decision by binary
        // search, else the greedy batch).  No tables: warp 0 walks the chunk
        // from its entry and then publishes the exit.
        if (w == 0) {
          int hh;
          int64_t FF;
          entry(hh, FF);
          CX_T(4);
          long long nbat = 0;
          while (hh < Cn) {
            const int k = stretch(hh, FF, Cn);
            if (k > 0) {
              const int np = k * Bm;
              for (int j = lane; j < np; j += 32) {
                const uint32_t l = sat_lat(FF + (int64_t)(j / Bm + 1) * TB - (int64_t)sA[hh + j]);
                out[hh + j] = l;
                ont += (int64_t)l <= p.L;
              }
              nbat += k;
              hh += np;
              FF += (int64_t)k * TB;
              continue;
            }
            int64_t t;
            int b = idle_decide(A, nloc, (int64_t)hh, Bm, p.L, sT, true, &t);
            int64_t fin;
            if (FF <= t) fin = t + sT[b - 1];
            else { b = count_upto(A, nloc, (int64_t)hh, Bm, FF); fin = FF + sT[b - 1]; }
            put(hh, b, fin, INT32_MAX);
            nbat++;
            hh += b;
            FF = fin;
          }
          publish(hh - Cn, FF);
          CX_T(6);
#ifdef PX_CHAIN_DEBUG
          if (lane == 0) {
            atomicAdd(a.dbg + 8, 1ull);
            atomicAdd(a.dbg + 9, (unsigned long long)nbat);
          }
#else
          (void)nbat;
#endif
        }
      } else {
      // idle decisions of every head (fact (ii): binary search)
      for (int i = tid; i < Cn; i += CHAIN_THREADS) {
        int64_t t;
        const int b = idle_decide(A, HN(i), (int64_t)i, HB(i), HL(i), HT(i), true, &t);
        sB[i] = (uint8_t)b;
        sTi[i] = (int32_t)(t - (int64_t)sA[i]);
      }
      __syncthreads();
      CX_T(1);
      // greedy batch at (hh, F), the device free at F after the idle decision
      // would have dispatched: min(Bmax, queued at F), Bmax without a search
      // when the Bmax-th query is already there
      auto greedy = [&](int hh, int64_t F) -> int {
        const int B_ = HB(hh);
        const int64_t N_ = HN(hh);
        return ((int64_t)hh + B_ - 1 < N_ && (int64_t)sA[hh + B_ - 1] <= F) ? B_ : count_upto(A, N_, (int64_t)hh, B_, F);
      };
      // the run of every head after its idle-branch decision (at most K
      // greedy batches are followed here -- backlogged stretches would make
      // this quadratic -- the rest is left to the link walk): inside the
      // head's segment (sNx: the next idle-branch head, -1: the run leaves the
      // segment (its state there is recomputed by the record walk), -3: ... onto an idle-branch head, -2: left to
      // the walk) and inside the chunk (sNc: the next idle-branch head, -1:
      // the run leaves the chunk, -2: left to the walk)
      for (int i = tid; i < Cn; i += CHAIN_THREADS) {
        const int se = (i / SEG + 1) * SEG < Cn ? (i / SEG + 1) * SEG : Cn;
        const int bi = sB[i];
        int64_t F = (int64_t)sA[i] + sTi[i] + HT(i)[bi - 1];
        int hh = i + bi;
        bool segdone = false;
        for (int st = 0;; st++) {
          const bool node = hh < Cn && F <= (int64_t)sA[hh] + sTi[hh];
          if (!segdone && hh >= se) {
            sNx[i] = node ? -3 : -1;
            segdone = true;
          }
          if (hh >= Cn) { sNc[i] = -1; break; }
          if (node) {
            if (!segdone) sNx[i] = (int16_t)hh;
            sNc[i] = (int16_t)hh;
            break;
          }
          if (st >= a.K) {
            if (!segdone) sNx[i] = -2;
            sNc[i] = -2;
            break;
          }
          const int g = greedy(hh, F);  // dispatched at F
          F += HT(hh)[g - 1];
          hh += g;
        }
      }
      __syncthreads();
      CX_T(2);
      // the last idle-branch head of every head's run inside its segment
      // (sJ): pointer jumping, in place (a pointer only ever moves further
      // along its own run) ...
      for (int i = tid; i < Cn; i += CHAIN_THREADS) {
        const int nx = sNx[i];
        sJ[i] = nx >= 0 ? (int16_t)nx : (int16_t)i;
      }
      for (bool more = true; more;) {
        __syncthreads();
        bool ch = false;
        for (int i = tid; i < Cn; i += CHAIN_THREADS) {
          const int j = sJ[i], jj = sJ[j];
          if (jj != j) { sJ[i] = (int16_t)jj; ch = true; }
        }
        more = __syncthreads_or(ch);
      }
      // ... and inside the chunk (sJc): a run whose last node r in its segment
      // reaches an idle-branch head further on (sNc[r], a later segment)
      // continues with that head's; segments from the last
      for (int sg = nseg - 1; sg >= 0; sg--) {
        const int s1 = (sg + 1) * SEG < Cn ? (sg + 1) * SEG : Cn;
        for (int i = sg * SEG + tid; i < s1; i += CHAIN_THREADS) {
          const int r = sJ[i], nc = sNc[r];
          sJc[i] = nc >= 0 ? sJc[nc] : (int16_t)r;
        }
        __syncthreads();
      }
      CX_T(3);
      if (w <= 1) {
        // warp 0, the link: the true run through the chunk, one hop per run
        // of idle-branch decisions (sJc), greedy batches between (full
        // batches 32 per ballot); the chunk's exit is published at once.
        // Warp 1, at the same time: the same run, one hop per segment (sJ),
        // recording the state at the first batch head of every segment for
        // the writers.
        int h;
        int64_t F;
#ifdef PX_CHAIN_DEBUG
        const long long cx_w0 = clock64();
#endif
        entry(h, F);
#ifdef PX_CHAIN_DEBUG
        if (lane == 0) atomicAdd(a.dbg + 18 + 3 * li, (unsigned long long)(clock64() - cx_w0));
#endif
        CX_T(4);
        int hh = h;
        int64_t FF = F;
        long long hops = 0;
        if (w == 0) {
        while (hh < Cn) {
          hops++;
          if (FF <= (int64_t)sA[hh] + sTi[hh]) {
            // the run's last idle-branch head in the chunk; then its greedy
            // batches (to the chunk's end when it leaves the chunk)
            const int r = sJc[hh];
            const int br = sB[r];
            FF = (int64_t)sA[r] + sTi[r] + HT(r)[br - 1];
            hh = r + br;
            if (sNc[r] == -1)
              while (hh < Cn) {
                const int g = greedy(hh, FF);
                FF += HT(hh)[g - 1];
                hh += g;
              }
            continue;
          }
          const int k = stretch(hh, FF, Cn);
          if (k > 0) {
            const int B_ = HB(hh);
            FF += (int64_t)k * HT(hh)[B_ - 1];
            hh += k * B_;
            continue;
          }
          const int g = count_upto(A, HN(hh), (int64_t)hh, HB(hh), FF);
          FF += HT(hh)[g - 1];
          hh += g;
        }
        publish(hh - Cn, FF);
#ifdef PX_CHAIN_DEBUG
        if (lane == 0) {  // per lane: link cycles, hops, wait cycles
          atomicAdd(a.dbg + 16 + 3 * li, (unsigned long long)(clock64() - cx_t));
          atomicAdd(a.dbg + 17 + 3 * li, (unsigned long long)hops);
        }
#endif
        CX_T(5);
        } else {
        int nrec = 0;  // segments [0, nrec) recorded (warp-uniform)
        auto rec = [&](int hq, int64_t Fq) {  // free time first, then the head (the writers' flag)
          const int upto = hq / SEG + 1 < nseg ? hq / SEG + 1 : nseg;
          for (int sg = nrec + lane; sg < upto; sg += 32) {
            sSegF[sg] = Fq;
            __threadfence_block();
            *(volatile int *)&sSegH[sg] = hq;
          }
          nrec = upto > nrec ? upto : nrec;
        };
        hh = h;
        FF = F;
        rec(hh, FF);
        while (hh < Cn) {
          if (FF <= (int64_t)sA[hh] + sTi[hh]) {
            const int r = sJ[hh];
            const int nx = sNx[r];
            if (nx == -2) { const int br = sB[r]; FF = (int64_t)sA[r] + sTi[r] + HT(r)[br - 1]; hh = r + br; rec(hh, FF); continue; }
            {  // the run of r to its segment's end (busy after r's batch, at most K greedy batches)
              const int ser = (r / SEG + 1) * SEG < Cn ? (r / SEG + 1) * SEG : Cn;
              const int br = sB[r];
              FF = (int64_t)sA[r] + sTi[r] + HT(r)[br - 1];
              hh = r + br;
              while (hh < ser) {
                const int g = greedy(hh, FF);
                FF += HT(hh)[g - 1];
                hh += g;
              }
            }
            rec(hh, FF);
            // a run leaving its segment busy: when its next idle-branch head
            // (sNc) lies in the segment it entered, no other segment starts
            // in between: continue there
            const int nc = sNc[r];
            if (nx == -1 && nc >= 0 && nc / SEG == hh / SEG) hh = nc;
            continue;
          }
          const int se = (hh / SEG + 1) * SEG < Cn ? (hh / SEG + 1) * SEG : Cn;
          const int k = stretch(hh, FF, se);
          if (k > 0) {
            const int B_ = HB(hh);
            FF += (int64_t)k * HT(hh)[B_ - 1];
            hh += k * B_;
            rec(hh, FF);
            continue;
          }
          const int g = count_upto(A, HN(hh), (int64_t)hh, HB(hh), FF);
          FF += HT(hh)[g - 1];
          hh += g;
          rec(hh, FF);
        }
        CX_T(7);
        }  // warp 1
#ifdef PX_CHAIN_DEBUG
        if (lane == 0 && w == 0) { atomicAdd(a.dbg + 8, 1ull); atomicAdd(a.dbg + 10, (unsigned long long)hops); }
#else
        (void)hops;
#endif
      }
      // the writers (warps 2..7, while warp 1 records): thread per segment,
      // from the true state at its first batch head, as soon as it is
      // recorded; a batch is written whole by the segment it starts in
      long long nbat = 0;
      for (int sg = tid - 64; sg < nseg; sg += CHAIN_THREADS - 64) {
        if (sg < 0) break;
        const int s1 = (sg + 1) * SEG < Cn ? (sg + 1) * SEG : Cn;
        int hh;
        while ((hh = *(volatile int *)&sSegH[sg]) < 0) __nanosleep(32);
        __threadfence_block();
        int64_t FF = *(volatile int64_t *)&sSegF[sg];
        while (hh < s1) {
          const int64_t ti = (int64_t)sA[hh] + sTi[hh];
          int b;
          int64_t fin;
          if (FF <= ti) { b = sB[hh]; fin = ti + HT(hh)[b - 1]; }
          else { b = greedy(hh, FF); fin = FF + HT(hh)[b - 1]; }
          if constexpr (EP) {  // the batch's epoch gives the SLO and the accuracy (F4)
            const int64_t Lh = HL(hh);
            unsigned on = 0;
            for (int j = 0; j < b; j++) {
              const uint32_t l = sat_lat(fin - (int64_t)sA[hh + j]);
              out[hh + j] = l;
              on += (int64_t)l <= Lh;
            }
            ont += on;
            nwr += (unsigned)b;
            accs += (unsigned long long)on * (unsigned)epp(hh)[3];
          } else {
            for (int j = 0; j < b; j++) {
              const uint32_t l = sat_lat(fin - (int64_t)sA[hh + j]);
              out[hh + j] = l;
              ont += (int64_t)l <= p.L;
            }
          }
          nbat++;
          hh += b;
          FF = fin;
        }
      }
      CX_T(6);
#ifdef PX_CHAIN_DEBUG
      atomicAdd(a.dbg + 9, (unsigned long long)nbat);
#else
      (void)nbat;
#endif
      }  // tables
      if (a.lcnt) {  // the lane's on-time count (violations = positions - on time, R6; accuracy = on time x A, R9)
        for (int o = 16; o; o >>= 1) ont += __shfl_xor_sync(0xffffffffu, ont, o);
        if ((tid & 31) == 0 && ont) atomicAdd(a.lcnt + li, ont);
      }
      if (EP && a.agg) {  // the scenario's counts (violations R6, on time, accuracy R9)
        for (int o = 16; o; o >>= 1) {
          ont += __shfl_xor_sync(0xffffffffu, ont, o);
          nwr += __shfl_xor_sync(0xffffffffu, nwr, o);
          accs += __shfl_xor_sync(0xffffffffu, accs, o);
        }
        if ((tid & 31) == 0 && nwr) {
          if (nwr > ont) atomicAdd((unsigned long long *)&a.agg[s], nwr - ont);
          if (ont) atomicAdd((unsigned long long *)&a.agg[a.S + s], ont);
          if (accs) atomicAdd((unsigned long long *)&a.agg[2 * a.S + s], accs);
        }
      }
    }
    __syncthreads();  // shared tables and sTicket are rewritten by the next unit
  }
}

// ---------------------------------------------------------------- host ----
static int env_int(const char *name, int dflt) {
  const char *v = getenv(name);
  return v && *v ? atoi(v) : dflt;
}

int px_replay(proteus_ctx *ctx, const uint32_t *d_arr, const uint8_t *d_fam, int64_t N, const int32_t *h_option,
              const int32_t *h_z, const int32_t *h_dev_type, int D, const int32_t *h_demand, const int32_t *h_slo,
              const proteus_scenario *h_sc, int S, uint32_t *d_lat_out, uint64_t *d_agg) {
  const int Q = ctx->Q, M = ctx->M;
  PX_CUDA(ctx, cudaMemsetAsync(d_agg, 0, ((size_t)3 * S + 1) * 8, ctx->stream));
  const size_t small = (size_t)(4 * D + 2 * Q + 2 * PX_MAXQ + 8 + 8 * S + 4 * (PX_MAXD + 2)) * 4 +
                       (size_t)S * sizeof(proteus_scenario) + (size_t)S * D * sizeof(LaneParam) +
                       (size_t)2 * (PX_MAXD + 2) * 8;
  char *sb = (char *)px_buf(ctx, B_R_MISC, small + 4096);
  if (!sb) return px_fail(ctx, PROTEUS_ENOMEM, "replay scratch");
  int32_t *d_opt = (int32_t *)sb, *d_z = d_opt + D, *d_dev = d_z + D, *d_dem = d_dev + D, *d_slo = d_dem + Q;
  int32_t *d_pat_off = d_slo + Q, *d_pat_len = d_pat_off + PX_MAXQ;
  uint32_t *d_flags = (uint32_t *)(d_pat_len + PX_MAXQ);  // [0] trace checks, [4] fix-up changes
  // [8][S] scenario lists: per routing mode rt, row rt = every scenario, row 2 + rt = the §5
  // scenarios (chunk / scan kernels), row 4 + rt = the baseline batchers (k_wc_lanes), row
  // 6 + rt = the AIMD ones (k_wc_spec chunk runs)
  int32_t *d_scl = (int32_t *)(d_flags + 8);
  int32_t *d_goff = d_scl + 8 * S;                        // [2][PX_MAXD + 2]
  int64_t *d_choff = (int64_t *)(((uintptr_t)(d_goff + 2 * (PX_MAXD + 2)) + 15) & ~(uintptr_t)15);  // [2][PX_MAXD + 2]
  proteus_scenario *d_sc = (proteus_scenario *)(d_choff + 2 * (PX_MAXD + 2));
  LaneParam *d_lp = (LaneParam *)(((uintptr_t)(d_sc + S) + 15) & ~(uintptr_t)15);
  // Bmax per (scenario, device), as k_lane_params (R4', R15); T(b) non-decreasing on the lane
  std::vector<int32_t> hB((size_t)S * D, 0), hT1(D, 0);
  std::vector<uint8_t> hmono((size_t)S * D, 0);
  for (int d = 0; d < D; d++) {
    if (h_option[d] <= 0) continue;
    const int32_t *Tr = ctx->lat.data() + ((size_t)h_dev_type[d] * M + (h_option[d] - 1)) * ctx->bmax;
    int depth = 0;
    while (depth < ctx->bmax && Tr[depth] > 0) depth++;
    hT1[d] = Tr[0];
    const int64_t base = h_slo[ctx->fam[h_option[d] - 1]];
    for (int s = 0; s < S; s++) {
      const int cap = h_sc[s].batch_cap;
      int B = (cap > 0 && cap < depth) ? cap : depth;
      if (h_sc[s].policy == 0 && B > 0) {  // the maximum allowed batch size (R4')
        const int64_t L = (int64_t)h_sc[s].slo_mult_milli * base / 1000;
        int Bn = 1;
        for (int b = 1; b <= B; b++) if (2 * (int64_t)Tr[b - 1] <= L) Bn = b;
        B = Bn;
      }
      hB[(size_t)s * D + d] = B;
      bool mono = true;
      for (int b = 1; b < B; b++) mono &= Tr[b] >= Tr[b - 1];
      hmono[(size_t)s * D + d] = mono ? 1 : 0;
    }
  }
  // the window path (k_win_*) takes the §5 scenarios whose lanes all have
  // Bmax <= WIN_EMAX; the chunk-run / stitch path below takes the rest
  const bool simple = env_int("PROTEUS_REPLAY_SIMPLE", 0) != 0;
  const bool use_win = !simple && env_int("PROTEUS_REPLAY_WINDOW", 0) != 0;
  std::vector<int32_t> wl[2];
  std::vector<char> is_win(S, 0);
  for (int s = 0; s < S; s++) {
    if (!use_win || h_sc[s].policy != 0) continue;
    int mb = 0;
    for (int d = 0; d < D; d++) mb = std::max(mb, hB[(size_t)s * D + d]);
    if (mb <= WIN_EMAX) { wl[h_sc[s].routing].push_back(s); is_win[s] = 1; }
  }
  std::vector<int32_t> scl[8];
  for (int s = 0; s < S; s++) {
    if (is_win[s]) continue;
    scl[h_sc[s].routing].push_back(s);
    scl[(h_sc[s].policy == 0 ? 2 : 4) + h_sc[s].routing].push_back(s);
    if (h_sc[s].policy == 2) scl[6 + h_sc[s].routing].push_back(s);
  }
  const bool any_old = !scl[0].empty() || !scl[1].empty();
  std::vector<int32_t> scl_all(8 * S, 0);
  for (int r = 0; r < 8; r++)
    for (size_t k = 0; k < scl[r].size(); k++) scl_all[r * S + k] = scl[r][k];
  PX_CUDA(ctx, cudaMemcpyAsync(d_opt, h_option, D * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_z, h_z, D * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_dev, h_dev_type, D * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_dem, h_demand, Q * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_slo, h_slo, Q * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_scl, scl_all.data(), 8 * S * 4, cudaMemcpyHostToDevice, ctx->stream));
  {  // the un-permute of the old path skips the window path's rows (routing -1)
    std::vector<proteus_scenario> sc2(h_sc, h_sc + S);
    for (int s = 0; s < S; s++) if (is_win[s]) sc2[s].routing = -1;
    PX_CUDA(ctx, cudaMemcpyAsync(d_sc, sc2.data(), S * sizeof(proteus_scenario), cudaMemcpyHostToDevice, ctx->stream));
    PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));  // sc2 is a stack copy
  }
  PX_CUDA(ctx, cudaMemsetAsync(d_flags, 0, 4, ctx->stream));
  if (N > 0) {
    PX_LAUNCH(ctx, "replay_check", k_check_trace, 1184, 256, 0, d_arr, d_fam, N, Q, d_flags);
    uint32_t flags = 0;
    PX_CUDA(ctx, cudaMemcpyAsync(&flags, d_flags, 4, cudaMemcpyDeviceToHost, ctx->stream));
    PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
    if (flags & 1) return px_fail(ctx, PROTEUS_ERANGE, "arrival timestamps not sorted");
    if (flags & 2) return px_fail(ctx, PROTEUS_EINVAL, "family id >= Q");
  }
  PX_LAUNCH(ctx, "replay_params", k_lane_params, (S * D + 127) / 128, 128, 0, S, D, M, ctx->bmax, d_opt, d_dev,
            ctx->d_fam, ctx->d_acc, ctx->d_lat, d_slo, d_sc, d_lp);
  const int64_t ntiles = (N + TILE - 1) / TILE;
  const unsigned tblocks = (unsigned)((ntiles + TILE_WARPS - 1) / TILE_WARPS);
  int64_t dsum = 0;
  for (int q = 0; q < Q; q++) dsum += h_demand[q];
  const size_t pat_cap = (size_t)dsum + (size_t)Q * D + 16;
  int64_t *devOff[2] = {nullptr, nullptr};
  const uint32_t *devArr[2] = {nullptr, nullptr}, *inv[2] = {nullptr, nullptr};
  int32_t *dbase_rt[2] = {nullptr, nullptr};
  const uint8_t *tgt_rt[2] = {nullptr, nullptr};
  for (int rt = 0; rt < 2; rt++) {
    if (scl[rt].empty() && wl[rt].empty()) continue;
    uint8_t *pat = (uint8_t *)px_buf(ctx, B_R_PAT, pat_cap);
    int32_t *hist = (int32_t *)px_buf(ctx, B_R_HIST, (size_t)(ntiles + 1) * (PX_MAXD + 2) * 4);
    int32_t *fbase = (int32_t *)px_buf(ctx, B_R_BASE, (size_t)(ntiles + 1) * (PX_MAXQ + 2) * 4);
    int32_t *dbase = (int32_t *)px_buf(ctx, rt ? B_R_DBASE1 : B_R_DBASE0, (size_t)(ntiles + 1) * (PX_MAXD + 2) * 4);
    uint8_t *tgt = (uint8_t *)px_buf(ctx, rt ? B_R_TGT1 : B_R_TGT, (size_t)N + 16);
    int64_t *off = (int64_t *)px_buf(ctx, rt ? B_R_OFF1 : B_R_OFF, (size_t)2 * (PX_MAXD + 2) * 8);
    // + whole trailing ring segment: k_stitch bulk-copies 4 KB segments
    // k_stitch's ring reads whole segments up to 2 past the head's: pad 3 segments
    uint32_t *darr = (uint32_t *)px_buf(ctx, rt ? B_R_DEVARR1 : B_R_DEVARR, ((size_t)N + 3 * RSEG) * 4);
    uint32_t *dinv = (uint32_t *)px_buf(ctx, rt ? B_R_DEVIDX1 : B_R_DEVIDX, (size_t)N * 4 + 16);
    if (!pat || !hist || !fbase || !dbase || !tgt || !off || !darr || !dinv)
      return px_fail(ctx, PROTEUS_ENOMEM, "routing buffers");
    int64_t *totals = off + (PX_MAXD + 2);
    PX_LAUNCH(ctx, "route_prepare", k_route_prepare, Q, 32, 0, rt, Q, D, M, ctx->bmax, d_opt, d_z, d_dev, d_dem,
              ctx->d_fam, ctx->d_lat, pat, d_pat_off, d_pat_len);
    if (N > 0) {
      PX_LAUNCH(ctx, "route_count", k_tile_count, tblocks, TILE_WARPS * 32, 0, d_fam, N, Q, hist);
      PX_LAUNCH(ctx, "route_scan", k_tile_scan, Q, 1024, 0, hist, ntiles, Q, fbase, totals);
      PX_LAUNCH(ctx, "route_target", k_route_target, tblocks, TILE_WARPS * 32, 0, d_fam, N, Q, fbase, pat, d_pat_off,
                d_pat_len, D, tgt, hist);
      PX_LAUNCH(ctx, "route_scan_dev", k_tile_scan, D + 1, 1024, 0, hist, ntiles, D + 1, dbase, totals);
      PX_LAUNCH(ctx, "route_offsets", k_dev_offsets, 1, 32, 0, totals, D + 1, off);
      PX_LAUNCH(ctx, "route_scatter", k_scatter, tblocks, TILE_WARPS * 32, 0, tgt, d_arr, N, D, dbase, off, darr,
                dinv);
    } else {
      PX_CUDA(ctx, cudaMemsetAsync(off, 0, (size_t)(PX_MAXD + 2) * 8, ctx->stream));
    }
    devOff[rt] = off; devArr[rt] = darr; inv[rt] = dinv; dbase_rt[rt] = dbase; tgt_rt[rt] = tgt;
  }
  if (N == 0) return 0;
  // ---- window path (k_win_tables, k_win_compose, k_win_write)
  if (!wl[0].empty() || !wl[1].empty()) {
    int WT = env_int("PROTEUS_REPLAY_WIN_TILES", 16);
    WT = WT < 1 ? 1 : WT > 32 ? 32 : WT;  // TQ = WT * TILE <= 16384 queries (shared-memory tiles)
    const int64_t TQ = (int64_t)WT * TILE;
    const int64_t nw = (ntiles + WT - 1) / WT;
    if (nw > 65535) return px_fail(ctx, PROTEUS_ERANGE, "replay windows");
    char *aux = (char *)px_buf(ctx, B_W_AUX, (size_t)S * D * (1 + 4 + 8) + (size_t)2 * S * 4 + 256);
    if (!aux) return px_fail(ctx, PROTEUS_ENOMEM, "window scratch");
    uint8_t *d_mono = (uint8_t *)aux;
    int64_t *d_recoff = (int64_t *)(((uintptr_t)(d_mono + (size_t)S * D) + 15) & ~(uintptr_t)15);
    int32_t *d_E = (int32_t *)(d_recoff + (size_t)S * D);
    int32_t *d_wl = d_E + (size_t)S * D;
    PX_CUDA(ctx, cudaMemcpyAsync(d_mono, hmono.data(), (size_t)S * D, cudaMemcpyHostToDevice, ctx->stream));
    std::vector<int64_t> recoff((size_t)S * D, 0);
    std::vector<int32_t> Ev((size_t)S * D, 0), wlv(2 * (size_t)S, 0);
    int64_t nrec = 0, lbase = 0;
    for (int rt = 0; rt < 2; rt++) {
      for (size_t i = 0; i < wl[rt].size(); i++) {
        wlv[(size_t)rt * S + i] = wl[rt][i];
        for (int d = 0; d < D; d++) {
          const int B = hB[(size_t)wl[rt][i] * D + d];
          const int E = B >= 1 ? std::min(B, WIN_EMAX) : 0;
          Ev[lbase + i * D + d] = E;
          recoff[lbase + i * D + d] = nrec;
          nrec += (int64_t)E * nw;
        }
      }
      lbase += (int64_t)wl[rt].size() * D;
    }
    WinRec *d_rec = (WinRec *)px_buf(ctx, B_W_REC, sizeof(WinRec) * (size_t)(nrec + 1));
    WinEntry *d_ent = (WinEntry *)px_buf(ctx, B_W_ENT, sizeof(WinEntry) * (size_t)(lbase * nw + 1));
    if (!d_rec || !d_ent) return px_fail(ctx, PROTEUS_ENOMEM, "window tables");
    PX_CUDA(ctx, cudaMemcpyAsync(d_recoff, recoff.data(), recoff.size() * 8, cudaMemcpyHostToDevice, ctx->stream));
    PX_CUDA(ctx, cudaMemcpyAsync(d_E, Ev.data(), Ev.size() * 4, cudaMemcpyHostToDevice, ctx->stream));
    PX_CUDA(ctx, cudaMemcpyAsync(d_wl, wlv.data(), wlv.size() * 4, cudaMemcpyHostToDevice, ctx->stream));
    PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));  // host vectors are staged
    const size_t sm1 = (size_t)(TQ + WIN_EXT) * 4 + (size_t)WIN_WARPS * TQ;
    const size_t sm3 = (size_t)TQ * 4 + (size_t)(TQ + (size_t)D * WIN_EXT) * 4;
    PX_CUDA(ctx, cudaFuncSetAttribute(k_win_tables, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm1));
    PX_CUDA(ctx, cudaFuncSetAttribute(k_win_write, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm3));
    int64_t loff = 0;
    for (int rt = 0; rt < 2; rt++) {
      const int nsc = (int)wl[rt].size();
      if (!nsc) continue;
      WinArgs wa;
      memset(&wa, 0, sizeof wa);
      wa.S = S; wa.D = D; wa.M = M; wa.bmax = ctx->bmax; wa.nsc = nsc; wa.WT = WT; wa.D1 = D + 1;
      wa.N = N; wa.nw = nw; wa.ntiles = ntiles;
      wa.option = d_opt; wa.dev_type = d_dev; wa.lat = ctx->d_lat; wa.sc_list = d_wl + (size_t)rt * S;
      wa.lp = d_lp; wa.mono = d_mono; wa.devOff = devOff[rt]; wa.dbase = dbase_rt[rt]; wa.devArr = devArr[rt];
      wa.inv = inv[rt]; wa.tgt = tgt_rt[rt]; wa.recoff = d_recoff + loff; wa.E = d_E + loff; wa.rec = d_rec;
      wa.ent = d_ent + loff * nw; wa.out = d_lat_out; wa.agg = d_agg;
      const int64_t items = (int64_t)nsc * D * nw;
      const bool dbg = env_int("PROTEUS_REPLAY_DEBUG", 0) != 0;
      if (dbg) {
        wa.dbg = (unsigned long long *)px_buf(ctx, B_R_VLAT, (size_t)nsc * D * 32 + 64);
        if (!wa.dbg) return px_fail(ctx, PROTEUS_ENOMEM, "debug counters");
        PX_CUDA(ctx, cudaMemsetAsync(wa.dbg, 0, (size_t)nsc * D * 32, ctx->stream));
      }
      (void)items;
      PX_LAUNCH(ctx, "replay_win_tables", k_win_tables, (unsigned)(nw * D), WIN_WARPS * 32, sm1, wa);
      PX_LAUNCH(ctx, "replay_win_compose", k_win_compose, (unsigned)(((int64_t)nsc * D + 3) / 4), 128, 0, wa);
      if (dbg) {
        std::vector<unsigned long long> hc((size_t)nsc * D * 4);
        std::vector<int64_t> hoff(D + 2);
        PX_CUDA(ctx, cudaMemcpyAsync(hoff.data(), devOff[rt], (D + 2) * 8, cudaMemcpyDeviceToHost, ctx->stream));
        PX_CUDA(ctx, cudaMemcpyAsync(hc.data(), wa.dbg, hc.size() * 8, cudaMemcpyDeviceToHost, ctx->stream));
        PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
        for (int i = 0; i < nsc; i++)
          for (int d = 0; d < D; d++) {
            const unsigned long long *c = &hc[((size_t)i * D + d) * 4];
            if (c[0] || c[1] || c[2])
              fprintf(stderr, "win rt %d sc %d (mult %d cap %d) dev %d: n=%lld Bmax=%d idle %llu backlog %llu walks %llu "
                      "walked %llu\n", rt, wl[rt][i], h_sc[wl[rt][i]].slo_mult_milli, h_sc[wl[rt][i]].batch_cap, d,
                      (long long)(hoff[d + 1] - hoff[d]), hB[(size_t)wl[rt][i] * D + d], c[0], c[1], c[2], c[3]);
          }
      }
      PX_LAUNCH(ctx, "replay_win_write", k_win_write, dim3((unsigned)nsc, (unsigned)nw), WIN_THREADS, sm3, wa);
      loff += (int64_t)nsc * D;
    }
  }
  if (!any_old) return 0;
  // chunk layout per routing mode (sizes only): the host reads the per-device counts
  int CH = env_int("PROTEUS_REPLAY_CHUNK", 4096);
  CH = CH < 1 ? 1 : CH > (1 << 20) ? (1 << 20) : CH;
  // fix-up rounds before the sequential stitch finishes whatever is left
  const int max_rounds = env_int("PROTEUS_REPLAY_ROUNDS", 0);
  int64_t h_off[2][PX_MAXD + 2];
  memset(h_off, 0, sizeof h_off);
  for (int rt = 0; rt < 2; rt++)
    if (devOff[rt])
      PX_CUDA(ctx, cudaMemcpyAsync(h_off[rt], devOff[rt], (D + 2) * 8, cudaMemcpyDeviceToHost, ctx->stream));
  uint32_t h_span[2] = {0, 0};  // first and last arrival (the chain path's rate estimate)
  PX_CUDA(ctx, cudaMemcpyAsync(&h_span[0], d_arr, 4, cudaMemcpyDeviceToHost, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(&h_span[1], d_arr + (N - 1), 4, cudaMemcpyDeviceToHost, ctx->stream));
  PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  int64_t NCH[2] = {0, 0};
  int32_t ngroups[2] = {0, 0};
  std::vector<int64_t> choff(2 * (PX_MAXD + 2), 0);
  std::vector<int32_t> goff(2 * (PX_MAXD + 2), 0);
  for (int rt = 0; rt < 2; rt++) {
    if (!devOff[rt]) continue;
    for (int d = 0; d < D; d++) {
      const int64_t nch = (h_off[rt][d + 1] - h_off[rt][d] + CH - 1) / CH;
      choff[rt * (PX_MAXD + 2) + d + 1] = choff[rt * (PX_MAXD + 2) + d] + nch;
      goff[rt * (PX_MAXD + 2) + d + 1] = goff[rt * (PX_MAXD + 2) + d] + (int32_t)((nch + 31) / 32);
    }
    NCH[rt] = choff[rt * (PX_MAXD + 2) + D];
    ngroups[rt] = goff[rt * (PX_MAXD + 2) + D];
  }
  PX_CUDA(ctx, cudaMemcpyAsync(d_choff, choff.data(), choff.size() * 8, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_goff, goff.data(), goff.size() * 4, cudaMemcpyHostToDevice, ctx->stream));
  // chain path (k_chain): the §5 lanes with T non-decreasing, 2 <= Bmax <= 255
  // and L < 2^30; the chunk runs + stitch take the other lanes
  const bool use_scan1 = !simple && env_int("PROTEUS_REPLAY_SCAN1", 1) != 0;
  const bool use_chain = !simple && env_int("PROTEUS_REPLAY_CHAIN", 1) != 0 && max_rounds == 0 &&
                         env_int("PROTEUS_REPLAY_TABLES", 0) == 0;
  int CHN = env_int("PROTEUS_REPLAY_CHAIN_C", 2048);
  CHN = CHN < 256 ? 256 : CHN > CHAIN_CMAX ? CHAIN_CMAX : CHN;  // shared-memory tables (~28 B per head)
  {
    int smax = 0;
    PX_CUDA(ctx, cudaDeviceGetAttribute(&smax, cudaDevAttrMaxSharedMemoryPerBlockOptin, ctx->device));
    const int seg0 = std::max(CHAIN_SEGMIN, env_int("PROTEUS_REPLAY_CHAIN_SEG", 128));
    while (CHN > 256 && chain_smem(CHN, ctx->bmax, std::min(CHN, seg0)) + 1024 > (size_t)smax) CHN -= 256;
  }
  const int chain_minb = std::max(2, env_int("PROTEUS_REPLAY_CHAIN_MINB", 2));
  std::vector<int32_t> clid[2], cnch[2];
  unsigned long long *d_units[2] = {nullptr, nullptr};  // chain ticket order per routing mode
  int64_t nunits[2] = {0, 0};
  std::vector<uint8_t> cmodev[2];
  int64_t cmax[2] = {0, 0};
  bool crest[2] = {true, true};  // lanes left to the chunk runs + stitch
  uint8_t *d_chainf = nullptr;  // skip flags [S][D]
  int32_t *d_rep = nullptr;      // row map [S][D + 1] (null: every lane its own row)
  int32_t *d_pairs[2] = {nullptr, nullptr};  // (duplicate, representative, device) per routing mode
  int64_t npair[2] = {0, 0};
  char *cbuf[2] = {nullptr, nullptr};  // per routing mode (chain_exoff)
  // Lanes (scenario, device) with the same policy, Bmax and SLO on a device
  // see the same arrivals under the same rule: one of them (the first
  // scenario) is replayed and the others read its row (rep[s][d], the row
  // holding lane (s, d); rep[s][D] = s for the sink).  skip[s][d]: the chunk
  // kernels leave the lane alone (a duplicate, or a chain lane).
  const bool dedup = !simple && !use_win && max_rounds == 0 && env_int("PROTEUS_REPLAY_DEDUP", 1) != 0 &&
                     env_int("PROTEUS_REPLAY_TABLES", 0) == 0 &&
                     env_int("PROTEUS_REPLAY_FINISH", 0) == 0 && env_int("PROTEUS_REPLAY_DEBUG", 0) == 0;
  std::vector<int32_t> hrep((size_t)S * (D + 1));
  std::vector<uint8_t> hskip((size_t)S * D, 0);
  for (int s = 0; s < S; s++)
    for (int d = 0; d <= D; d++) hrep[(size_t)s * (D + 1) + d] = s;
  auto lane_L = [&](int s, int d) -> int64_t {
    return (int64_t)h_sc[s].slo_mult_milli * h_slo[ctx->fam[h_option[d] - 1]] / 1000;
  };
  if (dedup) {
    for (int rt = 0; rt < 2; rt++)
      for (int d = 0; d < D; d++) {
        if (h_option[d] <= 0) continue;
        std::vector<std::pair<std::array<int64_t, 3>, int>> seen;
        for (int s : scl[rt]) {
          int B = hB[(size_t)s * D + d];
          if (h_sc[s].policy == 0 && B == 1 && use_scan1) continue;  // the Bmax = 1 scan writes every row
          const int64_t L = lane_L(s, d);
          if (h_sc[s].policy == 1) {  // Nexus batches Bn: the largest b <= Bmax with 2 T(b) <= L, at least 1 (R14)
            const int32_t *Tr = ctx->lat.data() + ((size_t)h_dev_type[d] * M + (h_option[d] - 1)) * ctx->bmax;
            int Bn = 1;
            for (int b = 1; b <= B; b++)
              if (2 * (int64_t)Tr[b - 1] <= L) Bn = b;
            B = Bn;
          }
          const std::array<int64_t, 3> key = {h_sc[s].policy, B, L};
          int r = -1;
          for (auto &e : seen) if (e.first == key) { r = e.second; break; }
          if (r < 0) { seen.push_back({key, s}); continue; }
          hrep[(size_t)s * (D + 1) + d] = r;
          hskip[(size_t)s * D + d] = 1;
        }
      }
  }
  if (use_chain) {
    // lanes whose idle batches are large: b^ = the largest b <= Bmax with
    // 1 + lambda (L - T(b + 1)) >= b (the queries arriving while the head
    // waits, lambda = the device's mean rate).  Small-batch lanes have long
    // serial walks per chunk here, while their chunk runs meet the true run at
    // once (the stitch accepts them), so they stay on the chunk runs + stitch.
    const double minbatch = (double)env_int("PROTEUS_REPLAY_CHAIN_MINBATCH", 0);
    const double minrho = (double)env_int("PROTEUS_REPLAY_CHAIN_RHO_PCT", 100) / 100.0;
    const double span = (double)h_span[1] - (double)h_span[0];
    std::vector<uint8_t> hchain((size_t)S * D, 0);
    for (int s = 0; s < S; s++) {
      if (is_win[s] || h_sc[s].policy != 0) continue;
      for (int d = 0; d < D; d++) {
        if (h_option[d] <= 0 || hskip[(size_t)s * D + d]) continue;
        const int B = hB[(size_t)s * D + d];
        const int64_t L = lane_L(s, d);
        if (B < chain_minb || B > 255 || !hmono[(size_t)s * D + d] || L >= (1ll << 30)) continue;
        const int32_t *Tr = ctx->lat.data() + ((size_t)h_dev_type[d] * M + (h_option[d] - 1)) * ctx->bmax;
        if (Tr[B - 1] >= (1 << 30)) continue;  // 32-bit idle finishes in the chunk tables
        const int rt = h_sc[s].routing;
        const int64_t nd = h_off[rt][d + 1] - h_off[rt][d];
        const double lam = span > 0 ? (double)nd / span : 1e30;
        int bh = 1;
        for (int b = 1; b <= B; b++)
          if (1.0 + lam * (double)(L - Tr[b < B ? b : B - 1]) >= (double)b) bh = b;
        // ... or lanes at or past overload at their batch cap (full batches
        // back to back: the chain walks them 32 batches per ballot)
        const double rho = lam * (double)Tr[B - 1] / (double)B;
        if (rho >= minrho) hchain[(size_t)s * D + d] = 2;
        else if (bh >= minbatch) hchain[(size_t)s * D + d] = 1;
        if (hchain[(size_t)s * D + d]) hskip[(size_t)s * D + d] = 1;
      }
    }
    for (int rt = 0; rt < 2; rt++) {
      if (!devOff[rt]) continue;
      bool rest = false;
      for (int d = 0; d < D; d++) {
        const int64_t nd = h_off[rt][d + 1] - h_off[rt][d];
        for (int k : scl[2 + rt]) {
          const size_t l = (size_t)k * D + d;
          if (nd > 0 && hchain[l]) {
            clid[rt].push_back((int32_t)l);
            cnch[rt].push_back((int32_t)((nd + CHN - 1) / CHN));
            cmodev[rt].push_back((uint8_t)(hchain[l] - 1));
            cmax[rt] = std::max(cmax[rt], (int64_t)cnch[rt].back());
          } else if (nd > 0 && !hskip[l] && !(use_scan1 && hB[l] == 1)) {
            rest = true;
          }
        }
      }
      crest[rt] = rest;
    }
  }
  if (!simple) {  // skip flags, row map and the chain lists in one buffer
    const size_t o_rep = ((size_t)S * D + 15) & ~(size_t)15;
    const size_t o_pr = o_rep + (((size_t)S * (D + 1) * 4 + 15) & ~(size_t)15);
    std::vector<int32_t> hpairs[2];
    for (int rt = 0; rt < 2; rt++)
      for (int s : scl[rt])
        for (int d = 0; d < D; d++)
          if (hrep[(size_t)s * (D + 1) + d] != s) {
            hpairs[rt].push_back(s);
            hpairs[rt].push_back(hrep[(size_t)s * (D + 1) + d]);
            hpairs[rt].push_back(d);
          }
    const size_t o_ch = o_pr + ((hpairs[0].size() + hpairs[1].size()) * 4 + 15) / 16 * 16;
    size_t part[2] = {0, 0}, need = o_ch;
    for (int rt = 0; rt < 2; rt++) {
      const size_t nl = clid[rt].size();
      if (nl) part[rt] = chain_exoff(nl) + nl * (size_t)cmax[rt] * 8;
      need += part[rt];
    }
    char *cb = (char *)px_buf(ctx, B_R_CHAIN, need + 64);
    if (!cb) return px_fail(ctx, PROTEUS_ENOMEM, "lane tables");
    d_chainf = (uint8_t *)cb;
    d_rep = (int32_t *)(cb + o_rep);
    PX_CUDA(ctx, cudaMemcpyAsync(d_chainf, hskip.data(), hskip.size(), cudaMemcpyHostToDevice, ctx->stream));
    PX_CUDA(ctx, cudaMemcpyAsync(d_rep, hrep.data(), hrep.size() * 4, cudaMemcpyHostToDevice, ctx->stream));
    for (int rt = 0; rt < 2; rt++) {
      d_pairs[rt] = (int32_t *)(cb + o_pr) + (rt ? hpairs[0].size() : 0);
      npair[rt] = (int64_t)hpairs[rt].size() / 3;
      if (npair[rt])
        PX_CUDA(ctx, cudaMemcpyAsync(d_pairs[rt], hpairs[rt].data(), hpairs[rt].size() * 4, cudaMemcpyHostToDevice,
                                     ctx->stream));
    }
    char *q = cb + o_ch;
    for (int rt = 0; rt < 2; rt++) {
      if (!part[rt]) continue;
      cbuf[rt] = q;
      const size_t nl = clid[rt].size();
      PX_CUDA(ctx, cudaMemcpyAsync(q, clid[rt].data(), nl * 4, cudaMemcpyHostToDevice, ctx->stream));
      PX_CUDA(ctx, cudaMemcpyAsync(q + nl * 4, cnch[rt].data(), nl * 4, cudaMemcpyHostToDevice, ctx->stream));
      PX_CUDA(ctx, cudaMemcpyAsync(q + nl * 8, cmodev[rt].data(), nl, cudaMemcpyHostToDevice, ctx->stream));
      PX_CUDA(ctx, cudaMemsetAsync(q + chain_ctroff(nl), 0, part[rt] - chain_ctroff(nl), ctx->stream));  // ticket, watchdog, exits
      // ticket order: every lane's chunks spread over the run in proportion to
      // its length (chunk c of a lane with n chunks at key c * maxch / n,
      // counting sort), so that long lanes keep several chunks in flight; a
      // chunk's predecessor always has a smaller key (an earlier ticket).
      // Uploaded once per lane layout (cached in the context).
      {
        const int64_t mx = cmax[rt];
        std::vector<int64_t> key;
        key.reserve(nl + 2);
        key.push_back((int64_t)nl);
        key.push_back(mx);
        size_t nu = 0;
        for (size_t l = 0; l < nl; l++) { key.push_back(cnch[rt][l]); nu += (size_t)cnch[rt][l]; }
        nunits[rt] = (int64_t)nu;
        d_units[rt] = (unsigned long long *)px_buf(ctx, B_R_UNITS0 + rt, nu * 8 + 16);
        if (!d_units[rt]) return px_fail(ctx, PROTEUS_ENOMEM, "chain tickets");
        if (key != ctx->chain_ukey[rt]) {
          std::vector<int64_t> cnt((size_t)mx + 1, 0);
          for (size_t l = 0; l < nl; l++)
            for (int64_t c = 0; c < cnch[rt][l]; c++) cnt[(size_t)(c * mx / cnch[rt][l]) + 1]++;
          for (int64_t k = 0; k < mx; k++) cnt[(size_t)k + 1] += cnt[(size_t)k];
          std::vector<unsigned long long> units(nu);
          for (size_t l = 0; l < nl; l++)
            for (int64_t c = 0; c < cnch[rt][l]; c++)
              units[(size_t)cnt[(size_t)(c * mx / cnch[rt][l])]++] = ((unsigned long long)l << 32) | (unsigned long long)c;
          PX_CUDA(ctx, cudaMemcpyAsync(d_units[rt], units.data(), nu * 8, cudaMemcpyHostToDevice, ctx->stream));
          PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));  // units is a host vector
          ctx->chain_ukey[rt] = key;
        }
      }
      q += part[rt];
    }
    PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));  // host vectors are staged
    if (!dedup) d_rep = nullptr;
  }
  const int64_t NS = (N + 31) & ~(int64_t)31;  // latd row stride
  // B_R_LAT stages host outputs; the stitch ring reads up to 3 segments past a row's last query
  uint32_t *latd = (uint32_t *)px_buf(ctx, B_R_LATD, (size_t)S * NS * 4 + 3 * RSEG * 4 + 64);
  if (!latd) return px_fail(ctx, PROTEUS_ENOMEM, "latency scratch");
  const int64_t nmax = NCH[0] > NCH[1] ? NCH[0] : NCH[1];
  ChunkSt *csb[2] = {nullptr, nullptr};  // chunk runs, double-buffered across fix-up rounds
  unsigned *d_changed = d_flags + 4;  // [0] chunk exits changed, [1] lanes left to the stitch
  unsigned *d_lstat = (unsigned *)px_buf(ctx, B_R_VOFF, (size_t)S * D * 24 + 64);
  if (!d_lstat) return px_fail(ctx, PROTEUS_ENOMEM, "lane statistics");
  int64_t *d_lstart = (int64_t *)(((uintptr_t)(d_lstat + 2 * (size_t)S * D) + 15) & ~(uintptr_t)15);
  PX_CUDA(ctx, cudaMemsetAsync(d_lstat, 0, (size_t)S * D * 8, ctx->stream));
  PX_CUDA(ctx, cudaMemsetAsync(d_lstart, 0xFF, (size_t)S * D * 16, ctx->stream));  // head -1: not scanned
  const bool use_bscan = !simple && env_int("PROTEUS_REPLAY_BSCAN", 0) != 0;
  if (!simple) {
    csb[0] = (ChunkSt *)px_buf(ctx, B_R_LANE, sizeof(ChunkSt) * (size_t)S * (nmax + 1));
    csb[1] = (ChunkSt *)px_buf(ctx, B_R_VEX, sizeof(ChunkSt) * (size_t)S * (nmax + 1));
    if (!csb[0] || !csb[1]) return px_fail(ctx, PROTEUS_ENOMEM, "chunk states");
    PX_CUDA(ctx, cudaFuncSetAttribute(k_stitch, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      (int)stitch_smem(ctx->bmax)));
  }
  for (int rt = 0; rt < 2; rt++) {
    if (scl[rt].empty()) continue;
    int32_t *d_ccov = nullptr;             // chain lanes whose counts k_chain folded (k_chain_agg)
    unsigned long long *d_lcnt = nullptr;
    LaneArgs la;
    memset(&la, 0, sizeof la);
    la.S = S; la.D = D; la.M = M; la.bmax = ctx->bmax; la.nsc = (int)scl[2 + rt].size(); la.CH = CH;
    la.N = N; la.NS = NS; la.NCH = nmax;  // one row stride for both routing modes
    la.WU = env_int("PROTEUS_REPLAY_WARMUP", 0);
    la.WU = la.WU < 0 ? 0 : la.WU;
    la.option = d_opt; la.dev_type = d_dev; la.lat = ctx->d_lat; la.sc_list = d_scl + (2 + rt) * S; la.lp = d_lp;
    la.devOff = devOff[rt]; la.choff = d_choff + rt * (PX_MAXD + 2); la.goff = d_goff + rt * (PX_MAXD + 2);
    la.devArr = devArr[rt]; la.latd = latd; la.cs = csb[0]; la.csp = nullptr; la.agg = d_agg;
    la.debug = env_int("PROTEUS_REPLAY_DEBUG", 0);
    la.maxchk = env_int("PROTEUS_REPLAY_CHECKS", 1 << 30);
    la.scan1 = use_scan1 ? 1 : 0;
    la.dmask = D >= 64 ? ~0ull : ((1ull << D) - 1);
    la.lstat = d_lstat;
    la.lstart = d_lstart;
    la.bsearch = env_int("PROTEUS_STITCH_BSEARCH", 0);
    la.skip = d_chainf;
    if (la.nsc > 0) {  // §5 scenarios
    if (use_scan1) {  // Bmax = 1 lanes: exact prefix-maximum scan
      Scan1Args sa;
      memset(&sa, 0, sizeof sa);
      sa.D = D; sa.nsc = la.nsc; sa.N = N; sa.NS = NS;
      std::vector<int32_t> t1(D, 0);
      int64_t nb = 0;
      for (int d = 0; d < D; d++) {
        sa.boff[d] = nb;
        bool any = false;
        for (int k : scl[2 + rt]) any |= hB[(size_t)k * D + d] == 1;
        if (!any) continue;
        t1[d] = hT1[d];
        nb += (h_off[rt][d + 1] - h_off[rt][d] + SCAN_BLK - 1) / SCAN_BLK;
      }
      sa.boff[D] = nb;
      if (nb > 0) {
        char *sb2 = (char *)px_buf(ctx, B_R_SCAN, (size_t)nb * 16 + (size_t)D * 4 + 64);
        if (!sb2) return px_fail(ctx, PROTEUS_ENOMEM, "scan buffers");
        sa.bmx = (int64_t *)sb2;
        sa.bpre = sa.bmx + nb;
        int32_t *d_t1 = (int32_t *)(sa.bpre + nb);
        PX_CUDA(ctx, cudaMemcpyAsync(d_t1, t1.data(), D * 4, cudaMemcpyHostToDevice, ctx->stream));
        sa.T1 = d_t1; sa.devOff = devOff[rt]; sa.devArr = devArr[rt]; sa.sc_list = d_scl + (2 + rt) * S; sa.lp = d_lp;
        sa.latd = latd;
        if (nb > 0x7fffffff) return px_fail(ctx, PROTEUS_ERANGE, "scan blocks");
        PX_LAUNCH(ctx, "replay_scan1", k_scan1_reduce, (unsigned)nb, 256, 0, sa);
        PX_LAUNCH(ctx, "replay_scan1", k_scan1_prefix, D, 32, 0, sa);
        PX_LAUNCH(ctx, "replay_scan1", k_scan1_apply, (unsigned)nb, 256, 0, sa);
      }
    }
    // chain lanes (k_chain): alongside the chunk runs + stitch when both have
    // lanes (on the main stream after the fork, at most CHAIN_OCC blocks per SM
    // so that stitch blocks still fit), else alone
    ChainArgs ca;
    memset(&ca, 0, sizeof ca);
    const bool chain_now = use_chain && !clid[rt].empty();
    // the chain lanes' counts are folded into its writers (k_chain_agg adds
    // them, k_count skips those lanes) when the counts come from the rows
    const bool fold_counts = (!d_lat_out || env_int("PROTEUS_REPLAY_FINISH", 0) == 0) &&
                             env_int("PROTEUS_REPLAY_CHAIN_COUNTS", 1) != 0;
    if (chain_now && fold_counts) {
      const int nl = (int)clid[rt].size();
      char *cc = (char *)px_buf(ctx, B_R_CCNT, (size_t)S * D * 4 + (size_t)nl * 8 + 64);
      if (!cc) return px_fail(ctx, PROTEUS_ENOMEM, "chain counts");
      std::vector<int32_t> cov((size_t)S * D, -1);
      for (int l = 0; l < nl; l++) cov[clid[rt][l]] = l;
      for (int k : scl[2 + rt])  // duplicates read their representative's row
        for (int d = 0; d < D; d++) {
          const int r = hrep[(size_t)k * (D + 1) + d];
          if (r != k && cov[(size_t)r * D + d] >= 0) cov[(size_t)k * D + d] = cov[(size_t)r * D + d];
        }
      ca.lcnt = (unsigned long long *)(cc + (((size_t)S * D * 4 + 15) & ~(size_t)15));
      d_ccov = (int32_t *)cc;
      d_lcnt = ca.lcnt;
      PX_CUDA(ctx, cudaMemcpyAsync(d_ccov, cov.data(), cov.size() * 4, cudaMemcpyHostToDevice, ctx->stream));
      PX_CUDA(ctx, cudaMemsetAsync(ca.lcnt, 0, (size_t)nl * 8, ctx->stream));
      PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));  // cov is a host vector
    }
    size_t smc = 0;
    int chain_nsm = 0, chain_occ = 0;
    if (chain_now) {
      const int nl = (int)clid[rt].size();
      ca.D = D; ca.M = M; ca.bmax = ctx->bmax; ca.nl = nl; ca.C = CHN;
      ca.K = std::max(0, env_int("PROTEUS_REPLAY_CHAIN_K", 16));
      ca.SEG = std::min(CHN, std::max(CHAIN_SEGMIN, env_int("PROTEUS_REPLAY_CHAIN_SEG", 128)));
      ca.NS = NS; ca.maxch = cmax[rt]; ca.nunits = nunits[rt];
      ca.lid = (const int32_t *)cbuf[rt]; ca.nch = ca.lid + nl; ca.cmode = (const uint8_t *)(cbuf[rt] + (size_t)nl * 8);
      ca.counter = (unsigned long long *)(cbuf[rt] + chain_ctroff(nl));
      ca.watchdog = (unsigned *)(ca.counter + 1);
      ca.ex = (unsigned long long *)(cbuf[rt] + chain_exoff(nl));
      ca.units = d_units[rt];
      ca.lp = d_lp; ca.option = d_opt; ca.dev_type = d_dev; ca.lat = ctx->d_lat;
      ca.devOff = devOff[rt]; ca.devArr = devArr[rt]; ca.latd = latd;
      smc = chain_smem(CHN, ctx->bmax, ca.SEG);
      PX_CUDA(ctx, cudaFuncSetAttribute(k_chain<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smc));
      PX_CUDA(ctx, cudaDeviceGetAttribute(&chain_nsm, cudaDevAttrMultiProcessorCount, ctx->device));
      const int orc = px_occupancy(ctx, (const void *)k_chain<false>, CHAIN_THREADS, smc, &chain_occ);
      if (orc) return orc;
      chain_occ = chain_occ > 0 ? chain_occ : 1;
#ifdef PX_CHAIN_DEBUG
      ca.dbg = (unsigned long long *)px_buf(ctx, B_R_VLAT, (16 + 3 * (size_t)nl) * 8);
      PX_CUDA(ctx, cudaMemsetAsync(ca.dbg, 0, (16 + 3 * (size_t)nl) * 8, ctx->stream));
#endif
    }
    auto launch_chain = [&](int occ_cap) -> int {
      const int64_t nb = std::min<int64_t>(ca.nunits, (int64_t)chain_nsm * std::min(chain_occ, occ_cap));
      PX_LAUNCH(ctx, "replay_chain", k_chain<false>, (unsigned)nb, CHAIN_THREADS, smc, ca);
      return 0;
    };
    const bool chain_beside = chain_now && !simple && ngroups[rt] > 0 && crest[rt] &&
                              env_int("PROTEUS_REPLAY_CHAIN_BESIDE", 0) != 0 &&
                              env_int("PROTEUS_REPLAY_OVERLAP", 1) != 0 && max_rounds == 0 && !la.debug;
    if (chain_now && !chain_beside) {
      const int rc = launch_chain(1 << 20);
      if (rc) return rc;
    }
    if (simple) {
      const int nl = la.nsc * D;
      PX_LAUNCH(ctx, "replay_lanes", k_lanes, (nl + LANE_THREADS - 1) / LANE_THREADS, LANE_THREADS, 0, la);
    } else if (ngroups[rt] > 0 && crest[rt]) {
      if ((ngroups[rt] + 3) / 4 > 65535 || (NCH[rt] + 3) / 4 > 65535)
        return px_fail(ctx, PROTEUS_ERANGE, "too many replay chunks");
      dim3 grid((unsigned)la.nsc, (unsigned)((ngroups[rt] + 3) / 4));
      // pipelining: the stitch runs on an auxiliary stream alongside the chunk
      // runs and waits for each chunk it reads (ready flags), so the critical
      // lanes start at once instead of after every chunk run of every lane
      const bool overlap = env_int("PROTEUS_REPLAY_OVERLAP", 1) != 0 && max_rounds == 0 && !use_bscan && !la.debug &&
                           env_int("PROTEUS_REPLAY_TABLES", 0) == 0;
      if (overlap) {
        unsigned *cready0 = (unsigned *)px_buf(ctx, B_R_READY, (size_t)S * nmax * 4 + (size_t)S * D * 4 + 64);
        if (!cready0) return px_fail(ctx, PROTEUS_ENOMEM, "chunk flags");
        unsigned *cready = cready0 + 4;  // cready[-1]: watchdog
        PX_CUDA(ctx, cudaMemsetAsync(cready0, 0, (size_t)S * nmax * 4 + 16, ctx->stream));
        if (!ctx->aux) {
          // the stitch on the highest-priority stream, the chunk runs on the lowest
          int lo = 0, hi = 0;
          PX_CUDA(ctx, cudaDeviceGetStreamPriorityRange(&lo, &hi));
          PX_CUDA(ctx, cudaStreamCreateWithPriority(&ctx->aux, cudaStreamNonBlocking, lo));
          PX_CUDA(ctx, cudaStreamCreateWithPriority(&ctx->aux_hi, cudaStreamNonBlocking, hi));
          PX_CUDA(ctx, cudaEventCreateWithFlags(&ctx->ev_fork, cudaEventDisableTiming));
          PX_CUDA(ctx, cudaEventCreateWithFlags(&ctx->ev_join, cudaEventDisableTiming));
          PX_CUDA(ctx, cudaEventCreateWithFlags(&ctx->ev_join2, cudaEventDisableTiming));
        }
        la.cready = cready;
        // stitch lanes longest first (device load, then Bmax): with the stitch on the
        // high-priority stream they hold the SMs from the start while the chunk runs
        // fill the rest (a stitch block needs > half an SM's shared memory, so an SM
        // never holds two, and chunk-run blocks always fit beside it: no deadlock)
        {
          std::vector<int32_t> ord((size_t)la.nsc * D);
          for (size_t i = 0; i < ord.size(); i++) ord[i] = (int32_t)i;
          std::stable_sort(ord.begin(), ord.end(), [&](int32_t x, int32_t y) {
            const int dx = x % D, dy = y % D;
            const int64_t nx = h_off[rt][dx + 1] - h_off[rt][dx], ny = h_off[rt][dy + 1] - h_off[rt][dy];
            if (nx != ny) return nx > ny;
            return hB[(size_t)scl[2 + rt][x / D] * D + dx] > hB[(size_t)scl[2 + rt][y / D] * D + dy];
          });
          int32_t *d_ord = (int32_t *)(cready0 + 4 + (size_t)S * nmax);
          PX_CUDA(ctx, cudaMemcpyAsync(d_ord, ord.data(), ord.size() * 4, cudaMemcpyHostToDevice, ctx->stream));
          PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));  // ord is a host vector
          la.lane_order = d_ord;
        }
        PX_CUDA(ctx, cudaEventRecord(ctx->ev_fork, ctx->stream));
        PX_CUDA(ctx, cudaStreamWaitEvent(ctx->aux, ctx->ev_fork, 0));
        PX_CUDA(ctx, cudaStreamWaitEvent(ctx->aux_hi, ctx->ev_fork, 0));
        if (chain_beside) {
          const int rc = launch_chain(std::max(1, env_int("PROTEUS_REPLAY_CHAIN_OCC", 2)));
          if (rc) return rc;
        }
        cudaStream_t main = ctx->stream;
        const int64_t warps = (int64_t)la.nsc * D;
        int rcs = 0;
        ctx->stream = ctx->aux;
        px_launch_begin(ctx, "replay_spec");
        k_spec<<<grid, 128, 0, ctx->stream>>>(la);
        rcs = px_launch_end(ctx);
        if (!rcs) {
          ctx->stream = ctx->aux_hi;
          px_launch_begin(ctx, "replay_stitch");
          k_stitch<<<(unsigned)((warps + 3) / 4), 128, stitch_smem(ctx->bmax), ctx->stream>>>(la);
          rcs = px_launch_end(ctx);
        }
        ctx->stream = main;
        if (rcs) return rcs;
        PX_CUDA(ctx, cudaEventRecord(ctx->ev_join, ctx->aux));
        PX_CUDA(ctx, cudaEventRecord(ctx->ev_join2, ctx->aux_hi));
        PX_CUDA(ctx, cudaStreamWaitEvent(ctx->stream, ctx->ev_join, 0));
        PX_CUDA(ctx, cudaStreamWaitEvent(ctx->stream, ctx->ev_join2, 0));
        unsigned wd = 0;
        PX_CUDA(ctx, cudaMemcpyAsync(&wd, cready - 1, 4, cudaMemcpyDeviceToHost, ctx->stream));
        PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
        if (wd) return px_fail(ctx, PROTEUS_EINTERNAL, "replay: pipelined stitch waited too long for a chunk run");
        la.cready = nullptr;
        la.lane_order = nullptr;
      } else {
      PX_LAUNCH(ctx, "replay_spec", k_spec, grid, 128, 0, la);
      // backlogged lanes (k_spec's statistics): full-batch prefix-maximum scan
      if (use_bscan) {
        std::vector<int32_t> lid;
        std::vector<int64_t> loff(1, 0);
        for (int k : scl[2 + rt])
          for (int d = 0; d < D; d++) {
            const int B = hB[(size_t)k * D + d];
            const int64_t nd = h_off[rt][d + 1] - h_off[rt][d];
            if (B < 2 || nd < B) continue;
            lid.push_back(k * D + d);
            loff.push_back(loff.back() + (nd / B + BSCAN_BLK - 1) / BSCAN_BLK);
          }
        const int nl = (int)lid.size();
        const int64_t nb = loff.back();
        if (nl > 0 && nb > 0) {
          if (nb > 0x7fffffff) return px_fail(ctx, PROTEUS_ERANGE, "scan blocks");
          char *bb = (char *)px_buf(ctx, B_R_BSCAN, (size_t)(nl + 1) * 8 + (size_t)nl * 4 + (size_t)nb * 16 +
                                                        (size_t)nl * 8 + 256);
          if (!bb) return px_fail(ctx, PROTEUS_ENOMEM, "scan buffers");
          BScanArgs ba;
          memset(&ba, 0, sizeof ba);
          int64_t *d_loff = (int64_t *)bb;
          ba.bmx = d_loff + (nl + 1);
          ba.bpre = ba.bmx + nb;
          ba.vio = (unsigned long long *)(ba.bpre + nb);
          int32_t *d_lid = (int32_t *)(ba.vio + nl);
          PX_CUDA(ctx, cudaMemcpyAsync(d_loff, loff.data(), loff.size() * 8, cudaMemcpyHostToDevice, ctx->stream));
          PX_CUDA(ctx, cudaMemcpyAsync(d_lid, lid.data(), lid.size() * 4, cudaMemcpyHostToDevice, ctx->stream));
          PX_CUDA(ctx, cudaMemsetAsync(ba.vio, 0xFF, (size_t)nl * 8, ctx->stream));
          ba.D = D; ba.nl = nl; ba.NS = NS; ba.loff = d_loff; ba.lid = d_lid; ba.devOff = devOff[rt];
          ba.devArr = devArr[rt]; ba.lat = ctx->d_lat; ba.option = d_opt; ba.dev_type = d_dev; ba.M = M;
          ba.bmax = ctx->bmax; ba.lp = d_lp; ba.lstat = d_lstat; ba.latd = latd; ba.lstart = d_lstart;
          PX_LAUNCH(ctx, "replay_bscan", k_bscan_reduce, (unsigned)nb, 256, 0, ba);
          PX_LAUNCH(ctx, "replay_bscan", k_bscan_prefix, nl, 32, 0, ba);
          PX_LAUNCH(ctx, "replay_bscan", k_bscan_verify, (unsigned)nb, 256, 0, ba);
          PX_LAUNCH(ctx, "replay_bscan", k_bscan_apply, (unsigned)nb, 256, 0, ba);
        }
      }
      if (la.debug) {  // diagnostic: speculative decisions per lane
        std::vector<unsigned> hs((size_t)2 * S * D);
        PX_CUDA(ctx, cudaMemcpyAsync(hs.data(), d_lstat, hs.size() * 4, cudaMemcpyDeviceToHost, ctx->stream));
        PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
        unsigned long long tot = 0, full = 0;
        for (int k : scl[2 + rt])
          for (int d = 0; d < D; d++) { tot += hs[2 * ((size_t)k * D + d) + 1]; full += hs[2 * ((size_t)k * D + d)]; }
        fprintf(stderr, "replay routing %d: %llu speculative decisions, %llu full-immediate\n", rt, tot, full);
        for (int d = 0; d < D; d++) {
          unsigned long long t = 0;
          for (int k : scl[2 + rt]) t += hs[2 * ((size_t)k * D + d) + 1];
          fprintf(stderr, "  device %d: n=%lld decisions=%llu\n", d, (long long)(h_off[rt][d + 1] - h_off[rt][d]), t);
        }
      }
      // fix-up rounds until no chunk exit changes (then every chunk is exact)
      int cur = 0;
      bool done = false;
      for (int r = 1; r <= max_rounds; r++) {
        la.csp = csb[cur];
        la.cs = csb[cur ^ 1];
        PX_CUDA(ctx, cudaMemsetAsync(d_changed, 0, 8, ctx->stream));
        dim3 gf((unsigned)la.nsc, (unsigned)((NCH[rt] + 3) / 4));
        PX_LAUNCH(ctx, "replay_fix", k_fix, gf, 128, 0, la, d_changed);
        cur ^= 1;
        unsigned changed[2] = {0, 0};
        PX_CUDA(ctx, cudaMemcpyAsync(changed, d_changed, 8, cudaMemcpyDeviceToHost, ctx->stream));
        PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
        if (la.debug) fprintf(stderr, "replay routing %d fix-up round %d: %u chunk exits changed\n", rt, r, changed[0]);
        if (changed[0] == 0) { done = changed[1] == 0; break; }
      }
      la.cs = csb[cur];
      la.csp = nullptr;
      if (!done) {  // the sequential stitch carries the true state through the rest
        // chunk tables for the lanes with large Bmax (slow-merging runs): the
        // stitch hops a chunk entered on the idle branch, k_rewrite replays it
        const int minB = env_int("PROTEUS_REPLAY_TABLES_MINB", 8);
        const bool tables = env_int("PROTEUS_REPLAY_TABLES", 0) != 0 && CH <= 8192;  // measured slower on c5
        std::vector<int32_t> tEv((size_t)la.nsc * D, 0);
        std::vector<int64_t> trecoff((size_t)la.nsc * D, 0);
        int64_t ntrec = 0;
        const int64_t nchd = nmax;
        if (tables) {
          for (int i = 0; i < la.nsc; i++)
            for (int d = 0; d < D; d++) {
              const int B = hB[(size_t)scl[2 + rt][i] * D + d];
              const int E = (B >= minB && B <= WIN_EMAX && B > 1) ? B : 0;
              tEv[(size_t)i * D + d] = E;
              trecoff[(size_t)i * D + d] = ntrec;
              ntrec += (int64_t)E * nchd;
            }
        }
        if (ntrec > 0) {
          char *aux = (char *)px_buf(ctx, B_W_AUX, (size_t)la.nsc * D * 12 + (size_t)S * D + 256);
          WinRec *d_trec = (WinRec *)px_buf(ctx, B_W_REC, sizeof(WinRec) * (size_t)ntrec + 64);
          WinEntry *d_rw = (WinEntry *)px_buf(ctx, B_W_ENT, sizeof(WinEntry) * (size_t)la.nsc * D * nchd + 64);
          if (!aux || !d_trec || !d_rw) return px_fail(ctx, PROTEUS_ENOMEM, "chunk tables");
          int64_t *d_trecoff = (int64_t *)aux;
          int32_t *d_tE = (int32_t *)(d_trecoff + (size_t)la.nsc * D);
          uint8_t *d_mono = (uint8_t *)(d_tE + (size_t)la.nsc * D);
          PX_CUDA(ctx, cudaMemcpyAsync(d_trecoff, trecoff.data(), trecoff.size() * 8, cudaMemcpyHostToDevice,
                                       ctx->stream));
          PX_CUDA(ctx, cudaMemcpyAsync(d_tE, tEv.data(), tEv.size() * 4, cudaMemcpyHostToDevice, ctx->stream));
          PX_CUDA(ctx, cudaMemcpyAsync(d_mono, hmono.data(), (size_t)S * D, cudaMemcpyHostToDevice, ctx->stream));
          PX_CUDA(ctx, cudaMemsetAsync(d_rw, 0, sizeof(WinEntry) * (size_t)la.nsc * D * nchd, ctx->stream));
          WinArgs wa;
          memset(&wa, 0, sizeof wa);
          wa.S = S; wa.D = D; wa.M = M; wa.bmax = ctx->bmax; wa.nsc = la.nsc; wa.WT = 1; wa.D1 = D + 1; wa.CHF = CH;
          wa.N = N; wa.nw = nchd; wa.ntiles = ntiles;
          wa.option = d_opt; wa.dev_type = d_dev; wa.lat = ctx->d_lat; wa.sc_list = la.sc_list; wa.lp = d_lp;
          wa.mono = d_mono; wa.devOff = devOff[rt]; wa.devArr = devArr[rt]; wa.recoff = d_trecoff; wa.E = d_tE;
          wa.rec = d_trec;
          const size_t smt = (size_t)(CH + WIN_EXT) * 4 + (size_t)WIN_WARPS * CH;
          PX_CUDA(ctx, cudaFuncSetAttribute(k_win_tables, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smt));
          PX_LAUNCH(ctx, "replay_tables", k_win_tables, (unsigned)(nchd * D), WIN_WARPS * 32, smt, wa);
          PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));  // host vectors staged
          la.trec = d_trec; la.trecoff = d_trecoff; la.tE = d_tE; la.rw = d_rw;
        }
        const int64_t warps = (int64_t)la.nsc * D;
        PX_LAUNCH(ctx, "replay_stitch", k_stitch, (unsigned)((warps + 3) / 4), 128, stitch_smem(ctx->bmax), la);
        if (ntrec > 0) {
          const int64_t nt = (int64_t)la.nsc * D * nchd;
          PX_LAUNCH(ctx, "replay_rewrite", k_rewrite, (unsigned)((nt + 127) / 128), 128, 0, la);
        }
        la.trec = nullptr; la.trecoff = nullptr; la.tE = nullptr; la.rw = nullptr;
      }
      }  // not pipelined
    }
    if (chain_now) {
#ifdef PX_CHAIN_DEBUG
      {
        unsigned long long hd[16];
        PX_CUDA(ctx, cudaMemcpyAsync(hd, ca.dbg, 16 * 8, cudaMemcpyDeviceToHost, ctx->stream));
        PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
        fprintf(stderr, "chain rt %d: lanes %d units %llu batches %llu hops %llu | cycles/unit load %.0f "
                "idle %.0f runs %.0f scan %.0f wait %.0f link %.0f rec %.0f write %.0f\n", rt, ca.nl, hd[8], hd[9],
                hd[10], hd[0] / (double)hd[8], hd[1] / (double)hd[8], hd[2] / (double)hd[8], hd[3] / (double)hd[8],
                hd[4] / (double)hd[8], hd[5] / (double)hd[8], hd[7] / (double)hd[8], hd[6] / (double)hd[8]);
        std::vector<unsigned long long> pl(3 * (size_t)ca.nl);
        PX_CUDA(ctx, cudaMemcpyAsync(pl.data(), ca.dbg + 16, pl.size() * 8, cudaMemcpyDeviceToHost, ctx->stream));
        PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
        std::vector<int> ord(ca.nl);
        for (int i = 0; i < ca.nl; i++) ord[i] = i;
        std::sort(ord.begin(), ord.end(), [&](int x, int y) { return pl[3 * x] > pl[3 * y]; });
        for (int k = 0; k < std::min(ca.nl, 12); k++) {
          const int l = ord[k], lid = clid[rt][l];
          fprintf(stderr, "  chain lane s=%d d=%d B=%d chunks=%d mode=%d: link Mcyc %.2f hops %llu wait Mcyc %.2f\n",
                  lid / D, lid % D, hB[lid], cnch[rt][l], (int)cmodev[rt][l], pl[3 * l] / 1e6, pl[3 * l + 1],
                  pl[3 * l + 2] / 1e6);
        }
      }
#endif
      unsigned wd = 0;
      PX_CUDA(ctx, cudaMemcpyAsync(&wd, ca.watchdog, 4, cudaMemcpyDeviceToHost, ctx->stream));
      PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
      if (wd) return px_fail(ctx, PROTEUS_EINTERNAL, "replay: chain wait for a previous chunk timed out");
    }
    }  // §5 scenarios
    if (!scl[4 + rt].empty()) {  // §8(f2) baseline batchers: chunk runs, then warp per (device, scenario)
      LaneArgs lb = la;
      lb.nsc = (int)scl[4 + rt].size();
      lb.sc_list = d_scl + (4 + rt) * S;
      lb.wst = nullptr;
      lb.wx = nullptr;
      // chunk runs for the AIMD scenarios only: an overloaded Nexus lane never finds the
      // device free, so its runs never meet (measured: no gain, +6 % for the runs)
      if (env_int("PROTEUS_REPLAY_WCSPEC", 1) && !scl[6 + rt].empty() && (NCH[rt] + 127) / 128 <= 65535 &&
          NCH[rt] > 0) {
        uint8_t *wst = (uint8_t *)px_buf(ctx, B_R_WST, (size_t)S * NS + 16);
        WcExit *wx = (WcExit *)px_buf(ctx, B_R_WEX, sizeof(WcExit) * (size_t)S * nmax + 16);
        if (!wst || !wx) return px_fail(ctx, PROTEUS_ENOMEM, "baseline chunk runs");
        for (int k : scl[4 + rt])
          PX_CUDA(ctx, cudaMemsetAsync(wst + (size_t)k * NS, 0, (size_t)NS, ctx->stream));
        lb.wst = wst;
        lb.wx = wx;
        LaneArgs la2 = lb;
        la2.nsc = (int)scl[6 + rt].size();
        la2.sc_list = d_scl + (6 + rt) * S;
        dim3 gs((unsigned)la2.nsc, (unsigned)((NCH[rt] + 127) / 128));
        PX_LAUNCH(ctx, "replay_baseline", k_wc_spec, gs, 128, 0, la2);
      }
      const int64_t warps = (int64_t)lb.nsc * D;
      // Nexus lanes predicted at or past overload at their batch size (rho =
      // lambda T(B) / B, lambda the device's mean rate): k_wc_lanes walks them
      // to their first overload stretch, the scan (k_nx_*) takes the stretch
      // as far as it is valid, the second walk the rest
      if (!simple && env_int("PROTEUS_REPLAY_NXSCAN", 0) != 0) {  // opt-in: measured slower on c5
        const double rho_min = env_int("PROTEUS_REPLAY_NXSCAN_RHO_PCT", 95) / 100.0;
        const double span = (double)h_span[1] - (double)h_span[0];
        std::vector<uint8_t> sel((size_t)S * D, 0);
        std::vector<int32_t> lid;
        std::vector<int64_t> loff(1, 0);
        for (int k : scl[4 + rt]) {
          if (h_sc[k].policy != 1) continue;
          for (int d = 0; d < D; d++) {
            if (h_option[d] <= 0 || hskip[(size_t)k * D + d]) continue;
            const int32_t *Tr = ctx->lat.data() + ((size_t)h_dev_type[d] * M + (h_option[d] - 1)) * ctx->bmax;
            const int64_t L = lane_L(k, d);
            int Bn = 1;
            for (int b = 1; b <= hB[(size_t)k * D + d]; b++)
              if (2 * (int64_t)Tr[b - 1] <= L) Bn = b;
            const int64_t nd = h_off[rt][d + 1] - h_off[rt][d];
            const double lam = span > 0 ? (double)nd / span : 0.0;
            if (nd < 2 * Bn || lam * (double)Tr[Bn - 1] / (double)Bn < rho_min) continue;
            sel[(size_t)k * D + d] = 1;
            lid.push_back(k * D + d);
            loff.push_back(loff.back() + (nd / Bn + NX_BLK) / NX_BLK);
          }
        }
        const int nl = (int)lid.size();
        const int64_t nb = loff.back();
        if (nl > 0) {
          if (nb > 0x7fffffff) return px_fail(ctx, PROTEUS_ERANGE, "scan blocks");
          const size_t o_loff = ((size_t)S * D + 15) & ~(size_t)15, o_lid = o_loff + (size_t)(nl + 1) * 8,
                       o_b = (o_lid + (size_t)nl * 4 + 15) & ~(size_t)15, o_vio = o_b + (size_t)nb * 16,
                       o_st = o_vio + (size_t)nl * 8, o_ik = o_st + (size_t)nl * 16,
                       tot = o_ik + (size_t)nb * NX_BLK * 4;
          char *nx = (char *)px_buf(ctx, B_R_NX, tot + 64);
          if (!nx) return px_fail(ctx, PROTEUS_ENOMEM, "Nexus scan buffers");
          PX_CUDA(ctx, cudaMemcpyAsync(nx, sel.data(), sel.size(), cudaMemcpyHostToDevice, ctx->stream));
          PX_CUDA(ctx, cudaMemcpyAsync(nx + o_loff, loff.data(), loff.size() * 8, cudaMemcpyHostToDevice, ctx->stream));
          PX_CUDA(ctx, cudaMemcpyAsync(nx + o_lid, lid.data(), lid.size() * 4, cudaMemcpyHostToDevice, ctx->stream));
          PX_CUDA(ctx, cudaMemsetAsync(nx + o_vio, 0xFF, (size_t)nl * 24, ctx->stream));  // vio, nxst
          NxArgs na;
          memset(&na, 0, sizeof na);
          na.D = D; na.nl = nl; na.NS = NS; na.loff = (const int64_t *)(nx + o_loff); na.lid = (const int32_t *)(nx + o_lid);
          na.devOff = devOff[rt]; na.devArr = devArr[rt]; na.lat = ctx->d_lat; na.option = d_opt; na.dev_type = d_dev;
          na.M = M; na.bmax = ctx->bmax; na.lp = d_lp; na.lstart = d_lstart; na.latd = latd;
          na.bmx = (int64_t *)(nx + o_b); na.bpre = na.bmx + nb; na.ik = (int32_t *)(nx + o_ik);
          na.vio = (unsigned long long *)(nx + o_vio);
          na.nxst = (int64_t *)(nx + o_st);
          lb.nxsel = (const uint8_t *)nx;
          lb.nxmode = 1;
          if (lb.wst) PX_LAUNCH(ctx, "replay_baseline", k_wc_lanes<true>, (unsigned)((warps + 3) / 4), 128, 0, lb);
          else PX_LAUNCH(ctx, "replay_baseline", k_wc_lanes<false>, (unsigned)((warps + 3) / 4), 128, 0, lb);
          PX_LAUNCH(ctx, "replay_nxscan", k_nx_reduce, (unsigned)nb, 256, 0, na);
          PX_LAUNCH(ctx, "replay_nxscan", k_nx_prefix, nl, 32, 0, na);
          PX_LAUNCH(ctx, "replay_nxscan", k_nx_verify, (unsigned)nb, 256, 0, na);
          PX_LAUNCH(ctx, "replay_nxscan", k_nx_apply, (unsigned)nb, 256, 0, na);
          PX_LAUNCH(ctx, "replay_nxscan", k_nx_commit, 1, 256, 0, na);
          lb.nxmode = 2;
          PX_LAUNCH(ctx, "replay_baseline", k_wc_lanes<false>, (unsigned)((warps + 3) / 4), 128, 0, lb);
          PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));  // sel / loff / lid are host vectors
        }
      }
      if (lb.nxmode == 2) {
        // done above
      } else if (lb.wst) PX_LAUNCH(ctx, "replay_baseline", k_wc_lanes<true>, (unsigned)((warps + 3) / 4), 128, 0, lb);
      else PX_LAUNCH(ctx, "replay_baseline", k_wc_lanes<false>, (unsigned)((warps + 3) / 4), 128, 0, lb);
    }
    if (!d_lat_out || env_int("PROTEUS_REPLAY_FINISH", 0) == 0) {  // counts from the device-major rows
      const int nall = (int)scl[rt].size();
      dim3 g(32, nall < 65535 ? nall : 65535);
      PX_LAUNCH(ctx, "replay_sink", k_sink, g, 256, 0, NS, S, D, d_scl + rt * S, nall, devOff[rt], latd, d_agg);
      dim3 cg((unsigned)((N + CNT_PER - 1) / CNT_PER), (unsigned)nall);
      if (d_ccov) {
        const int n5 = (int)scl[2 + rt].size();
        PX_LAUNCH(ctx, "replay_count", k_chain_agg, (n5 * D + 255) / 256, 256, 0, S, D, n5, d_scl + (2 + rt) * S, d_ccov,
                  d_lcnt, devOff[rt], d_lp, d_agg);
      }
      PX_LAUNCH(ctx, "replay_count", k_count, cg, 256, 0, N, NS, S, D, d_scl + rt * S, devOff[rt], d_lp, d_rep, latd,
                d_agg, d_ccov);
    }
    if (d_lat_out && d_rep && npair[rt] > 0) {  // the duplicate lanes' rows, for the un-permute
      int64_t maxn = 1;
      for (int d = 0; d < D; d++) maxn = std::max(maxn, h_off[rt][d + 1] - h_off[rt][d]);
      const unsigned gx = (unsigned)std::min<int64_t>(64, (maxn + 4095) / 4096);
      for (int64_t k0 = 0; k0 < npair[rt]; k0 += 65535) {
        const unsigned gy = (unsigned)std::min<int64_t>(65535, npair[rt] - k0);
        PX_LAUNCH(ctx, "replay_dupcopy", k_dupcopy, dim3(gx, gy), 256, 0, NS, d_pairs[rt] + 3 * k0, devOff[rt], latd);
      }
    }
  }
  if (d_lat_out) {
    const int64_t nb = (N + 256 * UNP_PER - 1) / (256 * UNP_PER);
    if (env_int("PROTEUS_REPLAY_FINISH", 0) == 0) {
      PX_LAUNCH(ctx, "replay_unpermute", k_unpermute, (unsigned)nb, 256, 0, N, NS, S, d_sc, inv[0], inv[1], latd,
                d_lat_out);
    } else {  // latencies in query order and the counts in one pass
      const int64_t nf = (N + 256 * FIN_PER - 1) / (256 * FIN_PER);
      PX_LAUNCH(ctx, "replay_finish", k_finish, (unsigned)nf, 256, 0, N, NS, S, D, d_sc, inv[0], inv[1], tgt_rt[0],
                tgt_rt[1], d_lp, latd, d_lat_out, d_agg);
    }
  }
  return 0;
}

// ============================================================ §8(f4) ======
// Closed loop (readings F1-F4): allocation e serves the queries
// arriving in epoch e = floor(a / epoch_us) (the per-second re-solve,
// P:707-723).  Routing restarts every epoch (SWRR over z[e] with
// the sink, R8); a device finishes one epoch's queue with that epoch's variant
// before serving the next epoch's queries (a batch holds one epoch), so a
// device's array is a sequence of (device, epoch) segments replayed with the
// §5 rule, the device state F carried from segment to segment.
//   phase A  every segment from an idle device, in parallel (k_ep_spec);
//   phase B  per (device, scenario), the true F carried over the epochs: a
//            segment whose first query arrives at or after F takes exactly the
//            idle run's decisions (t = max(F, a_head) = a_head) and is kept,
//            otherwise it is replayed from F (k_ep_stitch).

// SWRR pattern per (epoch, family): weights w[(e * Q + q) * (D + 1) + d] (the
// sink is member D), one warp per pattern (as k_route_prepare)
__global__ void k_ep_patterns(int EQ, int D, const int32_t *__restrict__ w, const int64_t *__restrict__ poff,
                              const int32_t *__restrict__ plen, uint8_t *pattern) {
  const int eq = blockIdx.x, lane = threadIdx.x;
  if (eq >= EQ) return;
  const int32_t Wq = plen[eq];
  int32_t wl[3], cur[3];
#pragma unroll
  for (int i = 0; i < 3; i++) {
    const int d = lane + 32 * i;
    wl[i] = d <= D ? w[(size_t)eq * (D + 1) + d] : 0;
    cur[i] = 0;
  }
  uint8_t *pat = pattern + poff[eq];
  for (int32_t k = 0; k < Wq; k++) {
    long long key = LLONG_MIN;
#pragma unroll
    for (int i = 0; i < 3; i++) {
      if (wl[i] == 0) continue;
      cur[i] += wl[i];
      const long long kk = ((long long)cur[i] << 32) | (0xFFFFFFFFu - (uint32_t)(lane + 32 * i));
      key = kk > key ? kk : key;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
      const long long v = __shfl_xor_sync(0xffffffffu, key, o);
      key = v > key ? v : key;
    }
    const int best = (int)(0xFFFFFFFFu - (uint32_t)(key & 0xFFFFFFFFll));
#pragma unroll
    for (int i = 0; i < 3; i++)
      if (best == lane + 32 * i) cur[i] -= Wq;
    if (lane == 0) pat[k] = (uint8_t)best;
  }
}

// per (epoch, family) counts; flags bit 3: an arrival beyond the last epoch
__global__ void k_ep_hist(const uint32_t *__restrict__ arr, const uint8_t *__restrict__ fam, int64_t N, int E,
                          int64_t epoch_us, int Q, int32_t *cntEQ, uint32_t *flags) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t e = (int64_t)arr[i] / epoch_us;
    if (e >= E) { atomicOr(flags, 8u); continue; }
    atomicAdd(cntEQ + e * Q + fam[i], 1);
  }
}

// family ordinal within the epoch -> target (as k_route_target, the ordinal
// made epoch-relative by the family's count before the epoch)
__global__ void k_ep_target(const uint8_t *__restrict__ fam, const uint32_t *__restrict__ arr, int64_t N, int Q,
                            int64_t epoch_us, const int32_t *__restrict__ famBase, const int32_t *__restrict__ fbEQ,
                            const uint8_t *__restrict__ pattern, const int64_t *__restrict__ poff,
                            const int32_t *__restrict__ plen, int D, uint8_t *target, int32_t *histDev) {
  __shared__ int32_t run[TILE_WARPS][PX_MAXQ];
  __shared__ int32_t cnt[TILE_WARPS][PX_MAXD + 2];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t tile = (int64_t)blockIdx.x * TILE_WARPS + w;
  const int64_t t0 = tile * TILE;
  if (t0 < N)
    for (int k = lane; k < Q; k += 32) run[w][k] = famBase[tile * Q + k];
  for (int k = lane; k <= D; k += 32) cnt[w][k] = 0;
  __syncthreads();
  if (t0 >= N) return;
  for (int c = 0; c < TILE; c += 32) {
    const int64_t i = t0 + c + lane;
    const bool valid = i < N;
    const int key = valid ? fam[i] : 255;
    const unsigned peers = __match_any_sync(0xffffffffu, key);
    const int rank = __popc(peers & ((1u << lane) - 1));
    int ord = 0;
    if (valid) ord = run[w][key] + rank;
    __syncwarp();
    if (valid && lane == __ffs(peers) - 1) run[w][key] += __popc(peers);
    int tgt = D;
    if (valid) {
      const int64_t eq = ((int64_t)arr[i] / epoch_us) * Q + key;
      const int len = plen[eq];
      tgt = len > 0 ? pattern[poff[eq] + ((ord - fbEQ[eq]) % len)] : D;
      target[i] = (uint8_t)tgt;
    }
    const unsigned tp = __match_any_sync(0xffffffffu, valid ? tgt : 255);
    if (valid && lane == __ffs(tp) - 1) cnt[w][tgt] += __popc(tp);
    __syncwarp();
  }
  for (int k = lane; k <= D; k += 32) histDev[tile * (D + 1) + k] = cnt[w][k];
}

// per (epoch, device) segment sizes (the sink is not a segment)
__global__ void k_ep_seghist(const uint8_t *__restrict__ target, const uint32_t *__restrict__ arr, int64_t N,
                             int64_t epoch_us, int D, int32_t *cntED) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    const int d = target[i];
    if (d < D) atomicAdd(cntED + ((int64_t)arr[i] / epoch_us) * D + d, 1);
  }
}

struct EpArgs {
  int E, D, M, bmax, S;
  int64_t NS;
  const int32_t *option;  // [E][D]
  const int32_t *dev_type, *lat, *acc, *fam_of_m, *slo;
  const proteus_scenario *sc;
  const int64_t *devOff;  // [D + 2]
  const int32_t *cntED, *segBase;  // [E][D]
  const uint32_t *devArr;
  uint32_t *latd;         // [S][NS]
  int64_t *exitF;         // [S][E][D]
};

struct EpLane {
  const int32_t *T;
  int Bmax;
  int64_t L;
};

__device__ __forceinline__ EpLane ep_lane(const EpArgs &a, int s, int e, int d) {
  EpLane r;
  const int o = a.option[(size_t)e * a.D + d];
  r.T = a.lat + ((size_t)a.dev_type[d] * a.M + (o - 1)) * a.bmax;
  int depth = 0;
  while (depth < a.bmax && r.T[depth] > 0) depth++;
  const int cap = a.sc[s].batch_cap;
  const int Bcap = (cap > 0 && cap < depth) ? cap : depth;
  r.L = (int64_t)a.sc[s].slo_mult_milli * a.slo[a.fam_of_m[o - 1]] / 1000;
  r.Bmax = 1;  // the maximum allowed batch size of the epoch's variant (reading R4')
  for (int b = 1; b <= Bcap; b++)
    if (2 * (int64_t)r.T[b - 1] <= r.L) r.Bmax = b;
  return r;
}

// replay one segment [st, st + n) of the device array from free time F; returns the exit F
__device__ __forceinline__ int64_t ep_walk(const EpArgs &a, int s, int e, int d, int64_t st, int64_t n, int64_t F) {
  const EpLane p = ep_lane(a, s, e, d);
  uint32_t *out = a.latd + (size_t)s * a.NS + st;
  if (p.Bmax < 1) {  // never routed to (z = 0 / depth 0); kept for safety
    for (int64_t j = 0; j < n; j++) out[j] = 0xFFFFFFFFu;
    return F;
  }
  GArr arr{a.devArr + st};
  int64_t h = 0;
  while (h < n) {
    int64_t t;
    const int b = decide(arr, n, h, F, p.Bmax, p.L, p.T, &t);
    F = t + p.T[b - 1];
    for (int j = 0; j < b; j++) out[h + j] = sat_lat(F - (int64_t)arr(h + j));
    h += b;
  }
  return F;
}

// the chain path's rule parameters per (scenario, epoch, device) (ep_lane):
// {Bmax, L, offset of the T(b) row in lat}; flags[0] |= 1 when a segment with
// queries is outside the chain's domain (Bmax outside [1, 255], T(b) not
// non-decreasing up to Bmax, L >= 2^30): the caller then takes the stitch
__global__ void k_ep_chparams(const __grid_constant__ EpArgs a, int32_t *epP, unsigned *flags) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= (int64_t)a.S * a.E * a.D) return;
  const int d = (int)(i % a.D), e = (int)((i / a.D) % a.E), s = (int)(i / ((int64_t)a.D * a.E));
  const int o = a.option[(size_t)e * a.D + d];
  int32_t *q = epP + i * 4;
  if (o <= 0) { q[0] = 1; q[1] = 0; q[2] = 0; q[3] = 0; return; }
  const EpLane p = ep_lane(a, s, e, d);
  q[0] = p.Bmax;
  q[1] = (int32_t)(p.L < (1ll << 30) ? p.L : 0);
  q[2] = (int32_t)(((size_t)a.dev_type[d] * a.M + (o - 1)) * a.bmax);
  q[3] = a.acc[o - 1];
  if (a.cntED[(size_t)e * a.D + d] > 0) {
    bool ok = p.Bmax >= 1 && p.Bmax <= 255 && p.L < (1ll << 30);
    for (int b = 1; ok && b < p.Bmax; b++) ok = p.T[b] >= p.T[b - 1];
    if (!ok) atomicOr(flags, 1u);
  }
}

// phase A: thread per (scenario, epoch, device) segment, from an idle device
__global__ void __launch_bounds__(128) k_ep_spec(const __grid_constant__ EpArgs a) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int s = blockIdx.y;
  if (i >= (int64_t)a.E * a.D) return;
  const int e = (int)(i / a.D), d = (int)(i % a.D);
  const int32_t n = a.cntED[i];
  if (n == 0) return;
  const int64_t st = a.devOff[d] + a.segBase[i];
  a.exitF[(size_t)s * a.E * a.D + i] = ep_walk(a, s, e, d, st, n, 0);
}

// phase B: warp per (scenario, device), the true state across the epochs.
// A re-walk takes one §5 decision per step with the lanes in parallel
// (decide_warp); arrivals come from a per-warp shared-memory ring over the
// device array.
__global__ void __launch_bounds__(128) k_ep_stitch(const __grid_constant__ EpArgs a) {
  __shared__ uint32_t sA[4][WC_RW];
  __shared__ uint32_t sL[4][WC_RW];  // the idle runs' latencies of the same positions
  __shared__ int32_t sT[4][PX_MAXB];
  const int wid = (int)((blockIdx.x * (unsigned)blockDim.x + threadIdx.x) >> 5), lane = threadIdx.x & 31;
  const int w = threadIdx.x >> 5;
  if (wid >= a.S * a.D) return;
  const int s = wid / a.D, d = wid % a.D;
  uint32_t *ring = sA[w];
  uint32_t *lring = sL[w];
  int32_t *T = sT[w];
  const int64_t dbase = a.devOff[d], dn = a.devOff[d + 1] - dbase;  // the device's array
  const uint32_t *arr = a.devArr + dbase;
  uint32_t *row = a.latd + (size_t)s * a.NS + dbase;
  int64_t b0 = -(int64_t)WC_RW;  // ring covers device positions [b0, b0 + WC_RW)
  auto fill = [&](int64_t from, int cnt) {
    for (int k = lane; k < cnt; k += 32) {
      const int64_t j = from + k;
      ring[j & (WC_RW - 1)] = j < dn ? __ldg(arr + j) : 0xFFFFFFFFu;
      lring[j & (WC_RW - 1)] = j < dn ? row[j] : 0u;  // positions >= the head: not rewritten yet
    }
  };
  auto A = [&](int64_t j) -> int64_t {  // j >= b0
    return j - b0 < WC_RW ? (int64_t)ring[j & (WC_RW - 1)] : (int64_t)__ldg(arr + j);
  };
  auto Lspec = [&](int64_t j) -> int64_t {  // the idle run's latency at j >= the head
    return j - b0 < WC_RW ? (int64_t)lring[j & (WC_RW - 1)] : (int64_t)row[j];
  };
  int64_t F = 0;  // R13
  for (int e = 0; e < a.E; e++) {
    const int64_t k = (int64_t)e * a.D + d;
    const int32_t n = a.cntED[k];
    if (n == 0) continue;
    const int64_t st = a.segBase[k];  // segment start in the device array
    const int64_t xF = a.exitF[(size_t)s * a.E * a.D + k];
    if (F <= (int64_t)__ldg(arr + st)) { F = xF; continue; }  // idle at the head: the idle run is the true one
    const EpLane p = ep_lane(a, s, e, d);
    __syncwarp();
    for (int i = lane; i < p.Bmax; i += 32) T[i] = p.T[i];
    __syncwarp();
    int64_t h = st, specPrev = 0;
    const int64_t en = st + n;
    bool met = false;
    while (h < en) {
      if (h - b0 >= WC_RW / 2 || h < b0) {  // slide / reload the ring
        const int64_t nb = h & ~(int64_t)(WC_RW / 2 - 1);
        __syncwarp();
        if (nb == b0 + WC_RW / 2) fill(b0 + WC_RW, WC_RW / 2);
        else fill(nb, WC_RW);
        b0 = nb;
        __syncwarp();
      }
      const int64_t a0 = A(h);
      if (h > st && F <= a0 && specPrev <= a0 && a0 + Lspec(h) != specPrev) { met = true; break; }
      const int B = p.Bmax;
      if (h + B <= en && A(h + B - 1) <= F) {
        // backlog: Bmax queued when the device frees -> a full batch leaves at
        // once (R4), so batch k of the stretch finishes at F + (k+1) T(Bmax)
        // while a_{h + (k+1) Bmax - 1} <= F + k T(Bmax); 32 batches per ballot
        const int64_t TB = T[B - 1];
        int done = 0;
        for (;;) {
          const int64_t hk = h + (int64_t)(done + lane) * B;
          const bool full = hk + B <= en && A(hk + B - 1) <= F + (int64_t)(done + lane) * TB;
          const unsigned m = __ballot_sync(0xffffffffu, full);
          const int r = m == 0xffffffffu ? 32 : __ffs(~m) - 1;
          const int64_t hs = h + (int64_t)done * B, ns = (int64_t)r * B;
          if (ns > 0) specPrev = A(hs + ns - 1) + Lspec(hs + ns - 1);
          __syncwarp();
          for (int64_t i = lane; i < ns; i += 32) {
            const int64_t kb = i / B;
            row[hs + i] = sat_lat(F + (done + kb + 1) * TB - A(hs + i));
          }
          done += r;
          if (r < 32 || h + (int64_t)(done + 32) * B - 1 - b0 >= WC_RW) break;  // stretch ends / ring edge
        }
        F += (int64_t)done * TB;
        h += (int64_t)done * B;
        continue;
      }
      int64_t t;
      auto Tl = [&](int j) -> int64_t { return (int64_t)T[j]; };
      const int b = decide_warp(A, en, h, F, p.Bmax, p.L, Tl, lane, &t);
      const int64_t Fn = t + T[b - 1];
      specPrev = A(h + b - 1) + Lspec(h + b - 1);
      __syncwarp();
      for (int i = lane; i < b; i += 32) row[h + i] = sat_lat(Fn - A(h + i));
      F = Fn;
      h += b;
    }
    if (met) F = xF;
  }
}

// per-scenario counts over the device-major rows (each position's epoch
// variant gives its SLO and accuracy); the sink segment is written dropped
__global__ void __launch_bounds__(256) k_ep_count(const __grid_constant__ EpArgs a, int64_t N, int64_t epoch_us,
                                                  uint64_t *agg, int sink_only) {
  __shared__ int64_t sOff[PX_MAXD + 2];
  __shared__ unsigned long long red[3][8];
  for (int k = threadIdx.x; k <= a.D + 1; k += blockDim.x) sOff[k] = a.devOff[k];
  __syncthreads();
  const int s = blockIdx.y;
  uint32_t *row = a.latd + (size_t)s * a.NS;
  unsigned long long v = 0, o = 0, ac = 0;
  const int64_t p0 = sink_only ? sOff[a.D] : 0;
  for (int64_t p = p0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < N; p += (int64_t)gridDim.x * blockDim.x) {
    int d = 0;
    while (p >= sOff[d + 1]) d++;
    if (d == a.D) { row[p] = 0xFFFFFFFFu; v++; continue; }
    const int e = (int)((int64_t)a.devArr[p] / epoch_us);
    const int opt = a.option[(size_t)e * a.D + d];
    const int64_t L = (int64_t)a.sc[s].slo_mult_milli * a.slo[a.fam_of_m[opt - 1]] / 1000;
    if ((int64_t)row[p] > L) v++;
    else { o++; ac += (unsigned long long)a.acc[opt - 1]; }
  }
  for (int k = 16; k; k >>= 1) {
    v += __shfl_xor_sync(0xffffffffu, v, k);
    o += __shfl_xor_sync(0xffffffffu, o, k);
    ac += __shfl_xor_sync(0xffffffffu, ac, k);
  }
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) { red[0][w] = v; red[1][w] = o; red[2][w] = ac; }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t[3] = {0, 0, 0};
    for (int k = 0; k < (int)(blockDim.x >> 5); k++) { t[0] += red[0][k]; t[1] += red[1][k]; t[2] += red[2][k]; }
    if (t[0]) atomicAdd((unsigned long long *)&agg[s], t[0]);
    if (t[1]) atomicAdd((unsigned long long *)&agg[a.S + s], t[1]);
    if (t[2]) atomicAdd((unsigned long long *)&agg[2 * a.S + s], t[2]);
  }
}

int px_replay_epochs(proteus_ctx *ctx, const uint32_t *d_arr, const uint8_t *d_fam, int64_t N, int E,
                     int64_t epoch_us, const int32_t *h_option, const int32_t *h_z, const int32_t *h_dev_type, int D,
                     const int32_t *h_demand, const int32_t *h_slo, const proteus_scenario *h_sc, int S,
                     uint32_t *d_lat_out, uint64_t *d_agg) {
  const int Q = ctx->Q, M = ctx->M;
  PX_CUDA(ctx, cudaMemsetAsync(d_agg, 0, ((size_t)3 * S + 1) * 8, ctx->stream));
  // F2: SWRR weights per (epoch, family) -- members z[e][d] of the hosting devices, the sink
  const size_t EQ = (size_t)E * Q;
  std::vector<int32_t> w(EQ * (D + 1), 0), plen(EQ, 0);
  std::vector<int64_t> poff(EQ + 1, 0);
  for (int e = 0; e < E; e++) {
    for (int q = 0; q < Q; q++) w[((size_t)e * Q + q) * (D + 1) + D] = h_demand[(size_t)e * Q + q];
    for (int d = 0; d < D; d++) {
      const int o = h_option[(size_t)e * D + d];
      if (o <= 0) continue;
      const int q = ctx->fam[o - 1];
      w[((size_t)e * Q + q) * (D + 1) + d] = h_z[(size_t)e * D + d];
      w[((size_t)e * Q + q) * (D + 1) + D] -= h_z[(size_t)e * D + d];
    }
  }
  for (size_t k = 0; k < EQ; k++) {
    int64_t t = 0;
    for (int d = 0; d <= D; d++) t += w[k * (D + 1) + d];
    plen[k] = (int32_t)t;
    poff[k + 1] = poff[k] + t;
  }
  const size_t small = EQ * (D + 1) * 4 + EQ * 4 + (EQ + 1) * 8 + (size_t)E * D * 4 * 4 + EQ * 4 * 2 + (size_t)Q * 4 +
                       (size_t)E * D * 4 + (size_t)S * sizeof(proteus_scenario) + 256 + 64 * 8;
  char *sb = (char *)px_buf(ctx, B_E_MISC, small + 4096);
  uint8_t *pat = (uint8_t *)px_buf(ctx, B_E_PAT, (size_t)poff[EQ] + 16);
  int64_t *exitF = (int64_t *)px_buf(ctx, B_E_EXIT, (size_t)S * E * D * 8 + 8);
  if (!sb || !pat || !exitF) return px_fail(ctx, PROTEUS_ENOMEM, "closed-loop buffers");
  char *cur = sb;
  auto take = [&](size_t bytes) { char *r = cur; cur += (bytes + 15) & ~(size_t)15; return r; };
  int32_t *d_w = (int32_t *)take(EQ * (D + 1) * 4);
  int32_t *d_plen = (int32_t *)take(EQ * 4);
  int64_t *d_poff = (int64_t *)take((EQ + 1) * 8);
  int32_t *d_opt = (int32_t *)take((size_t)E * D * 4);
  int32_t *d_dev = (int32_t *)take((size_t)D * 4);
  int32_t *d_slo = (int32_t *)take((size_t)Q * 4);
  int32_t *d_cntEQ = (int32_t *)take(EQ * 4);
  int32_t *d_fbEQ = (int32_t *)take((EQ + Q) * 4);
  int32_t *d_cntED = (int32_t *)take((size_t)E * D * 4);
  int32_t *d_segBase = (int32_t *)take(((size_t)E + 1) * D * 4);
  int64_t *d_tot = (int64_t *)take(64 * 8);
  uint32_t *d_flags = (uint32_t *)take(16);
  proteus_scenario *d_sc = (proteus_scenario *)take((size_t)S * sizeof(proteus_scenario));
  if ((size_t)(cur - sb) > small + 4096) return px_fail(ctx, PROTEUS_EINTERNAL, "closed-loop scratch layout");
  PX_CUDA(ctx, cudaMemcpyAsync(d_w, w.data(), w.size() * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_plen, plen.data(), EQ * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_poff, poff.data(), (EQ + 1) * 8, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_opt, h_option, (size_t)E * D * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_dev, h_dev_type, (size_t)D * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_slo, h_slo, (size_t)Q * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_sc, h_sc, (size_t)S * sizeof(proteus_scenario), cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemsetAsync(d_flags, 0, 16, ctx->stream));
  PX_CUDA(ctx, cudaMemsetAsync(d_cntEQ, 0, EQ * 4, ctx->stream));
  PX_CUDA(ctx, cudaMemsetAsync(d_cntED, 0, (size_t)E * D * 4, ctx->stream));
  if (EQ > 0x7fffffff) return px_fail(ctx, PROTEUS_ERANGE, "epochs x families");
  PX_LAUNCH(ctx, "loop_patterns", k_ep_patterns, (unsigned)EQ, 32, 0, (int)EQ, D, d_w, d_poff, d_plen, pat);
  if (N > 0) {
    PX_LAUNCH(ctx, "replay_check", k_check_trace, 1184, 256, 0, d_arr, d_fam, N, Q, d_flags);
    PX_LAUNCH(ctx, "loop_hist", k_ep_hist, 1184, 256, 0, d_arr, d_fam, N, E, epoch_us, Q, d_cntEQ, d_flags);
    uint32_t flags = 0;
    PX_CUDA(ctx, cudaMemcpyAsync(&flags, d_flags, 4, cudaMemcpyDeviceToHost, ctx->stream));
    PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
    if (flags & 1) return px_fail(ctx, PROTEUS_ERANGE, "arrival timestamps not sorted");
    if (flags & 2) return px_fail(ctx, PROTEUS_EINVAL, "family id >= Q");
    if (flags & 8) return px_fail(ctx, PROTEUS_ERANGE, "an arrival lies beyond the last epoch");
  }
  const int64_t ntiles = (N + TILE - 1) / TILE;
  const unsigned tblocks = (unsigned)((ntiles + TILE_WARPS - 1) / TILE_WARPS);
  int32_t *hist = (int32_t *)px_buf(ctx, B_R_HIST, (size_t)(ntiles + 1) * (PX_MAXD + 2) * 4);
  int32_t *fbase = (int32_t *)px_buf(ctx, B_R_BASE, (size_t)(ntiles + 1) * (PX_MAXQ + 2) * 4);
  int32_t *dbase = (int32_t *)px_buf(ctx, B_R_DBASE0, (size_t)(ntiles + 1) * (PX_MAXD + 2) * 4);
  uint8_t *tgt = (uint8_t *)px_buf(ctx, B_R_TGT, (size_t)N + 16);
  int64_t *off = (int64_t *)px_buf(ctx, B_R_OFF, (size_t)2 * (PX_MAXD + 2) * 8);
  uint32_t *darr = (uint32_t *)px_buf(ctx, B_R_DEVARR, (size_t)N * 4 + 16);
  uint32_t *dinv = (uint32_t *)px_buf(ctx, B_R_DEVIDX, (size_t)N * 4 + 16);
  const int64_t NS = (N + 31) & ~(int64_t)31;
  uint32_t *latd = (uint32_t *)px_buf(ctx, B_R_LATD, (size_t)S * NS * 4 + 8192);
  if (!hist || !fbase || !dbase || !tgt || !off || !darr || !dinv || !latd)
    return px_fail(ctx, PROTEUS_ENOMEM, "routing buffers");
  int64_t *totals = off + (PX_MAXD + 2);
  if (N == 0) {
    PX_CUDA(ctx, cudaMemsetAsync(off, 0, (size_t)(PX_MAXD + 2) * 8, ctx->stream));
    return 0;
  }
  PX_LAUNCH(ctx, "loop_route", k_tile_scan, Q, 1024, 0, d_cntEQ, (int64_t)E, Q, d_fbEQ, d_tot);
  PX_LAUNCH(ctx, "loop_route", k_tile_count, tblocks, TILE_WARPS * 32, 0, d_fam, N, Q, hist);
  PX_LAUNCH(ctx, "loop_route", k_tile_scan, Q, 1024, 0, hist, ntiles, Q, fbase, totals);
  PX_LAUNCH(ctx, "loop_route", k_ep_target, tblocks, TILE_WARPS * 32, 0, d_fam, d_arr, N, Q, epoch_us, fbase, d_fbEQ,
            pat, d_poff, d_plen, D, tgt, hist);
  PX_LAUNCH(ctx, "loop_route", k_tile_scan, D + 1, 1024, 0, hist, ntiles, D + 1, dbase, totals);
  PX_LAUNCH(ctx, "loop_route", k_dev_offsets, 1, 32, 0, totals, D + 1, off);
  PX_LAUNCH(ctx, "loop_route", k_scatter, tblocks, TILE_WARPS * 32, 0, tgt, d_arr, N, D, dbase, off, darr, dinv);
  PX_LAUNCH(ctx, "loop_route", k_ep_seghist, 1184, 256, 0, tgt, d_arr, N, epoch_us, D, d_cntED);
  PX_LAUNCH(ctx, "loop_route", k_tile_scan, D, 1024, 0, d_cntED, (int64_t)E, D, d_segBase, d_tot);
  EpArgs ea;
  memset(&ea, 0, sizeof ea);
  ea.E = E; ea.D = D; ea.M = M; ea.bmax = ctx->bmax; ea.S = S; ea.NS = NS;
  ea.option = d_opt; ea.dev_type = d_dev; ea.lat = ctx->d_lat; ea.acc = ctx->d_acc; ea.fam_of_m = ctx->d_fam;
  ea.slo = d_slo; ea.sc = d_sc; ea.devOff = off; ea.cntED = d_cntED; ea.segBase = d_segBase; ea.devArr = darr;
  ea.latd = latd; ea.exitF = exitF;
  if (S > 65535) return px_fail(ctx, PROTEUS_EINVAL, "S");
  const int64_t nseg = (int64_t)E * D;
  // the chain path (k_chain<true>): per-chunk tables of the idle-branch
  // decisions with each head's epoch parameters, a chained scan of chunk
  // exits; the chunk runs + stitch otherwise
  bool chained = false;
  if (env_int("PROTEUS_LOOP_CHAIN", 1) != 0 && E <= 65535 && ctx->bmax <= 255 && N < (1ll << 31)) {
    int C = std::max(256, std::min(CHAIN_CMAX, env_int("PROTEUS_REPLAY_CHAIN_C", 2048)));
    const int SEG = std::min(C, std::max(CHAIN_SEGMIN, env_int("PROTEUS_REPLAY_CHAIN_SEG", 128)));
    {  // the chunk's tables must fit the block's shared memory (the per-head epoch arrays included)
      int smax = 0;
      PX_CUDA(ctx, cudaDeviceGetAttribute(&smax, cudaDevAttrMaxSharedMemoryPerBlockOptin, ctx->device));
      while (C > 256 && chain_smem(C, ctx->bmax, SEG, true) + 1024 > (size_t)smax) C -= 256;
    }
    int32_t *epP = (int32_t *)px_buf(ctx, B_E_CHAIN, (size_t)S * E * D * 16 + 64);
    if (!epP) return px_fail(ctx, PROTEUS_ENOMEM, "closed-loop chain parameters");
    PX_CUDA(ctx, cudaMemsetAsync(d_flags, 0, 4, ctx->stream));
    const int64_t np = (int64_t)S * E * D;
    PX_LAUNCH(ctx, "loop_chain", k_ep_chparams, (unsigned)((np + 255) / 256), 256, 0, ea, epP, d_flags);
    int64_t h_off[PX_MAXD + 2];
    uint32_t fl = 0;
    PX_CUDA(ctx, cudaMemcpyAsync(h_off, off, (D + 2) * 8, cudaMemcpyDeviceToHost, ctx->stream));
    PX_CUDA(ctx, cudaMemcpyAsync(&fl, d_flags, 4, cudaMemcpyDeviceToHost, ctx->stream));
    PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
    if (!(fl & 1)) {
      std::vector<int32_t> lid, nch;
      int64_t mx = 1;
      for (int sc = 0; sc < S; sc++)
        for (int d = 0; d < D; d++) {
          const int64_t nd = h_off[d + 1] - h_off[d];
          if (nd <= 0) continue;
          lid.push_back(sc * D + d);
          nch.push_back((int32_t)((nd + C - 1) / C));
          mx = std::max(mx, (int64_t)nch.back());
        }
      const size_t nl = lid.size();
      if (nl > 0) {
        const size_t part = chain_exoff(nl) + nl * (size_t)mx * 8;
        char *q = (char *)px_buf(ctx, B_E_UNITS, part + 64);
        if (!q) return px_fail(ctx, PROTEUS_ENOMEM, "closed-loop chain buffers");
        std::vector<uint8_t> cm(nl, 0);
        PX_CUDA(ctx, cudaMemcpyAsync(q, lid.data(), nl * 4, cudaMemcpyHostToDevice, ctx->stream));
        PX_CUDA(ctx, cudaMemcpyAsync(q + nl * 4, nch.data(), nl * 4, cudaMemcpyHostToDevice, ctx->stream));
        PX_CUDA(ctx, cudaMemcpyAsync(q + nl * 8, cm.data(), nl, cudaMemcpyHostToDevice, ctx->stream));
        PX_CUDA(ctx, cudaMemsetAsync(q + chain_ctroff(nl), 0, part - chain_ctroff(nl), ctx->stream));
        // ticket order (as px_replay's): chunks spread in proportion to the lane's length
        size_t nu = 0;
        for (size_t l = 0; l < nl; l++) nu += (size_t)nch[l];
        std::vector<int64_t> cnt((size_t)mx + 1, 0);
        for (size_t l = 0; l < nl; l++)
          for (int64_t c = 0; c < nch[l]; c++) cnt[(size_t)(c * mx / nch[l]) + 1]++;
        for (int64_t k = 0; k < mx; k++) cnt[(size_t)k + 1] += cnt[(size_t)k];
        std::vector<unsigned long long> units(nu);
        for (size_t l = 0; l < nl; l++)
          for (int64_t c = 0; c < nch[l]; c++)
            units[(size_t)cnt[(size_t)(c * mx / nch[l])]++] = ((unsigned long long)l << 32) | (unsigned long long)c;
        unsigned long long *du = (unsigned long long *)px_buf(ctx, B_R_UNITS0, nu * 8 + 16);
        if (!du) return px_fail(ctx, PROTEUS_ENOMEM, "closed-loop chain tickets");
        ctx->chain_ukey[0].clear();  // B_R_UNITS0 now holds this order, not px_replay's
        PX_CUDA(ctx, cudaMemcpyAsync(du, units.data(), nu * 8, cudaMemcpyHostToDevice, ctx->stream));
        ChainArgs ca;
        memset(&ca, 0, sizeof ca);
        ca.D = D; ca.M = M; ca.bmax = ctx->bmax; ca.nl = (int)nl; ca.C = C; ca.SEG = SEG;
        ca.K = std::max(0, env_int("PROTEUS_REPLAY_CHAIN_K", 16));
        ca.NS = NS; ca.maxch = mx; ca.nunits = (int64_t)nu; ca.units = du;
        ca.lid = (const int32_t *)q; ca.nch = ca.lid + nl; ca.cmode = (const uint8_t *)(q + nl * 8);
        ca.counter = (unsigned long long *)(q + chain_ctroff(nl));
        ca.watchdog = (unsigned *)(ca.counter + 1);
        ca.ex = (unsigned long long *)(q + chain_exoff(nl));
        ca.lat = ctx->d_lat; ca.devOff = off; ca.devArr = darr; ca.latd = latd;
        ca.E = E; ca.epoch_us = epoch_us; ca.epP = epP; ca.segBase = d_segBase; ca.cntED = d_cntED;
        ca.agg = d_agg; ca.S = S;
        const size_t smc = chain_smem(C, ctx->bmax, SEG, true);
        PX_CUDA(ctx, cudaFuncSetAttribute(k_chain<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smc));
        int nsm = 0, occ = 0;
        PX_CUDA(ctx, cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, ctx->device));
        const int orc = px_occupancy(ctx, (const void *)k_chain<true>, CHAIN_THREADS, smc, &occ);
        if (orc) return orc;
        const int64_t nb = std::min<int64_t>((int64_t)nu, (int64_t)nsm * std::max(occ, 1));
        PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));  // host vectors are staged
        PX_LAUNCH(ctx, "loop_chain", k_chain<true>, (unsigned)nb, CHAIN_THREADS, smc, ca);
        unsigned wd = 0;
        PX_CUDA(ctx, cudaMemcpyAsync(&wd, ca.watchdog, 4, cudaMemcpyDeviceToHost, ctx->stream));
        PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
        if (wd) return px_fail(ctx, PROTEUS_EINTERNAL, "closed loop: chain wait for a previous chunk timed out");
      }
      chained = true;
    }
  }
  if (!chained) {
    PX_LAUNCH(ctx, "loop_spec", k_ep_spec, dim3((unsigned)((nseg + 127) / 128), (unsigned)S), 128, 0, ea);
    PX_LAUNCH(ctx, "loop_stitch", k_ep_stitch, (unsigned)((S * D + 3) / 4), 128, 0, ea);
  }
  // counts: the chain writers folded every device's; k_ep_count takes the rest (the sink)
  PX_LAUNCH(ctx, "loop_count", k_ep_count, dim3(296, (unsigned)S), 256, 0, ea, N, epoch_us, d_agg, chained ? 1 : 0);
  if (d_lat_out) {
    const int64_t nb = (N + 256 * UNP_PER - 1) / (256 * UNP_PER);
    PX_LAUNCH(ctx, "loop_unpermute", k_unpermute, (unsigned)nb, 256, 0, N, NS, S, d_sc, dinv, dinv, latd, d_lat_out);
  }
  return 0;
}
