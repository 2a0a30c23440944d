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
// One block.  Weights and the SWRR pattern of every family (R8).
//   routing 0: member weight z_d for hosting devices with z_d > 0, sink weight
//              s_q - sum z (unmet demand, reading R7)
//   routing 1: weight 1 per hosting device that fits batch 1 (depth >= 1); no sink
__global__ void k_route_prepare(int routing, int Q, int D, int M, int bmax, const int32_t *__restrict__ option,
                                const int32_t *__restrict__ z, const int32_t *__restrict__ dev_type,
                                const int32_t *__restrict__ demand, const int32_t *__restrict__ fam_of_m,
                                const int32_t *__restrict__ lat, uint8_t *pattern, int32_t *pat_off,
                                int32_t *pat_len) {
  __shared__ int32_t W[PX_MAXQ];
  const int q = threadIdx.x;
  int32_t w[PX_MAXD + 1];
  int32_t cur[PX_MAXD + 1];
  if (q < Q) {
    int64_t tot = 0, zsum = 0;
    for (int d = 0; d < D; d++) {
      w[d] = 0;
      const int o = option[d];
      if (o <= 0 || fam_of_m[o - 1] != q) continue;
      if (routing == 0) {
        w[d] = z[d];
        zsum += z[d];
      } else {
        w[d] = lat[((size_t)dev_type[d] * M + (o - 1)) * bmax] > 0 ? 1 : 0;
      }
      tot += w[d];
    }
    w[D] = routing == 0 ? (int32_t)(demand[q] - zsum) : 0;
    tot += w[D];
    W[q] = (int32_t)tot;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int32_t acc = 0;
    for (int k = 0; k < Q; k++) { pat_off[k] = acc; pat_len[k] = W[k]; acc += W[k]; }
  }
  __syncthreads();
  if (q >= Q) return;
  const int32_t Wq = W[q];
  uint8_t *pat = pattern + pat_off[q];
  for (int d = 0; d <= D; d++) cur[d] = 0;
  for (int32_t k = 0; k < Wq; k++) {
    int best = -1;
    for (int d = 0; d <= D; d++) {
      if (w[d] == 0) continue;
      cur[d] += w[d];
      if (best < 0 || cur[d] > cur[best]) best = d;
    }
    cur[best] -= Wq;
    pat[k] = (uint8_t)best;
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
struct SpecExit {
  int64_t F;
  int32_t ov;  // exit head - chunk end (overhang of the last batch into the next chunk)
  int32_t mer;  // phase runs: offset from the chunk start where the run met run 0 (else the chunk length)
};

struct LaneParam {  // per (scenario, device)
  int32_t Bmax;     // min(cap, depth) (R4); 0 for idle devices
  uint32_t A;       // accuracy of the hosted variant
  int64_t L;        // scenario SLO of the hosted family (R12)
};

__global__ void k_lane_params(int S, int D, int M, int bmax, const int32_t *__restrict__ option,
                              const int32_t *__restrict__ dev_type, const int32_t *__restrict__ fam_of_m,
                              const int32_t *__restrict__ acc, const int32_t *__restrict__ lat,
                              const int32_t *__restrict__ slo_base, const proteus_scenario *__restrict__ sc,
                              LaneParam *lp) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= S * D) return;
  const int s = i / D, d = i % D;
  LaneParam p = {0, 0, 0};
  const int o = option[d];
  if (o > 0) {
    const int32_t *T = lat + ((size_t)dev_type[d] * M + (o - 1)) * bmax;
    int depth = 0;
    while (depth < bmax && T[depth] > 0) depth++;
    const int cap = sc[s].batch_cap;
    p.Bmax = (cap > 0 && cap < depth) ? cap : depth;
    p.A = (uint32_t)acc[o - 1];
    p.L = (int64_t)sc[s].slo_mult_milli * slo_base[fam_of_m[o - 1]] / 1000;
  }
  lp[i] = p;
}

struct LaneArgs {
  int S, D, M, bmax, nsc, CH;
  int64_t N, NCH;
  const int32_t *option, *dev_type, *lat, *sc_list;
  const LaneParam *lp;
  const int64_t *devOff;  // [D + 2]; segment D = the sink
  const int64_t *choff;   // [D + 1] chunk offsets
  const int32_t *goff;    // [D + 1] phase-A warp-group offsets
  const uint32_t *devArr;
  uint32_t *latd;         // [S][N] device-major
  SpecExit *ex;           // [S][NCH]
  uint64_t *agg;          // [3][S]
  int maxchk;             // convergence checks per chunk (free decisions only)
  int rmax;               // phase runs: lanes with 2 <= Bmax <= rmax speculate Bmax runs per chunk
  uint32_t *vlat;         // latencies of the phase runs r >= 1 (lane base voff[lane] + (r - 1) n)
  SpecExit *vex;          // their exit states (lane base voff[S D + lane] + (r - 1) nch)
  const int64_t *voff;    // [2][S * D]
  long long debug;        // > 0: k_stitch prints lanes slower than this many cycles (diagnostic)
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
  uint32_t *out = a.latd + (size_t)s * a.N + st;
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

// number of speculative runs per chunk of a lane (see k_spec)
__host__ __device__ __forceinline__ int n_phase_runs(int Bmax, int rmax) {
  return Bmax < 2 ? 1 : Bmax < rmax ? Bmax : rmax;
}

// ---- phase A: speculative chunks
// Each device array is cut into chunks of CH queries.  One warp per (device,
// scenario, 32 consecutive chunks); lane = chunk, replayed from an idle
// device (the true state at the start of the trace, R13).  All lanes follow
// the same rule parameters, so the warp stays close to converged.
// Launched twice: run 0 (rbase 0, gridDim.z 1), then the phase runs r >= 1
// (rbase 1), which stop as soon as they meet run 0 (same batch end, same
// finish) and take run 0's exit; `mer` records where.
__global__ void __launch_bounds__(128) k_spec(const __grid_constant__ LaneArgs a, int rbase) {
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
  const int s = a.sc_list[blockIdx.x];
  const LaneParam p = a.lp[s * a.D + d];
  const int64_t off = a.devOff[d], n = a.devOff[d + 1] - off;
  const int64_t nch = a.choff[d + 1] - a.choff[d];
  const int64_t c = (int64_t)(g - sG[d]) * 32 + lane;
  const int r = blockIdx.z + rbase;  // phase run r: first batch starts at st + r
  if (r > 0 && r >= n_phase_runs(p.Bmax, a.rmax)) return;
  if (c < nch) {
    const int64_t st = c * a.CH, en = st + a.CH < n ? st + a.CH : n;
    const int64_t lane_id = (int64_t)s * a.D + d;
    uint32_t *out = r == 0 ? a.latd + (size_t)s * a.N + off : a.vlat + a.voff[lane_id] + (int64_t)(r - 1) * n;
    int64_t h = st + r, F = 0;
    SpecExit e;
    e.mer = (int32_t)(en - st);
    bool met = false;
    if (p.Bmax < 1) {
      for (int64_t j = st; j < en; j++) out[j] = 0xFFFFFFFFu;
      h = en;
    } else {
      const int32_t *T = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
      GArr arr{a.devArr + off};
      const uint32_t *run0 = a.latd + (size_t)s * a.N + off;
      while (h < en) {
        int64_t t;
        const int b = decide(arr, n, h, F, p.Bmax, p.L, T, &t);
        const int64_t Fn = t + T[b - 1];
        const int64_t jend = h + b < en ? h + b : en;
        for (int64_t j = h; j < jend; j++) out[j] = sat_lat(Fn - (int64_t)arr(j));
        const int64_t j2 = h + b;
        // met run 0: it also ends a batch at j2 - 1 finishing at Fn (the next
        // batch always finishes later); tested after batches the device waited for
        if (r > 0 && t > F && j2 < en && (int64_t)arr(j2 - 1) + run0[j2 - 1] == Fn &&
            (int64_t)arr(j2) + run0[j2] != Fn) {
          met = true;
          e.mer = (int32_t)(j2 - st);
          break;
        }
        F = Fn;
        h = j2;
      }
    }
    if (met) {
      const SpecExit e0 = a.ex[(size_t)s * a.NCH + a.choff[d] + c];
      e.F = e0.F;
      e.ov = e0.ov;
    } else {
      e.F = F;
      e.ov = (int32_t)(h - en);
    }
    if (r == 0) a.ex[(size_t)s * a.NCH + a.choff[d] + c] = e;
    else a.vex[a.voff[(int64_t)a.S * a.D + lane_id] + (int64_t)(r - 1) * nch + c] = e;
  }
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
#define SPECCAP 1024                 // chunk length limit of the stitch
#define RSEG 1024                    // ring segment (queries), one bulk copy
#define RING (4 * RSEG)              // per-warp arrival ring
#define SPB (SPECCAP + 8)            // speculative-latency buffer (+ alignment lead)
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
  return ((size_t)RING + 2 * SPB + 12 + 64 * SUMAX + bmax + 3) & ~(size_t)3;
}
static size_t stitch_smem(int bmax) { return 4 * stitch_wstride(bmax) * 4; }

__global__ void __launch_bounds__(128) k_stitch(const __grid_constant__ LaneArgs a) {
  // shared memory per warp: arrival ring [RING], spec latencies [2][SPB],
  // mbarriers [4 ring + 2 spec], T [bmax]
  extern __shared__ __align__(16) uint32_t ssm[];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int64_t gw = (int64_t)blockIdx.x * 4 + w;
  if (gw >= (int64_t)a.nsc * a.D) return;
  const int s = a.sc_list[gw / a.D], d = (int)(gw % a.D);
  const LaneParam p = a.lp[s * a.D + d];
  const int64_t off = a.devOff[d], n = a.devOff[d + 1] - off;
  const int64_t nch = a.choff[d + 1] - a.choff[d];
  if (p.Bmax < 1 || nch < 2) return;
  uint32_t *wsm = ssm + (size_t)w * stitch_wstride(a.bmax);
  uint32_t *ring = wsm;
  uint32_t *specbuf = wsm + RING;
  uint64_t *bars = (uint64_t *)(wsm + RING + 2 * SPB);  // [0..3] ring slots, [4..5] spec buffers
  int64_t *FeS = (int64_t *)(wsm + RING + 2 * SPB + 12);  // [32 SUMAX] stretch batch finishes
  int32_t *T = (int32_t *)(wsm + RING + 2 * SPB + 12 + 64 * SUMAX);
  const int32_t *Tg = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
  for (int k = lane; k < a.bmax; k += 32) T[k] = Tg[k];
  if (lane < 6) mbar_init(bars + lane);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  uint32_t *out = a.latd + (size_t)s * a.N + off;
  const uint32_t *src = out;  // the speculative run the current chunk is matched against
  int64_t mr = 0;             // ... whose own latencies cover [h, mr), run 0's from mr on
  const SpecExit *ex = a.ex + (size_t)s * a.NCH + a.choff[d];
  const int64_t CH = a.CH;
  int64_t h = (CH < n ? CH : n) + ex[0].ov, F = ex[0].F;
  // Arrivals stream through a 4-segment ring by TMA bulk copies of whole
  // 1024-query segments of the routed array (segment g >> 10 of the absolute
  // index g = off + j sits in slot (g >> 10) & 3, so ring[g & (RING - 1)] is
  // query g).  Segments up to the one 2 past h's are in flight; a slot is
  // refilled only after its previous segment has been waited for and lies
  // 2 segments behind h (the stitch reads back at most Bmax - 1 <= 1023).
  const int64_t sg0 = (off + CH) >> 10;  // first segment ever read (chunk 1 starts at CH)
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
      if (lane == 0) bulk_load(ring + (sg_iss & 3) * RSEG, a.devArr + sg_iss * RSEG, RSEG * 4, bars + (sg_iss & 3));
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
  auto put = [&](int64_t j, int64_t Fb) { out[j] = sat_lat(Fb - AR(j)); };
  // Speculative latencies of chunk c (run 0) are bulk-copied into buffer
  // (c - 1) & 1 while chunk c - 1 is stitched.
  uint32_t *specL = specbuf;
  int64_t spec_base = -1;
  auto spec_issue = [&](int64_t c) {
    if (c >= nch) return;
    const int bi = (int)((c - 1) & 1);
    if (c >= 3) mbar_wait(bars + 4 + bi, (uint32_t)(((c - 3) >> 1) & 1));  // previous use consumed
    __syncwarp();
    if (lane == 0) {
      const int64_t st = c * CH, en = st + CH < n ? st + CH : n;
      const uintptr_t g = (uintptr_t)(out + st), g0 = g & ~(uintptr_t)15;
      const uint32_t bytes = (uint32_t)(((g - g0) + (uintptr_t)(en - st) * 4 + 15) & ~(uintptr_t)15);
      bulk_load(specbuf + bi * SPB, (const void *)g0, bytes, bars + 4 + bi);
    }
  };
  spec_issue(1);
  // j in [h, en): always inside the cached window [spec_base, en)
  auto spec_F = [&](int64_t j) -> int64_t { return AR(j) + specL[(int32_t)(j - spec_base)]; };
  const int64_t TB = T[p.Bmax - 1];
  // the 32-bit decision needs L < C / 2 and every T(b) < C (so W_k < C and
  // t + T(b) < 2^31); per-lane W_k = L - T(k + 2) and T(k + 1) for the
  // first two ballot rounds stay in registers
  int32_t tmax = 0;
  for (int k = lane; k < p.Bmax; k += 32) tmax = T[k] > tmax ? T[k] : tmax;
  tmax = __reduce_max_sync(0xffffffffu, tmax);
  const bool lean = p.L < LEAN_C / 2 && tmax < LEAN_C;
  const int32_t W0 = lane + 1 < p.Bmax ? (int32_t)p.L - T[lane + 1] : 0;
  const int32_t W1 = lane + 33 < p.Bmax ? (int32_t)p.L - T[lane + 33] : 0;
  const int32_t T0 = lane < p.Bmax ? T[lane] : 0;
  const int32_t T1 = lane + 32 < p.Bmax ? T[lane + 32] : 0;
  const int R = n_phase_runs(p.Bmax, a.rmax);
  const int64_t lane_id = (int64_t)s * a.D + d;
  const uint32_t *vl = R > 1 ? a.vlat + a.voff[lane_id] : nullptr;
  const SpecExit *vx = R > 1 ? a.vex + a.voff[(int64_t)a.S * a.D + lane_id] : nullptr;
  const int SU = p.Bmax >= 16 ? 1 : p.Bmax >= 8 ? 2 : SUMAX;  // batches per lane in a full-batch stretch
  const uint32_t bmagic = (uint32_t)((1ull << 32) / (uint64_t)p.Bmax + 1);  // q / Bmax = umulhi(q, bmagic), q < 2^16
  // SW: a full batch needs its last arrival <= max(F_i, a[h_i] + SW) (see the stretch)
  int32_t tbig = 0;
  for (int k = lane; k + 1 < p.Bmax; k += 32) tbig = T[k] > tbig ? T[k] : tbig;
  tbig = __reduce_max_sync(0xffffffffu, tbig);
  const int64_t SW = tbig <= TB ? (p.L - TB > 0 ? p.L - TB : 0) : INT64_MIN / 4;
  bool lastfull = true;
  long long dbg_t0 = clock64(), dbg_dec = 0, dbg_jump = 0, dbg_match = 0, dbg_chk = 0;
  long long dbg_sec[5] = {0, 0, 0, 0, 0}, dbg_tk = 0;
  for (int64_t c0 = 1; c0 < nch; c0 += 32) {
    int64_t pF = 0;
    int pov = 0;
    if (c0 + lane < nch) {
      const SpecExit e = ex[c0 + lane];
      pF = e.F;
      pov = e.ov;
    }
    const int cnt = nch - c0 < 32 ? (int)(nch - c0) : 32;
    for (int k = 0; k < cnt; k++) {
      const int64_t st = (c0 + k) * CH, en = st + CH < n ? st + CH : n;
      const int64_t eF = __shfl_sync(0xffffffffu, pF, k);
      const int eov = __shfl_sync(0xffffffffu, pov, k);
      const int64_t c = c0 + k;
      spec_issue(c + 1);
      need(h, (h < en ? h : en) + p.Bmax + 1);
      if (h > st) {  // queries of this chunk in the last batch of the previous one
        const int64_t hi = h < en ? h : en;
        for (int64_t j = st + lane; j < hi; j += 32) put(j, F);
      }
      if (h >= en) continue;
      // match against the run whose first batch starts where the true one
      // does: phase r = h - st (run 0 = the chunk's own start)
      const int ovr = (int)(h - st);
      const bool var = ovr > 0 && ovr < R;
      int64_t xF = eF;
      int xov = eov;
      mr = st;
      src = out;
      if (var) {
        src = vl + (int64_t)(ovr - 1) * n;
        const SpecExit ve = vx[(int64_t)(ovr - 1) * nch + c];
        xF = ve.F;
        xov = ve.ov;
        mr = st + ve.mer;
      }
      if ((ovr == 0 || var) && F <= AR(h)) {  // speculative start = true state
        for (int64_t j = h + lane; j < mr; j += 32) out[j] = src[j];
        h = en + xov;
        F = xF;
        PX_DBG(dbg_match++);
        continue;
      }
      int checks = a.maxchk;
      // the speculative latencies of [h, en) are cached at the first meeting
      // test of the chunk: the true run has only rewritten positions < h
      spec_base = -1;
      auto spec_cache = [&]() {
        if (spec_base >= 0) return;
        const int bi = (int)((c - 1) & 1);
        specL = specbuf + bi * SPB;
        mbar_wait(bars + 4 + bi, (uint32_t)(((c - 1) >> 1) & 1));  // run 0's, prefetched
        if (!var) {
          spec_base = st - (int64_t)(((uintptr_t)(out + st) & 15) >> 2);
          return;
        }
        __syncwarp();  // a phase run's: plain loads over the prefetched copy
        spec_base = h;
        const int64_t m = en - h;
        for (int64_t i = lane; i < m; i += 32) specL[i] = (h + i < mr ? src : out)[h + i];
        __syncwarp();
      };
      bool spec_ready = false;  // latency cache of this chunk loaded (at its first meeting test)
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
            r.sp = test && h + k < en ? specL[(int32_t)(h + k - spec_base)] : 0u;
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
              spec_cache();
              spec_ready = true;
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
            // the rest of the chunk is the speculative run's (phase runs: their own latencies up to mr)
            for (int64_t jj = h + lane; jj < mr; jj += 32) out[jj] = specL[jj - spec_base];
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
          spec_cache();
          spec_ready = true;
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
          // the rest of the chunk is the speculative run's (phase runs: their own latencies up to mr)
          for (int64_t jj = h + lane; jj < mr; jj += 32) out[jj] = specL[jj - spec_base];
          h = en + xov;
          F = xF;
          break;
        }
      }
    }
  }
  if (a.debug && lane == 0) {
    const long long cyc = clock64() - dbg_t0;
    if (cyc > a.debug) printf("stitch s=%d d=%d n=%lld Bmax=%d L=%lld nch=%lld cycles=%lld dec=%lld jump=%lld match=%lld chk=%lld "
                              "sdec=%lld schk=%lld swr=%lld sloop=%lld sring=%lld\n", s, d,
                              (long long)n, p.Bmax, (long long)p.L, (long long)nch, cyc, dbg_dec, dbg_jump, dbg_match, dbg_chk,
                              dbg_sec[0], dbg_sec[1], dbg_sec[2], dbg_sec[3], dbg_sec[4]);
  }
}

// dropped queries (the sink segment, device index D): latency UINT32_MAX (R7)
__global__ void k_sink(int64_t N, int S, int D, const int32_t *__restrict__ sc_list, int nsc, const int64_t *devOff,
                       uint32_t *latd, uint64_t *agg) {
  for (int k = blockIdx.y; k < nsc; k += gridDim.y) {
    const int64_t st = devOff[D], n = devOff[D + 1] - st;
    const int s = sc_list[k];
    uint32_t *row = latd + (size_t)s * N + st;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
      row[j] = 0xFFFFFFFFu;
  }
}

// a13: per scenario, violations (latency > the SLO of the device's family, R6;
// dropped queries included), on-time count and the serving variant's accuracy
// summed over on-time queries (R9), over the device-major rows.
__global__ void k_count(int64_t N, int S, int D, const int32_t *__restrict__ sc_list, const int64_t *__restrict__ devOff,
                        const LaneParam *__restrict__ lp, const uint32_t *__restrict__ latd, uint64_t *agg) {
  __shared__ int64_t sOff[PX_MAXD + 2], sL[PX_MAXD + 1];
  __shared__ uint32_t sA[PX_MAXD + 1];
  __shared__ unsigned long long red[3][32];
  const int s = sc_list[blockIdx.y];
  for (int k = threadIdx.x; k <= D + 1; k += blockDim.x) sOff[k] = devOff[k];
  for (int k = threadIdx.x; k <= D; k += blockDim.x) {
    sL[k] = k < D ? lp[s * D + k].L : -1;  // the sink: every latency is a violation
    sA[k] = k < D ? lp[s * D + k].A : 0;
  }
  __syncthreads();
  const uint32_t *row = latd + (size_t)s * N;
  unsigned long long viol = 0, ont = 0, accs = 0;
  const int64_t per = (N + gridDim.x - 1) / gridDim.x;
  const int64_t lo = (int64_t)blockIdx.x * per, hi = lo + per < N ? lo + per : N;
  int d = 0;
  for (int64_t p0 = lo; p0 < hi; p0 += 4 * blockDim.x) {
    while (d < D && sOff[d + 1] <= p0) d++;  // segment of this step's first position (uniform)
    uint32_t l[4];
#pragma unroll
    for (int k = 0; k < 4; k++) {
      const int64_t p = p0 + threadIdx.x + (int64_t)k * blockDim.x;
      l[k] = p < hi ? row[p] : 0;
    }
#pragma unroll
    for (int k = 0; k < 4; k++) {
      const int64_t p = p0 + threadIdx.x + (int64_t)k * blockDim.x;
      if (p >= hi) continue;
      int dd = d;
      while (dd < D && sOff[dd + 1] <= p) dd++;
      if ((int64_t)l[k] > sL[dd]) viol++;
      else { ont++; accs += sA[dd]; }
    }
  }
  for (int o = 16; o; o >>= 1) {
    viol += __shfl_xor_sync(0xffffffffu, viol, o);
    ont += __shfl_xor_sync(0xffffffffu, ont, o);
    accs += __shfl_xor_sync(0xffffffffu, accs, o);
  }
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) { red[0][w] = viol; red[1][w] = ont; red[2][w] = accs; }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long v = 0, o2 = 0, a2 = 0;
    for (int k = 0; k < (int)(blockDim.x >> 5); k++) { v += red[0][k]; o2 += red[1][k]; a2 += red[2][k]; }
    if (v) atomicAdd((unsigned long long *)&agg[s], v);
    if (o2) atomicAdd((unsigned long long *)&agg[S + s], o2);
    if (a2) atomicAdd((unsigned long long *)&agg[2 * S + s], a2);
  }
}

// per-query order: out[s][i] = latd[s][inv(i)] (coalesced stores, gathered loads
// that walk ~D sequential streams)
#define UNP_PER 16
__global__ void __launch_bounds__(256) k_unpermute(int64_t N, int S, const proteus_scenario *__restrict__ sc,
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
    const size_t r = (size_t)s * N;
    const bool m1 = rt[s] != 0;
    uint32_t v[UNP_PER];
#pragma unroll
    for (int k = 0; k < UNP_PER; k++)
      if (i0 + 256 * k < N) v[k] = latd[r + (m1 ? p1[k] : p0[k])];
#pragma unroll
    for (int k = 0; k < UNP_PER; k++)
      if (i0 + 256 * k < N) out[r + i0 + 256 * k] = v[k];
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
  const size_t small = (size_t)(4 * D + 2 * Q + 2 * PX_MAXQ + 8 + 2 * S + 4 * (PX_MAXD + 2)) * 4 +
                       (size_t)S * sizeof(proteus_scenario) + (size_t)S * D * sizeof(LaneParam) +
                       (size_t)2 * (PX_MAXD + 2) * 8;
  char *sb = (char *)px_buf(ctx, B_R_MISC, small + 4096);
  if (!sb) return px_fail(ctx, PROTEUS_ENOMEM, "replay scratch");
  int32_t *d_opt = (int32_t *)sb, *d_z = d_opt + D, *d_dev = d_z + D, *d_dem = d_dev + D, *d_slo = d_dem + Q;
  int32_t *d_pat_off = d_slo + Q, *d_pat_len = d_pat_off + PX_MAXQ;
  uint32_t *d_flags = (uint32_t *)(d_pat_len + PX_MAXQ);
  int32_t *d_scl = (int32_t *)(d_flags + 8);              // [2][S] scenario lists per routing mode
  int32_t *d_goff = d_scl + 2 * S;                        // [2][PX_MAXD + 2]
  int64_t *d_choff = (int64_t *)(((uintptr_t)(d_goff + 2 * (PX_MAXD + 2)) + 15) & ~(uintptr_t)15);  // [2][PX_MAXD + 2]
  proteus_scenario *d_sc = (proteus_scenario *)(d_choff + 2 * (PX_MAXD + 2));
  LaneParam *d_lp = (LaneParam *)(((uintptr_t)(d_sc + S) + 15) & ~(uintptr_t)15);
  std::vector<int32_t> scl[2];
  for (int s = 0; s < S; s++) scl[h_sc[s].routing].push_back(s);
  std::vector<int32_t> scl_all(2 * S, 0);
  for (int rt = 0; rt < 2; rt++)
    for (size_t k = 0; k < scl[rt].size(); k++) scl_all[rt * S + k] = scl[rt][k];
  PX_CUDA(ctx, cudaMemcpyAsync(d_opt, h_option, D * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_z, h_z, D * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_dev, h_dev_type, D * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_dem, h_demand, Q * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_slo, h_slo, Q * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_scl, scl_all.data(), 2 * S * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(d_sc, h_sc, S * sizeof(proteus_scenario), cudaMemcpyHostToDevice, ctx->stream));
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
  for (int rt = 0; rt < 2; rt++) {
    if (scl[rt].empty()) continue;
    uint8_t *pat = (uint8_t *)px_buf(ctx, B_R_PAT, pat_cap);
    int32_t *hist = (int32_t *)px_buf(ctx, B_R_HIST, (size_t)(ntiles + 1) * (PX_MAXD + 2) * 4);
    int32_t *fbase = (int32_t *)px_buf(ctx, B_R_BASE, (size_t)(ntiles + 1) * (PX_MAXQ + 2) * 4);
    int32_t *dbase = (int32_t *)px_buf(ctx, B_R_DBASE0, (size_t)(ntiles + 1) * (PX_MAXD + 2) * 4);
    uint8_t *tgt = (uint8_t *)px_buf(ctx, B_R_TGT, (size_t)N + 16);
    int64_t *off = (int64_t *)px_buf(ctx, rt ? B_R_OFF1 : B_R_OFF, (size_t)2 * (PX_MAXD + 2) * 8);
    // + whole trailing ring segment: k_stitch bulk-copies 4 KB segments
    uint32_t *darr = (uint32_t *)px_buf(ctx, rt ? B_R_DEVARR1 : B_R_DEVARR, ((size_t)N + 2 * RSEG) * 4);
    uint32_t *dinv = (uint32_t *)px_buf(ctx, rt ? B_R_DEVIDX1 : B_R_DEVIDX, (size_t)N * 4 + 16);
    if (!pat || !hist || !fbase || !dbase || !tgt || !off || !darr || !dinv)
      return px_fail(ctx, PROTEUS_ENOMEM, "routing buffers");
    int64_t *totals = off + (PX_MAXD + 2);
    PX_LAUNCH(ctx, "route_prepare", k_route_prepare, 1, 32, 0, rt, Q, D, M, ctx->bmax, d_opt, d_z, d_dev, d_dem,
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
    devOff[rt] = off; devArr[rt] = darr; inv[rt] = dinv;
  }
  if (N == 0) return 0;
  // chunk layout per routing mode (sizes only): the host reads the per-device counts
  int CH = env_int("PROTEUS_REPLAY_CHUNK", 1024);
  CH = CH < 1 ? 1 : CH > SPECCAP ? SPECCAP : CH;  // the stitch caches one chunk
  const bool simple = env_int("PROTEUS_REPLAY_SIMPLE", 0) != 0;
  int64_t h_off[2][PX_MAXD + 2];
  for (int rt = 0; rt < 2; rt++)
    if (devOff[rt])
      PX_CUDA(ctx, cudaMemcpyAsync(h_off[rt], devOff[rt], (D + 2) * 8, cudaMemcpyDeviceToHost, ctx->stream));
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
  uint32_t *latd = (uint32_t *)px_buf(ctx, B_R_LATD, (size_t)S * N * 4 + 64);  // B_R_LAT stages host outputs
  if (!latd) return px_fail(ctx, PROTEUS_ENOMEM, "latency scratch");
  SpecExit *ex = nullptr;
  // phase runs (k_spec): lanes with 2 <= Bmax <= rmax also speculate each
  // chunk from its (r + 1)-th query, r < Bmax, so the true run (which enters
  // a chunk up to Bmax - 1 queries late) always has a run that starts with it
  const int rmax = simple ? 1 : env_int("PROTEUS_REPLAY_PHASES", 1);
  uint32_t *vlat = nullptr;
  SpecExit *vex = nullptr;
  int64_t *d_voff = nullptr;
  int rz = 1;
  if (!simple) {
    std::vector<int64_t> voff(2 * (size_t)S * D, 0);
    int64_t vtot = 0, vxtot = 0;
    for (int s = 0; s < S; s++) {
      const int rt = h_sc[s].routing;
      for (int d = 0; d < D; d++) {
        int Bmax = 0;
        if (h_option[d] > 0) {
          const int32_t *Tr = ctx->lat.data() + ((size_t)h_dev_type[d] * M + (h_option[d] - 1)) * ctx->bmax;
          int depth = 0;
          while (depth < ctx->bmax && Tr[depth] > 0) depth++;
          const int cap = h_sc[s].batch_cap;
          Bmax = (cap > 0 && cap < depth) ? cap : depth;  // as k_lane_params
        }
        const int R = n_phase_runs(Bmax, rmax);
        const int64_t nd = h_off[rt][d + 1] - h_off[rt][d], nchd = (nd + CH - 1) / CH;
        voff[(size_t)s * D + d] = vtot;
        voff[(size_t)S * D + (size_t)s * D + d] = vxtot;
        vtot += (int64_t)(R - 1) * nd;
        vxtot += (int64_t)(R - 1) * nchd;
        if (R > rz && nchd > 1) rz = R;
      }
    }
    if (rz > 1) {
      vlat = (uint32_t *)px_buf(ctx, B_R_VLAT, (size_t)vtot * 4 + 16);
      vex = (SpecExit *)px_buf(ctx, B_R_VEX, sizeof(SpecExit) * (size_t)(vxtot + 1));
      d_voff = (int64_t *)px_buf(ctx, B_R_VOFF, voff.size() * 8);
      if (!vlat || !vex || !d_voff) return px_fail(ctx, PROTEUS_ENOMEM, "phase-run buffers");
      PX_CUDA(ctx, cudaMemcpyAsync(d_voff, voff.data(), voff.size() * 8, cudaMemcpyHostToDevice, ctx->stream));
    }
    const int64_t nmax = NCH[0] > NCH[1] ? NCH[0] : NCH[1];
    ex = (SpecExit *)px_buf(ctx, B_R_LANE, sizeof(SpecExit) * (size_t)S * (nmax + 1));
    if (!ex) return px_fail(ctx, PROTEUS_ENOMEM, "speculation states");
    PX_CUDA(ctx, cudaFuncSetAttribute(k_stitch, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      (int)stitch_smem(ctx->bmax)));
  }
  for (int rt = 0; rt < 2; rt++) {
    if (scl[rt].empty()) continue;
    LaneArgs la;
    memset(&la, 0, sizeof la);
    la.S = S; la.D = D; la.M = M; la.bmax = ctx->bmax; la.nsc = (int)scl[rt].size(); la.CH = CH;
    la.N = N; la.NCH = NCH[0] > NCH[1] ? NCH[0] : NCH[1];  // one row stride for both routing modes
    la.option = d_opt; la.dev_type = d_dev; la.lat = ctx->d_lat; la.sc_list = d_scl + rt * S; la.lp = d_lp;
    la.devOff = devOff[rt]; la.choff = d_choff + rt * (PX_MAXD + 2); la.goff = d_goff + rt * (PX_MAXD + 2);
    la.devArr = devArr[rt]; la.latd = latd; la.ex = ex; la.agg = d_agg;
    la.debug = env_int("PROTEUS_REPLAY_DEBUG", 0);
    la.maxchk = env_int("PROTEUS_REPLAY_CHECKS", 1 << 30);
    la.rmax = rz > 1 ? rmax : 1;
    la.vlat = vlat; la.vex = vex; la.voff = d_voff;
    if (simple) {
      const int nl = la.nsc * D;
      PX_LAUNCH(ctx, "replay_lanes", k_lanes, (nl + LANE_THREADS - 1) / LANE_THREADS, LANE_THREADS, 0, la);
    } else {
      if (ngroups[rt] > 0) {
        if ((ngroups[rt] + 3) / 4 > 65535) return px_fail(ctx, PROTEUS_ERANGE, "too many replay chunks");
        dim3 grid((unsigned)la.nsc, (unsigned)((ngroups[rt] + 3) / 4));
        PX_LAUNCH(ctx, "replay_spec", k_spec, grid, 128, 0, la, 0);
        if (rz > 1) {
          dim3 gv(grid.x, grid.y, (unsigned)(rz - 1));
          PX_LAUNCH(ctx, "replay_spec_phase", k_spec, gv, 128, 0, la, 1);
        }
      }
      const int64_t warps = (int64_t)la.nsc * D;
      PX_LAUNCH(ctx, "replay_stitch", k_stitch, (unsigned)((warps + 3) / 4), 128,
                stitch_smem(ctx->bmax), la);
    }
    dim3 g(32, la.nsc < 65535 ? la.nsc : 65535);
    PX_LAUNCH(ctx, "replay_sink", k_sink, g, 256, 0, N, S, D, d_scl + rt * S, la.nsc, devOff[rt], latd, d_agg);
    int nsm = 0;
    PX_CUDA(ctx, cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, ctx->device));
    int64_t cbx = (N + 4095) / 4096;
    const int64_t cap_bx = ((int64_t)nsm * 64 + la.nsc - 1) / la.nsc;
    if (cbx > cap_bx) cbx = cap_bx > 0 ? cap_bx : 1;
    dim3 cg((unsigned)cbx, (unsigned)la.nsc);
    PX_LAUNCH(ctx, "replay_count", k_count, cg, 256, 0, N, S, D, d_scl + rt * S, devOff[rt], d_lp, latd, d_agg);
  }
  if (d_lat_out) {
    int nsm = 0;
    PX_CUDA(ctx, cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, ctx->device));
    const int64_t nb = (N + 256 * UNP_PER - 1) / (256 * UNP_PER);
    PX_LAUNCH(ctx, "replay_unpermute", k_unpermute, (unsigned)nb, 256, 0, N, S, d_sc, inv[0], inv[1], latd, d_lat_out);
  }
  return 0;
}
