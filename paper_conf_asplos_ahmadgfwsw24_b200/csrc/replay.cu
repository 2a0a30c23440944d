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

// stable scatter into device-major arrays
__global__ void k_scatter(const uint8_t *__restrict__ target, const uint32_t *__restrict__ arr, int64_t N, int D,
                          const int32_t *__restrict__ devBase, const int64_t *__restrict__ devOff, uint32_t *devArr,
                          uint32_t *devIdx) {
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
    if (valid) { devArr[pos] = arr[i]; devIdx[pos] = (uint32_t)i; }
  }
}

// --------------------------------------------------------------- lanes ----
struct SpecExit {
  int64_t F;
  int32_t ov;  // exit head - window end (overhang of the last batch into the next window)
  int32_t pad;
};

struct LaneArgs {
  int S, D, M, bmax, Q;
  int64_t N, ntiles;
  const int32_t *option, *dev_type, *fam_of_m, *acc, *lat, *slo_base;
  const proteus_scenario *sc;
  // one routing mode
  int nsc, win_tiles, nwin, use_tile;
  const int32_t *sc_list;
  const int64_t *devOff;   // [D + 2]
  const int32_t *devBase;  // [ntiles + 1][D + 1]
  const uint32_t *devArr, *devIdx;
  uint32_t *lat_out;       // [S][N]
  SpecExit *ex;            // [S][D][nwin]
};

struct LaneP {
  int Bmax;
  int64_t L;
};

__device__ __forceinline__ LaneP lane_params(const LaneArgs &a, int s, int d, const int32_t *T) {
  int depth = 0;
  while (depth < a.bmax && T[depth] > 0) depth++;
  const proteus_scenario sc = a.sc[s];
  LaneP p;
  p.Bmax = (sc.batch_cap > 0 && sc.batch_cap < depth) ? sc.batch_cap : depth;  // R4
  p.L = (int64_t)sc.slo_mult_milli * a.slo_base[a.fam_of_m[a.option[d] - 1]] / 1000;  // R12
  return p;
}

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

struct PtrArr {
  const uint32_t *p;
  __device__ __forceinline__ uint32_t operator()(int64_t j) const { return p[j]; }
};

// ---- fallback: one thread per (device, scenario) walks the whole array
__global__ void __launch_bounds__(LANE_THREADS) k_lanes(const __grid_constant__ LaneArgs a) {
  const int lane_id = blockIdx.x * blockDim.x + threadIdx.x;
  if (lane_id >= a.nsc * a.D) return;
  const int s = a.sc_list[lane_id / a.D], d = lane_id % a.D;
  if (a.option[d] <= 0) return;
  const int64_t st = a.devOff[d], n = a.devOff[d + 1] - st;
  if (n == 0) return;
  const uint32_t *idx = a.devIdx + st;
  const int32_t *T = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
  const LaneP p = lane_params(a, s, d, T);
  uint32_t *out = a.lat_out + (size_t)s * a.N;
  if (p.Bmax < 1) {  // cannot run even batch 1: never routed to (z = 0 / depth 0), kept for safety
    for (int64_t j = 0; j < n; j++) out[idx[j]] = 0xFFFFFFFFu;
    return;
  }
  PtrArr arr{a.devArr + st};
  int64_t h = 0, F = 0;  // R13
  while (h < n) {
    int64_t t;
    const int b = decide(arr, n, h, F, p.Bmax, p.L, T, &t);
    F = t + T[b - 1];
    for (int j = 0; j < b; j++) out[idx[h + j]] = sat_lat(F - (int64_t)arr(h + j));
    h += b;
  }
}

// ---- phase A: speculative windows
// grid (nwin, scenario groups of 32, device groups of 32); warp = device,
// lane = scenario.  A window's arrivals and query indices of every device are
// staged in shared memory.  With use_tile (one device group) the window's
// output rows of the block's 32 scenarios are assembled in shared memory
// (initialised to "dropped" so sink queries need no extra pass) and flushed
// with coalesced stores.
__global__ void k_spec(const __grid_constant__ LaneArgs a) {
  extern __shared__ uint32_t sm[];
  __shared__ int sOff[33], sStage[32];
  const int c = blockIdx.x, sg = blockIdx.y, dg = blockIdx.z;
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  const int d = dg * 32 + w;
  const int win = a.win_tiles * TILE;
  const int64_t i0 = (int64_t)c * win;
  const int wlen = (int)(a.N - i0 < win ? a.N - i0 : win);
  const int stage_cap = win + nw * a.bmax;
  const int tstride = win + 1;                                   // padded rows: no bank conflicts
  uint32_t *tile = sm;                                          // [32][tstride] if use_tile
  int32_t *sT = (int32_t *)(sm + (a.use_tile ? 32 * tstride : 0));  // [nw][bmax]
  uint32_t *sA = (uint32_t *)(sT + nw * a.bmax);                // staged arrivals [stage_cap]
  uint32_t *sI = sA + stage_cap;                                // staged query indices [stage_cap]
  const int64_t tile0 = (int64_t)c * a.win_tiles;
  const int64_t tile1 = tile0 + a.win_tiles < a.ntiles ? tile0 + a.win_tiles : a.ntiles;
  const bool dvalid = d < a.D;
  const int64_t n_d = dvalid ? a.devOff[d + 1] - a.devOff[d] : 0;
  const int64_t st = dvalid ? a.devBase[tile0 * (a.D + 1) + d] : 0;
  const int64_t en = dvalid ? a.devBase[tile1 * (a.D + 1) + d] : 0;
  const int64_t len = en - st;
  const bool host = dvalid && a.option[d] > 0 && len > 0;
  const int64_t look = n_d - en < a.bmax ? n_d - en : a.bmax;
  const int stage = host ? (int)(len + look) : 0;
  if (lane == 0) sStage[w] = stage;
  if (a.use_tile)
    for (int k = threadIdx.x; k < 32 * tstride; k += blockDim.x) tile[k] = 0xFFFFFFFFu;
  __syncthreads();
  if (threadIdx.x == 0) {
    int acc = 0;
    for (int k = 0; k < nw; k++) { sOff[k] = acc; acc += sStage[k]; }
    sOff[nw] = acc;
  }
  __syncthreads();
  uint32_t *arr = sA + sOff[w];
  uint32_t *ixs = sI + sOff[w];
  const int32_t *T = sT + w * a.bmax;
  if (host) {
    const uint32_t *src = a.devArr + a.devOff[d] + st, *isrc = a.devIdx + a.devOff[d] + st;
    for (int k = lane; k < stage; k += 32) {
      arr[k] = src[k];
      ixs[k] = k < len ? isrc[k] : 0;
    }
    const int32_t *row = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
    for (int k = lane; k < a.bmax; k += 32) sT[w * a.bmax + k] = row[k];
  }
  __syncthreads();
  const int si = sg * 32 + lane;
  if (host && si < a.nsc) {
    const int s = a.sc_list[si];
    const LaneP p = lane_params(a, s, d, T);
    uint32_t *out = a.use_tile ? tile + (size_t)lane * tstride : a.lat_out + (size_t)s * a.N;
    const uint32_t obase = a.use_tile ? (uint32_t)i0 : 0u;
    int64_t h = 0, F = 0;
    if (p.Bmax < 1) {
      if (!a.use_tile)
        for (int64_t j = 0; j < len; j++) out[ixs[j] - obase] = 0xFFFFFFFFu;
      h = len;
    } else {
      PtrArr A{arr};
      while (h < len) {
        int64_t t;
        const int b = decide(A, stage, h, F, p.Bmax, p.L, T, &t);
        F = t + T[b - 1];
        const int64_t jend = h + b < len ? h + b : len;
        for (int64_t j = h; j < jend; j++) out[ixs[j] - obase] = sat_lat(F - (int64_t)arr[j]);
        h += b;
      }
    }
    SpecExit e;
    e.F = F;
    e.ov = (int32_t)(h - len);
    e.pad = 0;
    a.ex[((size_t)s * a.D + d) * a.nwin + c] = e;
  }
  if (!a.use_tile) return;
  __syncthreads();
  for (int r = 0; r < 32; r++) {
    if (sg * 32 + r >= a.nsc) break;
    uint32_t *row = a.lat_out + (size_t)a.sc_list[sg * 32 + r] * a.N + i0;
    const uint32_t *tr = tile + (size_t)r * tstride;
    for (int k = threadIdx.x; k < wlen; k += blockDim.x) row[k] = tr[k];
  }
}

// ---- phase B: exact stitch, one warp per (device, scenario)
// The true state (h, F) is carried from window to window.  A window whose
// speculative start (its first query, device idle) equals the true state is
// already right.  Otherwise the true run is replayed batch by batch until it
// meets the speculative run: after a batch [h, j2) finishing at Fn, if the
// speculative run also has a batch ending at j2 - 1 with finish Fn (its
// latency + arrival) and a new batch at j2, both runs are in the same state
// (j2, Fn) and agree from there on.  Only batches that the device waited for
// (t > F) are tested: a batch dispatched the moment the previous one finished
// can only meet a run that had already met.  Backlogged stretches (Bmax
// queued when the device frees) are full batches back to back -- batch k
// finishes at F + (k+1) T(Bmax) -- and are taken 32 batches per step with a
// ballot.  The device's arrivals and query indices stream through a
// shared-memory ring; window bounds and exit states are fetched 32 windows
// at a time.
#define SBUF 2048
#define SAHEAD 1088

struct BufArr {
  const uint32_t *buf, *g;
  int64_t base;
  __device__ __forceinline__ uint32_t operator()(int64_t j) const {
    const int64_t o = j - base;
    return (o >= 0 && o < SBUF) ? buf[o] : __ldg(g + j);
  }
};

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

// decide() with the counting done 32 arrivals at a time by the warp
template <class Arr>
__device__ __forceinline__ int decide_warp(const Arr &A, int64_t n, int64_t h, int64_t F, int Bmax, int64_t L,
                                           const int32_t *T, int lane, int64_t *t_out) {
  const int64_t ah = A(h);
  int64_t t = F > ah ? F : ah;
  int q = count_le(A, n, h, 1, Bmax, t, lane);
  int b;
  for (;;) {
    if (q >= Bmax) { b = Bmax; break; }
    const int64_t W = ah + L - T[q];
    if (t >= W) { b = q; break; }
    if (h + q < n) {
      const int64_t nx = A(h + q);
      if (nx <= W) {
        t = nx;
        q = count_le(A, n, h, q, Bmax, t, lane);
        continue;
      }
    }
    t = W;
    b = q;
    break;
  }
  *t_out = t;
  return b;
}

// The same decision with the serial Case-2 loop replaced by one ballot over
// up to 32 queue states: state k holds k + 1 queries at tau_k = max(t0,
// a[h + k]); it is "complete" when the next arrival comes strictly later (or
// the queue is at Bmax), and the batch leaves at the first complete state that
// must dispatch now (k + 1 = Bmax, or tau_k >= Tmax_wait(k + 2)) or whose
// timer Tmax_wait(k + 2) fires before the next arrival.  Ts[b - 1] = T(b).
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
      const int64_t ts = __shfl_sync(0xffffffffu, now ? tau : W, src);
      *t_out = ts;
      return kb + src + 1;
    }
  }
}

__global__ void __launch_bounds__(128) k_stitch(const __grid_constant__ LaneArgs a) {
  extern __shared__ uint32_t ssm[];  // [4 warps][2][SBUF], then [4 warps][bmax] latencies T
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int64_t gw = (int64_t)blockIdx.x * 4 + w;
  if (gw >= (int64_t)a.nsc * a.D || a.nwin < 2) return;
  const int s = a.sc_list[gw / a.D], d = (int)(gw % a.D);
  if (a.option[d] <= 0) return;
  const int64_t n = a.devOff[d + 1] - a.devOff[d];
  if (n == 0) return;
  uint32_t *bufA = ssm + (size_t)w * 2 * SBUF, *bufI = bufA + SBUF;
  const uint32_t *garr = a.devArr + a.devOff[d], *gix = a.devIdx + a.devOff[d];
  const int32_t *Tg = a.lat + ((size_t)a.dev_type[d] * a.M + (a.option[d] - 1)) * a.bmax;
  int32_t *T = (int32_t *)(ssm + 4 * 2 * SBUF) + w * a.bmax;
  for (int k = lane; k < a.bmax; k += 32) T[k] = Tg[k];
  __syncwarp();
  const LaneP p = lane_params(a, s, d, T);
  if (p.Bmax < 1) return;
  uint32_t *out = a.lat_out + (size_t)s * a.N;
  const SpecExit *ex = a.ex + ((size_t)s * a.D + d) * a.nwin;
  BufArr A{bufA, garr, -(int64_t)(4 * SBUF)};
  auto ensure = [&](int64_t h) {
    if (h >= A.base && h + SAHEAD <= A.base + SBUF) return;
    __syncwarp();
    A.base = h & ~(int64_t)31;
    for (int k = lane; k < SBUF; k += 32) {
      const int64_t j = A.base + k;
      bufA[k] = j < n ? garr[j] : 0xFFFFFFFFu;
      bufI[k] = j < n ? gix[j] : 0u;
    }
    __syncwarp();
  };
  auto IX = [&](int64_t j) -> uint32_t {
    const int64_t o = j - A.base;
    return (o >= 0 && o < SBUF) ? bufI[o] : __ldg(gix + j);
  };
  auto write_batch = [&](int64_t lo, int64_t hi, int64_t Fb) {
    for (int64_t j = lo + lane; j < hi; j += 32) out[IX(j)] = sat_lat(Fb - (int64_t)A(j));
  };
  const int64_t TB = T[p.Bmax - 1];
  const int64_t nwin = a.nwin;
  auto tile_of = [&](int64_t c) { return c * a.win_tiles < a.ntiles ? c * a.win_tiles : a.ntiles; };
  int64_t h = a.devBase[tile_of(1) * (a.D + 1) + d] + ex[0].ov, F = ex[0].F;
  for (int64_t c0 = 1; c0 < nwin; c0 += 32) {
    // lane k prefetches window c0 + k: its start, end and speculative exit
    const int64_t ck = c0 + lane;
    int64_t pst = 0, pen = 0, pF = 0;
    int pov = 0;
    if (ck < nwin) {
      pst = a.devBase[tile_of(ck) * (a.D + 1) + d];
      pen = a.devBase[tile_of(ck + 1) * (a.D + 1) + d];
      const SpecExit e = ex[ck];
      pF = e.F;
      pov = e.ov;
    }
    const int cnt = nwin - c0 < 32 ? (int)(nwin - c0) : 32;
    for (int k = 0; k < cnt; k++) {
      const int64_t st = __shfl_sync(0xffffffffu, pst, k), en = __shfl_sync(0xffffffffu, pen, k);
      const int64_t eF = __shfl_sync(0xffffffffu, pF, k);
      const int eov = __shfl_sync(0xffffffffu, pov, k);
      if (en == st) continue;
      if (h > st) {  // queries of this window in the last batch of the previous one
        ensure(st);
        write_batch(st, h < en ? h : en, F);
      }
      if (h >= en) continue;
      ensure(h);
      if (h == st && F <= (int64_t)A(st)) {  // speculative start = true state
        h = en + eov;
        F = eF;
        continue;
      }
      int checks = 4;  // meeting tests per window (each costs a global round trip)
      while (h < en) {
        ensure(h);
        if (F > (int64_t)A(h) && h + p.Bmax - 1 < n && (int64_t)A(h + p.Bmax - 1) <= F) {
          // backlog: full batches back to back
          int64_t kmax = (en - h + p.Bmax - 1) / p.Bmax;
          const int64_t room = (A.base + SBUF - h) / p.Bmax;
          if (kmax > room) kmax = room;
          if (kmax > 32) kmax = 32;
          const int64_t idx = h + (int64_t)(lane + 1) * p.Bmax - 1;
          const bool ok = lane < kmax && idx < n && (int64_t)A(idx) <= F + (int64_t)lane * TB;
          const unsigned bal = __ballot_sync(0xffffffffu, ok);
          const int r = bal == 0xffffffffu ? 32 : __ffs(~bal) - 1;
          const int64_t nq = (int64_t)r * p.Bmax;
          for (int64_t i = lane; i < nq; i += 32) {
            const int64_t kk = i / p.Bmax, j = h + i;
            out[IX(j)] = sat_lat(F + (kk + 1) * TB - (int64_t)A(j));
          }
          h += nq;
          F += (int64_t)r * TB;
          continue;
        }
        int64_t t;
        const int b = decide_par(A, n, h, F, p.Bmax, p.L, T, lane, &t);
        const int64_t Fn = t + T[b - 1];
        const int64_t j2 = h + b;
        bool conv = false;
        if (t > F && j2 < en && checks > 0) {
          checks--;
          const int64_t f1 = (int64_t)A(j2 - 1) + out[IX(j2 - 1)];
          const int64_t f2 = (int64_t)A(j2) + out[IX(j2)];
          conv = f1 == Fn && f2 != Fn;
        }
        __syncwarp();
        write_batch(h, j2 < en ? j2 : en, Fn);
        h = j2;
        F = Fn;
        if (conv) {
          h = en + eov;
          F = eF;
          break;
        }
      }
    }
  }
}

// dropped queries (the sink segment, device index D): latency UINT32_MAX (R7)
__global__ void k_sink(int64_t N, int D, const int32_t *__restrict__ sc_list, int nsc, const int64_t *devOff,
                       const uint32_t *devIdx, uint32_t *lat_out) {
  for (int k = blockIdx.y; k < nsc; k += gridDim.y) {
    const int64_t st = devOff[D], n = devOff[D + 1] - st;
    uint32_t *row = lat_out + (size_t)sc_list[k] * N;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
      row[devIdx[st + j]] = 0xFFFFFFFFu;
  }
}

// ------------------------------------------------------------- counts ----
// a13: per scenario, violations (latency > SLO of the query's family, R6;
// dropped included), on-time count and the serving variant's accuracy summed
// over on-time queries (R9).
__global__ void k_count(int64_t N, int S, int D, int Q, const proteus_scenario *__restrict__ sc,
                        const int32_t *__restrict__ slo_base, const int32_t *__restrict__ option,
                        const int32_t *__restrict__ acc, const uint8_t *__restrict__ fam,
                        const uint8_t *__restrict__ tgt0, const uint8_t *__restrict__ tgt1,
                        const uint32_t *__restrict__ lat, uint64_t *agg) {
  __shared__ int64_t sL[PX_MAXQ];
  __shared__ uint32_t sA[PX_MAXD + 1];
  __shared__ unsigned long long red[3][32];
  const int s = blockIdx.y;
  const proteus_scenario scn = sc[s];
  if (threadIdx.x < Q) sL[threadIdx.x] = (int64_t)scn.slo_mult_milli * slo_base[threadIdx.x] / 1000;
  if (threadIdx.x <= D) sA[threadIdx.x] = threadIdx.x < D && option[threadIdx.x] > 0 ? acc[option[threadIdx.x] - 1] : 0;
  __syncthreads();
  const uint8_t *tgt = scn.routing ? tgt1 : tgt0;
  const uint32_t *row = lat + (size_t)s * N;
  unsigned long long viol = 0, ont = 0, accs = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t l = row[i];
    if ((int64_t)l > sL[fam[i]]) viol++;
    else { ont++; accs += sA[tgt[i]]; }
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
  const size_t small = (size_t)(4 * D + 2 * Q + 2 * PX_MAXQ + 8 + 2 * S) * 4 + (size_t)S * sizeof(proteus_scenario);
  char *sb = (char *)px_buf(ctx, B_R_MISC, small + 4096);
  if (!sb) return px_fail(ctx, PROTEUS_ENOMEM, "replay scratch");
  int32_t *d_opt = (int32_t *)sb, *d_z = d_opt + D, *d_dev = d_z + D, *d_dem = d_dev + D, *d_slo = d_dem + Q;
  int32_t *d_pat_off = d_slo + Q, *d_pat_len = d_pat_off + PX_MAXQ;
  uint32_t *d_flags = (uint32_t *)(d_pat_len + PX_MAXQ);
  int32_t *d_scl = (int32_t *)(d_flags + 8);  // [2][S] scenario lists per routing mode
  proteus_scenario *d_sc = (proteus_scenario *)(((uintptr_t)(d_scl + 2 * S) + 15) & ~(uintptr_t)15);
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
  const int64_t ntiles = (N + TILE - 1) / TILE;
  const unsigned tblocks = (unsigned)((ntiles + TILE_WARPS - 1) / TILE_WARPS);
  int64_t dsum = 0;
  for (int q = 0; q < Q; q++) dsum += h_demand[q];
  const size_t pat_cap = (size_t)dsum + (size_t)Q * D + 16;
  const int64_t *devOff[2] = {nullptr, nullptr};
  const int32_t *devBase[2] = {nullptr, nullptr};
  const uint32_t *devArr[2] = {nullptr, nullptr}, *devIdx[2] = {nullptr, nullptr};
  const uint8_t *tgts[2] = {nullptr, nullptr};
  for (int rt = 0; rt < 2; rt++) {
    if (scl[rt].empty()) continue;
    uint8_t *pat = (uint8_t *)px_buf(ctx, B_R_PAT, pat_cap);
    int32_t *hist = (int32_t *)px_buf(ctx, B_R_HIST, (size_t)(ntiles + 1) * (PX_MAXD + 2) * 4);
    int32_t *fbase = (int32_t *)px_buf(ctx, B_R_BASE, (size_t)(ntiles + 1) * (PX_MAXQ + 2) * 4);
    int32_t *dbase = (int32_t *)px_buf(ctx, rt ? B_R_DBASE1 : B_R_DBASE0, (size_t)(ntiles + 1) * (PX_MAXD + 2) * 4);
    uint8_t *tgt = (uint8_t *)px_buf(ctx, rt ? B_R_TGT1 : B_R_TGT, (size_t)N + 16);
    int64_t *off = (int64_t *)px_buf(ctx, rt ? B_R_OFF1 : B_R_OFF, (size_t)2 * (PX_MAXD + 2) * 8);
    uint32_t *darr = (uint32_t *)px_buf(ctx, rt ? B_R_DEVARR1 : B_R_DEVARR, (size_t)N * 4 + 16);
    uint32_t *didx = (uint32_t *)px_buf(ctx, rt ? B_R_DEVIDX1 : B_R_DEVIDX, (size_t)N * 4 + 16);
    if (!pat || !hist || !fbase || !dbase || !tgt || !off || !darr || !didx)
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
                didx);
    } else {
      PX_CUDA(ctx, cudaMemsetAsync(off, 0, (size_t)(PX_MAXD + 2) * 8, ctx->stream));
    }
    devOff[rt] = off; devArr[rt] = darr; devIdx[rt] = didx; devBase[rt] = dbase; tgts[rt] = tgt;
  }
  if (N == 0) return 0;
  // the stitch reads speculative latencies, so rows exist even when the caller wants none
  uint32_t *lat = d_lat_out;
  if (!lat) {
    lat = (uint32_t *)px_buf(ctx, B_R_LAT, (size_t)S * N * 4);
    if (!lat) return px_fail(ctx, PROTEUS_ENOMEM, "latency scratch");
  }
  const int win_tiles = env_int("PROTEUS_REPLAY_WIN_TILES", 2);
  const int nwin = (int)((ntiles + win_tiles - 1) / win_tiles);
  const int win = win_tiles * TILE;
  const int dpb = D < 32 ? D : 32;
  const int ndg = (D + 31) / 32;
  int use_tile = ndg == 1 && !env_int("PROTEUS_REPLAY_NO_TILE", 0);
  auto spec_smem = [&](int tile) {
    return ((size_t)(tile ? 32 * (win + 1) : 0) + (size_t)dpb * ctx->bmax + 2 * ((size_t)win + (size_t)dpb * ctx->bmax)) * 4;
  };
  if (use_tile && spec_smem(1) > 200 * 1024) use_tile = 0;
  const size_t smem = spec_smem(use_tile);
  const bool simple = env_int("PROTEUS_REPLAY_SIMPLE", 0) != 0 || smem > 200 * 1024;
  SpecExit *ex = nullptr;
  if (!simple) {
    ex = (SpecExit *)px_buf(ctx, B_R_LANE, sizeof(SpecExit) * (size_t)S * D * nwin);
    if (!ex) return px_fail(ctx, PROTEUS_ENOMEM, "speculation states");
    if (smem > 48 * 1024)
      PX_CUDA(ctx, cudaFuncSetAttribute(k_spec, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    PX_CUDA(ctx, cudaFuncSetAttribute(k_stitch, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      4 * 2 * SBUF * 4 + 4 * ctx->bmax * 4));
  }
  for (int rt = 0; rt < 2; rt++) {
    if (scl[rt].empty()) continue;
    LaneArgs la;
    memset(&la, 0, sizeof la);
    la.S = S; la.D = D; la.M = M; la.bmax = ctx->bmax; la.Q = Q; la.N = N; la.ntiles = ntiles;
    la.option = d_opt; la.dev_type = d_dev; la.fam_of_m = ctx->d_fam; la.acc = ctx->d_acc; la.lat = ctx->d_lat;
    la.slo_base = d_slo; la.sc = d_sc;
    la.nsc = (int)scl[rt].size(); la.win_tiles = win_tiles; la.nwin = nwin; la.use_tile = simple ? 0 : use_tile;
    la.sc_list = d_scl + rt * S;
    la.devOff = devOff[rt]; la.devBase = devBase[rt]; la.devArr = devArr[rt]; la.devIdx = devIdx[rt];
    la.lat_out = lat; la.ex = ex;
    if (simple) {
      const int nl = la.nsc * D;
      PX_LAUNCH(ctx, "replay_lanes", k_lanes, (nl + LANE_THREADS - 1) / LANE_THREADS, LANE_THREADS, 0, la);
    } else {
      dim3 grid(nwin, (la.nsc + 31) / 32, ndg);
      PX_LAUNCH(ctx, "replay_spec", k_spec, grid, dpb * 32, smem, la);
      const int64_t warps = (int64_t)la.nsc * D;
      PX_LAUNCH(ctx, "replay_stitch", k_stitch, (unsigned)((warps + 3) / 4), 128, 4 * 2 * SBUF * 4 + 4 * ctx->bmax * 4,
                la);
    }
    if (simple || !la.use_tile) {
      dim3 g(64, la.nsc < 65535 ? la.nsc : 65535);
      PX_LAUNCH(ctx, "replay_sink", k_sink, g, 256, 0, N, D, d_scl + rt * S, la.nsc, devOff[rt], devIdx[rt], lat);
    }
  }
  int nsm = 0;
  PX_CUDA(ctx, cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, ctx->device));
  int bx = (int)((N + 255) / 256);
  const int cap_bx = (nsm * 8 + S - 1) / S;
  if (bx > cap_bx) bx = cap_bx > 0 ? cap_bx : 1;
  dim3 cg(bx, S);
  PX_LAUNCH(ctx, "replay_count", k_count, cg, 256, 0, N, S, D, Q, d_sc, d_slo, d_opt, ctx->d_acc, d_fam,
            tgts[0] ? tgts[0] : tgts[1], tgts[1] ? tgts[1] : tgts[0], lat, d_agg);
  return 0;
}
