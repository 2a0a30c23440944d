// solve_factored.cu -- mode 2, the family-factored exact search (a8) and the
// batched per-second re-solve (a10).
//
// Eqs. 1, 3 and 5 make a device serve only the family of the
// variant it hosts, so a placement's value is the sum over families of the
// family's water-fill value, which depends only on the family's count vector
// n[t][v] (devices of type t hosting variant v).  The search is therefore
//   g_q(u) = max over count vectors of family q with usage u (u_t = sum_v n[t][v])
//   G_q(b) = max_{u <= b} g_q(u) + G_{q+1}(b - u),  G_Q = 0,  optimum G_0(N),
// and the canonical solution is the lexicographically smallest tensor n
// (q-major, then t, then v) among optima (reading C9), reconstructed family
// by family.  Variants with P = 0 on a type are never used by that solution
// (reading C16) and are left out of the type's count vectors.
//
// Kernels:
//  k_fact_lists  one thread per (family, type): the type's count vectors in
//                lexicographic order (rank), their capacity vector in fill
//                order, their usage, and a stable bucketing by usage.
//  k_fact_g      one warp per (vector, family, usage u): the product of the
//                per-type usage buckets, water-filled and reduced to the best
//                (score desc, lexicographic rank asc).
//  k_fact_dp     one block per vector: the budget DP over the usage lattice,
//                reconstruction, materialisation (a9).
#include <algorithm>

#include "internal.cuh"

#define FG_WARPS 8
#ifndef DP_THREADS
#define DP_THREADS 256  // c4 fact_dp: 128 1.95 ms, 256 1.97, 512 2.20 (barrier stalls)
#endif

struct FactLayout {
  int32_t Q, T, VM, U;
  int32_t Nt[PX_MAXT];
  int32_t ustride[PX_MAXT];           // u key = sum_t u_t * ustride[t], type T-1 stride 1
  int64_t list_off[PX_MAXQ][PX_MAXT]; // entry offset of list (q, t)
  int32_t V[PX_MAXQ], off[PX_MAXQ];
  // device arrays
  int32_t *L;          // [Q][T] list lengths
  int32_t *bstart;     // [Q][T][PX_MAXD + 2] bucket starts by usage
  int32_t *bucket;     // [entries] ranks ordered by (usage, rank)
  int32_t *ecap;       // [entries][VM] capacity vector in fill (slot) order
  uint8_t *ecnt;       // [entries][16] counts in caller's variant order
  int32_t *esum;       // [entries]
  uint32_t fmask[PX_MAXQ];  // bit t: family q has a variant with P > 0 on type t (else u_t = 0)
  int32_t morder[PX_MAXQ];  // family q's DP work list: row of items
  int32_t nitems[PX_MAXQ];  // its length
  int64_t istride;          // row stride of items
  const int2 *items;        // [rows][istride] DP work items (lattice indexing only, see k_fact_dp)
};

// ------------------------------------------------------------- lists ----
__global__ void k_fact_lists(const __grid_constant__ FactLayout f, const int32_t *__restrict__ P,
                             const int32_t *__restrict__ slot_of, int M) {
  const int id = blockIdx.x * blockDim.x + threadIdx.x;
  if (id >= f.Q * f.T) return;
  const int q = id / f.T, t = id % f.T;
  const int V = f.V[q], N = f.Nt[t];
  const int64_t base = f.list_off[q][t];
  int feas[PX_MAXV], capv[PX_MAXV], jof[PX_MAXV];
  for (int v = 0; v < V; v++) {
    const int m = f.off[q] + v;
    capv[v] = P[t * M + m];
    feas[v] = capv[v] > 0;
    jof[v] = slot_of[m] - q * f.VM;
  }
  int n[PX_MAXV];
  for (int v = 0; v < V; v++) n[v] = 0;
  int cnt_by_sum[PX_MAXD + 2];
  for (int u = 0; u <= N + 1; u++) cnt_by_sum[u] = 0;
  int r = 0, sum = 0;
  for (;;) {
    // emit entry r
    int32_t *cap = f.ecap + (base + r) * f.VM;
    for (int j = 0; j < f.VM; j++) cap[j] = 0;
    for (int v = 0; v < V; v++) {
      cap[jof[v]] = n[v] * capv[v];
      f.ecnt[(base + r) * 16 + v] = (uint8_t)n[v];
    }
    for (int v = V; v < 16; v++) f.ecnt[(base + r) * 16 + v] = 0;
    f.esum[base + r] = sum;
    cnt_by_sum[sum]++;
    r++;
    // lexicographic successor: rightmost feasible position that can grow,
    // later positions reset to 0
    int i = V - 1;
    for (; i >= 0; i--) {
      if (!feas[i]) continue;
      int pre = 0;
      for (int k = 0; k < i; k++) pre += n[k];
      if (pre + n[i] + 1 <= N) break;
    }
    if (i < 0) break;
    n[i]++;
    for (int k = i + 1; k < V; k++) n[k] = 0;
    sum = 0;
    for (int k = 0; k < V; k++) sum += n[k];
  }
  f.L[id] = r;
  int32_t *bs = f.bstart + (size_t)id * (PX_MAXD + 2);
  int acc = 0;
  for (int u = 0; u <= N; u++) { bs[u] = acc; acc += cnt_by_sum[u]; }
  bs[N + 1] = acc;
  for (int u = 0; u <= N; u++) cnt_by_sum[u] = bs[u];
  for (int k = 0; k < r; k++) f.bucket[base + cnt_by_sum[f.esum[base + k]]++] = k;
}

// ----------------------------------------------------------------- g ----
__device__ __forceinline__ void warp_best_f(uint64_t &s, uint64_t &i) {
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    uint64_t s2 = __shfl_xor_sync(0xffffffffu, s, o);
    uint64_t i2 = __shfl_xor_sync(0xffffffffu, i, o);
    if (px_better(s2, i2, s, i)) { s = s2; i = i2; }
  }
}

__global__ void __launch_bounds__(FG_WARPS * 32) k_fact_g(const __grid_constant__ FactLayout f, int n_vec,
                                                          const int32_t *__restrict__ demand,
                                                          const int32_t *__restrict__ slot_acc, BestRec *g) {
  const int lane = threadIdx.x & 31;
  const int64_t item = (int64_t)blockIdx.x * FG_WARPS + (threadIdx.x >> 5);
  const int64_t nitems = (int64_t)n_vec * f.Q * f.U;
  if (item >= nitems) return;
  const int ukey = (int)(item % f.U);
  const int q = (int)((item / f.U) % f.Q);
  const int vec = (int)(item / ((int64_t)f.U * f.Q));
  const int T = f.T, VM = f.VM;
  int bsz[PX_MAXT], bst[PX_MAXT];
  int64_t lstride[PX_MAXT];
  int64_t prod = 1;
  {
    int64_t ls = 1;
    for (int t = T - 1; t >= 0; t--) {
      const int ut = (ukey / f.ustride[t]) % (f.Nt[t] + 1);
      const int32_t *bs = f.bstart + ((size_t)q * T + t) * (PX_MAXD + 2);
      bst[t] = bs[ut];
      bsz[t] = bs[ut + 1] - bs[ut];
      prod *= bsz[t];
      lstride[t] = ls;
      ls *= f.L[q * T + t];
    }
  }
  const int s = demand[(size_t)vec * f.Q + q];
  uint64_t best_s = 0, best_i = ~0ull;
  for (int64_t k = lane; k < prod; k += 32) {
    int64_t x = k;
    int cap[PX_MAXV];
    for (int j = 0; j < VM; j++) cap[j] = 0;
    uint64_t sub = 0;
    for (int t = T - 1; t >= 0; t--) {
      const int o = (int)(x % bsz[t]);
      x /= bsz[t];
      const int r = f.bucket[f.list_off[q][t] + bst[t] + o];
      sub += (uint64_t)r * lstride[t];
      const int32_t *ec = f.ecap + (f.list_off[q][t] + r) * VM;
      for (int j = 0; j < VM; j++) cap[j] += ec[j];
    }
    int rem = s;
    uint64_t acc = 0;
    for (int j = 0; j < VM; j++) {
      const int tk = min(rem, cap[j]);
      acc += (uint64_t)(uint32_t)slot_acc[q * VM + j] * (uint32_t)tk;
      rem -= tk;
    }
    const uint64_t sc = px_pack((uint32_t)(s - rem), acc);
    if (px_better(sc, sub, best_s, best_i)) { best_s = sc; best_i = sub; }
  }
  warp_best_f(best_s, best_i);
  if (lane == 0) {
    BestRec &o = g[item];
    o.score = best_s;
    o.index = best_i;  // ~0 when no count vector has this usage
  }
}

// Batched variant for many demand vectors: the count vectors of a (family,
// usage) cell and their capacity vectors do not depend on the demand, only
// the water-fill does.  One warp per (family, usage, 64 vectors), two vectors
// per lane.  The warp materialises the cell's candidates GV_TILE at a time in
// shared memory as cumulative capacities C_j = cap_0 + ... + cap_{j-1} in
// fill order (lanes decode 2 each, type T-1 fastest so ranks ascend), then
// every lane water-fills each of them for its own vectors.  The fill is
// written in summation-by-parts form: with m_j = min(s, C_j) the fill takes
// m_{j+1} - m_j from slot j, so
//   served = m_VM,   accsum = sum_{j=1..VM} m_j (A_{j-1} - A_j)   (A_VM = 0)
// -- the same integers as the sequential fill (take = min(rem, cap)), two
// instructions per slot and no serial dependence between slots.  Each lane
// keeps the first maximum in candidate order (= lowest lexicographic rank)
// as a candidate ordinal and decodes its rank once at the end.
#ifndef GV_TILE
#define GV_TILE 64
#endif
#ifndef GV_NV
#define GV_NV 2  // demand vectors per lane (2: 5.54 ms on c4; 1: 6.28, 4: 5.90, 8: 6.73)
#endif
__device__ __forceinline__ uint64_t madw(uint32_t a, uint32_t b, uint64_t c) {
  uint64_t r;
  asm("mad.wide.u32 %0, %1, %2, %3;" : "=l"(r) : "r"(a), "r"(b), "l"(c));
  return r;
}

template <int VMT, int NV>
__global__ void __launch_bounds__(128) k_fact_gv(const __grid_constant__ FactLayout f, int n_vec,
                                                 const int32_t *__restrict__ demand,
                                                 const int32_t *__restrict__ slot_acc,
                                                 const int32_t *__restrict__ cell_order, BestRec *g) {
  constexpr int CS = (VMT + 3) & ~3;  // cumulative-capacity row stride (int4 loads)
  __shared__ __align__(16) int32_t tc[4][GV_TILE][CS];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int item = blockIdx.x * 4 + w;
  if (item >= f.Q * f.U) return;
  // cells by decreasing candidate count: the warps of a block get similar
  // work and the largest cells start first
  const int cell = cell_order[item];
  const int q = cell / f.U, ukey = cell % f.U;
  uint32_t sv[NV];  // demands of this lane's vectors blockIdx.y * 32 NV + lane + 32 i
#pragma unroll
  for (int i = 0; i < NV; i++) {
    const int vec = blockIdx.y * 32 * NV + lane + 32 * i;
    sv[i] = vec < n_vec ? (uint32_t)demand[(size_t)vec * f.Q + q] : 0u;
  }
  const int T = f.T, VM = f.VM;
  // per type: start and size of the cell's usage bucket (register-resident:
  // compile-time type indices, guarded by t < T)
  int bsz[PX_MAXT], bst[PX_MAXT];
  int64_t prod = 1;
#pragma unroll
  for (int t = 0; t < PX_MAXT; t++) {
    bsz[t] = 1;
    bst[t] = 0;
    if (t < T) {
      const int ut = (ukey / f.ustride[t]) % (f.Nt[t] + 1);
      const int32_t *bs = f.bstart + ((size_t)q * T + t) * (PX_MAXD + 2);
      bst[t] = bs[ut];
      bsz[t] = bs[ut + 1] - bs[ut];
      prod *= bsz[t];
    }
  }
  uint32_t dA[VMT];  // A_{j-1} - A_j for j = 1..VMT (fill order: non-increasing; pads 0)
#pragma unroll
  for (int j = 0; j < VMT; j++) {
    const uint32_t a0 = j < VM ? (uint32_t)slot_acc[q * VM + j] : 0u;
    const uint32_t a1 = j + 1 < VM ? (uint32_t)slot_acc[q * VM + j + 1] : 0u;
    dA[j] = a0 - a1;
  }
  uint32_t blo[NV], bhi[NV];  // packed best scores (first candidate always taken)
  int32_t kbest[NV];
#pragma unroll
  for (int i = 0; i < NV; i++) { blo[i] = 0; bhi[i] = 0; kbest[i] = 0; }
  for (int64_t k0 = 0; k0 < prod; k0 += GV_TILE) {
    for (int r = lane; r < GV_TILE; r += 32) {
      const int64_t k = k0 + r;
      if (k >= prod) break;
      uint32_t x = (uint32_t)k;  // < 2^31 (host check)
      int cap[VMT];
#pragma unroll
      for (int j = 0; j < VMT; j++) cap[j] = 0;
#pragma unroll
      for (int t = PX_MAXT - 1; t >= 0; t--) {
        if (t < T) {
          const uint32_t o = x % (uint32_t)bsz[t];
          x /= (uint32_t)bsz[t];
          const int rk = f.bucket[f.list_off[q][t] + bst[t] + o];
          const int32_t *ec = f.ecap + (f.list_off[q][t] + rk) * VM;
#pragma unroll
          for (int j = 0; j < VMT; j++) cap[j] += j < VM ? ec[j] : 0;
        }
      }
      int acc = 0;
#pragma unroll
      for (int j = 0; j < VMT; j++) {
        acc += cap[j];
        tc[w][r][j] = acc;
      }
    }
    __syncwarp();
    const int nt = prod - k0 < GV_TILE ? (int)(prod - k0) : GV_TILE;
#pragma unroll 2
    for (int r = 0; r < nt; r++) {
      int32_t C[CS];
#pragma unroll
      for (int j = 0; j < CS; j += 4) *(int4 *)&C[j] = *(const int4 *)&tc[w][r][j];
      const int32_t kk = (int32_t)(k0 + r);
#pragma unroll
      for (int i = 0; i < NV; i++) {
        uint64_t a = 0;
        uint32_t m = 0;
#pragma unroll
        for (int j = 0; j < VMT; j++) {
          m = min(sv[i], (uint32_t)C[j]);
          a = madw(m, dA[j], a);
        }
        // packed score (served << 42) + accsum as (hi, lo) words; served = m_VM
        const uint32_t h = (uint32_t)(a >> 32) + (m << (PX_ACC_BITS - 32)), l = (uint32_t)a;
        if (h > bhi[i] || (h == bhi[i] && l > blo[i])) { bhi[i] = h; blo[i] = l; kbest[i] = kk; }
      }
    }
    __syncwarp();
  }
  // rank (lexicographic sub-index) of the chosen candidates
  auto sub_of = [&](uint32_t k) -> uint64_t {
    uint64_t sub = 0, ls = 1;
#pragma unroll
    for (int t = PX_MAXT - 1; t >= 0; t--) {
      if (t < T) {
        const uint32_t o = k % (uint32_t)bsz[t];
        k /= (uint32_t)bsz[t];
        sub += (uint64_t)f.bucket[f.list_off[q][t] + bst[t] + o] * ls;
        ls *= (uint64_t)f.L[q * T + t];
      }
    }
    return sub;
  };
  const bool none = prod == 0;  // no count vector has this usage
#pragma unroll
  for (int i = 0; i < NV; i++) {
    const int vec = blockIdx.y * 32 * NV + lane + 32 * i;
    if (vec < n_vec) {
      BestRec &out = g[((size_t)vec * f.Q + q) * f.U + ukey];
      out.score = ((uint64_t)bhi[i] << 32) | blo[i];
      out.index = none ? ~0ull : sub_of(kbest[i]);
    }
  }
}

// ---------------------------------------------------------------- DP ----
__device__ __forceinline__ void ukey_decode(const FactLayout &f, int key, int *u) {
  for (int t = 0; t < f.T; t++) u[t] = (key / f.ustride[t]) % (f.Nt[t] + 1);
}

__global__ void __launch_bounds__(DP_THREADS) k_fact_dp(const __grid_constant__ FactLayout f,
                                                         const BestRec *__restrict__ g, uint64_t *Gbuf,
                                                         const int32_t *__restrict__ demand,
                                                         const int32_t *__restrict__ dev_type, int D,
                                                         const int32_t *__restrict__ Pdev, int K,
                                                         const int32_t *__restrict__ slot_code,
                                                         const int32_t *__restrict__ slot_acc, SolRec *out) {
  // Budget DP with the stages in shared memory: G_q(b) = max over u <= b of
  // g_q(u) + G_{q+1}(b - u).  The boxes {u <= b} -- restricted to u_t = 0 on
  // the types where family q has no feasible variant, the only usages it can
  // have -- are cut into work items (b, outer digits of u), each a run of the
  // innermost type's digit (contiguous keys); items are listed round-robin
  // over budgets, so the threads of a warp update different budgets with a
  // shared-memory atomicMax, and every thread gets a similar share.  The key
  // of b - u is key(b) - key(u) (keys are linear).  Every stage is also
  // written to global memory for the reconstruction.  A score of ~0 marks "no
  // count vector with this usage" (a real score has accsum < 10^6 * served <
  // 2^42 - 1, so it is never ~0).
  extern __shared__ uint64_t dsm[];
  const int vec = blockIdx.x;
  const int Q = f.Q, U = f.U, T = f.T;
  const BestRec *gv = g + (size_t)vec * Q * U;
  uint64_t *G = Gbuf + (size_t)vec * (Q + 1) * U;
  uint64_t *Gn = dsm, *gq = dsm + U, *Gc = dsm + 2 * U;
  const uint64_t NONE = ~0ull;
  for (int b = threadIdx.x; b < U; b += blockDim.x) { Gn[b] = 0; Gc[b] = 0; G[(size_t)Q * U + b] = 0; }
  for (int q = Q - 1; q >= 0; q--) {
    for (int u = threadIdx.x; u < U; u += blockDim.x) {
      const BestRec e = gv[(size_t)q * U + u];
      gq[u] = e.index == ~0ull ? NONE : e.score;
    }
    __syncthreads();
    const int2 *it = f.items + (size_t)f.morder[q] * f.istride;
    const int n_it = f.nitems[q];
    const bool inner = T >= 1 && ((f.fmask[q] >> (T - 1)) & 1u);
    const int Nin = f.Nt[T - 1] + 1;
    for (int i = threadIdx.x; i < n_it; i += blockDim.x) {
      const int2 w = it[i];  // (budget key b, key of the usage's outer digits)
      const int b = w.x, up = w.y;
      const int lim_in = inner ? b % Nin : 0;  // innermost type: stride 1
      uint64_t best = 0;  // partial maxima are >= 0; u = 0 is always a usage
      for (int x = 0; x <= lim_in; x++) {
        const uint64_t gs = gq[up + x];
        if (gs == NONE) continue;
        const uint64_t c = gs + Gn[b - up - x];
        best = c > best ? c : best;
      }
      atomicMax((unsigned long long *)&Gc[b], (unsigned long long)best);
    }
    __syncthreads();
    for (int b = threadIdx.x; b < U; b += blockDim.x) {
      G[(size_t)q * U + b] = Gc[b];
      Gn[b] = 0;  // becomes the next stage's accumulator
    }
    __syncthreads();
    uint64_t *tmp = Gn; Gn = Gc; Gc = tmp;
  }
  // reconstruction (warp 0): lexicographically smallest count tensor
  __shared__ uint64_t pick_sub[PX_MAXQ];
  if (threadIdx.x < 32) {
    const int lane = threadIdx.x;
    int bv[PX_MAXT];
    for (int t = 0; t < T; t++) bv[t] = f.Nt[t];
    for (int q = 0; q < Q; q++) {
      int bkey = 0, box = 1, lim[PX_MAXT];
      for (int t = 0; t < T; t++) {
        bkey += bv[t] * f.ustride[t];
        lim[t] = (f.fmask[q] >> t) & 1u ? bv[t] : 0;
        box *= lim[t] + 1;
      }
      const uint64_t target = G[(size_t)q * U + bkey];
      uint64_t bsub = ~0ull;
      uint64_t bu = 0;
      for (int i = lane; i < box; i += 32) {
        int x = i, uk = 0, rk = 0;
        for (int t = T - 1; t >= 0; t--) {
          const int ut = x % (lim[t] + 1);
          x /= lim[t] + 1;
          uk += ut * f.ustride[t];
        }
        rk = bkey - uk;
        const BestRec e = gv[(size_t)q * U + uk];
        if (e.index == ~0ull) continue;
        if (e.score + G[(size_t)(q + 1) * U + rk] == target && e.index < bsub) { bsub = e.index; bu = (uint64_t)uk; }
      }
      for (int o = 16; o; o >>= 1) {
        const uint64_t s2 = __shfl_xor_sync(0xffffffffu, bsub, o), u2 = __shfl_xor_sync(0xffffffffu, bu, o);
        if (s2 < bsub) { bsub = s2; bu = u2; }
      }
      if (lane == 0) pick_sub[q] = bsub;
      int uu[PX_MAXT];
      ukey_decode(f, (int)bu, uu);
      for (int t = 0; t < T; t++) bv[t] -= uu[t];
    }
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  // materialise (a9): family q's pick is the mixed-radix number of its
  // per-type lexicographic ranks (type 0 most significant)
  SolRec &r = out[vec];
  int status = 0;
  for (int q = 0; q < Q; q++)
    if (pick_sub[q] == ~0ull) status = 2;
  int32_t lopt[PX_MAXD], lz[PX_MAXD];  // thread-local: no global read-after-write
  for (int d = 0; d < D; d++) { lopt[d] = 0; lz[d] = 0; }
  for (int t = 0; t < T && !status; t++) {
    int d = 0;
    for (int q = 0; q < Q; q++) {
      uint64_t ls = 1;
      for (int t2 = T - 1; t2 > t; t2--) ls *= (uint64_t)f.L[q * T + t2];
      const int rk = (int)((pick_sub[q] / ls) % (uint64_t)f.L[q * T + t]);
      const uint8_t *ec = f.ecnt + (f.list_off[q][t] + rk) * 16;
      for (int v = 0; v < f.V[q]; v++)
        for (int k = 0; k < ec[v]; k++) {
          while (d < D && dev_type[d] != t) d++;
          if (d >= D) { status = 3; break; }
          lopt[d] = 1 + f.off[q] + v;
          d++;
        }
    }
  }
  int64_t served = 0, accsum = 0, stot = 0;
  uint64_t score = 0;
  const int32_t *s = demand + (size_t)vec * Q;
  for (int q = 0; q < Q; q++) {
    int rem = s[q];
    uint64_t acc = 0;
    stot += s[q];
    for (int j = 0; j < f.VM; j++) {
      const int code = slot_code[q * f.VM + j];
      if (!code) continue;
      const int A = slot_acc[q * f.VM + j];
      for (int d = 0; d < D; d++) {
        if (lopt[d] != code) continue;
        const int tk = min(rem, Pdev[d * K + code]);
        lz[d] = tk;
        rem -= tk;
        acc += (uint64_t)A * (uint64_t)tk;
      }
    }
    served += s[q] - rem;
    accsum += (int64_t)acc;
    score += px_pack((uint32_t)(s[q] - rem), acc);
  }
  for (int d = 0; d < D; d++) { r.option[d] = lopt[d]; r.z[d] = lz[d]; }
  if (score != G[U - 1]) status = status ? status : 1;
  uint64_t ncand = 0;
  for (int q = 0; q < Q; q++) {
    uint64_t p = 1;
    for (int t = 0; t < T; t++) p *= (uint64_t)f.L[q * T + t];
    ncand += p;
  }
  r.score = score;
  r.index = ~0ull;
  r.served = served;
  r.unmet = stot - served;
  r.accsum = accsum;
  r.eff = served > 0 ? (int32_t)(accsum / served) : 0;
  r.n_candidates = ncand;
  r.status = status;
}

// -------------------------------------------------------------- host ----
int px_solve_factored(proteus_ctx *ctx, const proteus_solve_args *a, const int32_t *h_dev_type,
                      const int32_t *d_dev, const int32_t *d_demand, int VM, const Tables &tab, const std::vector<int32_t> &h_P,
                      SolRec *d_sol) {
  const int Q = ctx->Q, T = ctx->T, D = a->D, K = 1 + ctx->M;
  FactLayout f;
  memset(&f, 0, sizeof f);
  f.Q = Q; f.T = T; f.VM = VM;
  for (int d = 0; d < D; d++) f.Nt[h_dev_type[d]]++;
  int64_t U = 1;
  for (int t = T - 1; t >= 0; t--) { f.ustride[t] = (int32_t)U; U *= f.Nt[t] + 1; }
  if (U > (1 << 22)) return px_fail(ctx, PROTEUS_ERANGE, "usage lattice %lld too large", (long long)U);
  f.U = (int32_t)U;
  // list capacity: count vectors with sum <= N_t over V_q variants (before pruning)
  int64_t total = 0;
  unsigned __int128 maxprod = 0;  // bound on the candidates of one (family, usage) cell
  for (int q = 0; q < Q; q++) {
    unsigned __int128 prod = 1;
    f.V[q] = ctx->V[q];
    f.off[q] = ctx->off[q];
    for (int t = 0; t < T; t++) {
      unsigned __int128 c = 1;
      for (int i = 1; i <= ctx->V[q]; i++) c = c * (unsigned)(f.Nt[t] + i) / (unsigned)i;
      if (c > (1u << 24)) return px_fail(ctx, PROTEUS_ERANGE, "count-vector list too large");
      f.list_off[q][t] = total;
      total += (int64_t)c;
      prod *= c;
    }
    if (prod > maxprod) maxprod = prod;
  }
  if (total > (1ll << 26)) return px_fail(ctx, PROTEUS_ERANGE, "count-vector lists too large");
  const size_t szL = (size_t)Q * T * 4, szB = (size_t)Q * T * (PX_MAXD + 2) * 4;
  const size_t szE = (size_t)total * (4 + (size_t)VM * 4 + 16 + 4);
  char *buf = (char *)px_buf(ctx, B_FACT0, szL + szB + szE + 64);
  if (!buf) return px_fail(ctx, PROTEUS_ENOMEM, "factored tables");
  // the count-vector lists depend only on the (cached) capacity tables and the
  // inventory: rebuilt only when those change
  const bool lists_ok = ctx->tab_valid && ctx->fact_lists_buf == (void *)buf && ctx->fact_lists_key == ctx->tab_key;
  f.L = (int32_t *)buf; buf += szL;
  f.bstart = (int32_t *)buf; buf += szB;
  f.bucket = (int32_t *)buf; buf += (size_t)total * 4;
  f.ecap = (int32_t *)buf; buf += (size_t)total * VM * 4;
  f.esum = (int32_t *)buf; buf += (size_t)total * 4;
  f.ecnt = (uint8_t *)buf;
  // DP work items (lattice indexing only), per distinct feasibility mask:
  // (budget b, key of the outer digits u_0..u_{T-2} <= b on the mask's
  // types), round r holding the r-th outer combination of every budget
  std::vector<uint32_t> masks;
  for (int q = 0; q < Q; q++) {
    uint32_t m = 0;
    for (int t = 0; t < T; t++)
      for (int v = 0; v < ctx->V[q]; v++)
        if (h_P[(size_t)t * ctx->M + ctx->off[q] + v] > 0) m |= 1u << t;
    f.fmask[q] = m;
    int row = -1;
    for (size_t k = 0; k < masks.size(); k++) if (masks[k] == m) row = (int)k;
    if (row < 0) { row = (int)masks.size(); masks.push_back(m); }
    f.morder[q] = row;
  }
  std::vector<int32_t> okey(f.Nt, f.Nt + T);
  okey.insert(okey.end(), masks.begin(), masks.end());
  if (ctx->dp_order_U != U || ctx->dp_order_key != okey) {
    std::vector<std::vector<int2>> rows(masks.size());
    for (size_t k = 0; k < masks.size(); k++) {
      std::vector<std::vector<int32_t>> combos(U);
      size_t maxc = 0;
      for (int b = 0; b < U; b++) {
        int lim[PX_MAXT], dig[PX_MAXT] = {0};
        for (int t = 0; t < T; t++) lim[t] = (masks[k] >> t) & 1u ? (b / f.ustride[t]) % (f.Nt[t] + 1) : 0;
        for (;;) {
          int key = 0;
          for (int t = 0; t + 1 < T; t++) key += dig[t] * f.ustride[t];
          combos[b].push_back(key);
          int t = T - 2;
          for (; t >= 0; t--) {
            if (dig[t] < lim[t]) { dig[t]++; break; }
            dig[t] = 0;
          }
          if (t < 0) break;
        }
        maxc = std::max(maxc, combos[b].size());
      }
      for (size_t r = 0; r < maxc; r++)
        for (int b = 0; b < U; b++)
          if (r < combos[b].size()) rows[k].push_back(make_int2(b, combos[b][r]));
      if (rows[k].size() > (1u << 26)) return px_fail(ctx, PROTEUS_ERANGE, "usage lattice too large for the DP");
    }
    size_t stride = 0;
    for (auto &r : rows) stride = std::max(stride, r.size());
    std::vector<int2> flat(rows.size() * stride, make_int2(0, 0));
    for (size_t k = 0; k < rows.size(); k++) std::copy(rows[k].begin(), rows[k].end(), flat.begin() + k * stride);
    char *pb = (char *)px_buf(ctx, B_FACT3, flat.size() * sizeof(int2) + 64);
    if (!pb) return px_fail(ctx, PROTEUS_ENOMEM, "DP work items");
    PX_CUDA(ctx, cudaMemcpyAsync(pb, flat.data(), flat.size() * sizeof(int2), cudaMemcpyHostToDevice, ctx->stream));
    ctx->dp_order = pb;
    ctx->dp_order_U = U;
    ctx->dp_order_key = okey;
    ctx->dp_items_stride = (int64_t)stride;
    ctx->dp_items_n.clear();
    for (auto &r : rows) ctx->dp_items_n.push_back((int32_t)r.size());
  }
  f.items = (const int2 *)ctx->dp_order;
  f.istride = ctx->dp_items_stride;
  for (int q = 0; q < Q; q++) f.nitems[q] = ctx->dp_items_n[f.morder[q]];
  const int n_vec = a->n_vec;
  BestRec *g = (BestRec *)px_buf(ctx, B_FACT1, sizeof(BestRec) * (size_t)n_vec * Q * U);
  uint64_t *G = (uint64_t *)px_buf(ctx, B_FACT2, 8 * (size_t)n_vec * (Q + 1) * U);
  if (!g || !G) return px_fail(ctx, PROTEUS_ENOMEM, "factored DP buffers");
  if (!lists_ok) {
    PX_LAUNCH(ctx, "fact_lists", k_fact_lists, (Q * T + 63) / 64, 64, 0, f, tab.P, tab.slot_of, ctx->M);
    ctx->fact_lists_buf = (void *)f.L;
    ctx->fact_lists_key = ctx->tab_key;
  }
  const int64_t nitems = (int64_t)n_vec * Q * U;
  // cell order of the batched g kernel: count vectors of family q with usage
  // u_t on type t = C(u_t + f - 1, f - 1) over the f feasible variants
  std::vector<int32_t> gkey(okey);
  gkey.insert(gkey.end(), ctx->V.begin(), ctx->V.end());
  for (int q = 0; q < Q; q++)
    for (int t = 0; t < T; t++) {
      int fq = 0;
      for (int v = 0; v < ctx->V[q]; v++) fq += h_P[(size_t)t * ctx->M + ctx->off[q] + v] > 0;
      gkey.push_back(fq);
    }
  if (ctx->gv_order_key != gkey) {
    std::vector<double> sz((size_t)Q * U);
    for (int q = 0; q < Q; q++) {
      int fq[PX_MAXT];
      for (int t = 0; t < T; t++) {
        fq[t] = 0;
        for (int v = 0; v < ctx->V[q]; v++) fq[t] += h_P[(size_t)t * ctx->M + ctx->off[q] + v] > 0;
      }
      for (int u = 0; u < U; u++) {
        double x = 1;
        for (int t = 0; t < T; t++) {
          const int ut = (u / f.ustride[t]) % (f.Nt[t] + 1);
          if (fq[t] == 0) { x *= ut == 0; continue; }
          double c = 1;  // C(ut + fq - 1, fq - 1)
          for (int i = 1; i < fq[t]; i++) c = c * (ut + i) / i;
          x *= c;
        }
        sz[(size_t)q * U + u] = x;
      }
    }
    std::vector<int32_t> ord((size_t)Q * U);
    for (size_t i = 0; i < ord.size(); i++) ord[i] = (int32_t)i;
    std::stable_sort(ord.begin(), ord.end(), [&](int32_t a, int32_t b) { return sz[a] > sz[b]; });
    char *ob = (char *)px_buf(ctx, B_FACT4, ord.size() * 4 + 64);
    if (!ob) return px_fail(ctx, PROTEUS_ENOMEM, "cell order");
    PX_CUDA(ctx, cudaMemcpyAsync(ob, ord.data(), ord.size() * 4, cudaMemcpyHostToDevice, ctx->stream));
    ctx->gv_order = ob;
    ctx->gv_order_key = gkey;
  }
  const int32_t *cell_order = (const int32_t *)ctx->gv_order;
  if (n_vec >= 8 && VM <= 8 && maxprod < ((unsigned __int128)1 << 31)) {  // candidate ordinals in int32
    dim3 grid((unsigned)((Q * U + 3) / 4), (unsigned)((n_vec + 32 * GV_NV - 1) / (32 * GV_NV)));
    auto kern = VM <= 3 ? k_fact_gv<3, GV_NV> : VM == 4 ? k_fact_gv<4, GV_NV> : VM == 5 ? k_fact_gv<5, GV_NV>
              : VM == 6 ? k_fact_gv<6, GV_NV> : k_fact_gv<8, GV_NV>;
    PX_LAUNCH(ctx, "fact_g", kern, grid, 128, 0, f, n_vec, d_demand, tab.slot_acc, cell_order, g);
  } else {
    PX_LAUNCH(ctx, "fact_g", k_fact_g, (unsigned)((nitems + FG_WARPS - 1) / FG_WARPS), FG_WARPS * 32, 0, f, n_vec,
              d_demand, tab.slot_acc, g);
  }
  const size_t dsmem = (size_t)3 * U * 8;
  if (dsmem > 200 * 1024) return px_fail(ctx, PROTEUS_ERANGE, "usage lattice %lld too large for the DP", (long long)U);
  if (dsmem > 48 * 1024)
    PX_CUDA(ctx, cudaFuncSetAttribute(k_fact_dp, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsmem));
  PX_LAUNCH(ctx, "fact_dp", k_fact_dp, n_vec, DP_THREADS, dsmem, f, g, G, d_demand, d_dev, D, tab.Pdev, K,
            tab.slot_code, tab.slot_acc, d_sol);
  return 0;
}
