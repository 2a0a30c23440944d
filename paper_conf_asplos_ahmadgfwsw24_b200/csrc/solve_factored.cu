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
#define DP_THREADS 512

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
  const int2 *pairs;   // DP: for each budget b, the keys (u, b - u) of every u <= b
  const int32_t *pstart;  // [U + 1] offsets into pairs
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
// the water-fill does.  One warp per (family, usage, 32 vectors): the warp
// materialises the cell's candidates 64 at a time in shared memory (capacity
// vector in fill order + lexicographic rank; lanes decode 2 each, type T-1
// fastest so ranks ascend), then every lane water-fills each of them for its
// own vector (broadcast loads) and keeps its first maximum.
#define GV_TILE 64
template <int VMT>
__global__ void __launch_bounds__(128) k_fact_gv(const __grid_constant__ FactLayout f, int n_vec,
                                                 const int32_t *__restrict__ demand,
                                                 const int32_t *__restrict__ slot_acc, BestRec *g) {
  __shared__ int32_t tcap[4][GV_TILE][VMT];
  __shared__ uint64_t tsub[4][GV_TILE];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int item = blockIdx.x * 4 + w;
  if (item >= f.Q * f.U) return;
  const int q = item / f.U, ukey = item % f.U;
  const int vec = blockIdx.y * 32 + lane;
  const bool active = vec < n_vec;
  const int s = active ? demand[(size_t)vec * f.Q + q] : 0;
  const int T = f.T, VM = f.VM;
  int bsz[PX_MAXT], bst[PX_MAXT];
  int64_t lstride[PX_MAXT], prod = 1;
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
  int A[VMT];
#pragma unroll
  for (int j = 0; j < VMT; j++) A[j] = j < VM ? slot_acc[q * VM + j] : 0;
  uint64_t best_s = 0, best_i = ~0ull;
  for (int64_t k0 = 0; k0 < prod; k0 += GV_TILE) {
    for (int r = lane; r < GV_TILE; r += 32) {
      const int64_t k = k0 + r;
      if (k >= prod) break;
      int64_t x = k;
      int cap[VMT];
#pragma unroll
      for (int j = 0; j < VMT; j++) cap[j] = 0;
      uint64_t sub = 0;
      for (int t = T - 1; t >= 0; t--) {
        const int o = (int)(x % bsz[t]);
        x /= bsz[t];
        const int rk = f.bucket[f.list_off[q][t] + bst[t] + o];
        sub += (uint64_t)rk * lstride[t];
        const int32_t *ec = f.ecap + (f.list_off[q][t] + rk) * VM;
#pragma unroll
        for (int j = 0; j < VMT; j++) cap[j] += j < VM ? ec[j] : 0;
      }
#pragma unroll
      for (int j = 0; j < VMT; j++) tcap[w][r][j] = cap[j];
      tsub[w][r] = sub;
    }
    __syncwarp();
    const int nt = prod - k0 < GV_TILE ? (int)(prod - k0) : GV_TILE;
    for (int r = 0; r < nt; r++) {
      int rem = s;
      uint64_t acc = 0;
#pragma unroll
      for (int j = 0; j < VMT; j++) {
        const int tk = min(rem, tcap[w][r][j]);
        acc += (uint64_t)(uint32_t)A[j] * (uint32_t)tk;
        rem -= tk;
      }
      const uint64_t sc = px_pack((uint32_t)(s - rem), acc);
      if (sc > best_s || best_i == ~0ull) { best_s = sc; best_i = tsub[w][r]; }
    }
    __syncwarp();
  }
  if (active) {
    BestRec &out = g[((size_t)vec * f.Q + q) * f.U + ukey];
    out.score = best_s;
    out.index = best_i;  // ~0 when no count vector has this usage
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
  // Budget DP with the current stage in shared memory: G_q(b) = max over
  // u <= b of g_q(u) + G_{q+1}(b - u).  One warp per budget b; lanes split the
  // box {u <= b}.  Every stage is also written to global memory for the
  // reconstruction.  A score of ~0 marks "no count vector with this usage"
  // (a real score has accsum < 10^6 * served < 2^42 - 1, so it is never ~0).
  extern __shared__ uint64_t dsm[];
  const int vec = blockIdx.x;
  const int Q = f.Q, U = f.U, T = f.T;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const BestRec *gv = g + (size_t)vec * Q * U;
  uint64_t *G = Gbuf + (size_t)vec * (Q + 1) * U;
  uint64_t *Gn = dsm, *gq = dsm + U;
  const uint64_t NONE = ~0ull;
  for (int b = threadIdx.x; b < U; b += blockDim.x) { Gn[b] = 0; G[(size_t)Q * U + b] = 0; }
  for (int q = Q - 1; q >= 0; q--) {
    for (int u = threadIdx.x; u < U; u += blockDim.x) {
      const BestRec e = gv[(size_t)q * U + u];
      gq[u] = e.index == ~0ull ? NONE : e.score;
    }
    __syncthreads();
    uint64_t *Gq = G + (size_t)q * U;
    for (int b = w; b < U; b += nw) {
      // lanes stride over the precomputed (u, b - u) key pairs of budget b
      uint64_t best = 0;
      bool have = false;
      const int pe = f.pstart[b + 1];
      for (int k = f.pstart[b] + lane; k < pe; k += 32) {
        const int2 pr = __ldg(&f.pairs[k]);
        const uint64_t gs = gq[pr.x];
        if (gs == NONE) continue;
        const uint64_t c = gs + Gn[pr.y];
        if (!have || c > best) { best = c; have = true; }
      }
      for (int o = 16; o; o >>= 1) {
        const uint64_t b2 = __shfl_xor_sync(0xffffffffu, best, o);
        const int h2 = __shfl_xor_sync(0xffffffffu, (int)have, o);
        if (h2 && (!have || b2 > best)) { best = b2; have = true; }
      }
      if (lane == 0) Gq[b] = best;  // u = 0 is always valid: have == true
    }
    __syncthreads();
    for (int b = threadIdx.x; b < U; b += blockDim.x) Gn[b] = Gq[b];
    __syncthreads();
  }
  // reconstruction (warp 0): lexicographically smallest count tensor
  __shared__ uint64_t pick_sub[PX_MAXQ];
  if (threadIdx.x < 32) {
    const int lane = threadIdx.x;
    int bv[PX_MAXT];
    for (int t = 0; t < T; t++) bv[t] = f.Nt[t];
    for (int q = 0; q < Q; q++) {
      int bkey = 0, box = 1;
      for (int t = 0; t < T; t++) { bkey += bv[t] * f.ustride[t]; box *= bv[t] + 1; }
      const uint64_t target = G[(size_t)q * U + bkey];
      uint64_t bsub = ~0ull;
      uint64_t bu = 0;
      for (int i = lane; i < box; i += 32) {
        int x = i, uk = 0, rk = 0;
        for (int t = T - 1; t >= 0; t--) {
          const int ut = x % (bv[t] + 1);
          x /= bv[t] + 1;
          uk += ut * f.ustride[t];
          rk += (bv[t] - ut) * f.ustride[t];
        }
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
  (void)h_P;
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
  for (int q = 0; q < Q; q++) {
    f.V[q] = ctx->V[q];
    f.off[q] = ctx->off[q];
    for (int t = 0; t < T; t++) {
      unsigned __int128 c = 1;
      for (int i = 1; i <= ctx->V[q]; i++) c = c * (unsigned)(f.Nt[t] + i) / (unsigned)i;
      if (c > (1u << 24)) return px_fail(ctx, PROTEUS_ERANGE, "count-vector list too large");
      f.list_off[q][t] = total;
      total += (int64_t)c;
    }
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
  // the DP's (u, b - u) key pairs of every budget b (lattice indexing only)
  if (ctx->dp_pairs_U != U || ctx->dp_pairs_key != std::vector<int32_t>(f.Nt, f.Nt + T)) {
    std::vector<int32_t> pst(U + 1);
    std::vector<int2> pr;
    for (int b = 0; b < U; b++) {
      pst[b] = (int32_t)pr.size();
      int bv[PX_MAXT], box = 1;
      for (int t = 0; t < T; t++) { bv[t] = (b / f.ustride[t]) % (f.Nt[t] + 1); box *= bv[t] + 1; }
      for (int x0 = 0; x0 < box; x0++) {
        int x = x0, uk = 0, rk = 0;
        for (int t = T - 1; t >= 0; t--) {
          const int ut = x % (bv[t] + 1);
          x /= bv[t] + 1;
          uk += ut * f.ustride[t];
          rk += (bv[t] - ut) * f.ustride[t];
        }
        pr.push_back(make_int2(uk, rk));
      }
      if (pr.size() > (1u << 26)) return px_fail(ctx, PROTEUS_ERANGE, "usage lattice too large for the DP");
    }
    pst[U] = (int32_t)pr.size();
    char *pb = (char *)px_buf(ctx, B_FACT3, pr.size() * sizeof(int2) + pst.size() * 4 + 64);
    if (!pb) return px_fail(ctx, PROTEUS_ENOMEM, "DP pairs");
    PX_CUDA(ctx, cudaMemcpyAsync(pb, pr.data(), pr.size() * sizeof(int2), cudaMemcpyHostToDevice, ctx->stream));
    PX_CUDA(ctx, cudaMemcpyAsync(pb + pr.size() * sizeof(int2), pst.data(), pst.size() * 4, cudaMemcpyHostToDevice,
                                 ctx->stream));
    ctx->dp_pairs = pb;
    ctx->dp_pairs_n = (int64_t)pr.size();
    ctx->dp_pairs_U = U;
    ctx->dp_pairs_key.assign(f.Nt, f.Nt + T);
  }
  f.pairs = (const int2 *)ctx->dp_pairs;
  f.pstart = (const int32_t *)((const char *)ctx->dp_pairs + ctx->dp_pairs_n * sizeof(int2));
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
  if (n_vec >= 8 && VM <= 8) {
    dim3 grid((unsigned)((Q * U + 3) / 4), (unsigned)((n_vec + 31) / 32));
    if (VM <= 3) PX_LAUNCH(ctx, "fact_g", k_fact_gv<3>, grid, 128, 0, f, n_vec, d_demand, tab.slot_acc, g);
    else if (VM == 4) PX_LAUNCH(ctx, "fact_g", k_fact_gv<4>, grid, 128, 0, f, n_vec, d_demand, tab.slot_acc, g);
    else if (VM == 5) PX_LAUNCH(ctx, "fact_g", k_fact_gv<5>, grid, 128, 0, f, n_vec, d_demand, tab.slot_acc, g);
    else if (VM == 6) PX_LAUNCH(ctx, "fact_g", k_fact_gv<6>, grid, 128, 0, f, n_vec, d_demand, tab.slot_acc, g);
    else PX_LAUNCH(ctx, "fact_g", k_fact_gv<8>, grid, 128, 0, f, n_vec, d_demand, tab.slot_acc, g);
  } else {
    PX_LAUNCH(ctx, "fact_g", k_fact_g, (unsigned)((nitems + FG_WARPS - 1) / FG_WARPS), FG_WARPS * 32, 0, f, n_vec,
              d_demand, tab.slot_acc, g);
  }
  const size_t dsmem = (size_t)2 * U * 8;
  if (dsmem > 200 * 1024) return px_fail(ctx, PROTEUS_ERANGE, "usage lattice %lld too large for the DP", (long long)U);
  if (dsmem > 48 * 1024)
    PX_CUDA(ctx, cudaFuncSetAttribute(k_fact_dp, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsmem));
  PX_LAUNCH(ctx, "fact_dp", k_fact_dp, n_vec, DP_THREADS, dsmem, f, g, G, d_demand, d_dev, D, tab.Pdev, K,
            tab.slot_code, tab.slot_acc, d_sol);
  return 0;
}
