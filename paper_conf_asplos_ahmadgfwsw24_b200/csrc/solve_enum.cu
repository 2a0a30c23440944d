// solve_enum.cu -- exhaustive allocation search, modes 0 (flat mixed radix) and
// 1 (per-type multiset): a2 candidate decode, a3 capacity aggregation, a4
// per-family water-fill, a5 score pack, a6 warp -> block -> grid argmax with
// lowest-index tie-break, a9 winner materialisation.
//
// Two scoring kernels:
//  * k_flat_pair<QM, VM>: mode 0 with families supplied in accuracy order and
//    Q <= QM, V_q <= VM.  Every thread owns a contiguous range of "prefixes"
//    (the options of devices 0..D-3); for each prefix it scores the K^2
//    candidates formed by the last two devices.  Capacities live in registers
//    (slots are compile-time indices), the per-device capacity of the last two
//    devices and the accuracies are launch parameters (constant bank), so a
//    candidate costs one 64-bit add + compare, or one joint water-fill when
//    both of the last two devices host the same family.
//  * k_enum_generic: any mode 0/1 instance within the ABI limits; decodes the
//    start index once (mixed radix over groups, combinadic unrank inside a
//    group) and walks successors, rescoring every candidate from scratch.
#include <algorithm>

#include "internal.cuh"

#ifndef FLAT_THREADS
// 512 x 1 block per SM (128 registers, 16 warps/SM).  Measured on the c2 batch
// (ms per 64 vectors) before the grid-wide bound: 384x1 16.8, 256x2 18.1,
// 512x1 17.3, 448x1 19.5, 352x1 18.5, 192x2 18.3, 128x4 18.9; with it (fewer
// flagged rows, so the spill-heavy re-scans matter less): 512x1 16.0,
// 384x1 16.4, 256x2 16.4
#define FLAT_THREADS 512
#endif
#define FLAT_NV 64  // demand vectors per flat launch (grid.x)
#ifndef FLAT_MINB
#define FLAT_MINB 1  // blocks per SM the register budget is sized for
#endif
#define GEN_THREADS 128

// ------------------------------------------------------------ reduce ----
__device__ __forceinline__ void warp_best(uint64_t &s, uint64_t &i) {
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    uint64_t s2 = __shfl_xor_sync(0xffffffffu, s, o);
    uint64_t i2 = __shfl_xor_sync(0xffffffffu, i, o);
    if (px_better(s2, i2, s, i)) { s = s2; i = i2; }
  }
}

// block-wide (score desc, index asc) maximum; result valid in thread 0
__device__ __forceinline__ void block_best(uint64_t &s, uint64_t &i) {
  __shared__ uint64_t ws[32], wi[32];
  warp_best(s, i);
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  if (lane == 0) { ws[w] = s; wi[w] = i; }
  __syncthreads();
  if (w == 0) {
    s = lane < nw ? ws[lane] : 0;
    i = lane < nw ? wi[lane] : ~0ull;
    warp_best(s, i);
  }
}

__global__ void k_best_final(const BestRec *__restrict__ in, int n, BestRec *out) {
  uint64_t s = 0, i = ~0ull;
  for (int k = threadIdx.x; k < n; k += blockDim.x)
    if (px_better(in[k].score, in[k].index, s, i)) { s = in[k].score; i = in[k].index; }
  block_best(s, i);
  if (threadIdx.x == 0) { out->score = s; out->index = i; }
}

// ------------------------------------------------------ group layout ----
// Candidates are tuples per group; a group's devices are interchangeable and
// take a non-decreasing option tuple (mode 0: every device is a group of one).
// Index = mixed radix over groups (group 0 most significant) of the tuple's
// lexicographic rank (reading C9).
struct EnumArgs {
  int32_t D, K, Q, VM, npos, ngroups;
  int32_t pos_dev[PX_MAXD];
  int32_t pos_group[PX_MAXD];
  int32_t group_start[PX_MAXD + 1];
  uint64_t group_stride[PX_MAXD];
  uint64_t lo, hi, per_thread;
  int32_t s[PX_MAXQ];
  int32_t V[PX_MAXQ];
  const int32_t *Pdev, *code_slot, *slot_acc, *slot_code;
  BestRec *out;
};

__device__ __forceinline__ uint64_t binom_dev(uint64_t n, uint64_t k) {
  if (k > n) return 0;
  if (k > n - k) k = n - k;
  unsigned __int128 r = 1;
  for (uint64_t i = 1; i <= k; i++) r = r * (n - k + i) / i;
  return (uint64_t)r;
}

// rank r -> non-decreasing tuple of length len over [0, K), lexicographic
__device__ void unrank_tuple(uint64_t r, int len, int K, int32_t *out) {
  int v = 0;
  for (int i = 0; i < len; i++) {
    int rest = len - i - 1;
    for (;; v++) {
      // tuples of length `rest` over symbols [v, K)
      uint64_t cnt = binom_dev((uint64_t)(K - v) + rest - 1, (uint64_t)rest);
      if (r < cnt) break;
      r -= cnt;
    }
    out[i] = v;
  }
}

__device__ void decode_index(const EnumArgs &a, uint64_t idx, int32_t *opt /* [npos] */) {
  for (int g = 0; g < a.ngroups; g++) {
    uint64_t r = idx / a.group_stride[g];
    idx -= r * a.group_stride[g];
    int gs = a.group_start[g], len = a.group_start[g + 1] - gs;
    unrank_tuple(r, len, a.K, opt + gs);
  }
}

// -------------------------------------------------- generic scoring ----
__global__ void __launch_bounds__(GEN_THREADS) k_enum_generic(const __grid_constant__ EnumArgs a) {
  __shared__ int32_t sAcc[PX_MAXQ * PX_MAXV];
  __shared__ int32_t sCS[PX_MAXM + 1];
  for (int i = threadIdx.x; i < a.Q * a.VM; i += blockDim.x) sAcc[i] = a.slot_acc[i];
  for (int i = threadIdx.x; i < a.K; i += blockDim.x) sCS[i] = a.code_slot[i];
  __syncthreads();
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  uint64_t c = a.lo + tid * a.per_thread;
  const uint64_t cend = c + a.per_thread < a.hi ? c + a.per_thread : a.hi;
  uint64_t best_s = 0, best_i = ~0ull;
  if (c < cend) {
    int32_t opt[PX_MAXD];
    int32_t cap[PX_MAXQ * PX_MAXV];
    for (int i = 0; i < a.Q * a.VM; i++) cap[i] = 0;
    decode_index(a, c, opt);
    for (int p = 0; p < a.npos; p++) {
      int o = opt[p];
      if (o) cap[sCS[o]] += __ldg(&a.Pdev[a.pos_dev[p] * a.K + o]);
    }
    for (;;) {
      uint64_t score = 0;
      for (int q = 0; q < a.Q; q++) {
        int rem = a.s[q];
        uint64_t acc = 0;
        for (int j = 0; j < a.V[q]; j++) {
          int t = min(rem, cap[q * a.VM + j]);
          acc += (uint64_t)(uint32_t)sAcc[q * a.VM + j] * (uint32_t)t;
          rem -= t;
        }
        score += px_pack((uint32_t)(a.s[q] - rem), acc);
      }
      if (px_better(score, c, best_s, best_i)) { best_s = score; best_i = c; }
      if (++c >= cend) break;
      // successor: rightmost group that can advance; its suffix is reset
      int p = a.npos - 1;
      for (;;) {
        int g = a.pos_group[p], gs = a.group_start[g], ge = a.group_start[g + 1];
        int i = ge - 1;
        while (i >= gs && opt[i] == a.K - 1) i--;
        if (i >= gs) {
          int nv = opt[i] + 1;
          for (int j = i; j < ge; j++) {
            int o = opt[j], dv = a.pos_dev[j];
            if (o) cap[sCS[o]] -= __ldg(&a.Pdev[dv * a.K + o]);
            opt[j] = nv;
            cap[sCS[nv]] += __ldg(&a.Pdev[dv * a.K + nv]);
          }
          break;
        }
        for (int j = gs; j < ge; j++) {
          int o = opt[j];
          if (o) cap[sCS[o]] -= __ldg(&a.Pdev[a.pos_dev[j] * a.K + o]);
          opt[j] = 0;
        }
        p = gs - 1;  // carry into the previous group (exists: c < hi)
      }
    }
  }
  block_best(best_s, best_i);
  if (threadIdx.x == 0) { a.out[blockIdx.x].score = best_s; a.out[blockIdx.x].index = best_i; }
}

// -------------------------------------------- specialised flat kernel ----
template <int QM, int VM>
struct FlatArgs {
  int32_t D, K;
  uint64_t p_lo, p_hi, per_thread;
  int32_t A[QM * VM];   // accuracy per slot
  int32_t PA[QM * VM];  // capacity of slot on device D-2
  int32_t PB[QM * VM];  // capacity of slot on device D-1
  int32_t code[QM * VM];
  int32_t s[FLAT_NV][QM];  // demand of each vector of the launch (grid.x)
  int64_t out_stride;      // rows of block winners per vector
  const int32_t *Pdev, *code_slot;
  BestRec *out;
  unsigned long long *gbound;  // per vector of the launch: best score any thread has found (0 at launch)
};

// water-fill of family q over slots q*VM..q*VM+VM-1, with capacity pa added
// to slot ja and pb to slot jb (compile-time; -1 = none) -> packed score
template <int QM, int VM>
__device__ __forceinline__ uint64_t fill(const int (&caps)[QM * VM], const FlatArgs<QM, VM> &a,
                                         const int32_t *sd, int q, int ja, int pa, int jb, int pb) {
  int rem = sd[q];
  uint64_t acc = 0;
#pragma unroll
  for (int j = 0; j < VM; j++) {
    int c = caps[q * VM + j] + (j == ja ? pa : 0) + (j == jb ? pb : 0);
    int t = min(rem, c);
    acc += (uint64_t)(uint32_t)a.A[q * VM + j] * (uint32_t)t;
    rem -= t;
  }
  return px_pack((uint32_t)(sd[q] - rem), acc);
}

template <int QM, int VM>
__global__ void __launch_bounds__(FLAT_THREADS, FLAT_MINB) k_flat_pair(const __grid_constant__ FlatArgs<QM, VM> a) {
  constexpr int S = QM * VM;
  extern __shared__ int32_t smem[];
  const int D = a.D, K = a.K;
  int32_t *sP = smem;          // [D][K]
  int32_t *sCS = smem + D * K; // [K]
  for (int i = threadIdx.x; i < D * K; i += blockDim.x) sP[i] = a.Pdev[i];
  for (int i = threadIdx.x; i < K; i += blockDim.x) sCS[i] = a.code_slot[i];
  __shared__ int32_t sDem[QM];  // this block's demand vector (grid.x)
  // grid.x = vector (fastest), grid.y = prefix range: the blocks of one vector
  // are spread over the whole launch, so most of them start with the
  // grid-wide bound of their vector already raised by the earlier ones
  const int vec = blockIdx.x, blk = blockIdx.y;
  if (threadIdx.x < QM) sDem[threadIdx.x] = a.s[vec][threadIdx.x];
  __syncthreads();
  const uint64_t tid = (uint64_t)blk * blockDim.x + threadIdx.x;
  uint64_t p = a.p_lo + tid * a.per_thread;
  const uint64_t pend = p + a.per_thread < a.p_hi ? p + a.per_thread : a.p_hi;
  const uint64_t KK = (uint64_t)K * K;
  uint64_t best_s = 0, best_i = ~0ull;
  if (p < pend) {
    int dig[PX_MAXD];
    {
      uint64_t x = p;
      for (int i = D - 3; i >= 0; i--) { dig[i] = (int)(x % K); x /= K; }
    }
    // capacities of devices 0..D-4 per slot: rebuilt only when a digit above
    // D-3 changes, kept in shared memory ([slot][thread], conflict-free) to
    // leave the registers to the candidate loop
    __shared__ int sCapsB[S][FLAT_THREADS];
    auto rebuild = [&]() {
      int cb[S];
#pragma unroll
      for (int s = 0; s < S; s++) cb[s] = 0;
      for (int i = 0; i < D - 3; i++) {
        const int o = dig[i];
        const int sl = sCS[o], pv = sP[i * K + o];
#pragma unroll
        for (int s = 0; s < S; s++) cb[s] += (sl == s) ? pv : 0;
      }
#pragma unroll
      for (int s = 0; s < S; s++) sCapsB[s][threadIdx.x] = cb[s];
    };
    rebuild();
    unsigned long long *gb = a.gbound + vec;
    for (;;) {
      // grid-wide lower bound: the best score any thread of this vector has
      // recorded so far (relaxed load, issued early; a stale value is only lower)
      uint64_t G;
      asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(G) : "l"(gb));
      const int o3 = dig[D - 3];
      const int sl3 = sCS[o3], p3 = sP[(D - 3) * K + o3];
      int caps[S];
#pragma unroll
      for (int s = 0; s < S; s++) caps[s] = sCapsB[s][threadIdx.x] + (sl3 == s ? p3 : 0);
      uint64_t Fq[QM];
      uint64_t base = 0;
#pragma unroll
      for (int q = 0; q < QM; q++) { Fq[q] = fill<QM, VM>(caps, a, sDem, q, -1, 0, -1, 0); base += Fq[q]; }
      uint64_t Fb[S];
#pragma unroll
      for (int s = 0; s < S; s++) Fb[s] = fill<QM, VM>(caps, a, sDem, s / VM, s % VM, a.PB[s], -1, 0) - Fq[s / VM];
      // The K^2 candidates of this prefix, one row per option of device D-2
      // (idle first).  Fast path per row: a candidate of another family than
      // the row's scores ba + Fb[sb] (Fb >= 0), so the row holds one above the
      // running best lb iff the largest such Fb exceeds lb - ba (M1 / M2
      // below: one compare for all of them); a same-family candidate is
      // scored through its joint water-fill.  The compares only flag the row.  A flagged row (it holds a better
      // candidate) is re-scanned in index order with strict >, so the first
      // (lowest-index) maximum is kept.  If lb < ba the row's first candidate
      // (sa, idle) = ba already flags the row, so the unsigned threshold never
      // matters when it wraps.  Pad slots (code 0, capacity 0) score exactly
      // like the idle option with the same index and never change the result.
      // Largest delta of device D-1 over all its options (M1, family fm1) and
      // over the options outside family fm1 (M2): a row of family qa holds an
      // other-family candidate above lb iff (qa == fm1 ? M2 : M1) > lb - ba.
      uint64_t M1 = 0, M2 = 0;
      int fm1 = -1;
#pragma unroll
      for (int q = 0; q < QM; q++) {
        uint64_t mq = Fb[q * VM];
#pragma unroll
        for (int j = 1; j < VM; j++) mq = Fb[q * VM + j] > mq ? Fb[q * VM + j] : mq;
        if (mq > M1) { M2 = M1; M1 = mq; fm1 = q; }
        else if (mq > M2) M2 = mq;
      }
      uint64_t lb = best_s;
      int lp = -1;
      if (best_i == ~0ull) { lb = base; lp = 0; }  // the thread's first candidate
      // Candidates below G cannot be the answer (G is the score of a real
      // candidate), so the threshold is raised to G - 1: the rows still flag
      // every candidate >= G (ties with G keep the lowest index), and the thread
      // that holds the first maximum records it -- its score M >= G always
      // exceeds the threshold until the thread has recorded M.  A thread that
      // records nothing reports (0, ~0), the neutral element of the argmax.
      if (G > 0 && G - 1 > lb) { lb = G - 1; lp = -1; }
      {
        const uint64_t thr = lb - base;
        if (base > lb || M1 > thr) {
          if (base > lb) { lb = base; lp = 0; }
#pragma unroll
          for (int sb = 0; sb < S; sb++)
            if (base + Fb[sb] > lb) { lb = base + Fb[sb]; lp = a.code[sb]; }
        }
      }
#pragma unroll
      for (int sa = 0; sa < S; sa++) {
        const int qa = sa / VM;
        const uint64_t ba = base + fill<QM, VM>(caps, a, sDem, qa, sa % VM, a.PA[sa], -1, 0) - Fq[qa];
        uint64_t jv[VM];  // same-family candidates (joint fills)
#pragma unroll
        for (int jb = 0; jb < VM; jb++)
          jv[jb] = base - Fq[qa] + fill<QM, VM>(caps, a, sDem, qa, sa % VM, a.PA[sa], jb, a.PB[qa * VM + jb]);
        const uint64_t thr = lb - ba;
        bool f0 = ba > lb || (qa == fm1 ? M2 : M1) > thr;
#pragma unroll
        for (int jb = 0; jb < VM; jb++) f0 |= jv[jb] > lb;
        if (f0) {
          if (ba > lb) { lb = ba; lp = a.code[sa] * K; }
#pragma unroll
          for (int sb = 0; sb < S; sb++) {
            const uint64_t c = (qa == sb / VM) ? jv[sb % VM] : ba + Fb[sb];
            if (c > lb) { lb = c; lp = a.code[sa] * K + a.code[sb]; }
          }
        }
      }
      if (lp >= 0) {
        best_s = lb;
        best_i = p * KK + (uint64_t)lp;
        if (lb > G) atomicMax(gb, (unsigned long long)lb);
      }
      if (++p >= pend) break;
      if (++dig[D - 3] == K) {
        dig[D - 3] = 0;
        for (int i = D - 4; i >= 0; i--) {
          if (++dig[i] < K) break;
          dig[i] = 0;
        }
        rebuild();
      }
    }
  }
  block_best(best_s, best_i);
  if (threadIdx.x == 0) {
    BestRec &o = a.out[(int64_t)vec * a.out_stride + blk];
    o.score = best_s;
    o.index = best_i;
  }
}

// ------------------------------------------------------- materialise ----
// a9: decode the winner, water-fill z in (accuracy desc, code asc, device asc)
// order (reading C10), report served / unmet / accsum / eff; re-check the score.
// a6 (grid level) is folded in: the block first reduces the per-block winners.
// Block v materialises vector v of a batch: its per-block results start at
// blocks + v * stride, its demand at dem_all + v * Q (dem_all NULL: a.s).
__global__ void k_materialize_enum(const __grid_constant__ EnumArgs a, const BestRec *__restrict__ blocks, int nb,
                                   uint64_t fixed_index, int use_fixed, uint64_t n_candidates, SolRec *out,
                                   int64_t stride, const int32_t *__restrict__ dem_all) {
  blocks += (int64_t)blockIdx.x * stride;
  out += blockIdx.x;
  __shared__ int32_t sS[PX_MAXQ];
  for (int q = threadIdx.x; q < a.Q; q += blockDim.x) sS[q] = dem_all ? dem_all[(int64_t)blockIdx.x * a.Q + q] : a.s[q];
  // the tables thread 0 walks, staged in shared memory (its loop is serial)
  __shared__ int32_t sPdev[8192];
  __shared__ int32_t sCode[PX_MAXQ * PX_MAXV], sAcc[PX_MAXQ * PX_MAXV];
  const bool staged = a.D * a.K <= 8192;
  if (staged)
    for (int k = threadIdx.x; k < a.D * a.K; k += blockDim.x) sPdev[k] = a.Pdev[k];
  for (int k = threadIdx.x; k < a.Q * a.VM; k += blockDim.x) { sCode[k] = a.slot_code[k]; sAcc[k] = a.slot_acc[k]; }
  uint64_t bs = 0, bi = ~0ull;
  if (!use_fixed)
    for (int k = threadIdx.x; k < nb; k += blockDim.x)
      if (px_better(blocks[k].score, blocks[k].index, bs, bi)) { bs = blocks[k].score; bi = blocks[k].index; }
  block_best(bs, bi);
  if (threadIdx.x != 0) return;
  SolRec &r = *out;
  const BestRec best_rec = {bs, bi};
  const BestRec *best = &best_rec;
  uint64_t idx = use_fixed ? fixed_index : best->index;
  if (idx == ~0ull) {  // empty shard: nothing scored
    for (int d = 0; d < a.D; d++) { r.option[d] = 0; r.z[d] = 0; }
    int64_t stot = 0;
    for (int q = 0; q < a.Q; q++) stot += sS[q];
    r.score = 0; r.index = idx; r.served = 0; r.unmet = stot; r.accsum = 0; r.eff = 0;
    r.n_candidates = n_candidates; r.status = 0;
    return;
  }
  int32_t opt[PX_MAXD], o[PX_MAXD], z[PX_MAXD];  // thread-local: no global read-after-write
  decode_index(a, idx, opt);
  for (int d = 0; d < a.D; d++) { o[d] = 0; z[d] = 0; }
  for (int p = 0; p < a.npos; p++) o[a.pos_dev[p]] = opt[p];
  int64_t served = 0, accsum = 0, stot = 0;
  uint64_t score = 0;
  for (int q = 0; q < a.Q; q++) {
    int rem = sS[q];
    uint64_t acc = 0;
    stot += sS[q];
    for (int j = 0; j < a.V[q]; j++) {
      const int code = sCode[q * a.VM + j];
      const int A = sAcc[q * a.VM + j];
      for (int d = 0; d < a.D; d++) {
        if (o[d] != code) continue;
        const int t = min(rem, staged ? sPdev[d * a.K + code] : __ldg(&a.Pdev[d * a.K + code]));
        z[d] = t;
        rem -= t;
        acc += (uint64_t)A * (uint64_t)t;
      }
    }
    served += sS[q] - rem;
    accsum += (int64_t)acc;
    score += px_pack((uint32_t)(sS[q] - rem), acc);
  }
  for (int d = 0; d < a.D; d++) { r.option[d] = o[d]; r.z[d] = z[d]; }
  r.score = score;
  r.index = idx;
  r.served = served;
  r.unmet = stot - served;
  r.accsum = accsum;
  r.eff = served > 0 ? (int32_t)(accsum / served) : 0;
  r.n_candidates = n_candidates;
  r.status = (!use_fixed && score != best->score) ? 1 : 0;
}

// ------------------------------------------------------------- host -----
template <int QM, int VM>
static int launch_flat(proteus_ctx *ctx, int D, int K, uint64_t p_lo, uint64_t p_hi, const int32_t *dev_type,
                       const int32_t *demand, int nvec, const std::vector<int32_t> &h_P,
                       const std::vector<int32_t> &h_slot_code, const Tables &tab, BestRec *d_blocks,
                       int64_t out_stride, unsigned long long *gbound, int *nblocks_out) {
  FlatArgs<QM, VM> a;
  memset(&a, 0, sizeof a);
  a.D = D; a.K = K;
  const int M = ctx->M;
  for (int s = 0; s < QM * VM; s++) {
    const int q = s / VM;
    const int code = q < ctx->Q ? h_slot_code[q * VM + s % VM] : 0;
    a.code[s] = code;
    a.A[s] = code ? ctx->acc[code - 1] : 0;
    a.PA[s] = code ? h_P[dev_type[D - 2] * M + code - 1] : 0;
    a.PB[s] = code ? h_P[dev_type[D - 1] * M + code - 1] : 0;
  }
  for (int v = 0; v < nvec; v++)
    for (int q = 0; q < QM; q++) a.s[v][q] = q < ctx->Q ? demand[(size_t)v * ctx->Q + q] : 0;
  a.out_stride = out_stride;
  a.Pdev = tab.Pdev;
  a.code_slot = tab.code_slot;
  a.out = d_blocks;
  a.gbound = gbound;
  PX_CUDA(ctx, cudaMemsetAsync(gbound, 0, sizeof(unsigned long long) * (size_t)nvec, ctx->stream));
  const size_t smem = (size_t)(D * K + K) * 4;
  auto kern = k_flat_pair<QM, VM>;
  if (smem > 48 * 1024) PX_CUDA(ctx, cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int nsm = 0, occ = 0;
  PX_CUDA(ctx, cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, ctx->device));
  {  // occupancy per (instantiation, shared-memory size), queried once
    static size_t occ_smem = ~(size_t)0;
    static int occ_val = 0;
    if (occ_smem != smem) {
      PX_CUDA(ctx, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_val, kern, FLAT_THREADS, smem));
      occ_smem = smem;
    }
    occ = occ_val;
  }
  if (occ < 1) occ = 1;
  const uint64_t np = p_hi - p_lo;
  uint64_t nb = (uint64_t)nsm * occ;
  const uint64_t need = (np + FLAT_THREADS - 1) / FLAT_THREADS;
  if (need < nb) nb = need ? need : 1;
  a.p_lo = p_lo; a.p_hi = p_hi;
  a.per_thread = (np + nb * FLAT_THREADS - 1) / (nb * FLAT_THREADS);
  if (a.per_thread == 0) a.per_thread = 1;
  // a multiple of K: every thread's prefix counter then carries (and rebuilds
  // the capacities of devices 0..D-4) in the same iteration -- no divergence
  if (a.per_thread > (uint64_t)K) a.per_thread = (a.per_thread + K - 1) / K * K;
  nb = (np + a.per_thread * FLAT_THREADS - 1) / (a.per_thread * FLAT_THREADS);
  if (nb == 0) nb = 1;
  PX_LAUNCH(ctx, "score_flat_pair", kern, dim3((unsigned)nvec, (unsigned)nb), FLAT_THREADS, smem, a);
  *nblocks_out = (int)nb;
  return 0;
}

typedef int (*flat_fn)(proteus_ctx *, int, int, uint64_t, uint64_t, const int32_t *, const int32_t *, int,
                       const std::vector<int32_t> &, const std::vector<int32_t> &, const Tables &, BestRec *, int64_t,
                       unsigned long long *, int *);

struct FlatInst { int QM, VM; flat_fn fn; };
static const FlatInst kFlat[] = {
    {1, 2, launch_flat<1, 2>}, {1, 3, launch_flat<1, 3>}, {1, 4, launch_flat<1, 4>}, {1, 5, launch_flat<1, 5>},
    {2, 2, launch_flat<2, 2>}, {2, 3, launch_flat<2, 3>}, {2, 4, launch_flat<2, 4>}, {2, 5, launch_flat<2, 5>},
    {3, 2, launch_flat<3, 2>}, {3, 3, launch_flat<3, 3>}, {3, 4, launch_flat<3, 4>}, {3, 5, launch_flat<3, 5>},
    {4, 2, launch_flat<4, 2>}, {4, 3, launch_flat<4, 3>}, {4, 4, launch_flat<4, 4>}, {4, 5, launch_flat<4, 5>},
};

static const FlatInst *pick_flat(int Q, int maxV) {
  const FlatInst *best = nullptr;
  for (const auto &f : kFlat)
    if (f.QM >= Q && f.VM >= maxV && (!best || f.QM * f.VM < best->QM * best->VM)) best = &f;
  return best;
}

int px_flat_template_vm(int Q, int maxV) {
  const FlatInst *f = pick_flat(Q, maxV);
  return f ? f->VM : 0;
}

static uint64_t mul_div(uint64_t a, uint64_t b, uint64_t c) {
  return (uint64_t)((unsigned __int128)a * b / c);
}

int px_solve_enum(proteus_ctx *ctx, const proteus_solve_args *args, const int32_t *h_dev_type,
                  const int32_t *h_slo, const int32_t *h_demand, int VM, const Tables &tab,
                  const std::vector<int32_t> &h_P, const std::vector<int32_t> &h_slot_code,
                  SolRec *d_sol, int32_t vec_lo, int32_t vec_hi, bool materialize_only, uint64_t mat_index,
                  bool use_flat, const int32_t *d_demand) {
  (void)h_slo;
  const int D = args->D, K = 1 + ctx->M, Q = ctx->Q, T = ctx->T;
  const int mode = args->mode;
  // group layout
  EnumArgs ea;
  memset(&ea, 0, sizeof ea);
  ea.D = D; ea.K = K; ea.Q = Q; ea.VM = VM;
  int np = 0, ng = 0;
  if (mode == 0) {
    for (int d = 0; d < D; d++) { ea.group_start[ng] = np; ea.pos_dev[np] = d; ea.pos_group[np] = ng; np++; ng++; }
  } else {
    for (int t = 0; t < T; t++) {
      int start = np;
      for (int d = 0; d < D; d++)
        if (h_dev_type[d] == t) { ea.pos_dev[np] = d; ea.pos_group[np] = ng; np++; }
      if (np > start) { ea.group_start[ng] = start; ng++; }
    }
  }
  ea.group_start[ng] = np;
  ea.npos = np; ea.ngroups = ng;
  {
    uint64_t stride = 1;
    for (int g = ng - 1; g >= 0; g--) {
      ea.group_stride[g] = stride;
      int len = ea.group_start[g + 1] - ea.group_start[g];
      unsigned __int128 c = 1;
      for (int i = 1; i <= len; i++) c = c * (unsigned)(K - 1 + i) / (unsigned)i;
      stride = (uint64_t)((unsigned __int128)stride * c);
    }
  }
  for (int q = 0; q < Q; q++) ea.V[q] = ctx->V[q];
  ea.Pdev = tab.Pdev; ea.code_slot = tab.code_slot; ea.slot_acc = tab.slot_acc; ea.slot_code = tab.slot_code;
  bool ovf = false;
  const uint64_t N = px_count_candidates(mode, D, h_dev_type, T, K, &ovf);
  const int world = args->shard_world > 0 ? args->shard_world : 1, rank = args->shard_world > 0 ? args->shard_rank : 0;
  const bool flat_ok = use_flat;
  int nsm = 0;
  PX_CUDA(ctx, cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, ctx->device));
  const size_t max_blocks = (size_t)nsm * 64;
  // per-block winners of every vector of the batch (one row each); one
  // materialise launch for the whole batch at the end (block = vector)
  const int64_t stride = (int64_t)max_blocks + 1;
  const int nv = materialize_only ? 1 : vec_hi - vec_lo;
  // per-block winners, then one grid-wide bound per vector (flat kernel)
  BestRec *d_blocks0 = (BestRec *)px_buf(ctx, B_BEST, sizeof(BestRec) * (size_t)stride * nv + 8 * (size_t)nv);
  if (!d_blocks0) return px_fail(ctx, PROTEUS_ENOMEM, "block results");
  uint64_t ncand_all = 0;
  int nb_all = 0, flat_nb = 0;
  for (int v = vec_lo; v < vec_hi; v++) {
    BestRec *d_blocks = d_blocks0 + (materialize_only ? 0 : (int64_t)(v - vec_lo) * stride);
    const int32_t *dem = h_demand + (size_t)v * Q;
    for (int q = 0; q < Q; q++) ea.s[q] = dem[q];
    SolRec *rec = d_sol + (materialize_only ? 0 : v - vec_lo);
    uint64_t ncand = 0;
    int nb_used = 0;
    if (!materialize_only) {
      int nb = 0;
      if (flat_ok) {
        const uint64_t NP = N / ((uint64_t)K * K);
        const uint64_t plo = mul_div(NP, rank, world), phi = mul_div(NP, rank + 1, world);
        ncand = (phi - plo) * (uint64_t)K * K;
        if ((v - vec_lo) % FLAT_NV == 0) {  // one launch per FLAT_NV vectors (grid.x = vector)
          const int nvec = vec_hi - v < FLAT_NV ? vec_hi - v : FLAT_NV;
          const FlatInst *f = pick_flat(Q, *std::max_element(ctx->V.begin(), ctx->V.end()));
          unsigned long long *gbound =
              (unsigned long long *)(d_blocks0 + (size_t)stride * nv) + (v - vec_lo);
          int rc = f->fn(ctx, D, K, plo, phi, h_dev_type, dem, nvec, h_P, h_slot_code, tab, d_blocks, stride,
                         gbound, &flat_nb);
          if (rc) return rc;
        }
        nb = flat_nb;
      } else {
        const uint64_t lo = mul_div(N, rank, world), hi = mul_div(N, rank + 1, world);
        ncand = hi - lo;
        int occ = 0;
        PX_CUDA(ctx, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_enum_generic, GEN_THREADS, 0));
        uint64_t nb64 = (uint64_t)nsm * (occ > 0 ? occ : 1);
        const uint64_t need = (ncand + GEN_THREADS - 1) / GEN_THREADS;
        if (need < nb64) nb64 = need ? need : 1;
        ea.lo = lo; ea.hi = hi;
        ea.per_thread = (ncand + nb64 * GEN_THREADS - 1) / (nb64 * GEN_THREADS);
        if (!ea.per_thread) ea.per_thread = 1;
        ea.out = d_blocks;
        PX_LAUNCH(ctx, "score_generic", k_enum_generic, (unsigned)nb64, GEN_THREADS, 0, ea);
        nb = (int)nb64;
      }
      nb_used = nb;
    }
    if (materialize_only) {
      PX_LAUNCH(ctx, "argmax_materialize", k_materialize_enum, 1, 1024, 0, ea, d_blocks, nb_used, mat_index, 1,
                ncand, rec, (int64_t)0, (const int32_t *)nullptr);
    } else {
      (void)rec;
      ncand_all = ncand;  // the same slice for every vector
      nb_all = nb_used;
    }
  }
  if (!materialize_only && nv > 0)
    PX_LAUNCH(ctx, "argmax_materialize", k_materialize_enum, (unsigned)nv, 1024, 0, ea, d_blocks0, nb_all,
              (uint64_t)0, 0, ncand_all, d_sol, stride, d_demand + (size_t)vec_lo * Q);
  return 0;
}
