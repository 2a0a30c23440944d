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
#ifndef FLAT_RK
#define FLAT_RK 1    // outer prefixes per thread per work item, in units of K
#endif
#ifndef FLAT_WAGG
#define FLAT_WAGG 1  // one grid-bound atomic per warp (0: per thread)
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
// k_flat_fam<QM, VM>: mode 0 with families supplied in accuracy order and
// Q <= QM, V_q <= VM.  The index is split as
//   idx = o K^3 + o3 K^2 + oA K + oB,
// o = the options of devices 0..D-4 ("outer prefix"), o3, oA, oB those of
// devices D-3, D-2, D-1.  A placement's value is the sum over families of
// the family's water-fill value (Eqs. 1, 3, 5 make a device serve only its
// variant's family), so for the K^2 candidates of a block (o, o3) everything
// is a function of per-family quantities of the block's capacities c_q:
//   F_q   = fill_q(c_q)                            (the (idle, idle) value)
//   MA_q  = max_j fill_q(c_q + PA_j e_j) - F_q       (device D-2 joins family q)
//   MB_q  = max_j fill_q(c_q + PB_j e_j) - F_q       (device D-1 joins family q)
//   J_q   = max_{i,j} fill_q(c_q + PA_i e_i + PB_j e_j) - F_q   (both join q)
// and the block's maximum is EXACT:
//   sum_q F_q + max(0, max_q MA_q, max_q MB_q, max_{qa != qb} MA_qa + MB_qb, max_q J_q)
// (a candidate with oA, oB in different families scores the separable sum).
// Devices D-3 and D-4 change one family's capacities per step, so between
// consecutive blocks only one family's state is recomputed ("incremental
// family carry"): the thread keeps the states of the outer prefix (devices
// 0..D-4) for every family, and per block recomputes only the family of o3.
// A block is skipped with one compare unless its maximum beats the running
// threshold; then (rarely) its lowest index reaching the maximum is found by
// a re-scan in index order, so the thread keeps its first maximum (reading
// C9).  Capacities of the outer prefix live in shared memory ([slot][thread],
// conflict-free), the per-family states in registers (compile-time indices),
// the last two devices' capacities and the accuracies in the constant bank.
template <int QM, int VM>
struct FlatArgs {
  int32_t D, K, nvec;
  uint64_t o_lo, o_hi, per_thread;  // outer prefixes [o_lo, o_hi); per thread per work item (a multiple of K)
  uint64_t n_items;                 // work items: (item / nvec)-th span of FLAT_THREADS * per_thread outer
                                    // prefixes of vector item % nvec
  unsigned long long *counter;      // work-item counter (0 at launch)
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

// water-fill of one family: capacities c[0..VM) in fill order (reading C10),
// demand s -> packed (served << 42) + accsum
template <int QM, int VM>
__device__ __forceinline__ uint64_t fam_fill(const int (&c)[VM], int s, const FlatArgs<QM, VM> &a, int q) {
  int rem = s;
  uint64_t acc = 0;
#pragma unroll
  for (int j = 0; j < VM; j++) {
    const int t = min(rem, c[j]);
    acc += (uint64_t)(uint32_t)a.A[q * VM + j] * (uint32_t)t;
    rem -= t;
  }
  // px_pack(served, acc) with served << 42 added to the high word only
  // (accsum < 2^42, so no carry crosses the halves)
  const uint32_t hi = (uint32_t)(acc >> 32) + ((uint32_t)(s - rem) << (PX_ACC_BITS - 32));
  return ((uint64_t)hi << 32) | (uint32_t)acc;
}

struct FamState {
  uint64_t F, MA, MB, J;
};

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

// SYM: devices D-2 and D-1 have the same capacities (same device type), so
// MB = MA and the joint fills are symmetric: 1 + V + V(V+1)/2 fills instead
// of 1 + 2V + V^2
template <int QM, int VM, bool SYM>
__device__ __forceinline__ FamState fam_state(const int (&c)[VM], int s, const FlatArgs<QM, VM> &a, int q) {
  FamState st;
  st.F = fam_fill<QM, VM>(c, s, a, q);
  uint64_t ma = st.F, mb = st.F, jm = st.F;
#pragma unroll
  for (int i = 0; i < VM; i++) {
    int ci[VM];
#pragma unroll
    for (int k = 0; k < VM; k++) ci[k] = c[k] + (k == i ? a.PA[q * VM + i] : 0);
    const uint64_t fa = fam_fill<QM, VM>(ci, s, a, q);
    ma = fa > ma ? fa : ma;
    if (!SYM) {
      int cb[VM];
#pragma unroll
      for (int k = 0; k < VM; k++) cb[k] = c[k] + (k == i ? a.PB[q * VM + i] : 0);
      const uint64_t fb = fam_fill<QM, VM>(cb, s, a, q);
      mb = fb > mb ? fb : mb;
    }
#pragma unroll
    for (int j = SYM ? i : 0; j < VM; j++) {
      int cj[VM];
#pragma unroll
      for (int k = 0; k < VM; k++) cj[k] = ci[k] + (k == j ? a.PB[q * VM + j] : 0);
      const uint64_t fj = fam_fill<QM, VM>(cj, s, a, q);
      jm = fj > jm ? fj : jm;
    }
  }
  st.MA = ma - st.F;
  st.MB = (SYM ? ma : mb) - st.F;
  st.J = jm - st.F;
  return st;
}

// The block's first candidate (index order: oA-major, then oB, idle first,
// slots = codes in order) scoring Mx; returns its oA * K + oB, -1 if none
// (an internal error, caught by the materialise check).  Rare: called when a
// block beats the thread's running maximum, so it is kept out of line.  No
// arrays indexed at run time (they would live in local memory): the block's
// capacities are read from shared memory, family fills recomputed.
template <int QM, int VM>
__device__ __noinline__ int flat_rescan(const FlatArgs<QM, VM> &a, const int *sCaps /* [S][FLAT_THREADS] */,
                                        const int32_t *sDem, int s3, int p3, uint64_t base, uint64_t Mx) {
  constexpr int S = QM * VM;
  const int K = a.K;
  // capacity of slot k with devices 0..D-3 placed, plus device D-2 (sa) / D-1 (sb) when given
  auto cap = [&](int k, int sa, int sb) -> int {
    return sCaps[k * FLAT_THREADS + threadIdx.x] + (k == s3 ? p3 : 0) + (k == sa ? a.PA[k] : 0) +
           (k == sb ? a.PB[k] : 0);
  };
  auto fill = [&](int q, int sa, int sb) -> uint64_t {  // family q's water-fill value
    int c[VM];
#pragma unroll
    for (int j = 0; j < VM; j++) c[j] = cap(q * VM + j, sa, sb);
    return fam_fill<QM, VM>(c, sDem[q], a, q);
  };
  if (base == Mx) return 0;  // (idle, idle)
  for (int sb = 0; sb < S; sb++) {
    const int qb = sb / VM;
    if (base - fill(qb, -1, -1) + fill(qb, -1, sb) == Mx) return a.code[sb];
  }
  for (int sa = 0; sa < S; sa++) {
    const int qa = sa / VM;
    const uint64_t Fa = fill(qa, -1, -1);
    const uint64_t ba = base - Fa + fill(qa, sa, -1);
    if (ba == Mx) return a.code[sa] * K;
    for (int sb = 0; sb < S; sb++) {
      const int qb = sb / VM;
      const uint64_t v = qb == qa ? base - Fa + fill(qa, sa, sb) : ba - fill(qb, -1, -1) + fill(qb, -1, sb);
      if (v == Mx) return a.code[sa] * K + a.code[sb];
    }
  }
  return -1;
}

template <int QM, int VM, bool SYM>
__global__ void __launch_bounds__(FLAT_THREADS, FLAT_MINB) k_flat_fam(const __grid_constant__ FlatArgs<QM, VM> a) {
  constexpr int S = QM * VM;
  extern __shared__ int32_t smem[];
  const int D = a.D, K = a.K;
  int32_t *sP = smem;          // [D][K]
  int32_t *sCS = smem + D * K; // [K]
  for (int i = threadIdx.x; i < D * K; i += blockDim.x) sP[i] = a.Pdev[i];
  for (int i = threadIdx.x; i < K; i += blockDim.x) sCS[i] = a.code_slot[i];
  __shared__ int32_t sDem[QM];  // the work item's demand vector
  __shared__ unsigned long long sItem;
  // capacities of devices 0..D-4 per slot ([slot][thread]: conflict-free)
  __shared__ int sCaps[S][FLAT_THREADS];
  const uint64_t K2 = (uint64_t)K * K, K3 = K2 * K;
  const int ND = D - 3;  // outer digits: devices 0..D-4
  // persistent blocks: work items taken in order, vectors interleaved (item %
  // nvec), so every vector's items spread over the launch and most start with
  // the grid-wide bound of their vector already raised by earlier items
  for (;;) {
    if (threadIdx.x == 0) sItem = atomicAdd(a.counter, 1ull);
    __syncthreads();
    const uint64_t item = sItem;
    if (item >= a.n_items) break;
    const int vec = (int)(item % a.nvec);
    const uint64_t chunk = item / a.nvec;
    if (threadIdx.x < QM) sDem[threadIdx.x] = a.s[vec][threadIdx.x];
    __syncthreads();
  uint64_t o = a.o_lo + (chunk * FLAT_THREADS + threadIdx.x) * a.per_thread;
  const uint64_t oend = o + a.per_thread < a.o_hi ? o + a.per_thread : a.o_hi;
  uint64_t best_s = 0, best_i = ~0ull;
  bool rec = false;
  if (o < oend) {
    // outer digits (touched at carries only): one byte each in a register when
    // they fit (ND <= 8, K <= 256: c1, c2), else a local array
    const bool pk = ND <= 8 && K <= 256;
    uint64_t dpk = 0;
    int dig_l[PX_MAXD];
    auto DG = [&](int i) -> int { return pk ? (int)((dpk >> (8 * i)) & 255u) : dig_l[i]; };
    auto DS = [&](int i, int v) {
      if (pk) dpk = (dpk & ~(0xFFull << (8 * i))) | ((uint64_t)v << (8 * i));
      else dig_l[i] = v;
    };
    {
      uint64_t x = o;
      for (int i = ND - 1; i >= 0; i--) { DS(i, (int)(x % K)); x /= K; }
    }
    FamState st[QM];
    uint64_t Fsum = 0;
    auto fam_from_smem = [&](int q) -> FamState {
      int c[VM];
#pragma unroll
      for (int j = 0; j < VM; j++) c[j] = sCaps[q * VM + j][threadIdx.x];
      return fam_state<QM, VM, SYM>(c, sDem[q], a, q);
    };
    auto rebuild = [&]() {  // all families from the outer digits
      int cb[S];
#pragma unroll
      for (int k = 0; k < S; k++) cb[k] = 0;
      for (int i = 0; i < ND; i++) {
        const int oo = DG(i);
        const int sl = sCS[oo], pv = sP[i * K + oo];
#pragma unroll
        for (int k = 0; k < S; k++) cb[k] += (sl == k) ? pv : 0;
      }
#pragma unroll
      for (int k = 0; k < S; k++) sCaps[k][threadIdx.x] = cb[k];
      Fsum = 0;
#pragma unroll
      for (int q = 0; q < QM; q++) { st[q] = fam_from_smem(q); Fsum += st[q].F; }
    };
    rebuild();
    unsigned long long *gb = a.gbound + vec;
    for (;;) {
      // the K blocks (o, o3) of this outer prefix.  Device D-3's option
      // touches one family q3 (warp-uniform; options are grouped by family,
      // so q3 changes QM + 1 times); the other families X are fixed, so their
      // part of the block maximum is folded once per q3: JX = max J, b1 / b2 =
      // the top two MB, MAX = max MA, CX = max over a != b in X of MA_a +
      // MB_b (b may be idle: gains are >= 0)
      int cq3 = -2;
      uint64_t baseX = 0, JX = 0, b1X = 0, MAX = 0, CX = 0;
      auto fold = [&](int q3) {
        baseX = Fsum;
        JX = 0;
        b1X = 0;
        MAX = 0;
        uint64_t b2 = 0;
        int f1 = -1;
#pragma unroll
        for (int q = 0; q < QM; q++) {
          if (q == q3) { baseX -= st[q].F; continue; }
          JX = st[q].J > JX ? st[q].J : JX;
          MAX = st[q].MA > MAX ? st[q].MA : MAX;
          if (st[q].MB > b1X) { b2 = b1X; b1X = st[q].MB; f1 = q; }
          else if (st[q].MB > b2) b2 = st[q].MB;
        }
        CX = 0;
#pragma unroll
        for (int q = 0; q < QM; q++) {
          if (q == q3) continue;
          const uint64_t v = st[q].MA + (q == f1 ? b2 : b1X);
          CX = v > CX ? v : CX;
        }
      };
      for (int o3 = 0; o3 < K; o3++) {
        uint64_t G;  // best score any thread of this vector has recorded (relaxed; stale = lower)
        asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(G) : "l"(gb));
        const int s3 = sCS[o3];  // warp-uniform (-1: idle)
        const int q3 = s3 >= 0 ? s3 / VM : -1;
        if (q3 != cq3) { fold(q3); cq3 = q3; }
        FamState m;  // family q3 with device D-3's capacity added
        uint64_t base = baseX, dmax;
        if (q3 >= 0) {
          int c[VM];
#pragma unroll
          for (int j = 0; j < VM; j++) c[j] = sCaps[q3 * VM + j][threadIdx.x] + (q3 * VM + j == s3 ? sP[(D - 3) * K + o3] : 0);
          m = fam_state<QM, VM, SYM>(c, sDem[q3], a, q3);
          base += m.F;
          // both in q3 (J), b alone, a in q3 with b in X or idle, a in X with b in q3, both in X
          const uint64_t mj = m.J > JX ? m.J : JX, mb = m.MB > b1X ? m.MB : b1X;
          const uint64_t c1 = m.MA + b1X, c2 = MAX + m.MB;
          dmax = mj > mb ? mj : mb;
          dmax = c1 > dmax ? c1 : dmax;
          dmax = c2 > dmax ? c2 : dmax;
          dmax = CX > dmax ? CX : dmax;
        } else {
          dmax = JX > b1X ? JX : b1X;
          dmax = CX > dmax ? CX : dmax;
        }
        const uint64_t Mx = base + dmax;
        // threshold: the thread's best so far (strict >: the first maximum is
        // kept), raised to G - 1 (nothing below the score G of a real
        // candidate can win; ties with G still record, reading C9)
        bool take;
        if (!rec) take = G == 0 || Mx > G - 1;
        else take = Mx > best_s && (G == 0 || Mx > G - 1);
        if (take) {
          const int lp = flat_rescan<QM, VM>(a, &sCaps[0][0], sDem, s3, s3 >= 0 ? sP[(D - 3) * K + o3] : 0, base,
                                             Mx);
          best_s = Mx;
          best_i = o * K3 + (uint64_t)o3 * K2 + (uint64_t)(lp < 0 ? 0 : lp);
          rec = true;
          if (Mx > G) {
#if FLAT_WAGG
            // raise the grid-wide bound once per warp (the largest new record
            // among the lanes here): early in a launch every thread records,
            // and one address per vector would serialise their atomics
            const unsigned am = __activemask();
            const uint32_t mh = __reduce_max_sync(am, (uint32_t)(Mx >> 32));
            const uint32_t ml = __reduce_max_sync(am, (uint32_t)(Mx >> 32) == mh ? (uint32_t)Mx : 0u);
            const uint64_t mv = ((uint64_t)mh << 32) | ml;
            if (lane_id() == __ffs(__ballot_sync(am, Mx == mv)) - 1) atomicMax(gb, (unsigned long long)mv);
#else
            atomicMax(gb, (unsigned long long)Mx);
#endif
          }
        }
      }
      if (++o >= oend) break;
      if (ND == 0) break;
      // next outer prefix: device D-4 advances (one or two families change)
      const int i4 = ND - 1;
      const int old = DG(i4);
      if (old + 1 == K) {
        DS(i4, 0);
        for (int i = i4 - 1; i >= 0; i--) {
          const int v = DG(i) + 1;
          if (v < K) { DS(i, v); break; }
          DS(i, 0);
        }
        rebuild();
      } else {
        DS(i4, old + 1);
        const int s_old = sCS[old], s_new = sCS[old + 1];
        if (s_old >= 0) sCaps[s_old][threadIdx.x] -= sP[i4 * K + old];
        sCaps[s_new][threadIdx.x] += sP[i4 * K + old + 1];
        const int q_old = s_old >= 0 ? s_old / VM : -1, q_new = s_new / VM;
#pragma unroll
        for (int q = 0; q < QM; q++)
          if (q == q_old || q == q_new) {
            Fsum -= st[q].F;
            st[q] = fam_from_smem(q);
            Fsum += st[q].F;
          }
      }
    }
  }
  block_best(best_s, best_i);
  if (threadIdx.x == 0) {
    BestRec &r = a.out[(int64_t)vec * a.out_stride + (int64_t)chunk];
    r.score = best_s;
    r.index = best_i;
  }
  __syncthreads();  // sItem / sDem / block_best's shared arrays are rewritten by the next item
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
int px_occupancy(proteus_ctx *ctx, const void *kern, int threads, size_t smem, int *occ) {
  // per context and device: cached by (kernel, shared memory)
  for (auto &e : ctx->occ_cache)
    if (e.first.first == kern && e.first.second == smem) { *occ = e.second; return 0; }
  PX_CUDA(ctx, cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, kern, threads, smem));
  ctx->occ_cache.push_back({{kern, smem}, *occ});
  return 0;
}

// o_lo, o_hi: outer prefixes (devices 0..D-4) of this slice
template <int QM, int VM>
static int launch_flat(proteus_ctx *ctx, int D, int K, uint64_t o_lo, uint64_t o_hi, const int32_t *dev_type,
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
  const size_t smem = (size_t)(D * K + K) * 4;
  bool sym = true;  // devices D-2 and D-1 of one type: the symmetric family states
  for (int s = 0; s < QM * VM; s++) sym &= a.PA[s] == a.PB[s];
  auto kern = sym ? k_flat_fam<QM, VM, true> : k_flat_fam<QM, VM, false>;
  if (smem > 48 * 1024) PX_CUDA(ctx, cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int nsm = 0, occ = 0;
  PX_CUDA(ctx, cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, ctx->device));
  int rc = px_occupancy(ctx, (const void *)kern, FLAT_THREADS, smem, &occ);
  if (rc) return rc;
  if (occ < 1) occ = 1;
  const uint64_t np = o_hi - o_lo;
  // work items of FLAT_THREADS threads x per_thread outer prefixes; per_thread
  // a multiple of K (o_lo is one too, px_solve_enum), so every thread's
  // device D-4 digit carries in the same iteration
  a.o_lo = o_lo; a.o_hi = o_hi;
  a.nvec = nvec;
  uint64_t pt = (uint64_t)K * FLAT_RK;
  const uint64_t per_vec_threads = (np + pt - 1) / pt;
  if (per_vec_threads * nvec < (uint64_t)nsm * occ * FLAT_THREADS) {  // small spaces: finer items
    pt = (np * nvec + (uint64_t)nsm * occ * FLAT_THREADS - 1) / ((uint64_t)nsm * occ * FLAT_THREADS);
    if (pt < 1) pt = 1;
  }
  a.per_thread = pt;
  const uint64_t span = pt * FLAT_THREADS;
  const uint64_t items_per_vec = (np + span - 1) / span;
  if (items_per_vec > (uint64_t)out_stride) return px_fail(ctx, PROTEUS_EINTERNAL, "flat: %llu work items per vector",
                                                           (unsigned long long)items_per_vec);
  a.n_items = items_per_vec * nvec;
  a.counter = gbound + nvec;
  PX_CUDA(ctx, cudaMemsetAsync(gbound, 0, sizeof(unsigned long long) * ((size_t)nvec + 1), ctx->stream));
  uint64_t nb = (uint64_t)nsm * occ;
  if (nb > a.n_items) nb = a.n_items;
  PX_LAUNCH(ctx, "score_flat_pair", kern, (unsigned)nb, FLAT_THREADS, smem, a);
  *nblocks_out = (int)items_per_vec;
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
  BestRec *d_blocks0 = (BestRec *)px_buf(ctx, B_BEST, sizeof(BestRec) * (size_t)stride * nv + 8 * ((size_t)nv + 1));
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
        // outer prefixes (devices 0..D-4), K^3 candidates each; rank slices
        // start on a multiple of K when there are enough
        const uint64_t K3 = (uint64_t)K * K * K;
        const uint64_t NO = N / K3;
        uint64_t plo, phi;
        if (NO % (uint64_t)K == 0 && NO / K >= (uint64_t)world) {
          plo = mul_div(NO / K, rank, world) * K;
          phi = mul_div(NO / K, rank + 1, world) * K;
        } else {
          plo = mul_div(NO, rank, world);
          phi = mul_div(NO, rank + 1, world);
        }
        ncand = (phi - plo) * K3;
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
