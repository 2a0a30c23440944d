// pareto.cu -- §8(f3): the Pareto frontier of Fig. 1b.  Every
// configuration of one family's variants on the D devices (each device hosts
// one variant, or also idles when allow_idle) has a system throughput capacity
// C = sum_d P(t_d, m_d) and a capacity-weighted accuracy sum_d P A / C (readings
// P1-P4 in DESIGN.md); the frontier is the set of configurations no other one
// beats in both.
//
//  k_pareto_opts   per (device, digit): P and P*A of the option (a1 table)
//  k_pareto_best   the candidates (mixed radix, device 0 most significant),
//                  thread-contiguous index ranges with odometer steps, reduced
//                  to the largest accuracy sum per capacity value (at equal
//                  capacity a larger sum dominates) in shared memory
//  k_pareto_front  one block: capacity c is a frontier point iff its best
//                  accuracy sum / c is strictly above every accuracy at a
//                  higher capacity (a suffix maximum of exact ratios), and the
//                  points are compacted in ascending capacity
//  k_pareto_index  second pass: the lowest index reaching each frontier point
#include <algorithm>

#include "internal.cuh"

#define PAR_THREADS 256
#define PAR_SMEM_CAP 12288  // capacity values kept in shared memory (else global atomics)

struct ParArgs {
  int D, K, idle;
  int64_t cmax;
  uint64_t lo, hi, per;            // index range of this call (shard) and per-thread share
  const int32_t *optP;             // [D][K]
  const int64_t *optPA;            // [D][K]
  long long *best;                 // [cmax + 1] largest accuracy sum per capacity (-1: none)
  const int32_t *slot;             // [cmax + 1] frontier slot of a capacity (-1: not on it)
  const long long *fbest;          // [slots] accuracy sum of each frontier point
  unsigned long long *fidx;        // [slots] lowest index (pass 2)
};

__global__ void k_pareto_opts(int D, int K, int idle, int M, int off, const int32_t *__restrict__ dev_type,
                              const int32_t *__restrict__ P, const int32_t *__restrict__ acc, int32_t *optP,
                              int64_t *optPA) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= D * K) return;
  const int d = i / K, o = i % K;
  if (idle && o == 0) { optP[i] = 0; optPA[i] = 0; return; }
  const int m = off + o - idle;
  const int32_t p = P[dev_type[d] * M + m];
  optP[i] = p;
  optPA[i] = (int64_t)p * acc[m];
}

// the candidates of this thread: a contiguous index range walked with an
// odometer; f(index, cap, accsum) per candidate
template <class F>
__device__ __forceinline__ void par_walk(const ParArgs &a, const int32_t *sP, const int64_t *sPA, F f) {
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  uint64_t i = a.lo + tid * a.per;
  if (i >= a.hi) return;
  const uint64_t iend = i + a.per < a.hi ? i + a.per : a.hi;
  int dig[PX_MAXD];
  int64_t cap = 0, as = 0;
  {
    uint64_t x = i;
    for (int d = a.D - 1; d >= 0; d--) {
      dig[d] = (int)(x % (uint64_t)a.K);
      x /= (uint64_t)a.K;
      cap += sP[d * a.K + dig[d]];
      as += sPA[d * a.K + dig[d]];
    }
  }
  const int dl = a.D - 1;
  const int32_t *Pl = sP + dl * a.K;   // the innermost device's options
  const int64_t *PAl = sPA + dl * a.K;
  int ol = dig[dl];                     // its digit, in a register
  for (;;) {
    f(i, cap, as);
    if (++i >= iend) break;
    if (++ol < a.K) {  // innermost digit
      cap += Pl[ol] - Pl[ol - 1];
      as += PAl[ol] - PAl[ol - 1];
      continue;
    }
    cap += Pl[0] - Pl[a.K - 1];  // carry: the innermost digit wraps to 0
    as += PAl[0] - PAl[a.K - 1];
    ol = 0;
    int d = dl - 1;
    for (; dig[d] == a.K - 1; d--) {  // outer digits at K - 1 wrap too
      cap += sP[d * a.K] - sP[d * a.K + a.K - 1];
      as += sPA[d * a.K] - sPA[d * a.K + a.K - 1];
      dig[d] = 0;
    }
    dig[d]++;
    cap += sP[d * a.K + dig[d]] - sP[d * a.K + dig[d] - 1];
    as += sPA[d * a.K + dig[d]] - sPA[d * a.K + dig[d] - 1];
  }
}

__global__ void __launch_bounds__(PAR_THREADS) k_pareto_best(const __grid_constant__ ParArgs a) {
  extern __shared__ __align__(16) unsigned char psm[];
  int64_t *sPA = (int64_t *)psm;
  int32_t *sP = (int32_t *)(sPA + a.D * a.K);
  long long *sbest = (long long *)(((uintptr_t)(sP + a.D * a.K) + 15) & ~(uintptr_t)15);
  const bool local = a.cmax + 1 <= PAR_SMEM_CAP;
  for (int k = threadIdx.x; k < a.D * a.K; k += blockDim.x) { sP[k] = a.optP[k]; sPA[k] = a.optPA[k]; }
  if (local)
    for (int64_t c = threadIdx.x; c <= a.cmax; c += blockDim.x) sbest[c] = -1;
  __syncthreads();
  long long *B = local ? sbest : a.best;
  par_walk(a, sP, sPA, [&](uint64_t, int64_t cap, int64_t as) {
    if (as > B[cap]) atomicMax(B + cap, (long long)as);
  });
  if (!local) return;
  __syncthreads();
  for (int64_t c = threadIdx.x; c <= a.cmax; c += blockDim.x)
    if (sbest[c] >= 0 && sbest[c] > a.best[c]) atomicMax(a.best + c, sbest[c]);
}

// exact accuracy order of (accsum a, capacity c); capacity 0 has accuracy 0 (P2)
__device__ __forceinline__ bool ratio_gt(long long a1, int64_t c1, long long a2, int64_t c2) {
  if (c1 == 0) return false;                 // 0 > x never
  if (c2 == 0) return a1 > 0;                // x > 0
  return (unsigned __int128)a1 * (uint64_t)c2 > (unsigned __int128)a2 * (uint64_t)c1;
}

// One block of 1024 threads.  Thread k owns capacities [k w, k w + w); the
// running maximum accuracy of everything above a capacity is the suffix
// maximum over threads (Hillis-Steele in shared memory) continued inside the
// thread's range from the top.
__global__ void __launch_bounds__(1024) k_pareto_front(int64_t cmax, const long long *__restrict__ best,
                                                       int32_t *slot, long long *fbest, int64_t *fcap,
                                                       unsigned long long *fidx, int32_t *nfront) {
  __shared__ long long sa[1024];
  __shared__ int64_t sc[1024];
  __shared__ int32_t scount[1024];
  const int k = threadIdx.x;
  const int64_t w = (cmax + 1 + 1023) / 1024;
  const int64_t c0 = (int64_t)k * w, c1 = c0 + w < cmax + 1 ? c0 + w : cmax + 1;
  long long ma = 0;  // maximum accuracy in the range as (accsum, capacity), none = (0, 0)
  int64_t mc = 0;
  for (int64_t c = c0; c < c1; c++)
    if (best[c] >= 0 && ratio_gt(best[c], c, ma, mc)) { ma = best[c]; mc = c; }
  sa[k] = ma;
  sc[k] = mc;
  __syncthreads();
  for (int o = 1; o < 1024; o <<= 1) {  // inclusive suffix maximum over threads k, k+1, ...
    long long a2 = 0;
    int64_t c2 = 0;
    if (k + o < 1024) { a2 = sa[k + o]; c2 = sc[k + o]; }
    __syncthreads();
    if (k + o < 1024 && ratio_gt(a2, c2, sa[k], sc[k])) { sa[k] = a2; sc[k] = c2; }
    __syncthreads();
  }
  long long ra = k + 1 < 1024 ? sa[k + 1] : 0;  // maximum above this thread's range
  int64_t rc = k + 1 < 1024 ? sc[k + 1] : 0;
  __syncthreads();
  int cnt = 0;
  for (int64_t c = c1 - 1; c >= c0; c--) {
    bool on = false;
    if (best[c] >= 0) {
      // on the frontier iff strictly more accurate than every higher capacity
      // (the all-zero point (0, 0) counts when nothing is above it)
      on = ratio_gt(best[c], c, ra, rc) || (rc == 0 && ra == 0 && c == 0);
      if (on) { ra = best[c]; rc = c; }
    }
    slot[c] = on ? 1 : -1;
    cnt += on;
  }
  scount[k] = cnt;
  __syncthreads();
  if (k == 0) {
    int acc = 0;
    for (int i = 0; i < 1024; i++) { const int v = scount[i]; scount[i] = acc; acc += v; }
    *nfront = acc;
  }
  __syncthreads();
  int pos = scount[k];
  for (int64_t c = c0; c < c1; c++) {
    if (slot[c] < 0) continue;
    slot[c] = pos;
    fbest[pos] = best[c];
    fcap[pos] = c;
    fidx[pos] = ~0ull;
    pos++;
  }
}

__global__ void __launch_bounds__(PAR_THREADS) k_pareto_index(const __grid_constant__ ParArgs a) {
  extern __shared__ __align__(16) unsigned char psm[];
  int64_t *sPA = (int64_t *)psm;
  int32_t *sP = (int32_t *)(sPA + a.D * a.K);
  int32_t *sslot = sP + a.D * a.K;
  const bool local = a.cmax + 1 <= PAR_SMEM_CAP;
  for (int k = threadIdx.x; k < a.D * a.K; k += blockDim.x) { sP[k] = a.optP[k]; sPA[k] = a.optPA[k]; }
  if (local)
    for (int64_t c = threadIdx.x; c <= a.cmax; c += blockDim.x) sslot[c] = a.slot[c];
  __syncthreads();
  const int32_t *S = local ? sslot : a.slot;
  par_walk(a, sP, sPA, [&](uint64_t i, int64_t cap, int64_t as) {
    const int sl = S[cap];
    if (sl >= 0 && as == a.fbest[sl]) atomicMin(a.fidx + sl, (unsigned long long)i);
  });
}

// ---------------------------------------------------------------- host ----
static uint64_t mul_div_u(uint64_t n, uint64_t r, uint64_t w) { return (uint64_t)(((unsigned __int128)n * r) / w); }

int px_pareto(proteus_ctx *ctx, int D, const int32_t *h_dev_type, const int32_t *d_dev, const int32_t *d_slo,
              int family, int allow_idle, int rank, int world, proteus_pareto_point *out, int32_t max_points,
              int32_t *n_points, uint64_t *n_configs) {
  const int T = ctx->T, M = ctx->M, V = ctx->V[family], off = ctx->off[family];
  const int K = V + (allow_idle ? 1 : 0);
  int VM = 0;
  for (int q = 0; q < ctx->Q; q++) VM = std::max(VM, ctx->V[q]);
  Tables tab;
  int rc = px_prepare_tables(ctx, D, d_dev, d_slo, VM, tab, false);
  if (rc) return rc;
  ctx->tab_valid = false;  // the cached solve tables were overwritten
  std::vector<int32_t> hP((size_t)T * M);
  PX_CUDA(ctx, cudaMemcpyAsync(hP.data(), tab.P, hP.size() * 4, cudaMemcpyDeviceToHost, ctx->stream));
  PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  // sizes: the index space and a bound on the capacity values (buffer sizing)
  unsigned __int128 n = 1;
  int64_t cmax = 0;
  for (int d = 0; d < D; d++) {
    n *= (unsigned)K;
    if (n > ((unsigned __int128)1 << 63)) return px_fail(ctx, PROTEUS_ERANGE, "configuration space exceeds 2^63");
    int32_t b = 0;
    for (int v = 0; v < V; v++) b = std::max(b, hP[(size_t)h_dev_type[d] * M + off + v]);
    cmax += b;
  }
  if (cmax >= (1ll << 26)) return px_fail(ctx, PROTEUS_ERANGE, "capacity range %lld too large", (long long)cmax);
  const uint64_t N = (uint64_t)n;
  const bool dist = px_comm_active(ctx);  // slices by communicator rank, combined by two all-reduces
  if (dist) { rank = ctx->comm_rank; world = ctx->comm_world; }
  const uint64_t lo = mul_div_u(N, rank, world), hi = mul_div_u(N, rank + 1, world);
  const size_t nc = (size_t)cmax + 1;
  char *b = (char *)px_buf(ctx, B_PARETO, (size_t)D * K * 12 + nc * (8 + 4 + 8 + 8 + 8) + 256);
  if (!b) return px_fail(ctx, PROTEUS_ENOMEM, "pareto buffers");
  ParArgs a;
  memset(&a, 0, sizeof a);
  int64_t *optPA = (int64_t *)b;
  int32_t *optP = (int32_t *)(optPA + (size_t)D * K);
  long long *best = (long long *)(((uintptr_t)(optP + (size_t)D * K) + 15) & ~(uintptr_t)15);
  long long *fbest = best + nc;
  int64_t *fcap = (int64_t *)(fbest + nc);
  unsigned long long *fidx = (unsigned long long *)(fcap + nc);
  int32_t *slot = (int32_t *)(fidx + nc);
  int32_t *d_nf = slot + nc;
  PX_CUDA(ctx, cudaMemsetAsync(best, 0xFF, nc * 8, ctx->stream));  // -1: no configuration
  PX_LAUNCH(ctx, "pareto_opts", k_pareto_opts, (D * K + 127) / 128, 128, 0, D, K, allow_idle ? 1 : 0, M, off, d_dev,
            tab.P, ctx->d_acc, optP, optPA);
  int nsm = 0;
  PX_CUDA(ctx, cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, ctx->device));
  const uint64_t cnt = hi - lo;
  const uint64_t threads = std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)nsm * 8 * PAR_THREADS, (cnt + 63) / 64));
  a.D = D; a.K = K; a.idle = allow_idle ? 1 : 0; a.cmax = cmax; a.lo = lo; a.hi = hi;
  a.per = (cnt + threads - 1) / threads;
  a.optP = optP; a.optPA = optPA; a.best = best; a.slot = slot; a.fbest = fbest; a.fidx = fidx;
  const unsigned blocks = (unsigned)((threads + PAR_THREADS - 1) / PAR_THREADS);
  const bool local = cmax + 1 <= PAR_SMEM_CAP;
  const size_t sm1 = (size_t)D * K * 12 + 16 + (local ? nc * 8 : 0);
  const size_t sm2 = (size_t)D * K * 12 + (local ? nc * 4 : 0);
  if (sm1 > 48 * 1024) PX_CUDA(ctx, cudaFuncSetAttribute(k_pareto_best, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm1));
  if (sm2 > 48 * 1024) PX_CUDA(ctx, cudaFuncSetAttribute(k_pareto_index, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm2));
  if (cnt > 0) PX_LAUNCH(ctx, "pareto_best", k_pareto_best, blocks, PAR_THREADS, sm1, a);
  // distributed: the largest accuracy sum per capacity over all slices (-1 = none)
  if (dist && (rc = px_comm_allreduce_u64(ctx, best, nc, PX_RED_MAX))) return rc;
  PX_LAUNCH(ctx, "pareto_front", k_pareto_front, 1, 1024, 0, cmax, best, slot, fbest, fcap, fidx, d_nf);
  int32_t nf = 0;
  if (dist) {  // every rank holds the same frontier; the lowest index per point over all slices
    PX_CUDA(ctx, cudaMemcpyAsync(&nf, d_nf, 4, cudaMemcpyDeviceToHost, ctx->stream));
    PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  }
  if (cnt > 0) PX_LAUNCH(ctx, "pareto_index", k_pareto_index, blocks, PAR_THREADS, sm2, a);
  if (dist && nf > 0 && (rc = px_comm_allreduce_u64(ctx, fidx, (size_t)nf, PX_RED_MIN))) return rc;
  PX_CUDA(ctx, cudaMemcpyAsync(&nf, d_nf, 4, cudaMemcpyDeviceToHost, ctx->stream));
  PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  const int k = std::min(nf, max_points);
  std::vector<long long> hb(k), hc(k);
  std::vector<unsigned long long> hi_(k);
  if (k > 0) {
    PX_CUDA(ctx, cudaMemcpyAsync(hb.data(), fbest, (size_t)k * 8, cudaMemcpyDeviceToHost, ctx->stream));
    PX_CUDA(ctx, cudaMemcpyAsync(hc.data(), fcap, (size_t)k * 8, cudaMemcpyDeviceToHost, ctx->stream));
    PX_CUDA(ctx, cudaMemcpyAsync(hi_.data(), fidx, (size_t)k * 8, cudaMemcpyDeviceToHost, ctx->stream));
    PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  }
  for (int i = 0; i < k; i++) {
    out[i].capacity = hc[i];
    out[i].accsum = hb[i];
    out[i].index = hi_[i];
  }
  *n_points = nf;
  *n_configs = dist ? N : cnt;
  return 0;
}
