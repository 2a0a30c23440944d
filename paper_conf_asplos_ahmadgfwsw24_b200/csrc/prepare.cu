// prepare.cu -- a1 (capacity estimate) and the per-call slot tables
// every scoring kernel reads.
#include "internal.cuh"

// One block.  Steps:
//  1. per (type t, variant m): depth = leading run of fitting batch sizes
//     (reading C7); b* = largest b <= depth with 2 lat(b) <= SLO (C5, C6);
//     P = floor(b* 10^6 / lat(b*)) (C4), 0 if no such b.
//  2. per family q: order its variants by (accuracy desc, code asc) -> slot
//     q*VM + j (reading C10 fill order); pad slots get code 0 / accuracy 0.
//  3. per (device d, code o): Pdev[d][o] = P[type_d][o-1] (0 for idle).
// With pclamp > 0 (the solve path) P is stored as min(P, pclamp): demand per
// vector is < 2^22 = pclamp, so a water-fill take min(rem, cap) and every z
// are unchanged, while slot sums of up to 64 devices stay far inside int32.
// The Fig. 1b frontier (pareto.cu) sums the exact capacities: pclamp = 0.
__global__ void k_prepare(int T, int Q, int M, int bmax, int D, int VM, const int32_t *__restrict__ lat,
                          const int32_t *__restrict__ acc, const int32_t *__restrict__ fam,
                          const int32_t *__restrict__ off, const int32_t *__restrict__ V,
                          const int32_t *__restrict__ dev_type, const int32_t *__restrict__ slo, int32_t pclamp,
                          Tables tab) {
  const int K = M + 1;
  for (int i = threadIdx.x; i < T * M; i += blockDim.x) {
    int t = i / M, m = i % M;
    const int32_t *row = lat + ((size_t)t * M + m) * bmax;
    int dep = 0;
    while (dep < bmax && row[dep] > 0) dep++;
    int64_t L = slo[fam[m]];
    int bs = 0;
    for (int b = dep; b >= 1; b--)
      if (2ll * row[b - 1] <= L) { bs = b; break; }
    tab.depth[i] = dep;
    int32_t P = bs ? (int32_t)(((int64_t)bs * 1000000ll) / row[bs - 1]) : 0;
    tab.P[i] = (pclamp > 0 && P > pclamp) ? pclamp : P;
  }
  for (int q = threadIdx.x; q < Q; q += blockDim.x) {
    for (int j = 0; j < VM; j++) { tab.slot_code[q * VM + j] = 0; tab.slot_acc[q * VM + j] = 0; }
    for (int v = 0; v < V[q]; v++) {
      int m = off[q] + v, a = acc[m], j = 0;
      for (int w = 0; w < V[q]; w++) {
        int a2 = acc[off[q] + w];
        if (a2 > a || (a2 == a && w < v)) j++;
      }
      tab.slot_of[m] = q * VM + j;
      tab.slot_code[q * VM + j] = m + 1;
      tab.slot_acc[q * VM + j] = a;
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i < D * K; i += blockDim.x) {
    int d = i / K, o = i % K;
    tab.Pdev[i] = o ? tab.P[dev_type[d] * M + (o - 1)] : 0;
  }
  for (int o = threadIdx.x; o < K; o += blockDim.x) tab.code_slot[o] = o ? tab.slot_of[o - 1] : -1;
}

int px_prepare_tables(proteus_ctx *ctx, int D, const int32_t *d_dev_type, const int32_t *d_slo, int VM,
                      Tables &tab, bool clamp) {
  const int T = ctx->T, Q = ctx->Q, M = ctx->M, K = M + 1;
  size_t n = (size_t)2 * T * M + M + 2 * Q * VM + K + (size_t)D * K;
  int32_t *b = (int32_t *)px_buf(ctx, B_TABLES, n * 4);
  if (!b) return px_fail(ctx, PROTEUS_ENOMEM, "tables");
  tab.P = b; b += T * M;
  tab.depth = b; b += T * M;
  tab.slot_of = b; b += M;
  tab.slot_code = b; b += Q * VM;
  tab.slot_acc = b; b += Q * VM;
  tab.code_slot = b; b += K;
  tab.Pdev = b;
  PX_LAUNCH(ctx, "prepare", k_prepare, 1, 256, 0, T, Q, M, ctx->bmax, D, VM, ctx->d_lat, ctx->d_acc, ctx->d_fam,
            ctx->d_off, ctx->d_V, d_dev_type, d_slo, clamp ? PX_PCLAMP : 0, tab);
  return 0;
}

// Size of the candidate space (host; pure counting, no method arithmetic):
// mode 0: K^D; mode 1: prod_t C(K + N_t - 1, N_t).
uint64_t px_count_candidates(int mode, int D, const int32_t *dev_type, int T, int K, bool *overflow) {
  unsigned __int128 n = 1;
  *overflow = false;
  if (mode == 0) {
    for (int d = 0; d < D; d++) {
      n *= (unsigned)K;
      if (n > (unsigned __int128)UINT64_MAX) { *overflow = true; return 0; }
    }
    return (uint64_t)n;
  }
  for (int t = 0; t < T; t++) {
    int Nt = 0;
    for (int d = 0; d < D; d++) Nt += dev_type[d] == t;
    unsigned __int128 c = 1;
    for (int i = 1; i <= Nt; i++) {
      c = c * (unsigned)(K - 1 + i) / (unsigned)i;
      if (c > (unsigned __int128)UINT64_MAX) { *overflow = true; return 0; }
    }
    n *= c;
    if (n > (unsigned __int128)UINT64_MAX) { *overflow = true; return 0; }
  }
  return (uint64_t)n;
}
