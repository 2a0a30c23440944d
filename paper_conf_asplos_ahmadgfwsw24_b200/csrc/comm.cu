// comm.cu -- the multi-GPU exchange of the path behind
// the C ABI: an NCCL communicator owned by the context, and the device kernels
// that combine per-rank results after a collective.
//
// NCCL is resolved at run time (dlopen of libnccl.so.2: the copy already loaded
// in the process -- torch's -- first, else the system one), so the library
// loads and every single-GPU call works without NCCL present; only
// proteus_comm_* needs it (PROTEUS_ENCCL otherwise).  All collectives run on
// the context's stream; nothing goes through the host between a kernel that
// produces a rank's result and the collective that exchanges it.
//
//   flat / multiset search: every rank scans slice `rank` of the index space,
//     materialises its winner per demand vector (SolRec), one ncclAllGather of
//     the SolRecs, then k_pick_solrec takes per vector the (score desc, index
//     asc) maximum -- the order of the in-GPU argmax (reading C9), so the
//     answer is the single-GPU one for every world size;
//   factored batched re-solve: vectors split by rank, one ncclAllGather of the
//     SolRecs, k_gather_vectors puts them back in vector order;
//   Fig. 1b frontier: one ncclAllReduce(MAX) of the per-capacity best
//     accuracy sums, every rank extracts the same frontier, one
//     ncclAllReduce(MIN) of the lowest index per frontier point (pareto.cu);
//   replay: scenarios assigned to ranks (px_scenario_owner), one
//     ncclAllReduce(SUM) of the zero-padded per-scenario aggregates.
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cstring>

#include "internal.cuh"

// ------------------------------------------------------------ loader ----
namespace {
struct NcclApi {
  bool tried = false, ok = false;
  std::string why;
  ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  const char *(*GetErrorString)(ncclResult_t) = nullptr;
};
NcclApi g_nccl;

bool nccl_load(std::string *why) {
  if (g_nccl.tried) {
    if (!g_nccl.ok) *why = g_nccl.why;
    return g_nccl.ok;
  }
  g_nccl.tried = true;
  const char *env = getenv("PROTEUS_NCCL_LIB");
  void *h = nullptr;
  if (env && *env) h = dlopen(env, RTLD_NOW | RTLD_GLOBAL);
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);  // the process's copy (torch's)
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
  if (!h) {
    g_nccl.why = std::string("libnccl.so.2 not found: ") + dlerror();
    *why = g_nccl.why;
    return false;
  }
#define PX_SYM(field, name)                                                  \
  *(void **)&g_nccl.field = dlsym(h, name);                                  \
  if (!g_nccl.field) {                                                       \
    g_nccl.why = std::string("libnccl lacks ") + name;                       \
    *why = g_nccl.why;                                                       \
    return false;                                                            \
  }
  PX_SYM(GetUniqueId, "ncclGetUniqueId");
  PX_SYM(CommInitRank, "ncclCommInitRank");
  PX_SYM(CommDestroy, "ncclCommDestroy");
  PX_SYM(AllGather, "ncclAllGather");
  PX_SYM(AllReduce, "ncclAllReduce");
  PX_SYM(GetErrorString, "ncclGetErrorString");
#undef PX_SYM
  g_nccl.ok = true;
  return true;
}
}  // namespace

#define PX_NCCL(ctx, call)                                                                                  \
  do {                                                                                                      \
    ncclResult_t r_ = (call);                                                                               \
    if (r_ != ncclSuccess) return px_fail(ctx, PROTEUS_ENCCL, "%s: %s", #call, g_nccl.GetErrorString(r_)); \
  } while (0)

// distributed while a communicator is attached and enabled -- world 1 too (the
// collectives then run over one rank: the same code path, testable on 1 GPU)
bool px_comm_active(const proteus_ctx *ctx) { return ctx->comm != nullptr && ctx->comm_on; }

int px_comm_allgather(proteus_ctx *ctx, const void *send, void *recv, size_t bytes) {
  px_launch_begin(ctx, "nccl_allgather");
  PX_NCCL(ctx, g_nccl.AllGather(send, recv, bytes, ncclUint8, (ncclComm_t)ctx->comm, ctx->stream));
  return px_launch_end(ctx);
}

int px_comm_allreduce_u64(proteus_ctx *ctx, void *buf, size_t count, int op) {
  px_launch_begin(ctx, "nccl_allreduce");
  const ncclRedOp_t o = op == PX_RED_SUM ? ncclSum : op == PX_RED_MAX ? ncclMax : ncclMin;
  PX_NCCL(ctx, g_nccl.AllReduce(buf, buf, count, op == PX_RED_MAX ? ncclInt64 : ncclUint64, o,
                                (ncclComm_t)ctx->comm, ctx->stream));
  return px_launch_end(ctx);
}

// ----------------------------------------------------------- kernels ----
// per vector: the (score desc, index asc) maximum over the world's records
// (reading C9); n_candidates = the sum of the slices'.  Thread 0 of a warp
// picks, the warp copies the winner's record.
__global__ void k_pick_solrec(const SolRec *__restrict__ gathered, int world, int n, SolRec *out) {
  const int v = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  if (v >= n) return;
  int best = 0;
  uint64_t bs = gathered[v].score, bi = gathered[v].index, nc = 0;
  int32_t st = 0;
  for (int r = 0; r < world; r++) {
    const SolRec &x = gathered[(size_t)r * n + v];
    nc += x.n_candidates;
    st |= x.status;
    if (px_better(x.score, x.index, bs, bi)) { bs = x.score; bi = x.index; best = r; }
  }
  const uint32_t *src = (const uint32_t *)&gathered[(size_t)best * n + v];
  uint32_t *dst = (uint32_t *)&out[v];
  for (int k = lane; k < (int)(sizeof(SolRec) / 4); k += 32) dst[k] = src[k];
  __syncwarp();
  if (lane == 0) {
    out[v].n_candidates = nc;
    out[v].status = st;
  }
}

// vectors split by rank (slice r = [n r / world, n (r+1) / world)), gathered
// with `stride` records per rank -> vector order
__global__ void k_gather_vectors(const SolRec *__restrict__ gathered, int world, int n, int stride, SolRec *out) {
  const int v = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  if (v >= n) return;
  int r = (int)(((int64_t)v * world) / n);  // candidate owner, then fix up
  while (r > 0 && ((int64_t)n * r) / world > v) r--;
  while (r + 1 < world && ((int64_t)n * (r + 1)) / world <= v) r++;
  const int lo = (int)(((int64_t)n * r) / world);
  const uint32_t *src = (const uint32_t *)&gathered[(size_t)r * stride + (v - lo)];
  uint32_t *dst = (uint32_t *)&out[v];
  for (int k = lane; k < (int)(sizeof(SolRec) / 4); k += 32) dst[k] = src[k];
}

int px_pick_solrec(proteus_ctx *ctx, const SolRec *d_gathered, int world, int n, SolRec *d_out) {
  PX_LAUNCH(ctx, "pick_solutions", k_pick_solrec, (n + 7) / 8, 256, 0, d_gathered, world, n, d_out);
  return 0;
}

int px_gather_vectors(proteus_ctx *ctx, const SolRec *d_gathered, int world, int n, int stride, SolRec *d_out) {
  PX_LAUNCH(ctx, "gather_vectors", k_gather_vectors, (n + 7) / 8, 256, 0, d_gathered, world, n, stride, d_out);
  return 0;
}

// Fig. 1b shard merge (reading P3): the union of the parts' frontier points;
// point i survives iff no point dominates it -- capacity >= and accuracy >=
// with one strict, accuracies accsum/cap compared by exact 128-bit
// cross-multiplication -- and, among equal points, it has the lowest index
// (then the lowest position).  Its output slot = the number of surviving
// points of lower capacity (survivors have distinct capacities).  O(P^2) in
// one block: P is a few thousand points at most.
__device__ __forceinline__ int acc_cmp(int64_t a1, int64_t c1, int64_t a2, int64_t c2) {
  // sign of a1/c1 - a2/c2 with capacity 0 meaning accuracy 0 (reading P2)
  if (c1 == 0 || c2 == 0) {
    const bool z1 = c1 == 0 || a1 == 0, z2 = c2 == 0 || a2 == 0;
    if (z1 && z2) return 0;
    return z1 ? -1 : 1;
  }
  const __int128 l = (__int128)a1 * c2, r = (__int128)a2 * c1;
  return l < r ? -1 : (l > r ? 1 : 0);
}

__global__ void k_pareto_merge(const proteus_pareto_point *__restrict__ pts, int n, int32_t *keep,
                               proteus_pareto_point *out, int32_t *n_out) {
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    const proteus_pareto_point p = pts[i];
    bool k = true;
    for (int j = 0; j < n && k; j++) {
      if (j == i) continue;
      const proteus_pareto_point q = pts[j];
      const int ac = acc_cmp(q.accsum, q.capacity, p.accsum, p.capacity);
      if (q.capacity >= p.capacity && ac >= 0) {
        if (q.capacity > p.capacity || ac > 0) k = false;                 // strictly dominated
        else if (q.index < p.index || (q.index == p.index && j < i)) k = false;  // equal point, lower index wins
      }
    }
    keep[i] = k;
  }
  __syncthreads();
  int cnt = 0;
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    if (!keep[i]) continue;
    int pos = 0;
    for (int j = 0; j < n; j++) pos += keep[j] && pts[j].capacity < pts[i].capacity;
    out[pos] = pts[i];
    cnt++;
  }
  atomicAdd(n_out, cnt);
}

int px_pareto_merge(proteus_ctx *ctx, const proteus_pareto_point *d_pts, int n, proteus_pareto_point *d_out,
                    int32_t *d_n) {
  int32_t *keep = (int32_t *)px_buf(ctx, B_C_KEEP, (size_t)n * 4 + 16);
  if (!keep) return px_fail(ctx, PROTEUS_ENOMEM, "merge buffer");
  PX_CUDA(ctx, cudaMemsetAsync(d_n, 0, 4, ctx->stream));
  PX_LAUNCH(ctx, "pareto_merge", k_pareto_merge, 1, 1024, 0, d_pts, n, keep, d_out, d_n);
  return 0;
}

// ----------------------------------------------- scenario assignment ----
// Relative cost of one replay scenario's lanes (host; a deterministic model
// from the measured 1-GPU time of every c5 scenario replayed alone,
// profiles/r02g_scenario_costs.json): §5 lanes with Bmax = 1
// are one exact prefix-max scan (0.7 ms); every other §5 scenario costs about
// the same (6-9.5 ms, the chain path's longest lane); Clipper AIMD 29-81 ms;
// Nexus 58-250 ms at batch cap 1 (the overload stretches) and 230-475 ms
// otherwise (sequential chains of the busy lanes).
static double scenario_cost(const proteus_scenario &s) {
  if (s.policy == 1) return s.batch_cap == 1 ? 12.0 : 62.0;  // Nexus early drop
  if (s.policy == 2) return 7.0;                              // Clipper AIMD
  return s.batch_cap == 1 ? 0.11 : 1.0;
}

// Longest-processing-time greedy: scenarios by decreasing cost (ties by
// index), each to the rank with the least load so far (ties: lowest rank).
void px_scenario_owner(const proteus_scenario *sc, int S, int world, int32_t *owner) {
  std::vector<int> ord(S);
  for (int s = 0; s < S; s++) ord[s] = s;
  std::stable_sort(ord.begin(), ord.end(),
                   [&](int a, int b) { return scenario_cost(sc[a]) > scenario_cost(sc[b]); });
  std::vector<double> load(world > 0 ? world : 1, 0.0);
  for (int s : ord) {
    int r = 0;
    for (int k = 1; k < (int)load.size(); k++)
      if (load[k] < load[r]) r = k;
    owner[s] = r;
    load[r] += scenario_cost(sc[s]);
  }
}

// ----------------------------------------------------------------- ABI ----
extern "C" {

int proteus_comm_unique_id(void *id_out) {
  if (!id_out) return PROTEUS_EINVAL;
  std::string why;
  if (!nccl_load(&why)) return PROTEUS_ENCCL;
  ncclUniqueId id;
  if (g_nccl.GetUniqueId(&id) != ncclSuccess) return PROTEUS_ENCCL;
  memcpy(id_out, &id, sizeof id);
  return PROTEUS_OK;
}

int proteus_comm_init(proteus_ctx *ctx, const void *nccl_unique_id, int world, int rank) {
  if (!ctx) return PROTEUS_EINVAL;
  ctx->err.clear();
  if (!nccl_unique_id || world < 1 || rank < 0 || rank >= world)
    return px_fail(ctx, PROTEUS_EINVAL, "comm_init: world %d rank %d", world, rank);
  std::string why;
  if (!nccl_load(&why)) return px_fail(ctx, PROTEUS_ENCCL, "%s", why.c_str());
  PX_CUDA(ctx, cudaSetDevice(ctx->device));
  if (ctx->comm) {
    g_nccl.CommDestroy((ncclComm_t)ctx->comm);
    ctx->comm = nullptr;
  }
  ncclUniqueId id;
  memcpy(&id, nccl_unique_id, sizeof id);
  ncclComm_t c = nullptr;
  PX_NCCL(ctx, g_nccl.CommInitRank(&c, world, id, rank));
  ctx->comm = c;
  ctx->comm_world = world;
  ctx->comm_rank = rank;
  ctx->comm_on = true;
  return PROTEUS_OK;
}

int proteus_comm_enable(proteus_ctx *ctx, int enable) {
  if (!ctx) return PROTEUS_EINVAL;
  if (enable && !ctx->comm) return px_fail(ctx, PROTEUS_EINVAL, "no communicator (proteus_comm_init)");
  ctx->comm_on = enable != 0;
  return PROTEUS_OK;
}

int proteus_comm_info(const proteus_ctx *ctx, int32_t *world, int32_t *rank) {
  if (!ctx) return PROTEUS_EINVAL;
  if (world) *world = ctx->comm ? ctx->comm_world : 1;
  if (rank) *rank = ctx->comm ? ctx->comm_rank : 0;
  return ctx->comm && ctx->comm_on ? 1 : 0;
}

int proteus_scenario_owner(const proteus_scenario *sc, int32_t S, int32_t world, int32_t *owner) {
  if (!sc || !owner || S < 0 || world < 1) return PROTEUS_EINVAL;
  px_scenario_owner(sc, S, world, owner);
  return PROTEUS_OK;
}

}  // extern "C"

void px_comm_destroy(proteus_ctx *ctx) {
  if (ctx->comm && g_nccl.ok) g_nccl.CommDestroy((ncclComm_t)ctx->comm);
  ctx->comm = nullptr;
}
