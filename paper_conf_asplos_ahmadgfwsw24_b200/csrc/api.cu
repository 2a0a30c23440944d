// api.cu -- the C ABI (include/proteus.h) and the host runtime around the
// kernels: context, grow-only device scratch, host/device pointer staging,
// validation (overflow guards) and kernel timing.  All arithmetic of the method
// runs in the kernels of prepare.cu, solve_enum.cu, solve_factored.cu and
// replay.cu.
#include <chrono>
#include <cstdarg>
#include <cstddef>
#include <cstdlib>
#include <cstring>

#include "internal.cuh"

// ---------------------------------------------------------------- utils ----
int px_fail(proteus_ctx *ctx, int code, const char *fmt, ...) {
  if (ctx) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    ctx->err = buf;
  }
  return code;
}

void *px_buf(proteus_ctx *ctx, int id, size_t bytes) {
  DevBuf &b = ctx->bufs[id];
  if (bytes == 0) bytes = 16;
  if (b.n < bytes) {
    if (b.p) {
      cudaStreamSynchronize(ctx->stream);
      cudaFree(b.p);
      b.p = nullptr;
      b.n = 0;
    }
    size_t n = bytes + bytes / 8;
    if (cudaMalloc(&b.p, n) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
    b.n = n;
  }
  return b.p;
}

bool px_is_device_ptr(const void *p) {
  if (!p) return false;
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

void px_launch_begin(proteus_ctx *ctx, const char *name) {
  ctx->launches++;
  if (!ctx->timing) return;
  cudaEvent_t a, b;
  if (ctx->ev_pool.size() >= 2) {
    a = ctx->ev_pool.back(); ctx->ev_pool.pop_back();
    b = ctx->ev_pool.back(); ctx->ev_pool.pop_back();
  } else {
    cudaEventCreate(&a);
    cudaEventCreate(&b);
  }
  cudaEventRecord(a, ctx->stream);
  ctx->tnames.push_back(name);
  ctx->tev.push_back(a);
  ctx->tev.push_back(b);
}

int px_launch_end(proteus_ctx *ctx) {
  cudaError_t e = cudaGetLastError();
  if (ctx->timing) cudaEventRecord(ctx->tev.back(), ctx->stream);
  if (e != cudaSuccess) return px_fail(ctx, PROTEUS_ECUDA, "kernel launch: %s", cudaGetErrorString(e));
  return 0;
}

static void timing_reset(proteus_ctx *ctx) {
  for (auto e : ctx->tev) ctx->ev_pool.push_back(e);
  ctx->tev.clear();
  ctx->tnames.clear();
  ctx->tms.clear();
}

static int timing_collect(proteus_ctx *ctx) {
  if (!ctx->timing) return 0;
  PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  ctx->tms.resize(ctx->tnames.size());
  for (size_t i = 0; i < ctx->tnames.size(); i++) {
    float ms = 0;
    cudaEventElapsedTime(&ms, ctx->tev[2 * i], ctx->tev[2 * i + 1]);
    ctx->tms[i] = ms;
  }
  return 0;
}

// copy n elements of T from a host-or-device pointer into host memory
template <class T>
static int to_host(proteus_ctx *ctx, const T *p, size_t n, std::vector<T> &out) {
  out.resize(n);
  if (n == 0) return 0;
  if (px_is_device_ptr(p)) {
    PX_CUDA(ctx, cudaMemcpyAsync(out.data(), p, n * sizeof(T), cudaMemcpyDeviceToHost, ctx->stream));
    PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  } else {
    memcpy(out.data(), p, n * sizeof(T));
  }
  return 0;
}

// device pointer for an input: the caller's if it is on the device, else a staged copy
template <class T>
static const T *to_device(proteus_ctx *ctx, const T *p, size_t n, int buf, int *rc) {
  *rc = 0;
  if (px_is_device_ptr(p)) return p;
  T *d = (T *)px_buf(ctx, buf, n * sizeof(T));
  if (!d) { *rc = px_fail(ctx, PROTEUS_ENOMEM, "device scratch (%zu bytes)", n * sizeof(T)); return nullptr; }
  if (n) {
    cudaError_t e = cudaMemcpyAsync(d, p, n * sizeof(T), cudaMemcpyHostToDevice, ctx->stream);
    if (e != cudaSuccess) { *rc = px_fail(ctx, PROTEUS_ECUDA, "H2D: %s", cudaGetErrorString(e)); return nullptr; }
  }
  return d;
}


// --------------------------------------------------------------- ABI -----
extern "C" {

int proteus_abi_version(void) { return PROTEUS_ABI_VERSION; }

int proteus_create(proteus_ctx **out, int cuda_device, void *cuda_stream) {
  if (!out) return PROTEUS_EINVAL;
  *out = nullptr;
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess || cuda_device < 0 || cuda_device >= n) {
    cudaGetLastError();
    return PROTEUS_ECUDA;
  }
  if (cudaSetDevice(cuda_device) != cudaSuccess) return PROTEUS_ECUDA;
  proteus_ctx *c = new proteus_ctx();
  c->device = cuda_device;
  c->stream = (cudaStream_t)cuda_stream;
  *out = c;
  return PROTEUS_OK;
}

void proteus_destroy(proteus_ctx *ctx) {
  if (!ctx) return;
  cudaSetDevice(ctx->device);
  cudaStreamSynchronize(ctx->stream);
  for (auto &b : ctx->bufs) if (b.p) cudaFree(b.p);
  for (int32_t *p : {ctx->d_lat, ctx->d_acc, ctx->d_fam, ctx->d_off, ctx->d_V}) if (p) cudaFree(p);
  for (auto e : ctx->tev) cudaEventDestroy(e);
  for (auto e : ctx->ev_pool) cudaEventDestroy(e);
  px_comm_destroy(ctx);
  if (ctx->aux) cudaStreamDestroy(ctx->aux);
  if (ctx->aux_hi) cudaStreamDestroy(ctx->aux_hi);
  if (ctx->ev_fork) cudaEventDestroy(ctx->ev_fork);
  if (ctx->ev_join) cudaEventDestroy(ctx->ev_join);
  if (ctx->ev_join2) cudaEventDestroy(ctx->ev_join2);
  delete ctx;
}

int proteus_set_stream(proteus_ctx *ctx, void *cuda_stream) {
  if (!ctx) return PROTEUS_EINVAL;
  ctx->stream = (cudaStream_t)cuda_stream;
  return PROTEUS_OK;
}

const char *proteus_last_error(const proteus_ctx *ctx) { return ctx ? ctx->err.c_str() : "null context"; }

int proteus_set_timing(proteus_ctx *ctx, int enable) {
  if (!ctx) return PROTEUS_EINVAL;
  ctx->timing = enable != 0;
  return PROTEUS_OK;
}

int proteus_kernel_times(const proteus_ctx *ctx, const char **names, float *ms, int cap) {
  if (!ctx) return PROTEUS_EINVAL;
  int n = (int)ctx->tms.size();
  for (int i = 0; i < n && i < cap; i++) {
    if (names) names[i] = ctx->tnames[i];
    if (ms) ms[i] = ctx->tms[i];
  }
  return n;
}

uint64_t proteus_launch_count(const proteus_ctx *ctx) { return ctx ? ctx->launches : 0; }

int proteus_load_profiles(proteus_ctx *ctx, const proteus_profiles *p) {
  if (!ctx || !p || !p->V || !p->acc_micro || !p->lat_us) return px_fail(ctx, PROTEUS_EINVAL, "null argument");
  ctx->err.clear();
  if (p->T < 1 || p->T > PX_MAXT || p->Q < 1 || p->Q > PX_MAXQ || p->bmax < 1 || p->bmax > PX_MAXB)
    return px_fail(ctx, PROTEUS_EINVAL, "T=%d Q=%d bmax=%d out of range", p->T, p->Q, p->bmax);
  PX_CUDA(ctx, cudaSetDevice(ctx->device));
  std::vector<int32_t> V, acc, lat;
  int rc;
  if ((rc = to_host(ctx, p->V, p->Q, V))) return rc;
  int M = 0;
  for (int q = 0; q < p->Q; q++) {
    if (V[q] < 1 || V[q] > PX_MAXV) return px_fail(ctx, PROTEUS_EINVAL, "V[%d]=%d out of range", q, V[q]);
    M += V[q];
  }
  if (M > PX_MAXM) return px_fail(ctx, PROTEUS_EINVAL, "sum V = %d > %d", M, PX_MAXM);
  if ((rc = to_host(ctx, p->acc_micro, M, acc))) return rc;
  for (int m = 0; m < M; m++)
    if (acc[m] < 1 || acc[m] > 1000000) return px_fail(ctx, PROTEUS_ERANGE, "acc_micro[%d]=%d not in [1, 1e6]", m, acc[m]);
  if ((rc = to_host(ctx, p->lat_us, (size_t)p->T * M * p->bmax, lat))) return rc;
  for (int32_t x : lat)
    if (x < 0) return px_fail(ctx, PROTEUS_EINVAL, "negative latency");
  std::vector<int32_t> fam(M), off(p->Q);
  for (int q = 0, m = 0; q < p->Q; q++) {
    off[q] = m;
    for (int v = 0; v < V[q]; v++) fam[m++] = q;
  }
  for (int32_t *ptr : {ctx->d_lat, ctx->d_acc, ctx->d_fam, ctx->d_off, ctx->d_V}) if (ptr) cudaFree(ptr);
  ctx->d_lat = ctx->d_acc = ctx->d_fam = ctx->d_off = ctx->d_V = nullptr;
  PX_CUDA(ctx, cudaMalloc(&ctx->d_lat, lat.size() * 4));
  PX_CUDA(ctx, cudaMalloc(&ctx->d_acc, M * 4));
  PX_CUDA(ctx, cudaMalloc(&ctx->d_fam, M * 4));
  PX_CUDA(ctx, cudaMalloc(&ctx->d_off, p->Q * 4));
  PX_CUDA(ctx, cudaMalloc(&ctx->d_V, p->Q * 4));
  PX_CUDA(ctx, cudaMemcpyAsync(ctx->d_lat, lat.data(), lat.size() * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(ctx->d_acc, acc.data(), M * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(ctx->d_fam, fam.data(), M * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(ctx->d_off, off.data(), p->Q * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(ctx->d_V, V.data(), p->Q * 4, cudaMemcpyHostToDevice, ctx->stream));
  PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  ctx->T = p->T; ctx->Q = p->Q; ctx->M = M; ctx->bmax = p->bmax;
  ctx->V = V; ctx->acc = acc; ctx->lat = lat; ctx->fam = fam; ctx->off = off;
  ctx->have_prof = true;
  ctx->prof_gen++;
  ctx->tab_valid = false;
  return PROTEUS_OK;
}

}  // extern "C"

// -------------------------------------------------------------- solve -----
struct SolveInputs {
  std::vector<int32_t> dev_type, slo, demand;
  const int32_t *d_dev = nullptr, *d_slo = nullptr, *d_dem = nullptr;
};

// Host copies of the small solve inputs (validation, launch parameters) and
// device pointers for the kernels: a device input is used in place and read
// back with a single synchronisation; a host input is staged to the device.
static int validate_solve(proteus_ctx *ctx, const proteus_solve_args *a, SolveInputs &in) {
  if (!ctx) return PROTEUS_EINVAL;
  ctx->err.clear();
  if (!a) return px_fail(ctx, PROTEUS_EINVAL, "null args");
  if (!ctx->have_prof) return px_fail(ctx, PROTEUS_EINVAL, "no profiles loaded");
  if (a->D < 1 || a->D > PX_MAXD) return px_fail(ctx, PROTEUS_EINVAL, "D=%d out of range [1, %d]", a->D, PX_MAXD);
  if (a->mode < 0 || a->mode > 2) return px_fail(ctx, PROTEUS_EINVAL, "mode %d", a->mode);
  if (a->n_vec < 1) return px_fail(ctx, PROTEUS_EINVAL, "n_vec=%d", a->n_vec);
  if (!a->device_type || !a->slo_us || !a->demand_qps) return px_fail(ctx, PROTEUS_EINVAL, "null array");
  if (a->shard_world < 0 || a->shard_rank < 0 || (a->shard_world > 0 && a->shard_rank >= a->shard_world))
    return px_fail(ctx, PROTEUS_EINVAL, "shard %d/%d", a->shard_rank, a->shard_world);
  PX_CUDA(ctx, cudaSetDevice(ctx->device));
  const int32_t *src[3] = {a->device_type, a->slo_us, a->demand_qps};
  std::vector<int32_t> *dst[3] = {&in.dev_type, &in.slo, &in.demand};
  const size_t cnt[3] = {(size_t)a->D, (size_t)ctx->Q, (size_t)a->n_vec * ctx->Q};
  const int32_t **dptr[3] = {&in.d_dev, &in.d_slo, &in.d_dem};
  bool dev[3], any_dev = false;
  for (int k = 0; k < 3; k++) {
    dst[k]->resize(cnt[k]);
    dev[k] = px_is_device_ptr(src[k]);
    if (dev[k]) {
      PX_CUDA(ctx, cudaMemcpyAsync(dst[k]->data(), src[k], cnt[k] * 4, cudaMemcpyDeviceToHost, ctx->stream));
      *dptr[k] = src[k];
      any_dev = true;
    } else {
      memcpy(dst[k]->data(), src[k], cnt[k] * 4);
    }
  }
  if (any_dev) PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  for (int d = 0; d < a->D; d++)
    if (in.dev_type[d] < 0 || in.dev_type[d] >= ctx->T)
      return px_fail(ctx, PROTEUS_EINVAL, "device_type[%d]=%d", d, in.dev_type[d]);
  for (int q = 0; q < ctx->Q; q++)
    if (in.slo[q] < 0) return px_fail(ctx, PROTEUS_EINVAL, "slo_us[%d] < 0", q);
  for (int v = 0; v < a->n_vec; v++) {
    int64_t sum = 0;
    for (int q = 0; q < ctx->Q; q++) {
      int32_t s = in.demand[(size_t)v * ctx->Q + q];
      if (s < 0) return px_fail(ctx, PROTEUS_EINVAL, "negative demand");
      sum += s;
    }
    if (sum >= (1 << 22)) return px_fail(ctx, PROTEUS_ERANGE, "sum of demand %lld >= 2^22", (long long)sum);
  }
  const int bufid[3] = {B_IN0, B_IN1, B_IN2};
  for (int k = 0; k < 3; k++) {
    if (dev[k]) continue;
    int32_t *d = (int32_t *)px_buf(ctx, bufid[k], cnt[k] * 4);
    if (!d) return px_fail(ctx, PROTEUS_ENOMEM, "input staging");
    PX_CUDA(ctx, cudaMemcpyAsync(d, dst[k]->data(), cnt[k] * 4, cudaMemcpyHostToDevice, ctx->stream));
    *dptr[k] = d;
  }
  return 0;
}

// Batched outputs (proteus_solve_batch): the solution records unpacked into
// the caller's device arrays (layout only), and the OR of their status words.
struct BatchPtrs {
  uint64_t *score, *index;
  int64_t *served, *unmet, *accsum;
  int32_t *eff, *option, *z;
};

__global__ void k_sol_unpack(const SolRec *__restrict__ sol, int n, int D, BatchPtrs o, int32_t *status) {
  const int i = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  if (i >= n) return;
  const SolRec &r = sol[i];
  if (lane == 0) {
    if (o.score) o.score[i] = r.score;
    if (o.index) o.index[i] = r.index;
    if (o.served) o.served[i] = r.served;
    if (o.unmet) o.unmet[i] = r.unmet;
    if (o.accsum) o.accsum[i] = r.accsum;
    if (o.eff) o.eff[i] = r.eff;
    if (r.status) atomicOr(status, 1 << (r.status & 15));
  }
  for (int d = lane; d < D; d += 32) {
    if (o.option) o.option[(size_t)i * D + d] = r.option[d];
    if (o.z) o.z[(size_t)i * D + d] = r.z[d];
  }
}

static int batch_out(proteus_ctx *ctx, const proteus_solve_args *a, const SolRec *d_sol, int n, proteus_batch *o) {
  void *ptrs[8] = {o->score, o->index, o->served, o->unmet, o->accsum, o->eff_acc_micro, o->option, o->z_qps};
  bool dev[8], any_host = false;
  for (int k = 0; k < 8; k++) {
    dev[k] = px_is_device_ptr(ptrs[k]);
    any_host |= ptrs[k] && !dev[k];
  }
  int32_t *d_status = (int32_t *)px_buf(ctx, B_IN3, 16);
  if (!d_status) return px_fail(ctx, PROTEUS_ENOMEM, "status word");
  PX_CUDA(ctx, cudaMemsetAsync(d_status, 0, 4, ctx->stream));
  BatchPtrs bp = {(uint64_t *)(dev[0] ? ptrs[0] : nullptr), (uint64_t *)(dev[1] ? ptrs[1] : nullptr),
                  (int64_t *)(dev[2] ? ptrs[2] : nullptr),  (int64_t *)(dev[3] ? ptrs[3] : nullptr),
                  (int64_t *)(dev[4] ? ptrs[4] : nullptr),  (int32_t *)(dev[5] ? ptrs[5] : nullptr),
                  (int32_t *)(dev[6] ? ptrs[6] : nullptr),  (int32_t *)(dev[7] ? ptrs[7] : nullptr)};
  PX_LAUNCH(ctx, "sol_unpack", k_sol_unpack, (n + 7) / 8, 256, 0, d_sol, n, a->D, bp, d_status);
  int32_t status = 0;
  std::vector<SolRec> h;
  if (any_host) {
    h.resize(n);
    PX_CUDA(ctx, cudaMemcpyAsync(h.data(), d_sol, sizeof(SolRec) * n, cudaMemcpyDeviceToHost, ctx->stream));
  }
  uint64_t n_cand = 0;
  PX_CUDA(ctx, cudaMemcpyAsync(&status, d_status, 4, cudaMemcpyDeviceToHost, ctx->stream));
  PX_CUDA(ctx, cudaMemcpyAsync(&n_cand, (const char *)d_sol + offsetof(SolRec, n_candidates), 8,
                               cudaMemcpyDeviceToHost, ctx->stream));
  PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  int rc = timing_collect(ctx);
  if (rc) return rc;
  if (status) return px_fail(ctx, PROTEUS_EINTERNAL, "internal check failed (status bits 0x%x)", status);
  o->n_candidates = n_cand;
  if (!any_host) return PROTEUS_OK;
  const int D = a->D;
  for (int i = 0; i < n; i++) {
    const SolRec &r = h[i];
    if (o->score && !dev[0]) o->score[i] = r.score;
    if (o->index && !dev[1]) o->index[i] = r.index;
    if (o->served && !dev[2]) o->served[i] = r.served;
    if (o->unmet && !dev[3]) o->unmet[i] = r.unmet;
    if (o->accsum && !dev[4]) o->accsum[i] = r.accsum;
    if (o->eff_acc_micro && !dev[5]) o->eff_acc_micro[i] = r.eff;
    if (o->option && !dev[6]) memcpy(o->option + (size_t)i * D, r.option, D * 4);
    if (o->z_qps && !dev[7]) memcpy(o->z_qps + (size_t)i * D, r.z, D * 4);
  }
  return PROTEUS_OK;
}

// families supplied in accuracy order (non-increasing within each family)?
static bool families_sorted(const proteus_ctx *ctx) {
  for (int q = 0; q < ctx->Q; q++)
    for (int v = 1; v < ctx->V[q]; v++)
      if (ctx->acc[ctx->off[q] + v] > ctx->acc[ctx->off[q] + v - 1]) return false;
  return true;
}

int px_flat_template_vm(int Q, int maxV);  // solve_enum.cu: VM of the specialised kernel, 0 if none

static int solve_common(proteus_ctx *ctx, const proteus_solve_args *a_in, proteus_solution *out, bool mat_only,
                        int32_t mat_vec, uint64_t mat_index, proteus_batch *bout = nullptr) {
  // PROTEUS_HOST_TIMING=1: host-side phase times of the call on stderr (diagnostic)
  static const bool htime = getenv("PROTEUS_HOST_TIMING") && atoi(getenv("PROTEUS_HOST_TIMING"));
  const auto ht0 = std::chrono::steady_clock::now();
  auto hts = [&](const char *what) {
    if (htime)
      fprintf(stderr, "solve %s %.1f us\n", what,
              std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - ht0).count());
  };
  SolveInputs in;
  int rc = validate_solve(ctx, a_in, in);
  if (rc) return rc;
  hts("validated");
  // distributed call (comm.cu): modes 0/1 scan the communicator rank's slice,
  // mode 2 solves the rank's slice of the demand vectors
  const bool dist = px_comm_active(ctx) && !mat_only;
  proteus_solve_args a_loc = *a_in;
  const proteus_solve_args *a = &a_loc;
  if (dist && a_in->mode != 2) {
    if (a_in->shard_world > 1) return px_fail(ctx, PROTEUS_EINVAL, "explicit shards in a distributed call");
    a_loc.shard_rank = ctx->comm_rank;
    a_loc.shard_world = ctx->comm_world;
  }
  if (!out && !bout) return px_fail(ctx, PROTEUS_EINVAL, "null out");
  if (mat_only && (a->mode == 2 || mat_vec < 0 || mat_vec >= a->n_vec))
    return px_fail(ctx, PROTEUS_EINVAL, "materialize: mode %d vec %d", a->mode, mat_vec);
  timing_reset(ctx);
  int K = 1 + ctx->M;
  int maxV = 0;
  for (int q = 0; q < ctx->Q; q++) maxV = ctx->V[q] > maxV ? ctx->V[q] : maxV;
  int VM = maxV;
  bool use_flat = false;
  if (a->mode == 0 && !(a->flags & PROTEUS_SOLVE_GENERIC) && a->D >= 3 && families_sorted(ctx)) {
    int vm = px_flat_template_vm(ctx->Q, maxV);
    if (vm) { VM = vm; use_flat = true; }
  }
  if (a->mode != 2) {
    bool ovf = false;
    uint64_t n = px_count_candidates(a->mode, a->D, in.dev_type.data(), ctx->T, K, &ovf);
    if (ovf || n > (1ull << 63)) return px_fail(ctx, PROTEUS_ERANGE, "candidate space exceeds 2^63");
    if (a->max_candidates && n > a->max_candidates)
      return px_fail(ctx, PROTEUS_ERANGE, "candidate space %llu > max_candidates %llu", (unsigned long long)n,
                     (unsigned long long)a->max_candidates);
  }
  const int32_t *d_dev = in.d_dev, *d_dem = in.d_dem;
  // Per-call tables (capacity a1, slot order, per-device capacity) depend only
  // on the profiles, the inventory and the SLOs: reused while those repeat.
  std::vector<int32_t> key;
  key.reserve(4 + in.dev_type.size() + in.slo.size());
  key.push_back((int32_t)ctx->prof_gen);
  key.push_back(a->D);
  key.push_back(VM);
  key.insert(key.end(), in.dev_type.begin(), in.dev_type.end());
  key.insert(key.end(), in.slo.begin(), in.slo.end());
  if (!ctx->tab_valid || key != ctx->tab_key) {
    ctx->tab_valid = false;
    if ((rc = px_prepare_tables(ctx, a->D, d_dev, in.d_slo, VM, ctx->tab, true))) return rc;
    // the launch parameters of the scoring kernels carry the capacity table
    ctx->tab_P.resize((size_t)ctx->T * ctx->M);
    ctx->tab_slot_code.resize((size_t)ctx->Q * VM);
    PX_CUDA(ctx, cudaMemcpyAsync(ctx->tab_P.data(), ctx->tab.P, ctx->tab_P.size() * 4, cudaMemcpyDeviceToHost,
                                 ctx->stream));
    PX_CUDA(ctx, cudaMemcpyAsync(ctx->tab_slot_code.data(), ctx->tab.slot_code, ctx->tab_slot_code.size() * 4,
                                 cudaMemcpyDeviceToHost, ctx->stream));
    PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
    ctx->tab_key = key;
    ctx->tab_valid = true;
  }
  const Tables &tab = ctx->tab;
  const std::vector<int32_t> &h_P = ctx->tab_P, &h_slot_code = ctx->tab_slot_code;
  int nout = mat_only ? 1 : a->n_vec;
  SolRec *d_sol = (SolRec *)px_buf(ctx, B_SOL, sizeof(SolRec) * nout);
  if (!d_sol) return px_fail(ctx, PROTEUS_ENOMEM, "solution buffer");
  if (a->mode == 2 && dist) {
    // vectors [lo, hi) on this rank, padded to `stride` records for the all-gather
    const int W = ctx->comm_world, R = ctx->comm_rank, n = a->n_vec;
    const int lo = (int)((int64_t)n * R / W), hi = (int)((int64_t)n * (R + 1) / W);
    const int stride = (n + W - 1) / W;
    SolRec *d_gat = (SolRec *)px_buf(ctx, B_C_GATHER, sizeof(SolRec) * (size_t)stride * (W + 1));
    if (!d_gat) return px_fail(ctx, PROTEUS_ENOMEM, "gather buffer");
    SolRec *d_mine = d_gat + (size_t)stride * W;
    if (hi > lo) {
      proteus_solve_args part = *a;
      part.n_vec = hi - lo;
      rc = px_solve_factored(ctx, &part, in.dev_type.data(), d_dev, d_dem + (size_t)lo * ctx->Q, VM, tab, h_P,
                             d_mine);
      if (rc) return rc;
    }
    if ((rc = px_comm_allgather(ctx, d_mine, d_gat, sizeof(SolRec) * (size_t)stride))) return rc;
    rc = px_gather_vectors(ctx, d_gat, W, n, stride, d_sol);
  } else if (a->mode == 2) {
    rc = px_solve_factored(ctx, a, in.dev_type.data(), d_dev, d_dem, VM, tab, h_P, d_sol);
  } else if (mat_only) {
    rc = px_solve_enum(ctx, a, in.dev_type.data(), in.slo.data(), in.demand.data(), VM, tab, h_P, h_slot_code,
                       d_sol, mat_vec, mat_vec + 1, true, mat_index, use_flat, d_dem);
  } else {
    rc = px_solve_enum(ctx, a, in.dev_type.data(), in.slo.data(), in.demand.data(), VM, tab, h_P, h_slot_code,
                       d_sol, 0, a->n_vec, false, 0, use_flat, d_dem);
    if (!rc && dist) {  // every rank's materialised winners -> the (score desc, index asc) maximum per vector
      const int W = ctx->comm_world;
      SolRec *d_gat = (SolRec *)px_buf(ctx, B_C_GATHER, sizeof(SolRec) * (size_t)nout * W);
      if (!d_gat) return px_fail(ctx, PROTEUS_ENOMEM, "gather buffer");
      if ((rc = px_comm_allgather(ctx, d_sol, d_gat, sizeof(SolRec) * (size_t)nout))) return rc;
      rc = px_pick_solrec(ctx, d_gat, W, nout, d_sol);
    }
  }
  if (rc) return rc;
  hts("launched");
  if (bout) {
    rc = batch_out(ctx, a, d_sol, nout, bout);
    hts("returned");
    return rc;
  }
  std::vector<SolRec> h(nout);
  PX_CUDA(ctx, cudaMemcpyAsync(h.data(), d_sol, sizeof(SolRec) * nout, cudaMemcpyDeviceToHost, ctx->stream));
  PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  if ((rc = timing_collect(ctx))) return rc;
  for (int i = 0; i < nout; i++)
    if (h[i].status != 0) return px_fail(ctx, PROTEUS_EINTERNAL, "internal check failed (vector %d, code %d)", i, h[i].status);
  for (int i = 0; i < nout; i++) {
    proteus_solution &o = out[i];
    o.score = h[i].score;
    o.index = h[i].index;
    o.served = h[i].served;
    o.unmet = h[i].unmet;
    o.accsum = h[i].accsum;
    o.eff_acc_micro = h[i].eff;
    o.n_candidates = h[i].n_candidates;
    // device outputs: copied on the stream from the device record (no host round trip), one sync below
    if (o.option) {
      if (px_is_device_ptr(o.option))
        PX_CUDA(ctx, cudaMemcpyAsync(o.option, d_sol[i].option, a->D * 4, cudaMemcpyDeviceToDevice, ctx->stream));
      else memcpy(o.option, h[i].option, a->D * 4);
    }
    if (o.z_qps) {
      if (px_is_device_ptr(o.z_qps))
        PX_CUDA(ctx, cudaMemcpyAsync(o.z_qps, d_sol[i].z, a->D * 4, cudaMemcpyDeviceToDevice, ctx->stream));
      else memcpy(o.z_qps, h[i].z, a->D * 4);
    }
  }
  PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  return PROTEUS_OK;
}

extern "C" {

int proteus_solve(proteus_ctx *ctx, const proteus_solve_args *args, proteus_solution *out) {
  return solve_common(ctx, args, out, false, 0, 0);
}

int proteus_solve_batch(proteus_ctx *ctx, const proteus_solve_args *args, proteus_batch *out) {
  if (!out) return px_fail(ctx, PROTEUS_EINVAL, "null out");
  return solve_common(ctx, args, nullptr, false, 0, 0, out);
}

int proteus_materialize(proteus_ctx *ctx, const proteus_solve_args *args, int32_t vec, uint64_t index,
                        proteus_solution *out) {
  return solve_common(ctx, args, out, true, vec, index);
}

int proteus_candidate_count(proteus_ctx *ctx, const proteus_solve_args *a, uint64_t *count) {
  if (!ctx || !a || !count) return PROTEUS_EINVAL;
  if (!ctx->have_prof) return px_fail(ctx, PROTEUS_EINVAL, "no profiles loaded");
  if (a->mode != 0 && a->mode != 1) return px_fail(ctx, PROTEUS_EINVAL, "mode %d", a->mode);
  std::vector<int32_t> dev;
  int rc;
  if ((rc = to_host(ctx, a->device_type, a->D, dev))) return rc;
  bool ovf = false;
  *count = px_count_candidates(a->mode, a->D, dev.data(), ctx->T, 1 + ctx->M, &ovf);
  return ovf ? px_fail(ctx, PROTEUS_ERANGE, "candidate space exceeds 2^64") : PROTEUS_OK;
}

// ------------------------------------------------------------ combine -----
int proteus_combine_solutions(proteus_ctx *ctx, int32_t world, int32_t n_vec, int32_t D, const proteus_batch *parts,
                              const uint64_t *part_candidates, proteus_batch *out) {
  if (!ctx) return PROTEUS_EINVAL;
  ctx->err.clear();
  if (world < 1 || n_vec < 1 || D < 1 || D > PX_MAXD || !parts || !out)
    return px_fail(ctx, PROTEUS_EINVAL, "combine: world %d n_vec %d D %d", world, n_vec, D);
  PX_CUDA(ctx, cudaSetDevice(ctx->device));
  timing_reset(ctx);
  // marshal the parts into the record layout the NCCL path gathers (host side: layout only)
  std::vector<SolRec> recs((size_t)world * n_vec);
  memset(recs.data(), 0, recs.size() * sizeof(SolRec));
  for (int r = 0; r < world; r++) {
    const proteus_batch &p = parts[r];
    if (!p.score || !p.index || !p.served || !p.unmet || !p.accsum || !p.eff_acc_micro || !p.option || !p.z_qps)
      return px_fail(ctx, PROTEUS_EINVAL, "combine: part %d lacks a field", r);
    std::vector<uint64_t> sc, ix;
    std::vector<int64_t> sv, um, ac;
    std::vector<int32_t> ef, op, zz;
    int rc;
    if ((rc = to_host(ctx, p.score, n_vec, sc)) || (rc = to_host(ctx, p.index, n_vec, ix)) ||
        (rc = to_host(ctx, p.served, n_vec, sv)) || (rc = to_host(ctx, p.unmet, n_vec, um)) ||
        (rc = to_host(ctx, p.accsum, n_vec, ac)) || (rc = to_host(ctx, p.eff_acc_micro, n_vec, ef)) ||
        (rc = to_host(ctx, p.option, (size_t)n_vec * D, op)) || (rc = to_host(ctx, p.z_qps, (size_t)n_vec * D, zz)))
      return rc;
    for (int v = 0; v < n_vec; v++) {
      SolRec &x = recs[(size_t)r * n_vec + v];
      x.score = sc[v]; x.index = ix[v]; x.served = sv[v]; x.unmet = um[v]; x.accsum = ac[v]; x.eff = ef[v];
      x.n_candidates = part_candidates ? part_candidates[r] : 0;
      memcpy(x.option, &op[(size_t)v * D], D * 4);
      memcpy(x.z, &zz[(size_t)v * D], D * 4);
    }
  }
  SolRec *d_gat = (SolRec *)px_buf(ctx, B_C_GATHER, sizeof(SolRec) * recs.size());
  SolRec *d_sol = (SolRec *)px_buf(ctx, B_SOL, sizeof(SolRec) * (size_t)n_vec);
  if (!d_gat || !d_sol) return px_fail(ctx, PROTEUS_ENOMEM, "combine buffers");
  PX_CUDA(ctx, cudaMemcpyAsync(d_gat, recs.data(), sizeof(SolRec) * recs.size(), cudaMemcpyHostToDevice, ctx->stream));
  int rc = px_pick_solrec(ctx, d_gat, world, n_vec, d_sol);
  if (rc) return rc;
  proteus_solve_args a;
  memset(&a, 0, sizeof a);
  a.D = D;
  return batch_out(ctx, &a, d_sol, n_vec, out);
}

int proteus_pareto_merge(proteus_ctx *ctx, const proteus_pareto_point *pts, int32_t n, proteus_pareto_point *out,
                         int32_t max_points, int32_t *n_points) {
  if (!ctx) return PROTEUS_EINVAL;
  ctx->err.clear();
  if (n < 0 || (n > 0 && !pts) || !n_points || max_points < 0 || (max_points > 0 && !out))
    return px_fail(ctx, PROTEUS_EINVAL, "pareto_merge arguments");
  PX_CUDA(ctx, cudaSetDevice(ctx->device));
  timing_reset(ctx);
  int rc;
  const proteus_pareto_point *d_pts = to_device(ctx, pts, (size_t)n, B_IN0, &rc);
  if (rc) return rc;
  proteus_pareto_point *d_out = (proteus_pareto_point *)px_buf(ctx, B_C_PTS, sizeof(proteus_pareto_point) * (size_t)(n + 1) + 16);
  if (!d_out) return px_fail(ctx, PROTEUS_ENOMEM, "merge output");
  int32_t *d_n = (int32_t *)(d_out + n + 1);
  if ((rc = px_pareto_merge(ctx, d_pts, n, d_out, d_n))) return rc;
  int32_t nf = 0;
  PX_CUDA(ctx, cudaMemcpyAsync(&nf, d_n, 4, cudaMemcpyDeviceToHost, ctx->stream));
  PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  const int k = nf < max_points ? nf : max_points;
  if (k > 0) {
    if (px_is_device_ptr(out))
      PX_CUDA(ctx, cudaMemcpyAsync(out, d_out, sizeof(proteus_pareto_point) * k, cudaMemcpyDeviceToDevice, ctx->stream));
    else
      PX_CUDA(ctx, cudaMemcpyAsync(out, d_out, sizeof(proteus_pareto_point) * k, cudaMemcpyDeviceToHost, ctx->stream));
    PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  }
  if ((rc = timing_collect(ctx))) return rc;
  *n_points = nf;
  return PROTEUS_OK;
}

// ------------------------------------------------------------- pareto -----
int proteus_pareto(proteus_ctx *ctx, const proteus_pareto_args *a, proteus_pareto_point *out, int32_t max_points,
                   int32_t *n_points, uint64_t *n_configs) {
  if (!ctx) return PROTEUS_EINVAL;
  ctx->err.clear();
  if (!a || !n_points || !n_configs || max_points < 0 || (max_points > 0 && !out))
    return px_fail(ctx, PROTEUS_EINVAL, "null argument");
  if (!ctx->have_prof) return px_fail(ctx, PROTEUS_EINVAL, "no profiles loaded");
  if (a->D < 1 || a->D > PX_MAXD || !a->device_type || !a->slo_us)
    return px_fail(ctx, PROTEUS_EINVAL, "D=%d out of range or null array", a->D);
  if (a->family < 0 || a->family >= ctx->Q) return px_fail(ctx, PROTEUS_EINVAL, "family %d", a->family);
  const int world = a->shard_world > 0 ? a->shard_world : 1, rank = a->shard_world > 0 ? a->shard_rank : 0;
  if (rank < 0 || rank >= world) return px_fail(ctx, PROTEUS_EINVAL, "shard %d/%d", rank, world);
  PX_CUDA(ctx, cudaSetDevice(ctx->device));
  timing_reset(ctx);
  std::vector<int32_t> dev, slo;
  int rc;
  if ((rc = to_host(ctx, a->device_type, a->D, dev)) || (rc = to_host(ctx, a->slo_us, ctx->Q, slo))) return rc;
  for (int d = 0; d < a->D; d++)
    if (dev[d] < 0 || dev[d] >= ctx->T) return px_fail(ctx, PROTEUS_EINVAL, "device_type[%d]=%d", d, dev[d]);
  for (int q = 0; q < ctx->Q; q++)
    if (slo[q] < 0) return px_fail(ctx, PROTEUS_EINVAL, "slo_us[%d] < 0", q);
  const int32_t *d_dev = to_device(ctx, dev.data(), dev.size(), B_IN0, &rc);
  if (rc) return rc;
  const int32_t *d_slo = to_device(ctx, slo.data(), slo.size(), B_IN1, &rc);
  if (rc) return rc;
  std::vector<proteus_pareto_point> h(max_points > 0 ? max_points : 1);
  int32_t np = 0;
  uint64_t nc = 0;
  if ((rc = px_pareto(ctx, a->D, dev.data(), d_dev, d_slo, a->family, a->allow_idle != 0, rank, world, h.data(),
                      max_points, &np, &nc)))
    return rc;
  if ((rc = timing_collect(ctx))) return rc;
  for (int i = 0; i < np && i < max_points; i++) out[i] = h[i];
  *n_points = np;
  *n_configs = nc;
  return PROTEUS_OK;
}

// ------------------------------------------------------------- replay -----

// Outputs of a replay: per-scenario aggregates [3][S] (+ the unsorted flag)
// from d_agg -- straight device-to-device into device outputs, one copy per
// array -- and the latency rows [S_run][N] into a host buffer.
static int replay_outputs(proteus_ctx *ctx, const uint64_t *d_agg, int S, int64_t N, int S_run, uint32_t *latency_us,
                          bool lat_dev, const uint32_t *d_lat, uint64_t *violations, uint64_t *on_time,
                          uint64_t *acc_sum) {
  uint64_t *outs[3] = {violations, on_time, acc_sum};
  for (int k = 0; k < 3; k++)
    if (outs[k] && px_is_device_ptr(outs[k]))
      PX_CUDA(ctx, cudaMemcpyAsync(outs[k], d_agg + (size_t)k * S, (size_t)S * 8, cudaMemcpyDeviceToDevice,
                                   ctx->stream));
  std::vector<uint64_t> agg((size_t)3 * S + 1);
  PX_CUDA(ctx, cudaMemcpyAsync(agg.data(), d_agg, ((size_t)3 * S + 1) * 8, cudaMemcpyDeviceToHost, ctx->stream));
  if (latency_us && !lat_dev && S_run > 0)
    PX_CUDA(ctx, cudaMemcpyAsync(latency_us, d_lat, (size_t)S_run * N * 4, cudaMemcpyDeviceToHost, ctx->stream));
  PX_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  int rc;
  if ((rc = timing_collect(ctx))) return rc;
  if (agg[3 * (size_t)S] != 0) return px_fail(ctx, PROTEUS_ERANGE, "arrival timestamps not sorted");
  for (int k = 0; k < 3; k++)
    if (outs[k] && !px_is_device_ptr(outs[k])) memcpy(outs[k], &agg[(size_t)k * S], (size_t)S * 8);
  return PROTEUS_OK;
}
// Distributed replay (comm.cu): this rank's scenarios only; their aggregates
// [3][S_own] (+ the unsorted flag) are scattered into a zero [3][S] (+ flag)
// vector that one all-reduce(SUM) completes on every rank.
__global__ void k_agg_scatter(const uint64_t *__restrict__ loc, int S_loc, const int32_t *__restrict__ map,
                              uint64_t *full, int S) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < 3 * S_loc) full[(size_t)(i / S_loc) * S + map[i % S_loc]] = loc[i];
  if (i == 0) full[(size_t)3 * S] = loc[(size_t)3 * S_loc];
}

struct ReplayShard {
  bool dist = false;
  std::vector<proteus_scenario> sc;  // this rank's scenarios (ascending scenario index)
  std::vector<int32_t> map;          // their scenario indices
};

static void replay_shard(proteus_ctx *ctx, const std::vector<proteus_scenario> &scv, ReplayShard &sh) {
  sh.dist = px_comm_active(ctx);
  if (!sh.dist) return;
  std::vector<int32_t> owner(scv.size());
  px_scenario_owner(scv.data(), (int)scv.size(), ctx->comm_world, owner.data());
  for (size_t s = 0; s < scv.size(); s++)
    if (owner[s] == ctx->comm_rank) { sh.sc.push_back(scv[s]); sh.map.push_back((int32_t)s); }
}

// combine a distributed replay's aggregates into d_full [3][S] + flag
static int replay_combine(proteus_ctx *ctx, const ReplayShard &sh, const uint64_t *d_loc, int S, uint64_t *d_full) {
  const int S_loc = (int)sh.map.size();
  PX_CUDA(ctx, cudaMemsetAsync(d_full, 0, ((size_t)3 * S + 1) * 8, ctx->stream));
  int32_t *d_map = (int32_t *)px_buf(ctx, B_C_PTS, (size_t)S_loc * 4 + 16);
  if (!d_map) return px_fail(ctx, PROTEUS_ENOMEM, "scenario map");
  if (S_loc) {
    PX_CUDA(ctx, cudaMemcpyAsync(d_map, sh.map.data(), (size_t)S_loc * 4, cudaMemcpyHostToDevice, ctx->stream));
    PX_LAUNCH(ctx, "agg_scatter", k_agg_scatter, (3 * S_loc + 255) / 256, 256, 0, d_loc, S_loc, d_map, d_full, S);
  }
  return px_comm_allreduce_u64(ctx, d_full, (size_t)3 * S + 1, PX_RED_SUM);
}

int proteus_replay(proteus_ctx *ctx, const uint32_t *arrival_us, const uint8_t *family, int64_t N,
                   const int32_t *option, const int32_t *z_qps, const int32_t *device_type, int32_t D,
                   const int32_t *demand_qps, const int32_t *slo_base_us, const proteus_scenario *sc, int32_t S,
                   uint32_t *latency_us, uint64_t *violations, uint64_t *on_time, uint64_t *acc_sum) {
  if (!ctx) return PROTEUS_EINVAL;
  ctx->err.clear();
  if (!ctx->have_prof) return px_fail(ctx, PROTEUS_EINVAL, "no profiles loaded");
  if (N < 0 || (N > 0 && (!arrival_us || !family))) return px_fail(ctx, PROTEUS_EINVAL, "trace");
  if (N >= (1ll << 32)) return px_fail(ctx, PROTEUS_ERANGE, "N >= 2^32");
  if (D < 1 || D > PX_MAXD || !option || !z_qps || !device_type || !demand_qps || !slo_base_us)
    return px_fail(ctx, PROTEUS_EINVAL, "allocation arguments");
  if (S < 1 || S > 4096 || !sc) return px_fail(ctx, PROTEUS_EINVAL, "S=%d", S);
  PX_CUDA(ctx, cudaSetDevice(ctx->device));
  timing_reset(ctx);
  int rc;
  std::vector<int32_t> opt, z, dev, dem, slo;
  std::vector<proteus_scenario> scv;
  if ((rc = to_host(ctx, option, D, opt)) || (rc = to_host(ctx, z_qps, D, z)) ||
      (rc = to_host(ctx, device_type, D, dev)) || (rc = to_host(ctx, demand_qps, ctx->Q, dem)) ||
      (rc = to_host(ctx, slo_base_us, ctx->Q, slo)) || (rc = to_host(ctx, sc, S, scv)))
    return rc;
  int64_t dsum = 0;
  for (int q = 0; q < ctx->Q; q++) {
    if (dem[q] < 0 || slo[q] < 0) return px_fail(ctx, PROTEUS_EINVAL, "negative demand/slo");
    dsum += dem[q];
  }
  if (dsum >= (1 << 22)) return px_fail(ctx, PROTEUS_ERANGE, "sum of demand >= 2^22");
  std::vector<int64_t> zsum(ctx->Q, 0);
  for (int d = 0; d < D; d++) {
    if (dev[d] < 0 || dev[d] >= ctx->T) return px_fail(ctx, PROTEUS_EINVAL, "device_type[%d]", d);
    if (opt[d] < 0 || opt[d] > ctx->M) return px_fail(ctx, PROTEUS_EINVAL, "option[%d]=%d", d, opt[d]);
    if (z[d] < 0 || (opt[d] == 0 && z[d] != 0)) return px_fail(ctx, PROTEUS_EINVAL, "z[%d]=%d", d, z[d]);
    if (opt[d]) zsum[ctx->fam[opt[d] - 1]] += z[d];
  }
  for (int q = 0; q < ctx->Q; q++)
    if (zsum[q] > dem[q]) return px_fail(ctx, PROTEUS_EINVAL, "sum z of family %d exceeds its demand", q);
  for (int s = 0; s < S; s++)
    if (scv[s].slo_mult_milli < 0 || scv[s].batch_cap < 0 || scv[s].routing < 0 || scv[s].routing > 1 ||
        scv[s].policy < 0 || scv[s].policy > 2)
      return px_fail(ctx, PROTEUS_EINVAL, "scenario %d", s);
  const uint32_t *d_arr = to_device(ctx, arrival_us, (size_t)N, B_IN0, &rc);
  if (rc) return rc;
  const uint8_t *d_fam = to_device(ctx, family, (size_t)N, B_IN1, &rc);
  if (rc) return rc;
  ReplayShard sh;
  replay_shard(ctx, scv, sh);
  const int S_run = sh.dist ? (int)sh.sc.size() : S;  // scenarios replayed here
  const proteus_scenario *sc_run = sh.dist ? sh.sc.data() : scv.data();
  uint32_t *d_lat = nullptr;
  bool lat_dev = latency_us && px_is_device_ptr(latency_us);
  if (latency_us) {
    d_lat = lat_dev ? latency_us : (uint32_t *)px_buf(ctx, B_R_LAT, (size_t)S_run * N * 4);
    if (!d_lat) return px_fail(ctx, PROTEUS_ENOMEM, "latency buffer");
  }
  // [3][S_run] + flag, then (distributed) the combined [3][S] + flag
  uint64_t *d_agg0 = (uint64_t *)px_buf(ctx, B_R_AGG, ((size_t)3 * S_run + 1 + (sh.dist ? 3 * (size_t)S + 1 : 0)) * 8);
  if (!d_agg0) return px_fail(ctx, PROTEUS_ENOMEM, "aggregate buffer");
  uint64_t *d_agg = d_agg0;
  if (S_run > 0) {
    rc = px_replay(ctx, d_arr, d_fam, N, opt.data(), z.data(), dev.data(), D, dem.data(), slo.data(), sc_run, S_run,
                   d_lat, d_agg);
    if (rc) return rc;
  } else {
    PX_CUDA(ctx, cudaMemsetAsync(d_agg, 0, 8, ctx->stream));
  }
  if (sh.dist) {
    d_agg = d_agg0 + 3 * (size_t)S_run + 1;
    if ((rc = replay_combine(ctx, sh, d_agg0, S, d_agg))) return rc;
  }
  return replay_outputs(ctx, d_agg, S, N, S_run, latency_us, lat_dev, d_lat, violations, on_time, acc_sum);
}

// -------------------------------------------------------- closed loop -----
int proteus_replay_epochs(proteus_ctx *ctx, const uint32_t *arrival_us, const uint8_t *family, int64_t N,
                          int32_t E, int64_t epoch_us, const int32_t *option, const int32_t *z_qps,
                          const int32_t *device_type, int32_t D, const int32_t *demand_qps,
                          const int32_t *slo_base_us, const proteus_scenario *sc, int32_t S, uint32_t *latency_us,
                          uint64_t *violations, uint64_t *on_time, uint64_t *acc_sum) {
  if (!ctx) return PROTEUS_EINVAL;
  ctx->err.clear();
  if (!ctx->have_prof) return px_fail(ctx, PROTEUS_EINVAL, "no profiles loaded");
  if (N < 0 || (N > 0 && (!arrival_us || !family))) return px_fail(ctx, PROTEUS_EINVAL, "trace");
  if (N >= (1ll << 32)) return px_fail(ctx, PROTEUS_ERANGE, "N >= 2^32");
  if (E < 1 || E > (1 << 24) || epoch_us < 1) return px_fail(ctx, PROTEUS_EINVAL, "E=%d epoch_us=%lld", E, (long long)epoch_us);
  if (D < 1 || D > PX_MAXD || !option || !z_qps || !device_type || !demand_qps || !slo_base_us)
    return px_fail(ctx, PROTEUS_EINVAL, "allocation arguments");
  if (S < 1 || S > 4096 || !sc) return px_fail(ctx, PROTEUS_EINVAL, "S=%d", S);
  PX_CUDA(ctx, cudaSetDevice(ctx->device));
  timing_reset(ctx);
  int rc;
  std::vector<int32_t> opt, z, dev, dem, slo;
  std::vector<proteus_scenario> scv;
  if ((rc = to_host(ctx, option, (size_t)E * D, opt)) || (rc = to_host(ctx, z_qps, (size_t)E * D, z)) ||
      (rc = to_host(ctx, device_type, D, dev)) || (rc = to_host(ctx, demand_qps, (size_t)E * ctx->Q, dem)) ||
      (rc = to_host(ctx, slo_base_us, ctx->Q, slo)) || (rc = to_host(ctx, sc, S, scv)))
    return rc;
  for (int q = 0; q < ctx->Q; q++)
    if (slo[q] < 0) return px_fail(ctx, PROTEUS_EINVAL, "negative slo");
  for (int d = 0; d < D; d++)
    if (dev[d] < 0 || dev[d] >= ctx->T) return px_fail(ctx, PROTEUS_EINVAL, "device_type[%d]", d);
  std::vector<int64_t> zsum(ctx->Q);
  for (int e = 0; e < E; e++) {
    int64_t dsum = 0;
    for (int q = 0; q < ctx->Q; q++) {
      if (dem[(size_t)e * ctx->Q + q] < 0) return px_fail(ctx, PROTEUS_EINVAL, "negative demand");
      dsum += dem[(size_t)e * ctx->Q + q];
      zsum[q] = 0;
    }
    if (dsum >= (1 << 22)) return px_fail(ctx, PROTEUS_ERANGE, "sum of demand >= 2^22 (epoch %d)", e);
    for (int d = 0; d < D; d++) {
      const int32_t o = opt[(size_t)e * D + d], zz = z[(size_t)e * D + d];
      if (o < 0 || o > ctx->M) return px_fail(ctx, PROTEUS_EINVAL, "option[%d][%d]=%d", e, d, o);
      if (zz < 0 || (o == 0 && zz != 0)) return px_fail(ctx, PROTEUS_EINVAL, "z[%d][%d]=%d", e, d, zz);
      if (o) zsum[ctx->fam[o - 1]] += zz;
    }
    for (int q = 0; q < ctx->Q; q++)
      if (zsum[q] > dem[(size_t)e * ctx->Q + q])
        return px_fail(ctx, PROTEUS_EINVAL, "sum z of family %d exceeds its demand (epoch %d)", q, e);
  }
  for (int s = 0; s < S; s++)
    if (scv[s].slo_mult_milli < 0 || scv[s].batch_cap < 0 || scv[s].routing != 0 || scv[s].policy != 0)
      return px_fail(ctx, PROTEUS_EINVAL, "scenario %d (closed loop: routing 0, policy 0)", s);
  const uint32_t *d_arr = to_device(ctx, arrival_us, (size_t)N, B_IN0, &rc);
  if (rc) return rc;
  const uint8_t *d_fam = to_device(ctx, family, (size_t)N, B_IN1, &rc);
  if (rc) return rc;
  ReplayShard sh;
  replay_shard(ctx, scv, sh);
  const int S_run = sh.dist ? (int)sh.sc.size() : S;  // scenarios replayed here
  const proteus_scenario *sc_run = sh.dist ? sh.sc.data() : scv.data();
  uint32_t *d_lat = nullptr;
  bool lat_dev = latency_us && px_is_device_ptr(latency_us);
  if (latency_us) {
    d_lat = lat_dev ? latency_us : (uint32_t *)px_buf(ctx, B_R_LAT, (size_t)S_run * N * 4);
    if (!d_lat) return px_fail(ctx, PROTEUS_ENOMEM, "latency buffer");
  }
  // [3][S_run] + flag, then (distributed) the combined [3][S] + flag
  uint64_t *d_agg0 = (uint64_t *)px_buf(ctx, B_R_AGG, ((size_t)3 * S_run + 1 + (sh.dist ? 3 * (size_t)S + 1 : 0)) * 8);
  if (!d_agg0) return px_fail(ctx, PROTEUS_ENOMEM, "aggregate buffer");
  uint64_t *d_agg = d_agg0;
  if (S_run > 0) {
    rc = px_replay_epochs(ctx, d_arr, d_fam, N, E, epoch_us, opt.data(), z.data(), dev.data(), D, dem.data(),
                          slo.data(), sc_run, S_run, d_lat, d_agg);
    if (rc) return rc;
  } else {
    PX_CUDA(ctx, cudaMemsetAsync(d_agg, 0, 8, ctx->stream));
  }
  if (sh.dist) {
    d_agg = d_agg0 + 3 * (size_t)S_run + 1;
    if ((rc = replay_combine(ctx, sh, d_agg0, S, d_agg))) return rc;
  }
  return replay_outputs(ctx, d_agg, S, N, S_run, latency_us, lat_dev, d_lat, violations, on_time, acc_sum);
}

}  // extern "C"
