// C ABI of the Multigrain forward (include/mg.h). Host-side: validation, plan lifetime,
// device upload, TMA descriptors, workspace, launches. Every step of the attention runs in the
// kernels of coarse_pp_sm100.cu, fine_mma.cu / fine_rows.cu and staged.cu; there is no CPU fallback.
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "kernels.cuh"
#include "mg.h"
#include "plan.hpp"

namespace {

thread_local std::string g_err;

mg_status fail(mg_status s, const std::string& msg) {
  g_err = msg;
  return s;
}
mg_status cuda_fail(cudaError_t e, const char* where) {
  return fail(MG_ERR_CUDA, std::string(where) + ": " + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ")");
}

PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(ptr);
  });
  return fn;
}

}  // namespace

struct mg_plan_s {
  mg::HostPlan hp;
  int device = -1;
  bool uploaded = false;
  int num_sms = 0;
  int num_sms_override = 0;
  int fine_kernel = 0;   // 0: mma.sync kernel (fine_mma.cu), 1: CUDA-core kernel (fine_rows.cu)
  int concurrency = 0;   // 0 default, 1 serial, 2 concurrent streams, 3 SM split (see mg_plan_opts)
  cudaStream_t side = nullptr;              // second stream of the concurrent mode
  // host-buffer forward: copy streams and per-chunk events (H2D of chunk c+1 and D2H of chunk c-1
  // overlap the forward of chunk c)
  cudaStream_t h2d = nullptr, d2h = nullptr;
  std::vector<cudaEvent_t> host_ev;
  cudaEvent_t host_event(size_t i) {
    while (host_ev.size() <= i) {
      cudaEvent_t e = nullptr;
      if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return nullptr;
      host_ev.push_back(e);
    }
    return host_ev[i];
  }
  cudaEvent_t fork_ev = nullptr, join_ev = nullptr;
  std::vector<void*> allocs;
  mg::Item* d_items = nullptr;
  mg::Item* d_items_split = nullptr;   // dense items split into column chunks (chosen per forward)
  int32_t* d_fine_sample = nullptr;    // batched plans: sample of each fine row
  mg::TileRef* d_trefs = nullptr;
  uint64_t* d_masks = nullptr;
  int32_t* d_strip_cols = nullptr;
  int32_t* d_global_rows = nullptr;
  int32_t* d_fine_slot = nullptr;
  int32_t* d_fine_rows = nullptr;
  int32_t* d_fine_row_ptr = nullptr;
  int32_t* d_fine_col = nullptr;
  int32_t* d_counter = nullptr;
  // stream-ordered workspaces
  float* d_part = nullptr;
  size_t part_cap = 0;      // in (row, bh) partial slots
  uint8_t* d_stage = nullptr;
  size_t stage_cap = 0;     // bytes
  uint8_t* d_dense = nullptr;   // split dense items: partials, then counters (zeroed at allocation)
  size_t dense_cap = 0;         // in (b*h) units
  // staged (paper-dataflow) path: canonical plan on the device, uploaded on first use
  bool staged_uploaded = false;
  int32_t *d_bsr_row_ptr = nullptr, *d_bsr_col = nullptr, *d_tile_row = nullptr, *d_csr_row_ptr = nullptr,
          *d_csr_col = nullptr;
  uint64_t* d_tile_masks = nullptr;
  uint8_t* d_row_is_global = nullptr;
  uint8_t* d_staged_ws = nullptr;   // S, P and O_csr buffers of mg_sparse_attention_fwd_staged
  cudaStream_t staged_side = nullptr;   // second stream of the multi-stream staged forward
  cudaEvent_t staged_ev = nullptr;
  size_t staged_ws_cap = 0;
  // TMA descriptors of the last forward's Q/K/V/O (re-encoded only when a tensor descriptor changes:
  // cuTensorMapEncodeTiled is host work on every call otherwise)
  struct Maps {
    mg_tensor q, k, v, o;
    bool valid = false, ok = false, gather_ok = false, store_ok = false;
    CUtensorMap tq, tk, tv, tq2, tk2, tv2, to;
    longlong3 rq, rk, rv;
  } maps;
  // diagnostics: device event-trace buffer of the coarse kernel (CTA 0)
  unsigned long long* trace = nullptr;
  int32_t trace_cap = 0;
  // profiling: per recorded call as few events as the call's kernels need (every timing event is
  // a point the stream must drain to, ~2-3 us each on B200, so a single-kernel call records 2):
  //   serial: E0 [fine] E1 [coarse] E2 (E1 only with both kernels);
  //   concurrent: E0 fork [fine on side] E1(side) [coarse] E2 join E3.
  struct ProfCall {
    int32_t first, last, fb, fe, cb, ce;   // event indices (-1: kernel absent)
  };
  bool profiling = false;
  std::vector<cudaEvent_t> prof_events;
  size_t prof_used = 0;
  std::vector<ProfCall> prof_calls;

  cudaEvent_t prof_event() {
    if (prof_used == prof_events.size()) {
      cudaEvent_t e = nullptr;
      if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
      prof_events.push_back(e);
    }
    return prof_events[prof_used++];
  }

  ~mg_plan_s() {
    for (cudaEvent_t e : prof_events) cudaEventDestroy(e);
    if (fork_ev) cudaEventDestroy(fork_ev);
    if (join_ev) cudaEventDestroy(join_ev);
    if (side) cudaStreamDestroy(side);
    for (cudaEvent_t e : host_ev) cudaEventDestroy(e);
    if (h2d) cudaStreamDestroy(h2d);
    if (d2h) cudaStreamDestroy(d2h);
    for (void* p : allocs) cudaFree(p);
    if (d_part) cudaFree(d_part);
    if (d_stage) cudaFree(d_stage);
    if (d_dense) cudaFree(d_dense);
    if (d_staged_ws) cudaFree(d_staged_ws);
    if (staged_side) cudaStreamDestroy(staged_side);
    if (staged_ev) cudaEventDestroy(staged_ev);
  }
};

namespace {

template <class T>
cudaError_t upload_vec(mg_plan_s* p, T** dst, const std::vector<T>& v) {
  const size_t bytes = std::max<size_t>(v.size() * sizeof(T), 16);
  cudaError_t e = cudaMalloc(reinterpret_cast<void**>(dst), bytes);
  if (e != cudaSuccess) return e;
  p->allocs.push_back(*dst);
  if (!v.empty()) e = cudaMemcpy(*dst, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice);
  return e;
}

mg_status upload(mg_plan_s* p) {
  if (p->uploaded) return MG_OK;
  if (!p->hp.kernel_ready) return fail(MG_ERR_UNSUPPORTED, "the forward requires block 64 or 128");
  cudaError_t e = cudaGetDevice(&p->device);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
  e = cudaDeviceGetAttribute(&p->num_sms, cudaDevAttrMultiProcessorCount, p->device);
  if (e != cudaSuccess) return cuda_fail(e, "cudaDeviceGetAttribute");
  int major = 0;
  cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, p->device);
  if (major != 10) return fail(MG_ERR_UNSUPPORTED, "this library is built for sm_100a (B200) only");
  const mg::HostPlan& h = p->hp;
  // the fine kernels' gather pointer issues one ring step per row start (fine_mma.cu issue_step):
  // every fine row must hold at least one entry (plan.cpp never lists an empty CSR row)
  for (size_t i = 0; i + 1 < h.fine_row_ptr.size(); ++i)
    if (h.fine_row_ptr[i + 1] <= h.fine_row_ptr[i]) return fail(MG_ERR_INTERNAL, "plan lists an empty fine row");
  if ((e = upload_vec(p, &p->d_items, h.items)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_items_split, h.items_split)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_fine_sample, h.fine_sample)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_trefs, h.trefs)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_masks, h.dev_masks)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_strip_cols, h.strip_cols)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_global_rows, h.global_rows)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_fine_slot, h.fine_slot)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_fine_rows, h.fine_rows)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_fine_row_ptr, h.fine_row_ptr)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_fine_col, h.fine_col)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_counter, std::vector<int32_t>(4, 0))) != cudaSuccess)
    return e == cudaErrorMemoryAllocation ? fail(MG_ERR_OUT_OF_MEMORY, "device allocation failed")
                                          : cuda_fail(e, "plan upload");
  p->uploaded = true;
  return MG_OK;
}

mg_status create_impl(int64_t L, int32_t heads, int32_t d, int32_t window, const int32_t* global_idx,
                      int64_t n_global, const int32_t* extra_idx, int64_t n_extra, const mg_plan_opts* opts,
                      mg_plan_t* plan_out, int64_t batch = 0, const int64_t* global_ptr = nullptr,
                      const int64_t* extra_ptr = nullptr) {
  if (!plan_out) return fail(MG_ERR_INVALID_ARG, "plan_out is null");
  *plan_out = nullptr;
  mg::PlanOptions po;
  int sms_override = 0, fine_kernel = 0, concurrency = 0;
  if (opts) {
    if (opts->block != 0) po.block = opts->block;
    po.force_all_fine = opts->force_all_fine != 0;
    if (opts->strip_max_cols != 0) po.strip_max_cols = opts->strip_max_cols < 0 ? 0 : opts->strip_max_cols;
    if (po.strip_max_cols > 128) return fail(MG_ERR_INVALID_ARG, "strip_max_cols must be <= 128");
    if (opts->num_sms < 0) return fail(MG_ERR_INVALID_ARG, "num_sms must be >= 0");
    sms_override = opts->num_sms;
    if (opts->fine_kernel < 0 || opts->fine_kernel > 1) return fail(MG_ERR_INVALID_ARG, "fine_kernel must be 0 or 1");
    fine_kernel = opts->fine_kernel;
    if (opts->concurrency < 0 || opts->concurrency > 3) return fail(MG_ERR_INVALID_ARG, "concurrency must be 0, 1, 2 or 3");
    concurrency = opts->concurrency;
    if (!(opts->tau >= 0.f && opts->tau <= 1.f)) return fail(MG_ERR_INVALID_ARG, "tau must be in [0, 1]");
    po.tau = opts->tau;
    if (opts->dense_chunk < -1) return fail(MG_ERR_INVALID_ARG, "dense_chunk must be >= -1");
    if (opts->dense_chunk < 0) po.dense_split = 1;
    if (opts->dense_chunk > 0) {
      po.dense_split = 2;
      po.dense_chunk = opts->dense_chunk;
    }
  }
  mg_plan_s* p = new (std::nothrow) mg_plan_s();
  if (!p) return fail(MG_ERR_OUT_OF_MEMORY, "host allocation failed");
  bool unsupported = false;
  std::string err;
  try {
    if (batch > 0)
      err = mg::build_batched_plan(p->hp, L, heads, d, window, batch, global_ptr, global_idx, extra_ptr, extra_idx, po,
                                   &unsupported);
    else
      err = mg::build_plan(p->hp, L, heads, d, window, global_idx, n_global, extra_idx, n_extra, po, &unsupported);
  } catch (const std::bad_alloc&) {
    delete p;
    return fail(MG_ERR_OUT_OF_MEMORY, "host allocation failed while building the plan");
  } catch (...) {
    delete p;
    return fail(MG_ERR_INTERNAL, "exception while building the plan");
  }
  if (!err.empty()) {
    delete p;
    return fail(unsupported ? MG_ERR_UNSUPPORTED : MG_ERR_INVALID_ARG, err);
  }
  p->num_sms_override = sms_override;
  p->fine_kernel = fine_kernel;
  p->concurrency = concurrency;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess) {
    ndev = 0;
    cudaGetLastError();
  }
  if (ndev > 0 && p->hp.kernel_ready) {
    const mg_status s = upload(p);
    if (s != MG_OK) {
      delete p;
      return s;
    }
  }
  *plan_out = p;
  return MG_OK;
}

mg_status check_tensor(const mg_tensor* t, const char* name, const mg_plan_s* p, bool host) {
  const std::string n(name);
  if (!t) return fail(MG_ERR_INVALID_ARG, n + " is null");
  if (!t->data) return fail(MG_ERR_INVALID_ARG, n + ".data is null");
  if (t->dtype != MG_BF16 && t->dtype != MG_FP16) return fail(MG_ERR_INVALID_ARG, n + ".dtype is not bf16/fp16");
  if (t->batch <= 0) return fail(MG_ERR_INVALID_ARG, n + ".batch must be > 0");
  if (t->heads != p->hp.heads) return fail(MG_ERR_INVALID_ARG, n + ".heads does not match the plan");
  if (t->seq_len != p->hp.L) return fail(MG_ERR_INVALID_ARG, n + ".seq_len does not match the plan");
  if (t->head_dim != p->hp.d) return fail(MG_ERR_INVALID_ARG, n + ".head_dim does not match the plan");
  if (t->stride_b < 0 || t->stride_h < 0 || t->stride_l < 0) return fail(MG_ERR_INVALID_ARG, n + ": negative stride");
  if ((t->stride_b % 8) || (t->stride_h % 8) || (t->stride_l % 8))
    return fail(MG_ERR_INVALID_ARG, n + ": strides must be multiples of 8 elements");
  if (reinterpret_cast<uintptr_t>(t->data) % 16) return fail(MG_ERR_INVALID_ARG, n + ".data must be 16-byte aligned");
  if (host) {
    // host tensors must be dense (either [B,H,L,d] or [B,L,H,d]) so they move as one span
    const int64_t total = t->batch * t->heads * t->seq_len * t->head_dim;
    const int64_t span = (t->batch - 1) * t->stride_b + (t->heads - 1) * t->stride_h +
                         (t->seq_len - 1) * t->stride_l + t->head_dim;
    if (span != total) return fail(MG_ERR_INVALID_ARG, n + ": host tensors must be dense");
  }
  return MG_OK;
}

mg_status check_all(const mg_plan_s* p, const mg_tensor* Q, const mg_tensor* K, const mg_tensor* V,
                    const mg_tensor* O, bool host) {
  mg_status s;
  if ((s = check_tensor(Q, "Q", p, host)) != MG_OK || (s = check_tensor(K, "K", p, host)) != MG_OK ||
      (s = check_tensor(V, "V", p, host)) != MG_OK || (s = check_tensor(O, "O", p, host)) != MG_OK)
    return s;
  if (K->batch != Q->batch || V->batch != Q->batch || O->batch != Q->batch)
    return fail(MG_ERR_INVALID_ARG, "Q/K/V/O batch sizes differ");
  if (K->dtype != Q->dtype || V->dtype != Q->dtype || O->dtype != Q->dtype)
    return fail(MG_ERR_UNSUPPORTED, "Q/K/V/O dtypes differ");
  if (p->hp.batch > 0 && Q->batch != p->hp.batch)
    return fail(MG_ERR_INVALID_ARG, "batch size differs from the batched plan's number of samples");
  if (!p->hp.kernel_ready) return fail(MG_ERR_UNSUPPORTED, "the forward requires block 64 or 128");
  if ((int64_t)Q->batch * p->hp.heads >=
      (int64_t(1) << 31) / std::max<int64_t>(1, (int64_t)std::max(p->hp.items.size(), p->hp.items_split.size())))
    return fail(MG_ERR_UNSUPPORTED, "batch * heads * work items exceeds int32");
  // the fine kernels address a gathered row as (uint32) col * stride_l elements
  if ((p->hp.L - 1) * std::max(K->stride_l, V->stride_l) >= (int64_t(1) << 32))
    return fail(MG_ERR_UNSUPPORTED, "(L - 1) * stride_l exceeds 2^32 elements");
  return MG_OK;
}

bool encode_map(CUtensorMap* m, const mg_tensor* t) {
  auto fn = tensor_map_encoder();
  if (!fn) return false;
  const int64_t s16 = 64;  // a harmless stride for extent-1 dimensions
  cuuint64_t dims[4] = {(cuuint64_t)t->head_dim, (cuuint64_t)t->seq_len, (cuuint64_t)t->heads, (cuuint64_t)t->batch};
  cuuint64_t strides[3] = {(cuuint64_t)std::max<int64_t>(t->stride_l, s16) * 2,
                           (cuuint64_t)std::max<int64_t>(t->stride_h, s16) * 2,
                           (cuuint64_t)std::max<int64_t>(t->stride_b, s16) * 2};
  cuuint32_t box[4] = {64, 128, 1, 1};
  cuuint32_t es[4] = {1, 1, 1, 1};
  const CUtensorMapDataType dt =
      t->dtype == MG_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16;
  const CUresult r = fn(m, dt, 4, t->data, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                        CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

// 2-D [rows, 64] view of a strided [B, H, L, d] tensor for TMA row gathers (tile::gather4, box
// 64 x 1) with a row stride of 64 elements; row(b, h, l) = b * r.x + h * r.y + l * r.z (+ 1 for the
// second 64 columns of a d = 128 row).
bool encode_map2d(CUtensorMap* m, const mg_tensor* t, longlong3* r) {
  auto fn = tensor_map_encoder();
  if (!fn) return false;
  auto gcd = [](int64_t a, int64_t b) {
    while (b) { const int64_t c = a % b; a = b; b = c; }
    return a;
  };
  // rows of 64 elements (a d = 128 row is two consecutive view rows): every stride must be a
  // multiple of 64 elements (true for dense [B,H,L,d] and [B,L,H,d])
  int64_t rs = 0;
  for (int64_t s : {t->stride_b, t->stride_h, t->stride_l})
    if (s > 0) rs = gcd(rs, s);
  if (rs <= 0 || rs % 64) return false;
  rs = 64;
  const int64_t span = (t->batch - 1) * t->stride_b + (t->heads - 1) * t->stride_h + (t->seq_len - 1) * t->stride_l + t->head_dim;
  const int64_t rows = (span + rs - 1) / rs;
  if (rows >= (int64_t(1) << 31)) return false;
  cuuint64_t dims[2] = {64, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)rs * 2};
  cuuint32_t box[2] = {64, 1};
  cuuint32_t es[2] = {1, 1};
  const CUtensorMapDataType dt =
      t->dtype == MG_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16;
  if (fn(m, dt, 2, t->data, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
         CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return false;
  *r = make_longlong3(t->stride_b / rs, t->stride_h / rs, t->stride_l / rs);
  return true;
}

mg::TensorView view(const mg_tensor* t) {
  return mg::TensorView{static_cast<uint16_t*>(t->data), t->stride_b, t->stride_h, t->stride_l};
}

// measured on B200: C4 serial vs concurrent
constexpr bool kConcurrentDefault = false;

// SM-split mode: coarse CTAs (one per SM) such that the coarse part takes about as long as the fine
// kernel would alone, from measured costs (C4): ~5,800 cycles per 128 x 128 tile for
// a coarse CTA sharing its SM with a fine block, ~6.4 cycles per CSR nnz and head per SM for the
// fine kernel. The environment variable MG_SPLIT_CTAS overrides it (A/B).
int coarse_split_ctas(const mg::HostPlan& h, int BH, int sms) {
  static const int env = [] {
    const char* e = std::getenv("MG_SPLIT_CTAS");
    return e ? std::atoi(e) : 0;
  }();
  if (env > 0) return env;
  int64_t tiles = 0;
  for (const mg::Item& it : h.items) tiles += it.ntiles;
  const double coarse_cta_cycles = (double)tiles * BH * 5800.0;
  const double fine_cycles = (double)h.fine_col.size() * BH * 6.4 / std::max(sms, 1);
  const int k = (int)std::ceil(coarse_cta_cycles / std::max(fine_cycles, 1.0));
  return std::max(1, std::min(k, sms));
}

mg_status fwd_impl(mg_plan_s* p, const mg_tensor* Q, const mg_tensor* K, const mg_tensor* V, mg_tensor* O,
                   cudaStream_t stream, const int32_t* valid_len = nullptr) {
  mg_status s = upload(p);
  if (s != MG_OK) return s;
  int dev = -1;
  cudaGetDevice(&dev);
  if (dev != p->device) return fail(MG_ERR_INVALID_ARG, "the plan was uploaded to another device");
  const mg::HostPlan& h = p->hp;
  const bool bf16 = Q->dtype == MG_BF16;
  // work units per item (and per fine row): every (b, h) of the batch, or for a batched plan (whose
  // items each belong to one sample) every head
  const int BH = (int)(h.batch > 0 ? h.heads : Q->batch * h.heads);
  const int nf = (int)h.fine_rows.size();
  const float scale_log2 = (float)(1.4426950408889634 / std::sqrt((double)h.d));
  cudaError_t e;
  // Concurrent coarse || fine (north_star item 5): chosen by measurement, only with
  // the tensor-core fine kernel and the paired-pipeline coarse kernel.
  const bool concurrent = nf > 0 && !h.items.empty() && p->fine_kernel == 0 &&
                          (p->concurrency >= 2 || (p->concurrency == 0 && kConcurrentDefault));
  // SM split (concurrency 3): the coarse kernel is launched first with a persistent grid of
  // coarse_split_ctas() CTAs (one per SM, beside which one fine block still fits), then the fine
  // kernel over the whole device with dynamically claimed rows, so its blocks that could not start
  // next to a coarse CTA take the remaining rows once that CTA leaves; rows with both parts merge as in
  // the concurrent mode
  const bool sm_split = concurrent && p->concurrency == 3;
  // fp32 partials of the CUDA-core CSR rows (fine -> coarse; and coarse -> fine plus one counter
  // per row when concurrent). Layout by capacity: [fine acc d][fine ml 2][coarse acc d][coarse ml 2]
  // floats per slot, then one int32 counter per slot (zeroed at allocation; even between forwards).
  const int D = h.d;
  const size_t need = ((size_t)BH * nf + 3) & ~size_t(3);   // multiple of 4: 16-byte aligned sections
  if (need > p->part_cap) {
    if (p->d_part) {
      if ((e = cudaFreeAsync(p->d_part, stream)) != cudaSuccess) return cuda_fail(e, "cudaFreeAsync");
      p->d_part = nullptr;
    }
    if ((e = cudaMallocAsync(reinterpret_cast<void**>(&p->d_part), need * (2 * D + 5) * sizeof(float), stream)) !=
        cudaSuccess)
      return e == cudaErrorMemoryAllocation ? fail(MG_ERR_OUT_OF_MEMORY, "workspace allocation failed")
                                            : cuda_fail(e, "cudaMallocAsync");
    if ((e = cudaMemsetAsync(p->d_part + need * (2 * D + 4), 0, need * sizeof(int32_t), stream)) != cudaSuccess)
      return cuda_fail(e, "cudaMemsetAsync");
    p->part_cap = need;
  }
  const size_t cap = p->part_cap;
  float* part_acc = p->d_part;
  float2* part_ml = reinterpret_cast<float2*>(p->d_part + cap * D);
  float* part_c_acc = p->d_part + cap * (D + 2);
  float2* part_c_ml = reinterpret_cast<float2*>(p->d_part + cap * (2 * D + 2));
  int32_t* part_flags = reinterpret_cast<int32_t*>(p->d_part + cap * (2 * D + 4));
  // split dense-row items (a work list with the global rows' column tiles in chunks): chosen when
  // the unsplit dense items would be few against the SMs (each would be a long serial chain), or
  // forced by the plan option; per (b*h, row group) chunk partials + chunk counters
  const bool use_split = h.dense_nsplit > 1 && h.n_dense_groups > 0 &&
                         (h.opts.dense_split == 2 ||
                          (h.opts.dense_split == 0 && (int64_t)h.n_dense_groups * BH * 2 <= p->num_sms));
  float* dense_part = nullptr;
  int32_t* dense_ctr = nullptr;
  if (use_split) {
    const size_t per_bh_part = (size_t)h.n_dense_groups * h.dense_nsplit * 128 * (D + 4) * sizeof(float);
    const size_t per_bh_ctr = (size_t)h.n_dense_groups * sizeof(int32_t);
    if ((size_t)BH > p->dense_cap) {
      if (p->d_dense) {
        if ((e = cudaFreeAsync(p->d_dense, stream)) != cudaSuccess) return cuda_fail(e, "cudaFreeAsync");
        p->d_dense = nullptr;
      }
      const size_t bytes = (size_t)BH * (per_bh_part + per_bh_ctr);
      if ((e = cudaMallocAsync(reinterpret_cast<void**>(&p->d_dense), bytes, stream)) != cudaSuccess)
        return e == cudaErrorMemoryAllocation ? fail(MG_ERR_OUT_OF_MEMORY, "workspace allocation failed")
                                              : cuda_fail(e, "cudaMallocAsync");
      if ((e = cudaMemsetAsync(p->d_dense + (size_t)BH * per_bh_part, 0, (size_t)BH * per_bh_ctr, stream)) != cudaSuccess)
        return cuda_fail(e, "cudaMemsetAsync");
      p->dense_cap = (size_t)BH;
    }
    dense_part = reinterpret_cast<float*>(p->d_dense);
    dense_ctr = reinterpret_cast<int32_t*>(p->d_dense + p->dense_cap * per_bh_part);
  }
  cudaStream_t fstream = stream;
  if (concurrent) {
    if (!p->side) {
      if ((e = cudaStreamCreateWithFlags(&p->side, cudaStreamNonBlocking)) != cudaSuccess ||
          (e = cudaEventCreateWithFlags(&p->fork_ev, cudaEventDisableTiming)) != cudaSuccess ||
          (e = cudaEventCreateWithFlags(&p->join_ev, cudaEventDisableTiming)) != cudaSuccess)
        return cuda_fail(e, "stream/event creation");
    }
    if ((e = cudaEventRecord(p->fork_ev, stream)) != cudaSuccess ||
        (e = cudaStreamWaitEvent(p->side, p->fork_ev, 0)) != cudaSuccess)
      return cuda_fail(e, "stream fork");
    fstream = p->side;
  }

  // profiling events (see mg_plan_s::ProfCall)
  const bool has_f = nf > 0, has_c = !h.items.empty();
  mg_plan_s::ProfCall pc{-1, -1, -1, -1, -1, -1};
  auto prof_rec = [&](cudaStream_t st) -> int32_t {
    cudaEvent_t ev = p->prof_event();
    if (!ev) return -1;
    cudaEventRecord(ev, st);
    return (int32_t)p->prof_used - 1;
  };
  if (p->profiling) {
    pc.first = prof_rec(stream);
    if (concurrent) cudaStreamWaitEvent(fstream, p->prof_events[pc.first], 0);
    if (has_f) pc.fb = pc.first;
    if (has_c && !has_f) pc.cb = pc.first;
  }
  // TMA descriptors of Q/K/V/O (re-encoded only when a tensor descriptor changes): the coarse kernel's
  // tiles and row gathers, the fine kernel's row gathers
  {
    mg_plan_s::Maps& mp = p->maps;
    if (!mp.valid || std::memcmp(&mp.q, Q, sizeof(mg_tensor)) || std::memcmp(&mp.k, K, sizeof(mg_tensor)) ||
        std::memcmp(&mp.v, V, sizeof(mg_tensor)) || std::memcmp(&mp.o, O, sizeof(mg_tensor))) {
      mp.q = *Q;
      mp.k = *K;
      mp.v = *V;
      mp.o = *O;
      mp.ok = encode_map(&mp.tq, Q) && encode_map(&mp.tk, K) && encode_map(&mp.tv, V);
      std::memset(&mp.tq2, 0, sizeof(CUtensorMap));
      std::memset(&mp.tk2, 0, sizeof(CUtensorMap));
      std::memset(&mp.tv2, 0, sizeof(CUtensorMap));
      std::memset(&mp.to, 0, sizeof(CUtensorMap));
      mp.gather_ok = encode_map2d(&mp.tq2, Q, &mp.rq) && encode_map2d(&mp.tk2, K, &mp.rk) &&
                     encode_map2d(&mp.tv2, V, &mp.rv);
      mp.store_ok = encode_map(&mp.to, O);
      mp.valid = true;
    }
  }
  auto launch_fine_part = [&]() -> mg_status {
  if (nf > 0) {
    mg::FineParams fp{};
    // Dynamic row chunks (two-head kernel): required by the SM split; otherwise when each warp of the
    // persistent grid has many rows (>= 64 head-pair rows per warp: C4 fine kernel 1.885 -> 1.850 ms),
    // while short row lists keep the static order (the start-up burst of claims on one counter costs
    // more than the balance gains: F9-RBR 0.072 vs 0.094 ms). MG_FINE_DYN=0/1 forces it (A/B).
    static const int fine_dyn_env = [] {
      const char* ev = std::getenv("MG_FINE_DYN");
      return ev ? std::atoi(ev) : -1;
    }();
    const int64_t rows2 = (int64_t)(BH / 2) * nf;
    const int64_t grid_warps = 4 * 3 * (int64_t)std::max(p->num_sms, 1);   // (two-head kernel: 3 blocks x 4 warps per SM)
    const bool dyn = sm_split || (fine_dyn_env < 0 ? rows2 >= 64 * grid_warps : fine_dyn_env == 1);
    fp.row_ctr = dyn ? p->d_counter + 2 : nullptr;
    fp.fine_rows = p->d_fine_rows;
    fp.row_ptr = p->d_fine_row_ptr;
    fp.cols = p->d_fine_col;
    fp.part_acc = part_acc;
    fp.part_ml = part_ml;
    fp.q = view(Q); fp.k = view(K); fp.v = view(V); fp.o = view(O);
    fp.H = h.heads; fp.BH = BH; fp.n_fine_rows = nf;
    fp.d = D;
    fp.fine_sample = h.batch > 0 ? p->d_fine_sample : nullptr;
    fp.scale_log2 = scale_log2;
    fp.concurrent = concurrent;
    fp.valid_len = valid_len;
    fp.part_c_acc = part_c_acc;
    fp.part_c_ml = part_c_ml;
    fp.part_flags = part_flags;
    // (the CUDA-core variant has no padding support: a padded forward always uses the MMA kernel)
    const int fsms = p->num_sms_override > 0 ? std::min(p->num_sms_override, p->num_sms) : p->num_sms;
    // (the CUDA-core variant takes d = 64 only: other forwards use the MMA kernel)
    // two heads per warp with TMA row gathers (tile::gather4): measured slower than the cp.async
    // gathers (C4 fine kernel 2.575 vs 1.887 ms), so only on request (MG_FINE_TMA=1, A/B)
    static const bool no_fine_tma = [] {
      const char* ev = std::getenv("MG_FINE_TMA");
      return !(ev && ev[0] == '1');
    }();
    const mg_plan_s::Maps& mp = p->maps;
    static const bool no_heads2 = [] {
      const char* ev = std::getenv("MG_FINE_HEADS2");
      return ev && ev[0] == '0';
    }();
    const bool fine_tma = !no_fine_tma && !no_heads2 && p->fine_kernel == 0 && D == 64 && (h.heads % 2) == 0 &&
                          mp.gather_ok;
    fp.rq = mp.rq;
    fp.rk = mp.rk;
    fp.rv = mp.rv;
    if (fine_tma)
      e = mg::launch_fine_tma2(fp, mp.tq2, mp.tk2, mp.tv2, bf16, fsms, fstream);
    else
      e = p->fine_kernel == 1 && !valid_len && D == 64 ? mg::launch_fine(fp, bf16, fstream)
                                                       : mg::launch_fine_mma(fp, bf16, fsms, fstream);
    if (e != cudaSuccess) return cuda_fail(e, "fine kernel launch");
  }
  if (p->profiling && has_f) {
    if (concurrent) {
      pc.fe = prof_rec(fstream);
      pc.cb = pc.first;
    } else if (has_c) {
      pc.fe = pc.cb = prof_rec(stream);
    }
  }
  return MG_OK;
  };
  auto launch_coarse_part = [&]() -> mg_status {
  if (!h.items.empty()) {
    mg_plan_s::Maps& mp = p->maps;
    if (!mp.ok)
      return fail(MG_ERR_CUDA, "cuTensorMapEncodeTiled failed (driver entry point unavailable or bad layout)");
    const CUtensorMap &tq = mp.tq, &tk = mp.tk, &tv = mp.tv;
    mg::CoarseParams cp{};
    cp.items = use_split ? p->d_items_split : p->d_items;
    cp.trefs = p->d_trefs;
    cp.masks = p->d_masks;
    cp.strip_cols = p->d_strip_cols;
    cp.global_rows = p->d_global_rows;
    cp.fine_slot = p->d_fine_slot;
    cp.part_acc = part_acc;
    cp.part_ml = part_ml;
    cp.counter = p->d_counter;
    cp.q = view(Q); cp.k = view(K); cp.v = view(V); cp.o = view(O);
    cp.L = h.L;
    cp.H = h.heads;
    cp.BH = BH;
    cp.d = D;
    cp.batched = h.batch > 0;
    cp.n_items = (int)(use_split ? h.items_split.size() : h.items.size());
    cp.n_dense_items = use_split ? h.n_dense_items_split : h.n_dense_items;
    cp.n_global = (int)h.global_rows.size();
    cp.n_fine_rows = nf;
    cp.total_units = cp.n_items * BH;
    cp.scale_log2 = scale_log2;
    cp.concurrent = concurrent;
    cp.valid_len = valid_len;
    cp.part_c_acc = part_c_acc;
    cp.part_c_ml = part_c_ml;
    cp.part_flags = part_flags;
    cp.dense_part = dense_part;
    cp.dense_ctr = dense_ctr;
    cp.n_dense_groups = h.n_dense_groups;
    cp.dense_nsplit = h.dense_nsplit;
    static const int dbg = [] {
      const char* e = std::getenv("MG_DEBUG_FLAGS");
      return e ? std::atoi(e) : 0;
    }();
    cp.debug_flags = dbg;
    cp.trace = p->trace;
    cp.trace_cap = p->trace_cap;
    // (the kernel resets its work counter itself: the last CTA to exit zeroes it)
    const int sms = p->num_sms_override > 0 ? std::min(p->num_sms_override, p->num_sms) : p->num_sms;
    {
      static const bool no_tma_gather = std::getenv("MG_NO_TMA_GATHER") != nullptr;   // A/B diagnostics
      cp.gather_tma = !no_tma_gather && mp.gather_ok;
      cp.rq = mp.rq;
      cp.rk = mp.rk;
      cp.rv = mp.rv;
      static const bool no_tma_store = std::getenv("MG_NO_TMA_STORE") != nullptr;   // A/B diagnostics
      cp.tma_store = !no_tma_store && mp.store_ok;
      // item-major band order in groups of at most 96 (b,h) units: C2's 96 heads' K/V windows stay in
      // L2 (C2 0.1419 -> 0.1375 ms); one group over C5's 768 heads re-reads K/V from DRAM (+7%)
      static const int group_env = [] {   // (A/B: MG_UNIT_GROUP=<heads per group>)
        const char* e = std::getenv("MG_UNIT_GROUP");
        return e ? std::atoi(e) : 0;
      }();
      cp.unit_group = mg::item_major_order() ? std::min(BH, group_env > 0 ? group_env : 96) : 0;
      const int grid = sm_split ? coarse_split_ctas(h, BH, sms) : mg::coarse_pp_ctas_per_sm(D) * sms;
      if ((e = mg::launch_coarse_pp(cp, tq, tk, tv, mp.tq2, mp.tk2, mp.tv2, mp.to, bf16, use_split,
                                    std::min(grid, cp.total_units), stream)) != cudaSuccess)
        return cuda_fail(e, "coarse kernel launch");
    }
  }
  if (p->profiling && concurrent) pc.ce = prof_rec(stream);
  return MG_OK;
  };
  if (sm_split) {
    if ((s = launch_coarse_part()) != MG_OK || (s = launch_fine_part()) != MG_OK) return s;
  } else {
    if ((s = launch_fine_part()) != MG_OK || (s = launch_coarse_part()) != MG_OK) return s;
  }
  if (concurrent) {
    if ((e = cudaEventRecord(p->join_ev, fstream)) != cudaSuccess ||
        (e = cudaStreamWaitEvent(stream, p->join_ev, 0)) != cudaSuccess)
      return cuda_fail(e, "stream join");
  }
  if (p->profiling) {
    pc.last = prof_rec(stream);
    if (has_f && pc.fe < 0) pc.fe = pc.last;
    if (has_c && pc.ce < 0) pc.ce = pc.last;
    if (pc.first < 0 || pc.last < 0) return fail(MG_ERR_CUDA, "cudaEventCreate failed");
    p->prof_calls.push_back(pc);
  }
  return MG_OK;
}


// ------------------------------------------------------------------ staged (paper dataflow) path
mg_status staged_upload(mg_plan_s* p) {
  mg_status s = upload(p);
  if (s != MG_OK) return s;
  if (p->staged_uploaded) return MG_OK;
  const mg::HostPlan& h = p->hp;
  std::vector<int32_t> tile_row(h.bsr_col.size());
  for (int64_t I = 0; I < h.nb(); ++I)
    for (int32_t t = h.bsr_row_ptr[I]; t < h.bsr_row_ptr[I + 1]; ++t) tile_row[t] = (int32_t)I;
  std::vector<uint8_t> is_g(h.L, 0);
  for (int32_t r : h.global_rows) is_g[r] = 1;
  cudaError_t e;
  if ((e = upload_vec(p, &p->d_bsr_row_ptr, h.bsr_row_ptr)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_bsr_col, h.bsr_col)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_tile_row, tile_row)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_tile_masks, h.tile_masks)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_csr_row_ptr, h.csr_row_ptr)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_csr_col, h.csr_col)) != cudaSuccess ||
      (e = upload_vec(p, &p->d_row_is_global, is_g)) != cudaSuccess)
    return e == cudaErrorMemoryAllocation ? fail(MG_ERR_OUT_OF_MEMORY, "device allocation failed")
                                          : cuda_fail(e, "staged plan upload");
  p->staged_uploaded = true;
  return MG_OK;
}

mg_staged_sizes staged_sizes(const mg::HostPlan& h) {
  mg_staged_sizes z;
  z.lpad = h.nb() * 128;
  z.tile_elems = (int64_t)h.bsr_col.size() * 128 * 128;
  z.csr_elems = (int64_t)h.csr_col.size();
  z.global_elems = (int64_t)h.global_rows.size() * z.lpad;
  z.ocsr_elems = h.L * 64;
  return z;
}

mg::StagedParams staged_params(const mg_plan_s* p, int64_t batch) {
  const mg::HostPlan& h = p->hp;
  mg::StagedParams sp{};
  sp.bsr_row_ptr = p->d_bsr_row_ptr;
  sp.bsr_col = p->d_bsr_col;
  sp.tile_row = p->d_tile_row;
  sp.tile_masks = p->d_tile_masks;
  sp.csr_row_ptr = p->d_csr_row_ptr;
  sp.csr_col = p->d_csr_col;
  sp.global_rows = p->d_global_rows;
  sp.row_is_global = p->d_row_is_global;
  sp.L = h.L;
  sp.nnz_csr = (int64_t)h.csr_col.size();
  sp.Lpad = h.nb() * 128;
  sp.H = h.heads;
  sp.BH = (int32_t)(batch * h.heads);
  sp.nb = (int32_t)h.nb();
  sp.n_tiles = (int32_t)h.bsr_col.size();
  sp.n_global = (int32_t)h.global_rows.size();
  sp.sf = (float)(1.0 / std::sqrt((double)h.d));
  return sp;
}

mg_status staged_check(mg_plan_s* p, const mg_tensor* t, const char* name) {
  mg_status s = check_tensor(t, name, p, false);
  if (s != MG_OK) return s;
  if (!p->hp.kernel_ready || p->hp.block != 128) return fail(MG_ERR_UNSUPPORTED, "the staged forward requires block == 128");
  if (p->hp.d != 64) return fail(MG_ERR_UNSUPPORTED, "the staged forward requires head_dim == 64");
  if (p->hp.batch > 0) return fail(MG_ERR_UNSUPPORTED, "the staged forward does not take batched plans");
  if ((int64_t)t->batch * p->hp.heads >= 65536) return fail(MG_ERR_UNSUPPORTED, "batch * heads must be < 65536");
  return staged_upload(p);
}

mg_status staged_buffers_ok(const mg_plan_s* p, const void* tiles, const void* csr, const void* glob) {
  const mg_staged_sizes z = staged_sizes(p->hp);
  if ((z.tile_elems && !tiles) || (z.csr_elems && !csr) || (z.global_elems && !glob))
    return fail(MG_ERR_INVALID_ARG, "a staged buffer of non-zero size is null");
  return MG_OK;
}

mg_status staged_sddmm_impl(mg_plan_s* p, const mg_tensor* Q, const mg_tensor* K, float* St, float* Sf, float* Sg,
                            cudaStream_t stream, cudaStream_t side) {
  mg::StagedParams sp = staged_params(p, Q->batch);
  sp.q = view(Q);
  sp.k = view(K);
  sp.S_t = St;
  sp.S_f = Sf;
  sp.S_g = Sg;
  cudaError_t e = mg::launch_staged_sddmm(sp, Q->dtype == MG_BF16, stream, side);
  return e == cudaSuccess ? MG_OK : cuda_fail(e, "staged SDDMM launch");
}

mg_status staged_softmax_impl(mg_plan_s* p, int64_t batch, mg_dtype dt, const float* St, const float* Sf,
                              const float* Sg, void* Pt, void* Pf, void* Pg, cudaStream_t stream) {
  mg::StagedParams sp = staged_params(p, batch);
  sp.S_t = const_cast<float*>(St);
  sp.S_f = const_cast<float*>(Sf);
  sp.S_g = const_cast<float*>(Sg);
  sp.P_t = static_cast<uint16_t*>(Pt);
  sp.P_f = static_cast<uint16_t*>(Pf);
  sp.P_g = static_cast<uint16_t*>(Pg);
  cudaError_t e = mg::launch_staged_softmax(sp, dt == MG_BF16, stream);
  return e == cudaSuccess ? MG_OK : cuda_fail(e, "staged SpSoftmax launch");
}

mg_status staged_spmm_impl(mg_plan_s* p, const void* Pt, const void* Pf, const void* Pg, const mg_tensor* V,
                           mg_tensor* O, float* Of, cudaStream_t stream, cudaStream_t side = nullptr) {
  mg::StagedParams sp = staged_params(p, V->batch);
  sp.v = view(V);
  sp.o = view(O);
  sp.P_t = static_cast<uint16_t*>(const_cast<void*>(Pt));
  sp.P_f = static_cast<uint16_t*>(const_cast<void*>(Pf));
  sp.P_g = static_cast<uint16_t*>(const_cast<void*>(Pg));
  sp.O_f = Of;
  cudaError_t e = mg::launch_staged_spmm(sp, V->dtype == MG_BF16, stream, side ? side : stream, p->staged_ev);
  return e == cudaSuccess ? MG_OK : cuda_fail(e, "staged SpMM launch");
}

}  // namespace

extern "C" {

int32_t mg_abi_version(void) { return MG_ABI_VERSION; }

const char* mg_last_error(void) { return g_err.c_str(); }

mg_status mg_plan_create(int64_t L, int32_t heads, int32_t d, int32_t window, const int32_t* global_idx,
                         int64_t n_global, const int32_t* extra_idx, int64_t n_extra, mg_plan_t* plan_out) {
  g_err.clear();
  return create_impl(L, heads, d, window, global_idx, n_global, extra_idx, n_extra, nullptr, plan_out);
}

mg_status mg_plan_create_ex(int64_t L, int32_t heads, int32_t d, int32_t window, const int32_t* global_idx,
                            int64_t n_global, const int32_t* extra_idx, int64_t n_extra, const mg_plan_opts* opts,
                            mg_plan_t* plan_out) {
  g_err.clear();
  return create_impl(L, heads, d, window, global_idx, n_global, extra_idx, n_extra, opts, plan_out);
}

mg_status mg_plan_create_batched(int64_t L, int32_t heads, int32_t d, int32_t window, int64_t batch,
                                 const int64_t* global_ptr, const int32_t* global_idx, const int64_t* extra_ptr,
                                 const int32_t* extra_idx, const mg_plan_opts* opts, mg_plan_t* plan_out) {
  g_err.clear();
  if (batch <= 0) return fail(MG_ERR_INVALID_ARG, "batch must be > 0");
  if (!global_ptr || !extra_ptr) return fail(MG_ERR_INVALID_ARG, "global_ptr / extra_ptr is null");
  return create_impl(L, heads, d, window, global_idx, 0, extra_idx, 0, opts, plan_out, batch, global_ptr, extra_ptr);
}

mg_status mg_plan_destroy(mg_plan_t plan) {
  g_err.clear();
  delete plan;
  return MG_OK;
}

mg_status mg_plan_info_get(mg_plan_t plan, mg_plan_info* info) {
  g_err.clear();
  if (!plan || !info) return fail(MG_ERR_INVALID_ARG, "null argument");
  const mg::HostPlan& h = plan->hp;
  std::memset(info, 0, sizeof(*info));
  info->L = h.L;
  info->heads = h.heads;
  info->d = h.d;
  info->window = h.window;
  info->block = h.block;
  info->n_row_blocks = h.nb();
  info->n_tiles = (int64_t)h.bsr_col.size();
  info->n_full_tiles = h.n_full_tiles;
  info->nnz_coarse = h.nnz_coarse;
  info->nnz_fine = (int64_t)h.csr_col.size();
  info->n_global = (int64_t)h.global_rows.size();
  info->nnz_total = h.nnz_coarse + info->nnz_fine + info->n_global * h.L;
  info->n_fine_rows = (int64_t)h.fine_rows.size();
  info->nnz_fine_strip = h.nnz_fine_strip;
  info->nnz_fine_cuda = (int64_t)h.fine_col.size();
  info->n_items = (int64_t)h.items.size();
  info->n_strip_tiles = h.n_strip_tiles;
  info->computed_scores = h.computed_scores;
  info->kernels_per_fwd = (h.fine_rows.empty() ? 0 : 1) + (h.items.empty() ? 0 : 1);
  return MG_OK;
}

mg_status mg_plan_export(mg_plan_t plan, int32_t* bsr_row_ptr, int32_t* bsr_col, uint64_t* tile_masks,
                         int32_t* csr_row_ptr, int32_t* csr_col, int32_t* global_rows) {
  g_err.clear();
  if (!plan) return fail(MG_ERR_INVALID_ARG, "plan is null");
  const mg::HostPlan& h = plan->hp;
  if (h.batch > 0) return fail(MG_ERR_UNSUPPORTED, "mg_plan_export: batched plans have one partition per sample");
  auto cp = [](auto* dst, const auto& v) {
    if (dst && !v.empty()) std::memcpy(dst, v.data(), v.size() * sizeof(v[0]));
  };
  cp(bsr_row_ptr, h.bsr_row_ptr);
  cp(bsr_col, h.bsr_col);
  cp(tile_masks, h.tile_masks);
  cp(csr_row_ptr, h.csr_row_ptr);
  cp(csr_col, h.csr_col);
  cp(global_rows, h.global_rows);
  return MG_OK;
}

mg_status mg_sparse_attention_fwd(mg_plan_t plan, const mg_tensor* Q, const mg_tensor* K, const mg_tensor* V,
                                  mg_tensor* O, void* stream) {
  g_err.clear();
  if (!plan) return fail(MG_ERR_INVALID_ARG, "plan is null");
  mg_status s = check_all(plan, Q, K, V, O, false);
  if (s != MG_OK) return s;
  return fwd_impl(plan, Q, K, V, O, static_cast<cudaStream_t>(stream));
}

mg_status mg_sparse_attention_fwd_padded(mg_plan_t plan, const mg_tensor* Q, const mg_tensor* K, const mg_tensor* V,
                                         mg_tensor* O, const int32_t* valid_len, void* stream) {
  g_err.clear();
  if (!plan) return fail(MG_ERR_INVALID_ARG, "plan is null");
  if (!valid_len) return fail(MG_ERR_INVALID_ARG, "valid_len is null");
  mg_status s = check_all(plan, Q, K, V, O, false);
  if (s != MG_OK) return s;
  return fwd_impl(plan, Q, K, V, O, static_cast<cudaStream_t>(stream), valid_len);
}

mg_status mg_sparse_attention_fwd_host(mg_plan_t plan, const mg_tensor* Q, const mg_tensor* K, const mg_tensor* V,
                                       mg_tensor* O, void* stream_) {
  g_err.clear();
  if (!plan) return fail(MG_ERR_INVALID_ARG, "plan is null");
  mg_status s = check_all(plan, Q, K, V, O, true);
  if (s != MG_OK) return s;
  if ((s = upload(plan)) != MG_OK) return s;
  cudaStream_t stream = static_cast<cudaStream_t>(stream_);
  const size_t bytes = (size_t)Q->batch * Q->heads * Q->seq_len * Q->head_dim * 2;
  cudaError_t e;
  if (4 * bytes > plan->stage_cap) {
    if (plan->d_stage) {
      if ((e = cudaFreeAsync(plan->d_stage, stream)) != cudaSuccess) return cuda_fail(e, "cudaFreeAsync");
      plan->d_stage = nullptr;
    }
    if ((e = cudaMallocAsync(reinterpret_cast<void**>(&plan->d_stage), 4 * bytes, stream)) != cudaSuccess)
      return e == cudaErrorMemoryAllocation ? fail(MG_ERR_OUT_OF_MEMORY, "staging allocation failed")
                                            : cuda_fail(e, "cudaMallocAsync");
    plan->stage_cap = 4 * bytes;
  }
  // Pipelined over batch chunks: the H2D copies of chunk c+1 (h2d stream) and the D2H copy of chunk
  // c-1 (d2h stream) overlap the forward of chunk c (`stream`); host tensors are dense, so a batch
  // chunk is one contiguous range of each. Batched plans (one pattern per sample) run as one chunk.
  const int64_t B = Q->batch;
  // a batch chunk is one contiguous byte range of every tensor only when the batch is the outermost
  // dimension of each (dense [B,H,L,d] or [B,L,H,d]); any other dense layout moves as one span
  bool batch_outer = true;
  for (const mg_tensor* t : {Q, K, V, static_cast<const mg_tensor*>(O)})
    batch_outer = batch_outer && t->stride_b == t->heads * t->seq_len * t->head_dim;
  const int64_t nchunk = (plan->hp.batch > 0 || !batch_outer) ? 1 : std::min<int64_t>(B, 8);
  const size_t per_b = bytes / (size_t)B;
  uint8_t* dst[4] = {plan->d_stage, plan->d_stage + bytes, plan->d_stage + 2 * bytes, plan->d_stage + 3 * bytes};
  const uint8_t* src[3] = {static_cast<const uint8_t*>(Q->data), static_cast<const uint8_t*>(K->data),
                           static_cast<const uint8_t*>(V->data)};
  if (!plan->h2d) {
    if ((e = cudaStreamCreateWithFlags(&plan->h2d, cudaStreamNonBlocking)) != cudaSuccess ||
        (e = cudaStreamCreateWithFlags(&plan->d2h, cudaStreamNonBlocking)) != cudaSuccess)
      return cuda_fail(e, "stream creation");
  }
  cudaEvent_t ev_start = plan->host_event(0), ev_end = plan->host_event(1);
  if (!ev_start || !ev_end || !plan->host_event(2 + 2 * nchunk)) return fail(MG_ERR_CUDA, "event creation failed");
  if ((e = cudaEventRecord(ev_start, stream)) != cudaSuccess ||
      (e = cudaStreamWaitEvent(plan->h2d, ev_start, 0)) != cudaSuccess ||
      (e = cudaStreamWaitEvent(plan->d2h, ev_start, 0)) != cudaSuccess)
    return cuda_fail(e, "stream fork");
  // every return after the fork joins the copy streams back into `stream` first, so that a caller
  // who synchronises `stream` after an error may free the pinned buffers the copies read
  auto join = [&]() {
    cudaEventRecord(ev_end, plan->h2d);
    cudaStreamWaitEvent(stream, ev_end, 0);
    cudaEventRecord(ev_end, plan->d2h);
    cudaStreamWaitEvent(stream, ev_end, 0);
  };
  auto fail_joined = [&](mg_status st) {
    const std::string msg = g_err;
    join();
    g_err = msg;
    return st;
  };
  for (int64_t c = 0; c < nchunk; ++c) {
    const int64_t b0 = B * c / nchunk, b1 = B * (c + 1) / nchunk;
    const size_t off = (size_t)b0 * per_b, len = (size_t)(b1 - b0) * per_b;
    cudaEvent_t ev_in = plan->host_event(2 + 2 * c), ev_done = plan->host_event(3 + 2 * c);
    for (int i = 0; i < 3; ++i)
      if ((e = cudaMemcpyAsync(dst[i] + off, src[i] + off, len, cudaMemcpyHostToDevice, plan->h2d)) != cudaSuccess)
        return fail_joined(cuda_fail(e, "H2D copy"));
    if ((e = cudaEventRecord(ev_in, plan->h2d)) != cudaSuccess || (e = cudaStreamWaitEvent(stream, ev_in, 0)) != cudaSuccess)
      return fail_joined(cuda_fail(e, "event"));
    mg_tensor dq = *Q, dk = *K, dv = *V, dO = *O;
    dq.data = dst[0] + off;
    dk.data = dst[1] + off;
    dv.data = dst[2] + off;
    dO.data = dst[3] + off;
    dq.batch = dk.batch = dv.batch = dO.batch = b1 - b0;
    if ((s = fwd_impl(plan, &dq, &dk, &dv, &dO, stream)) != MG_OK) return fail_joined(s);
    if ((e = cudaEventRecord(ev_done, stream)) != cudaSuccess || (e = cudaStreamWaitEvent(plan->d2h, ev_done, 0)) != cudaSuccess)
      return fail_joined(cuda_fail(e, "event"));
    if ((e = cudaMemcpyAsync(static_cast<uint8_t*>(O->data) + off, dst[3] + off, len, cudaMemcpyDeviceToHost,
                             plan->d2h)) != cudaSuccess)
      return fail_joined(cuda_fail(e, "D2H copy"));
  }
  if ((e = cudaEventRecord(ev_end, plan->h2d)) != cudaSuccess || (e = cudaStreamWaitEvent(stream, ev_end, 0)) != cudaSuccess ||
      (e = cudaEventRecord(ev_end, plan->d2h)) != cudaSuccess || (e = cudaStreamWaitEvent(stream, ev_end, 0)) != cudaSuccess)
    return cuda_fail(e, "stream join");
  return MG_OK;
}


mg_status mg_staged_get_sizes(mg_plan_t plan, mg_staged_sizes* out) {
  g_err.clear();
  if (!plan || !out) return fail(MG_ERR_INVALID_ARG, "null argument");
  *out = staged_sizes(plan->hp);
  return MG_OK;
}

mg_status mg_staged_sddmm(mg_plan_t plan, const mg_tensor* Q, const mg_tensor* K, float* S_tiles, float* S_csr,
                          float* S_global, void* stream) {
  g_err.clear();
  if (!plan) return fail(MG_ERR_INVALID_ARG, "plan is null");
  mg_status s;
  if ((s = staged_check(plan, Q, "Q")) != MG_OK || (s = staged_check(plan, K, "K")) != MG_OK) return s;
  if (K->batch != Q->batch || K->dtype != Q->dtype) return fail(MG_ERR_INVALID_ARG, "Q/K batch or dtype differ");
  if ((s = staged_buffers_ok(plan, S_tiles, S_csr, S_global)) != MG_OK) return s;
  return staged_sddmm_impl(plan, Q, K, S_tiles, S_csr, S_global, static_cast<cudaStream_t>(stream),
                           static_cast<cudaStream_t>(stream));
}

mg_status mg_staged_softmax(mg_plan_t plan, int64_t batch, mg_dtype dtype, const float* S_tiles, const float* S_csr,
                            const float* S_global, void* P_tiles, void* P_csr, void* P_global, void* stream) {
  g_err.clear();
  if (!plan) return fail(MG_ERR_INVALID_ARG, "plan is null");
  if (batch <= 0) return fail(MG_ERR_INVALID_ARG, "batch must be > 0");
  if (dtype != MG_BF16 && dtype != MG_FP16) return fail(MG_ERR_INVALID_ARG, "dtype is not bf16/fp16");
  if (!plan->hp.kernel_ready || plan->hp.block != 128) return fail(MG_ERR_UNSUPPORTED, "the staged forward requires block == 128");
  if (plan->hp.d != 64) return fail(MG_ERR_UNSUPPORTED, "the staged forward requires head_dim == 64");
  if (plan->hp.batch > 0) return fail(MG_ERR_UNSUPPORTED, "the staged forward does not take batched plans");
  mg_status s;
  if ((s = staged_upload(plan)) != MG_OK) return s;
  if ((s = staged_buffers_ok(plan, S_tiles, S_csr, S_global)) != MG_OK ||
      (s = staged_buffers_ok(plan, P_tiles, P_csr, P_global)) != MG_OK)
    return s;
  return staged_softmax_impl(plan, batch, dtype, S_tiles, S_csr, S_global, P_tiles, P_csr, P_global,
                             static_cast<cudaStream_t>(stream));
}

mg_status mg_staged_spmm(mg_plan_t plan, const void* P_tiles, const void* P_csr, const void* P_global,
                         const mg_tensor* V, mg_tensor* O, float* O_csr, void* stream) {
  g_err.clear();
  if (!plan) return fail(MG_ERR_INVALID_ARG, "plan is null");
  mg_status s;
  if ((s = staged_check(plan, V, "V")) != MG_OK || (s = staged_check(plan, O, "O")) != MG_OK) return s;
  if (O->batch != V->batch || O->dtype != V->dtype) return fail(MG_ERR_INVALID_ARG, "V/O batch or dtype differ");
  if ((s = staged_buffers_ok(plan, P_tiles, P_csr, P_global)) != MG_OK) return s;
  if (!plan->hp.csr_col.empty() && !O_csr) return fail(MG_ERR_INVALID_ARG, "O_csr is null");
  return staged_spmm_impl(plan, P_tiles, P_csr, P_global, V, O, O_csr, static_cast<cudaStream_t>(stream));
}

mg_status mg_sparse_attention_fwd_staged_ex(mg_plan_t plan, const mg_tensor* Q, const mg_tensor* K, const mg_tensor* V,
                                            mg_tensor* O, int32_t flags, void* stream_) {
  g_err.clear();
  if (flags & ~MG_STAGED_MULTI_STREAM) return fail(MG_ERR_INVALID_ARG, "unknown staged flags");
  if (!plan) return fail(MG_ERR_INVALID_ARG, "plan is null");
  mg_status s = check_all(plan, Q, K, V, O, false);
  if (s != MG_OK) return s;
  if ((s = staged_check(plan, Q, "Q")) != MG_OK) return s;
  cudaStream_t stream = static_cast<cudaStream_t>(stream_);
  const mg_staged_sizes z = staged_sizes(plan->hp);
  const size_t BH = (size_t)Q->batch * plan->hp.heads;
  auto al = [](size_t b) { return (b + 255) & ~size_t(255); };
  const size_t bt = al(BH * z.tile_elems * 4), bf = al(BH * z.csr_elems * 4), bg = al(BH * z.global_elems * 4);
  const size_t pt = al(BH * z.tile_elems * 2), pf = al(BH * z.csr_elems * 2), pg = al(BH * z.global_elems * 2);
  const size_t bo = al(BH * z.ocsr_elems * 4);
  const size_t need = bt + bf + bg + pt + pf + pg + bo;
  cudaError_t e;
  if (need > plan->staged_ws_cap) {
    if (plan->d_staged_ws) {
      if ((e = cudaFreeAsync(plan->d_staged_ws, stream)) != cudaSuccess) return cuda_fail(e, "cudaFreeAsync");
      plan->d_staged_ws = nullptr;
    }
    if ((e = cudaMallocAsync(reinterpret_cast<void**>(&plan->d_staged_ws), need, stream)) != cudaSuccess)
      return e == cudaErrorMemoryAllocation ? fail(MG_ERR_OUT_OF_MEMORY, "staged workspace allocation failed")
                                            : cuda_fail(e, "cudaMallocAsync");
    plan->staged_ws_cap = need;
  }
  uint8_t* w = plan->d_staged_ws;
  float* St = reinterpret_cast<float*>(w);
  float* Sf = reinterpret_cast<float*>(w + bt);
  float* Sg = reinterpret_cast<float*>(w + bt + bf);
  void* Pt = w + bt + bf + bg;
  void* Pf = w + bt + bf + bg + pt;
  void* Pg = w + bt + bf + bg + pt + pf;
  float* Of = reinterpret_cast<float*>(w + bt + bf + bg + pt + pf + pg);
  cudaStream_t side = stream;
  const bool multi = (flags & MG_STAGED_MULTI_STREAM) && !plan->hp.csr_col.empty();
  if (multi) {
    if (!plan->staged_side) {
      if ((e = cudaStreamCreateWithFlags(&plan->staged_side, cudaStreamNonBlocking)) != cudaSuccess)
        return cuda_fail(e, "stream creation");
    }
    side = plan->staged_side;
  }
  if (!plan->staged_ev && (e = cudaEventCreateWithFlags(&plan->staged_ev, cudaEventDisableTiming)) != cudaSuccess)
    return cuda_fail(e, "event creation");
  // fork: the side stream starts after everything before this call on `stream`
  auto sync_into = [&](cudaStream_t from, cudaStream_t to) {
    cudaError_t r = cudaEventRecord(plan->staged_ev, from);
    return r == cudaSuccess ? cudaStreamWaitEvent(to, plan->staged_ev, 0) : r;
  };
  if (multi && (e = sync_into(stream, side)) != cudaSuccess) return cuda_fail(e, "stream fork");
  if ((s = staged_sddmm_impl(plan, Q, K, St, Sf, Sg, stream, side)) != MG_OK) return s;
  if (multi && (e = sync_into(side, stream)) != cudaSuccess) return cuda_fail(e, "stream join");
  if ((s = staged_softmax_impl(plan, Q->batch, (mg_dtype)Q->dtype, St, Sf, Sg, Pt, Pf, Pg, stream)) != MG_OK) return s;
  if (multi && (e = sync_into(stream, side)) != cudaSuccess) return cuda_fail(e, "stream fork");
  // (launch_staged_spmm joins the side stream back before the row blocks that read O_csr)
  return staged_spmm_impl(plan, Pt, Pf, Pg, V, O, Of, stream, side);
}

mg_status mg_sparse_attention_fwd_staged(mg_plan_t plan, const mg_tensor* Q, const mg_tensor* K, const mg_tensor* V,
                                         mg_tensor* O, void* stream) {
  return mg_sparse_attention_fwd_staged_ex(plan, Q, K, V, O, 0, stream);
}

mg_status mg_plan_autotune(int64_t L, int32_t heads, int32_t d, int32_t window, const int32_t* global_idx,
                           int64_t n_global, const int32_t* extra_idx, int64_t n_extra, const mg_tensor* Q,
                           const mg_tensor* K, const mg_tensor* V, mg_tensor* O, void* stream_, mg_plan_t* plan_out,
                           mg_plan_opts* chosen, double* best_ms) {
  g_err.clear();
  if (!plan_out) return fail(MG_ERR_INVALID_ARG, "plan_out is null");
  *plan_out = nullptr;
  cudaStream_t stream = static_cast<cudaStream_t>(stream_);
  cudaEvent_t ev[2] = {nullptr, nullptr};
  cudaError_t e;
  if ((e = cudaEventCreate(&ev[0])) != cudaSuccess || (e = cudaEventCreate(&ev[1])) != cudaSuccess) {
    if (ev[0]) cudaEventDestroy(ev[0]);
    return cuda_fail(e, "cudaEventCreate");
  }
  mg_plan_t best = nullptr;
  mg_plan_opts best_opts{};
  double best_t = 0.0;
  mg_status status = MG_OK;
  const int32_t blocks[2] = {128, 64};
  const float taus[4] = {0.f, 0.1f, 0.25f, 0.5f};
  for (int32_t b : blocks) {
    for (float tau : taus) {
      mg_plan_opts o{};
      o.block = b;
      o.tau = tau;
      mg_plan_t cand = nullptr;
      mg_status s = create_impl(L, heads, d, window, global_idx, n_global, extra_idx, n_extra, &o, &cand);
      if (s == MG_OK) s = check_all(cand, Q, K, V, O, false);
      std::vector<float> ts;
      for (int i = 0; i < 7 && s == MG_OK; ++i) {
        if (cudaEventRecord(ev[0], stream) != cudaSuccess) s = fail(MG_ERR_CUDA, "cudaEventRecord");
        if (s == MG_OK) s = fwd_impl(cand, Q, K, V, O, stream);
        if (s == MG_OK && (e = cudaEventRecord(ev[1], stream)) != cudaSuccess) s = cuda_fail(e, "cudaEventRecord");
        if (s == MG_OK && (e = cudaEventSynchronize(ev[1])) != cudaSuccess) s = cuda_fail(e, "cudaEventSynchronize");
        float ms = 0.f;
        if (s == MG_OK && i >= 2) {
          cudaEventElapsedTime(&ms, ev[0], ev[1]);
          ts.push_back(ms);
        }
      }
      if (s != MG_OK) {
        delete cand;
        if (best) delete best;
        best = nullptr;
        status = s;
        break;
      }
      std::sort(ts.begin(), ts.end());
      const double med = ts[ts.size() / 2];
      if (!best || med < best_t) {
        if (best) delete best;
        best = cand;
        best_t = med;
        best_opts = o;
      } else {
        delete cand;
      }
    }
    if (status != MG_OK) break;
  }
  cudaEventDestroy(ev[0]);
  cudaEventDestroy(ev[1]);
  if (status != MG_OK) return status;
  *plan_out = best;
  if (chosen) *chosen = best_opts;
  if (best_ms) *best_ms = best_t;
  return MG_OK;
}

mg_status mg_plan_set_profiling(mg_plan_t plan, int32_t enable) {
  g_err.clear();
  if (!plan) return fail(MG_ERR_INVALID_ARG, "plan is null");
  plan->profiling = enable != 0;
  plan->prof_used = 0;
  plan->prof_calls.clear();
  return MG_OK;
}

mg_status mg_plan_get_profile_calls(mg_plan_t plan, mg_profile* out, double* per_call_ms, int64_t cap) {
  g_err.clear();
  if (!plan || !out) return fail(MG_ERR_INVALID_ARG, "null argument");
  if (cap < 0 || (cap > 0 && !per_call_ms)) return fail(MG_ERR_INVALID_ARG, "bad per-call buffer");
  std::memset(out, 0, sizeof(*out));
  auto ms = [&](int32_t a, int32_t b) {
    float t = 0.f;
    if (a >= 0 && b >= 0) cudaEventElapsedTime(&t, plan->prof_events[a], plan->prof_events[b]);
    return (double)t;
  };
  int64_t i = 0;
  for (const auto& c : plan->prof_calls) {
    cudaError_t e = cudaEventSynchronize(plan->prof_events[c.last]);
    if (e != cudaSuccess) return cuda_fail(e, "cudaEventSynchronize");
    out->fine_ms += ms(c.fb, c.fe);
    out->coarse_ms += ms(c.cb, c.ce);
    const double tot = ms(c.first, c.last);
    out->total_ms += tot;
    if (i < cap) per_call_ms[i] = tot;
    ++i;
  }
  out->calls = (int64_t)plan->prof_calls.size();
  plan->prof_used = 0;
  plan->prof_calls.clear();
  return MG_OK;
}

mg_status mg_plan_get_profile(mg_plan_t plan, mg_profile* out) {
  return mg_plan_get_profile_calls(plan, out, nullptr, 0);
}

mg_status mg_plan_set_trace(mg_plan_t plan, void* device_buffer, int64_t capacity_events) {
  g_err.clear();
  if (!plan || (device_buffer == nullptr) != (capacity_events == 0) ||
      (device_buffer != nullptr && capacity_events < 128) || capacity_events > (int64_t(1) << 30))
    return fail(MG_ERR_INVALID_ARG, "bad trace buffer");
  plan->trace = static_cast<unsigned long long*>(device_buffer);
  plan->trace_cap = (int32_t)capacity_events;
  return MG_OK;
}

mg_status mg_selftest_umma(int32_t mode, const void* A, const void* B, float* D, void* stream) {
  g_err.clear();
  if (!A || !B || !D || (mode != 0 && mode != 1)) return fail(MG_ERR_INVALID_ARG, "bad selftest arguments");
  const cudaError_t e = mg::launch_selftest_umma(mode, A, B, D, static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? MG_OK : cuda_fail(e, "selftest launch");
}

}  // extern "C"
