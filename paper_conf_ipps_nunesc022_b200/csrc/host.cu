// host.cu -- the C ABI of include/csmv.h: device memory, launches, stats.
//
// Every transaction step runs in the fused kernel (kernel.cu); the host only
// allocates, initialises, launches and copies results.  Nothing here falls
// back to the CPU: without an sm_100a device csmv_create fails.  The one
// host-side computation is the zipf CDF (setup); the KV preload runs on the
// device (launch_kv_preload).
#include <cuda_runtime.h>

#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/csmv.h"
#include "kernel.cuh"

using namespace csmvd;

namespace {

thread_local char g_err[512] = "";

int set_err(int code, const char* fmt, ...) __attribute__((format(printf, 2, 3)));
int set_err(int code, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof g_err, fmt, ap);
  va_end(ap);
  return code;
}

#define CK(call)                                                                                 \
  do {                                                                                           \
    cudaError_t e_ = (call);                                                                     \
    if (e_ != cudaSuccess)                                                                       \
      return set_err(CSMV_ECUDA, "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__); \
  } while (0)

// zipf CDF (docs/GENERATOR.md section 2), built on the host in IEEE double
std::vector<uint64_t> build_zipf(uint32_t n, uint32_t theta_milli) {
  std::vector<uint64_t> cdf(n);
  const double theta = (double)theta_milli / 1000.0;
  double h = 0.0;
  for (uint32_t r = 1; r <= n; ++r) h += std::pow((double)r, -theta);
  double s = 0.0;
  for (uint32_t i = 0; i < n; ++i) {
    s += std::pow((double)(i + 1), -theta);
    const double x = std::ldexp(s / h, 64);
    cdf[i] = (x >= 18446744073709551616.0) ? UINT64_MAX : (uint64_t)x;
  }
  cdf[n - 1] = UINT64_MAX;
  return cdf;
}

uint32_t nslot_for(uint32_t k) { return k <= 2 ? 2 : k <= 4 ? 4 : k <= 8 ? 8 : 16; }

}  // namespace

struct csmv {
  int kind = CSMV_KIND_BANK;
  uint64_t n_items = 0;  // bank: accounts; KV: all items (3S + T)
  uint32_t K = 0, nslot = 0;
  int device = 0, sm_count = 0;
  cudaStream_t stream = nullptr;
  bool loaded = false;
  // bank store
  uint64_t* d_rings = nullptr;
  int32_t* d_init = nullptr;  // csmv_load staging (allocated once: no pool growth inside a timed load)
  // KV store
  uint32_t kv_S = 0, kv_A = 0, kv_T = 0, kv_keys = 0;
  uint32_t* d_kvstage = nullptr;  // csmv_load_kv staging + scratch (kept: no allocation inside a timed load)
  size_t kvstage_bytes = 0;
  uint64_t *d_key = nullptr, *d_val = nullptr, *d_lru = nullptr, *d_clk = nullptr;
  // shared
  uint32_t* d_lastw = nullptr;
  uint32_t* d_gts = nullptr;
  Ctl* d_ctl = nullptr;
  DevStats* d_stats = nullptr;
  uint32_t* d_done = nullptr;
  // per-client-warp message slots, sized for the full grid
  uint32_t max_cw = 0, maxid = 2;
  uint32_t* d_req_seq = nullptr;
  ReqHdr* d_req_hdr = nullptr;
  uint32_t* d_req_ids = nullptr;
  uint32_t* d_req_cnt = nullptr;
  Resp* d_resp = nullptr;
  uint32_t* d_req_vals = nullptr;  // CSMV_COMMIT_ONLYCS (bank)
  // CSMV_SERVER_PART message slots (allocated on first use): 8 servers x max_cw
  uint32_t *d_mreq_seq = nullptr, *d_mdec_seq = nullptr, *d_mdack = nullptr;
  Resp* d_mresp = nullptr;
  uint64_t* d_mdec = nullptr;
  uint64_t* d_jv_ws = nullptr;     // CSMV_COMMIT_JVSTM global ATR (allocated on first use)
  csmv_trace_rec* d_trace = nullptr;  // CSMV_DBG_TRACE (allocated on first use)
  bool last_traced = false;
  uint32_t* d_jv_tag = nullptr;
  uint32_t* d_tk = nullptr;  // CSMV_RETRY_FIFO: u32 next[T] + u64 serving[T] (allocated on first use)
  // logs
  csmv_log_rec* d_log = nullptr;
  uint64_t log_cap = 0;
  uint32_t* d_vals = nullptr;
  uint64_t vals_cap = 0;
  uint64_t last_n_tx = 0;
  uint32_t last_log_mode = 0, last_max_vals = 0;
  // zipf table cache
  uint64_t* d_zipf = nullptr;
  uint32_t zipf_n = 0, zipf_theta = 0;

  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  csmv_stats_t last{};
};

static void free_all(csmv* h) {
  void* ps[] = {h->d_rings, h->d_key, h->d_val, h->d_lru, h->d_clk, h->d_lastw, h->d_gts, h->d_ctl,
                h->d_stats, h->d_done, h->d_req_seq, h->d_req_hdr, h->d_req_ids, h->d_req_cnt,
                h->d_resp, h->d_log, h->d_vals, h->d_zipf, h->d_req_vals, h->d_jv_ws, h->d_jv_tag, h->d_init,
                h->d_kvstage, h->d_trace, h->d_mreq_seq, h->d_mdec_seq, h->d_mdack, h->d_mresp, h->d_mdec, h->d_tk};
  for (void* q : ps) cudaFree(q);
  if (h->ev0) cudaEventDestroy(h->ev0);
  if (h->ev1) cudaEventDestroy(h->ev1);
}

extern "C" {

int csmv_abi_version(void) { return CSMV_ABI_VERSION; }

const char* csmv_last_error(void) { return g_err; }

static int device_check(int* dev, int* sms) {
  int n = 0;
  cudaError_t e = cudaGetDeviceCount(&n);
  if (e != cudaSuccess || n == 0)
    return set_err(CSMV_ECUDA, "no CUDA device (%s); there is no CPU fallback",
                   e == cudaSuccess ? "0 devices" : cudaGetErrorString(e));
  CK(cudaGetDevice(dev));
  cudaDeviceProp pr;
  CK(cudaGetDeviceProperties(&pr, *dev));
  if (pr.major != 10 || pr.minor != 0)
    return set_err(CSMV_ECUDA, "device %s is sm_%d%d; this library is built for sm_100a only", pr.name,
                   pr.major, pr.minor);
  if (!pr.cooperativeLaunch) return set_err(CSMV_ECUDA, "device lacks cooperative launch");
  *sms = pr.multiProcessorCount;
  return CSMV_OK;
}

// allocations common to both store kinds
static bool alloc_common(csmv* h) {
  h->max_cw = (uint32_t)(h->sm_count - 1) * kWarps;
  if (cudaMalloc(&h->d_lastw, h->n_items * sizeof(uint32_t)) != cudaSuccess) return false;
  if (cudaMalloc(&h->d_gts, 64) != cudaSuccess) return false;
  if (cudaMalloc(&h->d_ctl, sizeof(Ctl)) != cudaSuccess) return false;
  if (cudaMalloc(&h->d_stats, sizeof(DevStats)) != cudaSuccess) return false;
  if (cudaMalloc(&h->d_done, sizeof(uint32_t) << kDoneLog2) != cudaSuccess) return false;
  if (cudaMalloc(&h->d_req_seq, h->max_cw * sizeof(uint32_t)) != cudaSuccess) return false;
  if (cudaMalloc(&h->d_req_hdr, h->max_cw * sizeof(ReqHdr)) != cudaSuccess) return false;
  if (cudaMalloc(&h->d_req_ids, (size_t)h->max_cw * h->maxid * 32 * sizeof(uint32_t)) != cudaSuccess) return false;
  if (cudaMalloc(&h->d_req_cnt, (size_t)h->max_cw * 32 * sizeof(uint32_t)) != cudaSuccess) return false;
  if (cudaMalloc(&h->d_resp, h->max_cw * sizeof(Resp)) != cudaSuccess) return false;
  cudaMemset(h->d_done, 0, sizeof(uint32_t) << kDoneLog2);
  cudaMemset(h->d_gts, 0, 64);
  cudaMemset(h->d_lastw, 0, h->n_items * sizeof(uint32_t));
  cudaEventCreate(&h->ev0);
  cudaEventCreate(&h->ev1);
  return cudaDeviceSynchronize() == cudaSuccess;
}

static csmv_t* create_fail(csmv* h, const char* what) {
  set_err(CSMV_ENOMEM, "csmv_create: allocation of %s failed (%s)", what, cudaGetErrorString(cudaGetLastError()));
  free_all(h);
  delete h;
  return nullptr;
}

csmv_t* csmv_create(uint64_t n_items, uint32_t n_versions) {
  g_err[0] = 0;
  if (n_items < 2 || n_items >= (1ull << 31) || n_versions < 1 || n_versions > 16) {
    set_err(CSMV_EINVAL, "csmv_create: need 2 <= n_items < 2^31 and 1 <= n_versions <= 16");
    return nullptr;
  }
  int dev = 0, sms = 0;
  if (device_check(&dev, &sms) != CSMV_OK) return nullptr;
  csmv* h = new csmv();
  h->kind = CSMV_KIND_BANK;
  h->n_items = n_items;
  h->K = n_versions;
  h->nslot = nslot_for(n_versions);
  h->device = dev;
  h->sm_count = sms;
  h->maxid = 2;
  if (cudaMalloc(&h->d_rings, n_items * h->nslot * sizeof(uint64_t)) != cudaSuccess) return create_fail(h, "rings");
  if (cudaMalloc(&h->d_init, n_items * sizeof(int32_t)) != cudaSuccess) return create_fail(h, "init staging");
  if (!alloc_common(h)) return create_fail(h, "control buffers");
  if (cudaMalloc(&h->d_req_vals, (size_t)h->max_cw * 128 * sizeof(uint32_t)) != cudaSuccess)
    return create_fail(h, "request values");
  return h;
}

csmv_t* csmv_create_kv(uint64_t n_slots, uint32_t ways, uint32_t n_versions) {
  g_err[0] = 0;
  if (ways < 1 || ways > kKvMaxWays || n_slots < ways || n_slots % ways || n_slots >= (1ull << 29) ||
      n_versions < 1 || n_versions > 16) {
    set_err(CSMV_EINVAL, "csmv_create_kv: need 1 <= ways <= %u, n_slots a multiple of ways below 2^29, "
                         "1 <= n_versions <= 16", kKvMaxWays);
    return nullptr;
  }
  int dev = 0, sms = 0;
  if (device_check(&dev, &sms) != CSMV_OK) return nullptr;
  csmv* h = new csmv();
  h->kind = CSMV_KIND_KV;
  h->kv_S = (uint32_t)n_slots;
  h->kv_A = ways;
  h->kv_T = (uint32_t)(n_slots / ways);
  h->n_items = 3ull * h->kv_S + h->kv_T;
  h->K = n_versions;
  h->nslot = nslot_for(n_versions);
  h->device = dev;
  h->sm_count = sms;
  h->maxid = kKvMaxId;
  const size_t S = h->kv_S, T = h->kv_T, NS = h->nslot;
  if (cudaMalloc(&h->d_key, S * NS * 4 * 8) != cudaSuccess) return create_fail(h, "key rings");
  if (cudaMalloc(&h->d_val, S * NS * 8 * 8) != cudaSuccess) return create_fail(h, "value rings");
  if (cudaMalloc(&h->d_lru, S * NS * 8) != cudaSuccess) return create_fail(h, "LRU rings");
  if (cudaMalloc(&h->d_clk, T * NS * 8) != cudaSuccess) return create_fail(h, "clock rings");
  if (!alloc_common(h)) return create_fail(h, "control buffers");
  return h;
}

void csmv_destroy(csmv_t* h) {
  if (!h) return;
  cudaStreamSynchronize(h->stream);
  free_all(h);
  delete h;
}

int csmv_set_stream(csmv_t* h, void* s) {
  if (!h) return set_err(CSMV_EINVAL, "null handle");
  h->stream = (cudaStream_t)s;
  return CSMV_OK;
}

int csmv_load(csmv_t* h, const int32_t* init, uint64_t n) {
  if (!h || !init) return set_err(CSMV_EINVAL, "csmv_load: null argument");
  if (h->kind != CSMV_KIND_BANK) return set_err(CSMV_EINVAL, "csmv_load: not a bank store");
  if (n != h->n_items)
    return set_err(CSMV_EINVAL, "csmv_load: n=%llu != n_items=%llu", (unsigned long long)n,
                   (unsigned long long)h->n_items);
  int32_t* d_init = h->d_init;
  CK(cudaMemcpyAsync(d_init, init, n * sizeof(int32_t), cudaMemcpyHostToDevice, h->stream));
  CK(launch_init_rings(h->d_rings, h->nslot, d_init, n, h->d_gts, h->stream));
  CK(cudaMemsetAsync(h->d_lastw, 0, n * sizeof(uint32_t), h->stream));
  // CTS restart at 1: stale done flags of an earlier run would publish GTS early
  CK(cudaMemsetAsync(h->d_done, 0, sizeof(uint32_t) << kDoneLog2, h->stream));
  CK(cudaStreamSynchronize(h->stream));
  h->loaded = true;
  return CSMV_OK;
}

static KParams kv_params(const csmv* h) {
  KParams p;
  memset(&p, 0, sizeof p);
  p.kind = CSMV_KIND_KV;
  p.K = h->K;
  p.gts = h->d_gts;
  p.kv_S = h->kv_S;
  p.kv_A = h->kv_A;
  p.kv_T = h->kv_T;
  p.kv_key = h->d_key;
  p.kv_val = h->d_val;
  p.kv_lru = h->d_lru;
  p.kv_clk = h->d_clk;
  return p;
}

int csmv_load_kv(csmv_t* h, uint64_t n_keys) {
  if (!h) return set_err(CSMV_EINVAL, "csmv_load_kv: null handle");
  if (h->kind != CSMV_KIND_KV) return set_err(CSMV_EINVAL, "csmv_load_kv: not a KV store");
  if (n_keys == 0 || n_keys >= (1ull << 32)) return set_err(CSMV_EINVAL, "csmv_load_kv: bad n_keys");
  const uint32_t S = h->kv_S, A = h->kv_A, T = h->kv_T;
  // PUT semantics per key, in key order (docs/GENERATOR.md 4), computed on
  // the device: a set's r-th insertion takes way r mod A (launch_kv_preload).
  uint32_t* d = nullptr;
  const size_t words = (size_t)S * 13 + T;
  const size_t scratch_words = 3 * (size_t)T + n_keys;
  size_t cub_bytes = 0;
  cudaError_t e = launch_kv_preload((uint32_t)n_keys, T, A, nullptr, nullptr, &cub_bytes, nullptr, nullptr, nullptr,
                                    nullptr, h->stream);
  if (e != cudaSuccess) return set_err(CSMV_ECUDA, "csmv_load_kv: %s", cudaGetErrorString(e));
  const size_t need = (words + scratch_words) * 4 + cub_bytes;
  if (h->kvstage_bytes < need) {
    cudaFree(h->d_kvstage);
    h->d_kvstage = nullptr;
    h->kvstage_bytes = 0;
    CK(cudaMalloc(&h->d_kvstage, need));
    h->kvstage_bytes = need;
  }
  d = h->d_kvstage;
  uint32_t* scratch = d + words;
  e = cudaMemsetAsync(d, 0, words * 4, h->stream);
  if (e == cudaSuccess)
    e = launch_kv_preload((uint32_t)n_keys, T, A, scratch, scratch + scratch_words, &cub_bytes, d,
                          d + (size_t)S * 4, d + (size_t)S * 12, d + (size_t)S * 13, h->stream);
  if (e == cudaSuccess)
    e = launch_init_kv(kv_params(h), h->nslot, d, d + (size_t)S * 4, d + (size_t)S * 12, d + (size_t)S * 13,
                       h->stream);
  if (e == cudaSuccess) e = cudaMemsetAsync(h->d_lastw, 0, h->n_items * 4, h->stream);
  if (e == cudaSuccess) e = cudaMemsetAsync(h->d_done, 0, sizeof(uint32_t) << kDoneLog2, h->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  if (e != cudaSuccess) return set_err(CSMV_ECUDA, "csmv_load_kv: %s", cudaGetErrorString(e));
  h->kv_keys = (uint32_t)n_keys;
  h->loaded = true;
  return CSMV_OK;
}

// guide buckets of the zipf search: 2^log2 with 2^log2 >= n, at most 2^22
static uint32_t zipf_guide_log2(uint32_t n) {
  uint32_t l = 0;
  while ((1u << l) < n && l < 22) ++l;
  return l;
}

static int prepare_zipf(csmv* h, uint32_t n, uint32_t theta) {
  if (h->d_zipf && h->zipf_n == n && h->zipf_theta == theta) return CSMV_OK;
  cudaFree(h->d_zipf);
  h->d_zipf = nullptr;
  std::vector<uint64_t> cdf = build_zipf(n, theta);
  // guide table (the cutpoint method): g[b] = pick(b * 2^(64-m)) for the
  // 2^m buckets of u plus g[2^m] = n-1, so that a pick in bucket b lies in
  // [g[b], g[b+1]] -- the same upper_bound, over a few entries instead of
  // all n (gen.cuh zipf_pick)
  const uint32_t m = zipf_guide_log2(n);
  std::vector<uint32_t> guide(((size_t)1 << m) + 1);
  uint32_t i = 0;
  for (uint64_t b = 0; b < ((uint64_t)1 << m); ++b) {
    const uint64_t u = m ? b << (64 - m) : 0;
    while (i < n - 1 && cdf[i] <= u) ++i;
    guide[b] = i;
  }
  guide[(size_t)1 << m] = n - 1;
  const size_t cb = (size_t)n * sizeof(uint64_t), gb = guide.size() * sizeof(uint32_t);
  CK(cudaMalloc(&h->d_zipf, cb + gb));
  CK(cudaMemcpy(h->d_zipf, cdf.data(), cb, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(reinterpret_cast<uint8_t*>(h->d_zipf) + cb, guide.data(), gb, cudaMemcpyHostToDevice));
  h->zipf_n = n;
  h->zipf_theta = theta;
  return CSMV_OK;
}

static int make_gen(csmv* h, const csmv_workload* w, uint64_t seed, GenParams* g) {
  memset(g, 0, sizeof *g);
  g->seed = seed;
  g->upd_thresh = ((uint64_t)w->p_update_ppm << 32) / 1000000ull;
  g->ro_period = w->ro_period;
  g->ro_reads = w->ro_reads;
  g->amount_max = w->amount_max;
  if (h->kind == CSMV_KIND_KV) {
    g->n_items = w->kv_keys ? w->kv_keys : h->kv_S;  // picks range over the key space
    g->ro_period = 0;
  } else {
    g->n_items = (uint32_t)h->n_items;
  }
  if (w->dist == CSMV_DIST_ZIPF) {
    int rc = prepare_zipf(h, g->n_items, w->zipf_theta_milli);
    if (rc) return rc;
    g->zipf_cdf = h->d_zipf;
    g->zipf_guide = reinterpret_cast<const uint32_t*>(h->d_zipf + g->n_items);
    g->guide_log2 = zipf_guide_log2(g->n_items);
  } else if (w->dist != CSMV_DIST_UNIFORM) {
    return set_err(CSMV_EINVAL, "unknown dist %u", w->dist);
  }
  return CSMV_OK;
}

int csmv_run(csmv_t* h, const csmv_workload* w, uint64_t n_tx, uint64_t seed) {
  if (!h || !w) return set_err(CSMV_EINVAL, "csmv_run: null argument");
  if (!h->loaded) return set_err(CSMV_ESTATE, "csmv_run: store not loaded");
  if (w->kind != (uint32_t)h->kind) return set_err(CSMV_EINVAL, "csmv_run: workload kind does not match the store");
  if (h->kind == CSMV_KIND_BANK && w->amount_max == 0) return set_err(CSMV_EINVAL, "csmv_run: amount_max must be >= 1");
  if (h->kind == CSMV_KIND_KV && w->log_mode == CSMV_LOG_FULL)
    return set_err(CSMV_EINVAL, "csmv_run: the KV workload logs digests only (use CSMV_LOG_DIGEST)");
  if (h->kind == CSMV_KIND_KV && w->kv_ways && w->kv_ways != h->kv_A)
    return set_err(CSMV_EINVAL, "csmv_run: kv_ways %u does not match the store's %u", w->kv_ways, h->kv_A);
  if (w->p_update_ppm > 1000000) return set_err(CSMV_EINVAL, "csmv_run: p_update_ppm > 10^6");
  if (w->log_mode > CSMV_LOG_FULL || w->publish > CSMV_PUBLISH_SERVER)
    return set_err(CSMV_EINVAL, "csmv_run: bad log_mode/publish");
  if (w->atr_mode > CSMV_ATR_LIST_NOCV) return set_err(CSMV_EINVAL, "csmv_run: unknown atr_mode %u", w->atr_mode);
  if (w->atr_mode != CSMV_ATR_HASH && (h->kind != CSMV_KIND_BANK || w->server != CSMV_SERVER_CTA))
    return set_err(CSMV_EINVAL, "csmv_run: the list ATR is built for the bank workload on the single-CTA server");
  if (n_tx >= (1ull << 32)) return set_err(CSMV_EINVAL, "csmv_run: n_tx must be < 2^32");
  // blind-write elision is safe only without blind writes: a bank
  // transfer reads both accounts it writes (RS = WS, so the validated
  // read-set already is RS u WS); a KV PUT writes its value (and, on a key
  // match or empty way, its LRU stamp) without reading it
  if (w->elide_ww > 1) return set_err(CSMV_EINVAL, "csmv_run: elide_ww must be 0 or 1");
  if (w->elide_ww && h->kind == CSMV_KIND_KV)
    return set_err(CSMV_EINVAL, "csmv_run: elide_ww refused: KV PUTs write blindly (value, LRU), so the "
                                "write-write check of P:115 cannot be omitted");
  if (w->retry_order > CSMV_RETRY_FIFO) return set_err(CSMV_EINVAL, "csmv_run: unknown retry_order %u", w->retry_order);
  if (w->retry_order == CSMV_RETRY_FIFO && h->kind != CSMV_KIND_KV)
    return set_err(CSMV_EINVAL, "csmv_run: CSMV_RETRY_FIFO is built for the KV workload (one set per PUT)");
  if (w->commit > CSMV_COMMIT_JVSTM) return set_err(CSMV_EINVAL, "csmv_run: unknown commit %u", w->commit);
  const bool jvstm = w->commit == CSMV_COMMIT_JVSTM;
  if (w->commit != CSMV_COMMIT_CSMV && (h->kind != CSMV_KIND_BANK || w->server != CSMV_SERVER_CTA))
    return set_err(CSMV_EINVAL, "csmv_run: the onlyCS / JVSTM-GPU ablations are built for the bank workload "
                                "with the single-CTA server setting");
  if (jvstm && !h->d_jv_ws) {
    CK(cudaMalloc(&h->d_jv_ws, sizeof(uint64_t) << kJvLog2));
    CK(cudaMalloc(&h->d_jv_tag, sizeof(uint32_t) << kJvLog2));
  }

  uint32_t gts0 = 0;
  CK(cudaMemcpyAsync(&gts0, h->d_gts, 4, cudaMemcpyDeviceToHost, h->stream));
  CK(cudaStreamSynchronize(h->stream));
  if ((uint64_t)gts0 + n_tx >= 0xFFFFFFFEull)
    return set_err(CSMV_EOVERFLOW, "csmv_run: timestamp space exhausted (GTS %u); reload", gts0);

  KParams p;
  memset(&p, 0, sizeof p);
  int rc = make_gen(h, w, seed, &p.gen);
  if (rc) return rc;

  // server: one CTA, a thread-block cluster of C CTAs (DSMEM), or
  // none (JVSTM-GPU: every CTA is a client)
  uint32_t n_srv = jvstm ? 0u : 1u, clog2 = 0, part_log2 = 0;
  const bool part = w->server == CSMV_SERVER_PART;
  if (part) {  // item-partitioned servers (server_part.cuh): S independent server CTAs
    n_srv = w->cluster_size ? w->cluster_size : 2u;
    if (n_srv < 2 || n_srv > 8 || (n_srv & (n_srv - 1)))
      return set_err(CSMV_EINVAL, "csmv_run: CSMV_SERVER_PART needs cluster_size (servers) = 2, 4 or 8");
    if (h->kind != CSMV_KIND_BANK || w->atr_mode != CSMV_ATR_HASH || w->commit != CSMV_COMMIT_CSMV ||
        (w->client_group && w->client_group != 1) || (w->debug_flags & CSMV_DBG_ALT_COMMIT))
      return set_err(CSMV_EINVAL, "csmv_run: CSMV_SERVER_PART is built for the bank workload with per-warp "
                                  "batches (atr_mode HASH, CSMV commit)");
    while ((1u << part_log2) < n_srv) ++part_log2;
  } else if (w->server == CSMV_SERVER_CLUSTER) {
    n_srv = w->cluster_size ? w->cluster_size : 16u;
    if (n_srv < 2 || n_srv > 16 || (n_srv & (n_srv - 1)))
      return set_err(CSMV_EINVAL, "csmv_run: cluster_size must be 2, 4, 8 or 16");
    while ((1u << clog2) < n_srv) ++clog2;
  } else if (w->server != CSMV_SERVER_CTA) {
    return set_err(CSMV_EINVAL, "csmv_run: unknown server kind %u", w->server);
  }
  // server CTA: warp 0 receiver, warps 1..n_workers workers, last warp publisher
  // (the last warp hosts the publisher unless it runs on a client CTA or the
  // clients publish: then it can be a 7th worker -- clamped below)
  uint32_t n_workers = w->server_workers ? w->server_workers : 4u;
  if (n_workers > kWarps - 1) n_workers = kWarps - 1;
  // bank + filter: the last warp of CTA 0 is the committer (server.cuh commit ring)
  const bool cmring = h->kind == CSMV_KIND_BANK && w->atr_mode == CSMV_ATR_HASH && w->commit == CSMV_COMMIT_CSMV &&
                      ((w->server == CSMV_SERVER_CLUSTER) != ((w->debug_flags & CSMV_DBG_ALT_COMMIT) != 0));
  if (cmring && n_workers > kWarps - 3) n_workers = kWarps - 3;
  // bank, one CTA, locked commit: self-receiving workers (no receiver warp)
  if (w->server_recv > CSMV_RECV_SELF) return set_err(CSMV_EINVAL, "csmv_run: unknown server_recv %u", w->server_recv);
  const bool kv_filt = h->kind == CSMV_KIND_KV && (h->kv_A > kKvFullWays || !(w->debug_flags & CSMV_DBG_KV_ITEMSETS));
  const bool selfrecv = w->server_recv == CSMV_RECV_SELF && w->server == CSMV_SERVER_CTA &&
                        (h->kind == CSMV_KIND_BANK ? w->atr_mode == CSMV_ATR_HASH && w->commit == CSMV_COMMIT_CSMV &&
                                                         !(w->debug_flags & CSMV_DBG_ALT_COMMIT)
                                                   : kv_filt);
  if (selfrecv) {  // warps 0..n_workers-1 workers, warp n_workers the publisher
    n_workers = w->server_workers ? w->server_workers : 4u;
    if (n_workers > kWarps - 1) n_workers = kWarps - 1;
  }
  // CTA-level batches: G client warps of one CTA per request
  const uint32_t group = w->client_group ? w->client_group : 1u;
  if (group != 1 && group != 2 && group != 4 && group != 8)
    return set_err(CSMV_EINVAL, "csmv_run: client_group must be 1, 2, 4 or 8");
  if (group > 1 && (h->kind != CSMV_KIND_BANK || w->atr_mode != CSMV_ATR_HASH || w->commit != CSMV_COMMIT_CSMV ||
                    selfrecv || (cmring && group > 4) || (!cmring && w->server != CSMV_SERVER_CTA)))
    return set_err(CSMV_EINVAL, "csmv_run: client_group > 1 needs the bank workload (atr_mode HASH, CSMV "
                                "commit) on the ticket-locked single-CTA server with a receiver warp (G = 2/4/8) "
                                "or on a commit ring (cluster server; G = 2/4)");
  uint32_t n_cw = w->client_warps ? w->client_warps : h->max_cw;
  if (n_cw > h->max_cw) n_cw = h->max_cw;
  if (n_cw == 0) return set_err(CSMV_EINVAL, "csmv_run: no client warps");

  // recent-commit table: 4 entries per bucket, striped over the server CTAs
  // (default 16384 entries = 144 KB per server CTA)
  uint32_t entries = w->atr_capacity ? w->atr_capacity : 16384u * n_srv;
  uint32_t rt_log2 = clog2 + 1;
  while ((4u << rt_log2) < entries && rt_log2 < 12 + clog2) ++rt_log2;
  // bank + CSMV_ATR_HASH reads the same smem as a recent-write filter of
  // 8 << rt_log2 slots (server.cuh); below ~1K slots a window of a few
  // batches saturates it and nearly every update would abort OVERFLOW
  const bool filt = h->kind == CSMV_KIND_BANK ? w->atr_mode == CSMV_ATR_HASH
                                              : (h->kv_A > kKvFullWays || !(w->debug_flags & CSMV_DBG_KV_ITEMSETS));
  if (filt && rt_log2 < 7 + clog2) rt_log2 = 7 + clog2;
  // cluster + commit ring: CTA 0 runs only the committer and the publisher,
  // CTAs 1..C-1 receive (server.cuh server_cta)
  const uint32_t n_serve = (cmring && n_srv > 1) ? n_srv - 1 : n_srv;
  const uint32_t per_srv = n_serve ? (n_cw + n_serve - 1) / n_serve : 0u;
  const uint32_t ring_log2 = cm_ring_log2(group, cmring);
  // eviction watermarks: only the KV item-set table (server_worker_generic) uses them
  const uint32_t ev_log2 = (h->kind == CSMV_KIND_KV && !filt) ? rt_log2 - clog2 : 2u;  // 16 B keeps what follows aligned
  // A/B knob (default off): keep the locked single-CTA bank server's 16-bit
  // filter under CSMV_FILT_TRIM_KB of shared memory in all, with a
  // non-power-of-two slot count, so that every SM's allocation (taken from
  // its unified L1) stays below a carveout step.  Measured neutral at 132 KB
  // (C2 527-537 vs 529-539 M tx/s, profiles/r02/raw/r02ai_ab_trim.jsonl),
  // unlike dropping the unused commit ring (+12 %).
#ifndef CSMV_FILT_TRIM_KB
#define CSMV_FILT_TRIM_KB 0
#endif
  uint32_t filt16_n = 0;
  const bool lock_filter = h->kind == CSMV_KIND_BANK && filt && n_srv == 1 && !cmring && w->commit == CSMV_COMMIT_CSMV;
  if (lock_filter && CSMV_FILT_TRIM_KB) {
    const size_t full = server_smem_bytes(rt_log2 - clog2, per_srv, ring_log2, ev_log2);
    const size_t other = full - (size_t)8 * rt_region_words(rt_log2 - clog2, 0);
    const size_t cap = (size_t)CSMV_FILT_TRIM_KB * 1024;
    if (full > cap && cap > other + 32768) filt16_n = (uint32_t)(((cap - other) / 2) & ~(size_t)255);
  }
  size_t smem = part ? part_smem_bytes(n_cw, part_bits_log2(h->n_items, part_log2)) : server_smem_bytes(rt_log2 - clog2, per_srv, ring_log2, ev_log2, filt16_n);
  if (h->kind == CSMV_KIND_KV && smem < kv_client_smem_bytes()) smem = kv_client_smem_bytes();
  if (smem > 227 * 1024) return set_err(CSMV_EINVAL, "csmv_run: ATR capacity too large for smem");

  // grid: server CTAs first, then client CTAs (client warps spread round-robin)
  p.kind = (uint32_t)h->kind;
  p.n_server_ctas = n_srv;
  p.clustered = w->server == CSMV_SERVER_CLUSTER;
  int cap = 0;
  CK(fused_capacity(p, h->nslot, smem, &cap));
  if (cap < (int)n_srv + (int)n_srv)
    return set_err(CSMV_ECUDA, "csmv_run: fused kernel cannot be resident (smem %zu, %d CTAs)", smem, cap);
  uint32_t max_client_ctas = (uint32_t)cap - n_srv;
  if (max_client_ctas > (uint32_t)h->sm_count - n_srv) max_client_ctas = (uint32_t)h->sm_count - n_srv;
  if (n_cw > max_client_ctas * kWarps) n_cw = max_client_ctas * kWarps;
  uint32_t n_ctas = n_cw < max_client_ctas ? n_cw : max_client_ctas;
  if (p.clustered) n_ctas = (n_ctas + n_srv - 1) / n_srv * n_srv;  // grid a multiple of the cluster
  if (p.clustered && n_ctas > max_client_ctas) n_ctas = max_client_ctas / n_srv * n_srv;
  if (n_ctas == 0) return set_err(CSMV_EINVAL, "csmv_run: no client CTA fits beside the server");
  // client warp cw runs on CTA cw mod n_ctas, warp cw / n_ctas: never more than the grid holds
  if (n_cw > n_ctas * kWarps) n_cw = n_ctas * kWarps;

  // logs
  uint32_t max_vals = 0;
  if (w->log_mode != CSMV_LOG_NONE) {
    if (n_tx > h->log_cap || !h->d_log) {
      cudaFree(h->d_log);
      h->d_log = nullptr;
      CK(cudaMalloc(&h->d_log, (n_tx ? n_tx : 1) * sizeof(csmv_log_rec)));
      h->log_cap = n_tx;
    }
    CK(cudaMemsetAsync(h->d_log, 0, n_tx * sizeof(csmv_log_rec), h->stream));
    if (w->log_mode == CSMV_LOG_FULL) {
      max_vals = w->ro_reads ? w->ro_reads : (uint32_t)h->n_items;
      if (max_vals < 2) max_vals = 2;
      const uint64_t words = n_tx * (uint64_t)max_vals;
      if (words > h->vals_cap || !h->d_vals) {
        cudaFree(h->d_vals);
        h->d_vals = nullptr;
        CK(cudaMalloc(&h->d_vals, (words ? words : 1) * sizeof(uint32_t)));
        h->vals_cap = words;
      }
      CK(cudaMemsetAsync(h->d_vals, 0, words * sizeof(uint32_t), h->stream));
    }
  }

  if (h->kind == CSMV_KIND_KV) {
    p = [&] {
      KParams q = kv_params(h);
      q.gen = p.gen;
      return q;
    }();
  }
  p.kind = (uint32_t)h->kind;
  p.rings = h->d_rings;
  p.n_items = (uint32_t)h->n_items;
  p.K = h->K;
  p.gts = h->d_gts;
  p.ctl = h->d_ctl;
  p.req_seq = h->d_req_seq;
  p.req_hdr = h->d_req_hdr;
  p.req_ids = h->d_req_ids;
  p.req_cnt = h->d_req_cnt;
  p.maxid = h->maxid;
  p.resp = h->d_resp;
  p.done_ring = h->d_done;
  p.stats = h->d_stats;
  p.log = h->d_log;
  p.vals = h->d_vals;
  p.max_vals = max_vals;
  p.log_mode = w->log_mode;
  p.n_tx = n_tx;
  p.n_cw = n_cw;
  p.n_client_ctas = n_ctas;
  p.n_server_ctas = n_srv;
  p.clog2 = clog2;
  p.clustered = w->server == CSMV_SERVER_CLUSTER;
  p.part_log2 = part_log2;
  p.part_bits_log2 = part ? part_bits_log2(h->n_items, part_log2) : 0u;
  if (part) {
    const size_t m = (size_t)8 * h->max_cw;
    if (!h->d_mreq_seq) {
      CK(cudaMalloc(&h->d_mreq_seq, m * 4));
      CK(cudaMalloc(&h->d_mdec_seq, m * 4));
      CK(cudaMalloc(&h->d_mdack, m * 4));
      CK(cudaMalloc(&h->d_mresp, m * sizeof(Resp)));
      CK(cudaMalloc(&h->d_mdec, (size_t)h->max_cw * 16));
    }
    CK(cudaMemsetAsync(h->d_mreq_seq, 0, m * 4, h->stream));
    CK(cudaMemsetAsync(h->d_mdec_seq, 0, m * 4, h->stream));
    CK(cudaMemsetAsync(h->d_mdack, 0, m * 4, h->stream));
    CK(cudaMemsetAsync(h->d_mresp, 0, m * sizeof(Resp), h->stream));
    CK(cudaMemsetAsync(h->d_mdec, 0, (size_t)h->max_cw * 16, h->stream));
    p.mstride = h->max_cw;
    p.mreq_seq = h->d_mreq_seq;
    p.mdec_seq = h->d_mdec_seq;
    p.mdack = h->d_mdack;
    p.mresp = h->d_mresp;
    p.mdec = h->d_mdec;
  }
  p.n_workers = n_workers;
  p.rt_log2 = rt_log2;
  p.lastw = h->d_lastw;
  p.publish = w->publish;
  p.ro_streak = w->ro_streak;
  p.combine = w->server_combine ? w->server_combine : 1u;
  p.atr_mode = w->atr_mode;
  p.backoff_max = w->backoff_max;
  p.debug = w->debug_flags;
  p.commit = w->commit;
  p.ro_adaptive = w->ro_adaptive;
  p.server_recv = w->server_recv;
  p.group = group;
  p.cm_ring_log2 = ring_log2;
  p.ev_log2 = ev_log2;
  p.filt16_n = filt16_n;
  p.gts_start = gts0;
  // round-tagged requests (ReqHdr, no client fence before the doorbell) on
  // the commit paths that check the tags: the self-receiving bank worker
  // (ticket-locked single CTA) and the KV filter workers
  {
    const uint64_t max_id = h->kind == CSMV_KIND_KV ? 3ull * h->kv_S + h->kv_T : h->n_items;
    const bool bank_lock = h->kind == CSMV_KIND_BANK && selfrecv;  // the self-receiving bank worker
    if (w->req_tagged > 1) return set_err(CSMV_EINVAL, "csmv_run: req_tagged must be 0 or 1");
    if (w->server_writeback > 1) return set_err(CSMV_EINVAL, "csmv_run: server_writeback must be 0 or 1");
    p.kv_swb = w->server_writeback && h->kind == CSMV_KIND_KV && kv_filt && h->maxid >= kSwbRow + kSwbRows + 1;
    p.bank_swb = w->server_writeback && h->kind == CSMV_KIND_BANK && selfrecv;
    p.req_tagged = w->req_tagged && (max_id <= (1ull << kIdItemBits)) &&
                   (bank_lock || (h->kind == CSMV_KIND_KV && kv_filt));
  }
  // the publisher takes the last warp slot of the first client CTA when no
  // client warp lives there (client warp cw runs on CTA cw % n_ctas, warp
  // cw / n_ctas): it then does not share the server SM with the critical
  // section.  CSMV_PUB_REMOTE=0 keeps it on the server CTA.
#ifndef CSMV_PUB_REMOTE
#define CSMV_PUB_REMOTE 1
#endif
  p.pub_remote = CSMV_PUB_REMOTE && w->publish == CSMV_PUBLISH_SERVER && !jvstm &&
                 (uint64_t)(kWarps - 1) * n_ctas >= n_cw;
  if (!selfrecv && !cmring && w->publish == CSMV_PUBLISH_SERVER && !p.pub_remote && p.n_workers > kWarps - 2)
    p.n_workers = kWarps - 2;  // the publisher needs the server CTA's last warp
  const bool traced = (w->debug_flags & CSMV_DBG_TRACE) != 0;
  if (traced && !h->d_trace) CK(cudaMalloc(&h->d_trace, sizeof(csmv_trace_rec) * kTraceCap));
  p.trace = h->d_trace;
  p.trace_item = w->trace_item;
  if (w->trace_item == 0xFFFFFFFFu)  // the hottest: zipf rank 0 (bank account 0, KV the set of key 0)
    p.trace_item = h->kind == CSMV_KIND_KV
                       ? (uint32_t)(((unsigned __int128)mix64(0ull ^ 0xA5A5A5A5A5A5A5A5ull) * h->kv_T) >> 64)
                       : 0u;
  p.req_vals = h->d_req_vals;
  p.jv_ws = h->d_jv_ws;
  p.jv_tag = h->d_jv_tag;
  p.jv_log2 = kJvLog2;
  p.watchdog_ns = (uint64_t)(w->watchdog_ms ? w->watchdog_ms : 20000u) * 1000000ull;

  CK(cudaMemsetAsync(h->d_ctl, 0, sizeof(Ctl), h->stream));
  if (part) CK(cudaMemcpyAsync(&h->d_ctl->cts_next, &gts0, 4, cudaMemcpyHostToDevice, h->stream));
  if (jvstm) {  // the global ATR starts empty at the current GTS
    CK(cudaMemcpyAsync(&h->d_ctl->jv_tail, &gts0, 4, cudaMemcpyHostToDevice, h->stream));
    CK(cudaMemsetAsync(h->d_jv_tag, 0, sizeof(uint32_t) << kJvLog2, h->stream));
  }
  if (w->retry_order == CSMV_RETRY_FIFO) {  // tickets restart at 0 every run (every one taken is served by its end)
    const size_t tkb = (size_t)h->kv_T * 12;
    if (!h->d_tk) CK(cudaMalloc(&h->d_tk, tkb));
    CK(cudaMemsetAsync(h->d_tk, 0, tkb, h->stream));
    p.kv_tk_serv = reinterpret_cast<uint64_t*>(h->d_tk);
    p.kv_tk_next = h->d_tk + 2 * (size_t)h->kv_T;
  }
  CK(cudaMemsetAsync(h->d_stats, 0, sizeof(DevStats), h->stream));
  CK(cudaMemsetAsync(h->d_req_seq, 0, n_cw * sizeof(uint32_t), h->stream));
  CK(cudaMemsetAsync(h->d_resp, 0, n_cw * sizeof(Resp), h->stream));
  CK(cudaEventRecord(h->ev0, h->stream));
  CK(launch_fused(p, h->nslot, n_srv + n_ctas, smem, h->stream));
  CK(cudaEventRecord(h->ev1, h->stream));
  CK(cudaStreamSynchronize(h->stream));

  Ctl ctl;
  DevStats ds;
  uint32_t gts1 = 0;
  CK(cudaMemcpy(&ctl, h->d_ctl, sizeof ctl, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(&ds, h->d_stats, sizeof ds, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(&gts1, h->d_gts, 4, cudaMemcpyDeviceToHost));
  float ms = 0.f;
  CK(cudaEventElapsedTime(&ms, h->ev0, h->ev1));

  csmv_stats_t& s = h->last;
  memset(&s, 0, sizeof s);
  s.committed_update = ds.committed_update;
  s.committed_ro = ds.committed_ro;
  for (int i = 0; i < (int)CSMV_N_ABORT; ++i)
    for (int k = 0; k < 2; ++k) s.aborts[i][k] = ds.aborts[i][k];
  s.batches = ds.batches;
  s.server_groups = ds.groups;
  s.rounds = ds.rounds;
  s.gts_start = gts0;
  s.gts_final = gts1;
  s.elapsed_ns = (uint64_t)((double)ms * 1e6);
  s.ro_checksum = ds.ro_checksum;
  if (h->kind == CSMV_KIND_KV) {
    s.store_bytes = (uint64_t)h->kv_S * h->nslot * (32 + 64 + 8) + (uint64_t)h->kv_T * h->nslot * 8;
    s.store_bytes_paper = (uint64_t)h->kv_S * ((4 + 20ull * h->K) + (4 + 36ull * h->K) + (4 + 8ull * h->K)) +
                          (uint64_t)h->kv_T * (4 + 8ull * h->K);
  } else {
    s.store_bytes = h->n_items * h->nslot * sizeof(uint64_t);
    s.store_bytes_paper = h->n_items * (4ull + 8ull * h->K);
  }
  s.server_lock_cycles = ds.lock_cycles;
  s.server_busy_cycles = ds.busy_cycles;
  for (int i = 0; i < 8; ++i) s.server_phase_cycles[i] = ds.phase[i];
  s.cas_failures = ds.cas_fail;
  for (int i = 0; i < 8; ++i) s.client_phase_cycles[i] = ds.client_phase[i];
  if (jvstm) ctl.tail_final = ctl.jv_tail;
  s.client_warps = n_cw;
  s.server_ctas = n_srv;
  s.server_workers = p.n_workers;
  s.atr_entries = 4u << rt_log2;
  s.sm_count = (uint32_t)h->sm_count;
  s.kernel_launches = 1;
  h->last_n_tx = n_tx;
  h->last_log_mode = w->log_mode;
  h->last_max_vals = max_vals;
  h->last_traced = traced;
  if (ctl.error) {
    h->loaded = false;
    return set_err(CSMV_ETIMEOUT, "csmv_run: device watchdog fired (loop %u; gts %u, cts %u); store state undefined",
                   ctl.where, gts1, part ? ctl.cts_next : ctl.tail_final);
  }
  if (s.committed_update + s.committed_ro != n_tx || gts1 != ctl.tail_final)
    return set_err(CSMV_ECUDA, "csmv_run: protocol error (committed %llu of %llu, gts %u, tail %u)",
                   (unsigned long long)(s.committed_update + s.committed_ro), (unsigned long long)n_tx, gts1,
                   ctl.tail_final);
  return CSMV_OK;
}

int csmv_stats(const csmv_t* h, csmv_stats_t* out) {
  if (!h || !out) return set_err(CSMV_EINVAL, "csmv_stats: null argument");
  *out = h->last;
  return CSMV_OK;
}

int csmv_get_log(const csmv_t* h, csmv_log_rec* buf, uint64_t cap, uint64_t* n_out) {
  if (!h || !buf) return set_err(CSMV_EINVAL, "csmv_get_log: null argument");
  if (h->last_log_mode == CSMV_LOG_NONE || !h->d_log) return set_err(CSMV_ESTATE, "csmv_get_log: last run had no log");
  if (cap < h->last_n_tx)
    return set_err(CSMV_EOVERFLOW, "csmv_get_log: cap %llu < n_tx %llu", (unsigned long long)cap,
                   (unsigned long long)h->last_n_tx);
  CK(cudaMemcpy(buf, h->d_log, h->last_n_tx * sizeof(csmv_log_rec), cudaMemcpyDeviceToHost));
  if (n_out) *n_out = h->last_n_tx;
  return CSMV_OK;
}

int csmv_get_vals(const csmv_t* h, uint32_t* buf, uint64_t cap_words, uint32_t* max_vals) {
  if (!h) return set_err(CSMV_EINVAL, "csmv_get_vals: null handle");
  if (h->last_log_mode != CSMV_LOG_FULL) return set_err(CSMV_ESTATE, "csmv_get_vals: last run not FULL");
  if (max_vals) *max_vals = h->last_max_vals;
  if (!buf) return CSMV_OK;
  const uint64_t words = h->last_n_tx * (uint64_t)h->last_max_vals;
  if (cap_words < words) return set_err(CSMV_EOVERFLOW, "csmv_get_vals: buffer too small");
  CK(cudaMemcpy(buf, h->d_vals, words * sizeof(uint32_t), cudaMemcpyDeviceToHost));
  return CSMV_OK;
}

int csmv_dump_store(const csmv_t* h, uint64_t* out, uint64_t cap) {
  if (!h || !out) return set_err(CSMV_EINVAL, "csmv_dump_store: null argument");
  if (h->kind != CSMV_KIND_BANK) return set_err(CSMV_EINVAL, "csmv_dump_store: not a bank store");
  if (cap < h->n_items * h->K) return set_err(CSMV_EOVERFLOW, "csmv_dump_store: cap too small");
  std::vector<uint64_t> raw(h->n_items * h->nslot);
  CK(cudaMemcpy(raw.data(), h->d_rings, raw.size() * sizeof(uint64_t), cudaMemcpyDeviceToHost));
  for (uint64_t i = 0; i < h->n_items; ++i)
    for (uint32_t j = 0; j < h->K; ++j) out[i * h->K + j] = raw[i * h->nslot + j];
  return CSMV_OK;
}

int csmv_dump_kv(const csmv_t* h, uint32_t* keys, uint32_t* vals, uint32_t* lru, uint32_t* clocks) {
  if (!h) return set_err(CSMV_EINVAL, "csmv_dump_kv: null handle");
  if (h->kind != CSMV_KIND_KV) return set_err(CSMV_EINVAL, "csmv_dump_kv: not a KV store");
  if (!h->loaded) return set_err(CSMV_ESTATE, "csmv_dump_kv: store not loaded");
  const size_t S = h->kv_S, T = h->kv_T;
  uint32_t* d = nullptr;
  CK(cudaMalloc(&d, (S * 13 + T) * 4));
  cudaError_t e = launch_kv_newest(kv_params(h), h->nslot, d, d + S * 4, d + S * 12, d + S * 13, h->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  if (e == cudaSuccess && keys) e = cudaMemcpy(keys, d, S * 16, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && vals) e = cudaMemcpy(vals, d + S * 4, S * 32, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && lru) e = cudaMemcpy(lru, d + S * 12, S * 4, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && clocks) e = cudaMemcpy(clocks, d + S * 13, T * 4, cudaMemcpyDeviceToHost);
  cudaFree(d);
  if (e != cudaSuccess) return set_err(CSMV_ECUDA, "csmv_dump_kv: %s", cudaGetErrorString(e));
  return CSMV_OK;
}

int csmv_gen_descs(csmv_t* h, const csmv_workload* w, uint64_t seed, uint64_t tx0, uint64_t n, uint32_t* out) {
  if (!h || !w || !out) return set_err(CSMV_EINVAL, "csmv_gen_descs: null argument");
  GenParams g;
  int rc = make_gen(h, w, seed, &g);
  if (rc) return rc;
  const uint32_t per = h->kind == CSMV_KIND_KV ? 10 : 6;
  uint32_t* d = nullptr;
  CK(cudaMalloc(&d, n * per * sizeof(uint32_t) + 4));
  cudaError_t e = h->kind == CSMV_KIND_KV ? launch_gen_kv_descs(g, tx0, n, d, h->stream)
                                          : launch_gen_descs(g, tx0, n, d, h->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  if (e == cudaSuccess) e = cudaMemcpy(out, d, n * per * sizeof(uint32_t), cudaMemcpyDeviceToHost);
  cudaFree(d);
  if (e != cudaSuccess) return set_err(CSMV_ECUDA, "csmv_gen_descs: %s", cudaGetErrorString(e));
  return CSMV_OK;
}

int csmv_get_trace(const csmv_t* h, csmv_trace_rec* buf, uint64_t cap, uint64_t* n_out) {
  if (!h || !buf || !n_out) return set_err(CSMV_EINVAL, "csmv_get_trace: null argument");
  if (!h->last_traced || !h->d_trace) return set_err(CSMV_ESTATE, "csmv_get_trace: last run was not traced");
  Ctl ctl;
  CK(cudaMemcpy(&ctl, h->d_ctl, sizeof ctl, cudaMemcpyDeviceToHost));
  const uint64_t n = ctl.trace_n < kTraceCap ? ctl.trace_n : kTraceCap;
  const uint64_t m = n < cap ? n : cap;
  if (m) CK(cudaMemcpy(buf, h->d_trace, m * sizeof(csmv_trace_rec), cudaMemcpyDeviceToHost));
  *n_out = ctl.trace_n;
  return CSMV_OK;
}

int csmv_zipf_table(uint32_t n, uint32_t theta_milli, uint64_t* out) {
  if (!out || n == 0) return set_err(CSMV_EINVAL, "csmv_zipf_table: bad argument");
  std::vector<uint64_t> c = build_zipf(n, theta_milli);
  memcpy(out, c.data(), n * sizeof(uint64_t));
  return CSMV_OK;
}

}  // extern "C"
