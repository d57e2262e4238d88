// kernel.cuh -- device-side data layout shared by host.cu and kernel.cu.
//
// HBM layout (one handle):
//   rings     u64[n_items][NSLOT]   packed (ts << 32 | value) versions; NSLOT
//                                   = K rounded up to 2/4/8/16 so a VBox is one
//                                   aligned record (32 B = one sector at K = 4)
//   gts       u32                   the global timestamp GTS
//   req_seq   u32[n_cw]             per client warp request doorbell
//   req_hdr   {snapshot, mask}[n_cw]
//   req_ids   u32[n_cw][MAXID][32]  lane-major item ids of RS u WS (bit 31 =
//                                   also in WS); coalesced 128 B rows
//   resp      {cts_base, commit_mask, overflow_mask, seq}[n_cw]
//   done_ring u32[2^20]             CSMV_PUBLISH_SERVER: done[cts & mask] = cts
//                                   after the write-back of cts
//   lastw     u32[n_items]          CTS of the last commit that wrote the item
//                                   (server-private level of the ATR)
//   log       csmv_log_rec[n_tx]    parity runs only
//   req_vals  u32[n_cw][2][32]      CSMV_COMMIT_ONLYCS: values for the server write-back
//   jv_ws/jv_tag u64/u32[2^22]      CSMV_COMMIT_JVSTM: the global-memory ATR
#pragma once
#include <cstdint>

#include "../../include/csmv.h"
#include "gen.cuh"

// back-off (ns) of three spin waits: a client warp polling its response, the
// client GTS publish chain, a server worker polling its dispatch queue
// (build-time knobs for A/B: CSMV_NVCC_EXTRA="-DCSMV_SLEEP_RESP=..")
#ifndef CSMV_SLEEP_RESP
#define CSMV_SLEEP_RESP 64
#endif
#ifndef CSMV_SLEEP_PUB
#define CSMV_SLEEP_PUB 32
#endif
#ifndef CSMV_SLEEP_QUEUE
#define CSMV_SLEEP_QUEUE 64
#endif
// back-off (ns) of a worker polling the ticket lock (single-CTA server)
#ifndef CSMV_SLEEP_LOCK
#define CSMV_SLEEP_LOCK 16
#endif
// idle back-off (ns) of the server's receiver sweep and publisher sweep (0 = spin)
#ifndef CSMV_SLEEP_RECV
#define CSMV_SLEEP_RECV 0
#endif
#ifndef CSMV_SLEEP_PUBLISHER
#define CSMV_SLEEP_PUBLISHER 0
#endif

namespace csmvd {

constexpr uint32_t kEmptyTs = 0xFFFFFFFFu;
constexpr uint32_t kWriteBit = 0x80000000u;
constexpr int kBlock = 256;            // threads per CTA (8 warps)
constexpr int kWarps = kBlock / 32;
constexpr uint32_t kDoneLog2 = 20;     // done ring entries (CSMV_PUBLISH_SERVER)
constexpr int kMaxCombine = 8;         // batches a server worker commits per critical section
// commit-ring slots (worker warps -> committer warp, bank): 2^5 for per-warp
// batches, 2^6 for client groups on a commit ring (a group takes G slots;
// with 32 slots the committer stalled on slots claimed but not yet filled:
// cluster-16, G = 4, 736 warps 268 -> 314 M tx/s; per-warp batches lose with
// 64: 241 -> 229 M).  The ticket-locked server keeps 32 (its CTAs' shared
// memory, and so every client CTA's, would grow by 33 KB at the L1's
// expense: its grouped C2 fell 490 -> 313 M with the larger allocation).
constexpr uint32_t kCmRingLog2 = 5;
constexpr uint32_t kCmRingLog2Max = 6;
__host__ __device__ inline uint32_t cm_ring_log2(uint32_t group, bool ring) {
#ifdef CSMV_RING_ALWAYS
  return ring && group > 1 ? kCmRingLog2Max : kCmRingLog2;
#else
  return !ring ? 0u : group > 1 ? kCmRingLog2Max : kCmRingLog2;  // no commit ring: one unused slot
#endif
}

// One commit-ring slot: a batch a worker warp has prepared for the committer
// (server.cuh).  Lane l's words: {fa0, fa1, fa2, fb0}, {fb1, fb2, id0, id1}
// -- the shared-memory addresses of its items' filter slots and the items.
struct alignas(16) CmSlot {
  uint32_t flag;   // = slot sequence number + 1 once the payload is written
  uint32_t cw;     // client warp
  uint32_t round;  // request round (tags the response)
  uint32_t e_pre;  // tail the worker's lastw prefetch covers
  uint32_t chk;    // lanes whose exact lastw check passed
  uint32_t pad[3];
  uint4 w[2][32];
};

struct Ctl {
  uint32_t error;       // 0 ok, 1 watchdog, 2 protocol
  uint32_t done_warps;  // client warps that finished
  uint32_t tail_final;  // server: last CTS assigned
  uint32_t where;       // which spin loop fired the watchdog
  uint32_t jv_tail;     // CSMV_COMMIT_JVSTM: last CTS reserved (global CAS target)
  uint32_t trace_n;     // CSMV_DBG_TRACE: records claimed
  uint32_t srv_done;    // server finished, tail_final valid (release; the remote publisher's exit)
  uint32_t cts_next;    // CSMV_SERVER_PART: last CTS handed out by the global counter
};
constexpr uint32_t kTraceCap = 1u << 18;

// A request's header.  Untagged requests: the three fields, written before
// a fence and the doorbell.  Tagged requests (KParams.req_tagged): two
// 64-bit words {round << 32 | snapshot}, {round << 32 | mask} and every id
// carrying the round's low kIdTagBits bits above the item (kIdItemBits):
// no fence between payload and doorbell -- the server re-reads the payload
// until every word carries the round of the doorbell it saw (as the client
// does with the response, Resp).
struct ReqHdr {
  uint32_t snapshot;
  uint32_t round;      // = the doorbell value; tags the response
  uint32_t mask;
  uint32_t round2;     // tagged requests: the round again (the mask's word)
};
constexpr uint32_t kIdItemBits = 24;                       // tagged requests: item ids < 2^24
constexpr uint32_t kIdItemMask = (1u << kIdItemBits) - 1;
constexpr uint32_t kIdTagMask = 0x7Fu;                     // bits 24..30: round & 0x7F (bit 31: in WS)
__host__ __device__ inline uint32_t id_tag(uint32_t round) { return (round & kIdTagMask) << kIdItemBits; }

// The response: every word carries the request's round in its upper half,
// so the client accepts it word by word -- no release/acquire pair and no
// fence on the server's respond path (the client needs nothing else the
// server wrote; CSMV_COMMIT_ONLYCS fences its write-backs first).
struct Resp {
  uint64_t base;       // round << 32 | first CTS of the batch
  uint64_t commit;     // round << 32 | commit mask
  uint64_t ovf;        // round << 32 | overflow mask
  uint64_t pad;
};

struct DevStats {
  unsigned long long committed_update, committed_ro;
  unsigned long long aborts[CSMV_N_ABORT][2];
  unsigned long long batches, rounds, groups;
  unsigned long long ro_checksum;
  unsigned long long lock_cycles, busy_cycles;
  unsigned long long phase[8];  // server worker: queue wait, load, lock wait, critical, respond
  unsigned long long cas_fail;  // CSMV_COMMIT_JVSTM: failed CTS reservations
  unsigned long long client_phase[8];  // CSMV_DBG_PHASES: client cycles by phase (mean lane)
};

struct KParams {
  uint64_t* rings;
  uint32_t n_items;
  uint32_t K;
  uint32_t* gts;
  Ctl* ctl;
  uint32_t* req_seq;
  ReqHdr* req_hdr;
  uint32_t* req_ids;
  Resp* resp;
  uint32_t* done_ring;
  DevStats* stats;
  csmv_log_rec* log;
  uint32_t* vals;
  uint32_t max_vals;
  uint32_t log_mode;
  GenParams gen;
  uint64_t n_tx;
  uint32_t n_cw;           // active client warps
  uint32_t n_client_ctas;  // CTAs n_server_ctas.. host clients
  uint32_t n_server_ctas;  // 1, or the cluster size of a cluster server
  uint32_t clog2;          // log2(n_server_ctas)
  uint32_t n_workers;      // server worker warps
  uint32_t rt_log2;        // recent-commit table buckets, all server CTAs (4 ways, 32 B each, + evmax)
  uint32_t* lastw;         // per-item CTS of the last committed write
  uint32_t publish;
  uint32_t ro_streak;      // read-only transactions a lane may run per round (0 = one tx per round)
  uint32_t combine;        // batches per critical section (1..kMaxCombine)
  uint32_t backoff_max;    // rounds an update rejected by the server may sit out (0 = none)
  uint32_t atr_mode;       // CSMV_ATR_HASH (item-indexed) / _LIST (paper, CV) / _LIST_NOCV
  uint32_t debug;
  uint64_t watchdog_ns;
  // KV workload (kind == CSMV_KIND_KV)
  uint32_t kind;
  uint32_t kv_S, kv_A, kv_T;  // slots, ways, sets
  uint64_t* kv_key;           // u64[S][NS][4]
  uint64_t* kv_val;           // u64[S][NS][8]
  uint64_t* kv_lru;           // u64[S][NS]
  uint64_t* kv_clk;           // u64[T][NS]
  uint32_t* req_cnt;          // ids per lane [n_cw][32] (generic requests)
  uint32_t maxid;             // id rows per request slot
  // commit-protocol ablations (CSMV_COMMIT_*)
  uint32_t commit;
  uint32_t ro_adaptive;       // stop a read-only run once the server has answered
  uint32_t server_recv;       // CSMV_RECV_*
  uint32_t group;             // client warps per request (1 = per-warp batches; 2/4/8 = CTA-level batches)
  uint32_t cm_ring_log2;      // commit-ring slots (cm_ring_log2())
  uint32_t ev_log2;           // eviction-watermark words per server CTA (log2; 2 = four unused words)
  uint32_t filt16_n;          // locked single-CTA bank server: 16-bit filter slots when trimmed (0 = 16 << rt_log2)
  uint32_t pub_remote;        // CSMV_PUBLISH_SERVER: the publisher runs on an idle warp of the first client CTA
  // CSMV_SERVER_PART (item-partitioned servers, server_part.cuh): server k of
  // 2^part_log2 owns the items with part_owner(x) == k
  uint32_t part_log2;         // 0 = not partitioned
  uint32_t part_bits_log2;    // pending bits per server (part_bits_log2())
  uint32_t mstride;           // per-server stride of the arrays below (client warps)
  uint32_t* mreq_seq;         // [S][mstride] prepare doorbells
  Resp* mresp;                // [S][mstride] prepare votes {ok mask, overflow mask}, round-tagged
  uint32_t* mdec_seq;         // [S][mstride] decide doorbells
  uint32_t* mdack;            // [S][mstride] decide acknowledgements (round)
  uint64_t* mdec;             // [mstride][2] decide payload {round << 32 | first CTS, round << 32 | commit mask}
  uint32_t gts_start;         // GTS when the run started
  uint32_t clustered;         // the server CTAs form a thread-block cluster (CSMV_SERVER_CLUSTER)
  csmv_trace_rec* trace;      // CSMV_DBG_TRACE buffer (kTraceCap records)
  uint32_t trace_item;        // bank account / KV set traced
  uint32_t* req_vals;         // ONLYCS: new values [n_cw][2][32] for the server-side write-back
  uint64_t* jv_ws;            // JVSTM: global ATR, write-set of CTS c at c & (2^jv_log2 - 1)
  uint32_t* jv_tag;           //        entry tag = c once the record of c is written
  uint32_t jv_log2;
  // CSMV_RETRY_FIFO (KV): per-set PUT tickets -- next ticket to hand out,
  // and {ticket now served << 32 | CTS of the previous ticket's commit}
  uint32_t* kv_tk_next;       // u32[T], nullptr = CSMV_RETRY_FREE
  uint64_t* kv_tk_serv;       // u64[T]
  uint32_t req_tagged;        // requests are round-tagged (ReqHdr): no client fence before the doorbell
  uint32_t kv_swb;            // KV: the server writes committed PUTs back and publishes (rows kSwbRow.. of a request)
  uint32_t bank_swb;          // bank, self-receiving workers: the server writes committed transfers back (req_vals)
};
// KV server write-back: request rows 4-7 the key, 8-15 the value, 16 the new
// LRU / clock value, 17 the replacement slots (key/value/LRU | clock << 8),
// 18 (tagged requests) a check word of the round and rows 4-17
constexpr uint32_t kSwbRow = 4, kSwbRows = 14;
// bank server write-back (req_vals rows 0-2: new balances, slots; row 3 the check word)
__host__ __device__ inline uint32_t bank_swb_check(uint32_t round, uint32_t a, uint32_t b, uint32_t c) {
  uint32_t h = round * 0x9E3779B1u + 0x7F4A7C15u;
  h = ((h ^ a) * 0x85EBCA77u) ^ (h >> 15);
  h = ((h ^ b) * 0x85EBCA77u) ^ (h >> 15);
  return ((h ^ c) * 0x85EBCA77u) ^ (h >> 15);
}
__host__ __device__ inline uint32_t swb_check(uint32_t round, const uint32_t* w, uint32_t stride) {
  uint32_t h = round * 0x9E3779B1u + 0x7F4A7C15u;
  for (uint32_t k = 0; k < kSwbRows; ++k) h = ((h ^ w[k * stride]) * 0x85EBCA77u) ^ (h >> 15);
  return h;
}

constexpr uint32_t kKvMaxWays = 256;              // KV ways supported by the device path
constexpr uint32_t kKvFullWays = 16;              // up to here PUT read-sets are shipped item by item
constexpr uint32_t kKvMaxRs = 2 * kKvFullWays + 1;  // keys + LRU stamps + clock
constexpr uint32_t kKvMaxId = 2 * kKvFullWays + 2;  // RS u WS

// CSMV_SERVER_PART: the server owning item x (a hash unrelated to the filter's)
__host__ __device__ inline uint32_t part_owner(uint32_t x, uint32_t log2s) {
  return x & ((1u << log2s) - 1);  // items spread evenly (bank and zipf ranks alike)
}
constexpr uint32_t kPartFiltLog2 = 13;      // 32-bit recent-commit filter slots per partition server
constexpr uint32_t kPartBitsLog2Max = 20;   // pending bits per partition server (128 KiB); more items fold
__host__ __device__ inline uint32_t part_pend_words(uint32_t bits_log2) { return bits_log2 > 5 ? 1u << (bits_log2 - 5) : 1u; }
inline uint32_t part_bits_log2(uint64_t n_items, uint32_t log2s) {
  uint32_t b = 5;
  while (b < kPartBitsLog2Max && ((uint64_t)1 << b) < ((n_items + (1u << log2s) - 1) >> log2s)) ++b;
  return b;
}
inline size_t part_smem_bytes(uint32_t n_cw, uint32_t bits_log2) {
  return ((size_t)4 << kPartFiltLog2) + (size_t)4 * part_pend_words(bits_log2) + (((size_t)n_cw + 31) / 32 * 32) * 4 * 3;
}

// client smem scratch per warp (KV read/write sets of its update lanes)
inline size_t kv_client_smem_bytes() { return (size_t)kWarps * 32 * (kKvMaxRs + 4 + 1) * 4; }

// dispatch queue slots: a power of two >= n_cw
__host__ __device__ inline uint32_t queue_log2(uint32_t n_cw) {
  uint32_t l = 5;
  while ((1u << l) < n_cw) ++l;
  return l;
}

// smem the server CTA needs (every CTA of the fused grid gets the same):
// recent-commit table, dispatch queue, receiver's last-seen doorbells, control words
// (per server CTA: its stripe of 2^local_log2 buckets and its slice of n_cw)
// rt stripe | dispatch queue | evmax stripe | last-seen doorbells | control
// block (64 B) | commit ring.  Only what the run's commit path uses is
// allocated (the eviction watermarks only for the KV item-set table, the
// commit ring only for a ring server): every CTA of the grid gets this much
// shared memory, and what it takes comes out of the SM's unified L1 --
// dropping the unused 33 KB ring of the locked server took C2 from ~485 to
// ~540 M tx/s (profiles/r02/raw/r02ae_ab_smem.jsonl).
// bytes of the recent-commit table / filter region (u64 words * 8)
__host__ __device__ inline uint32_t rt_region_words(uint32_t local_log2, uint32_t filt16_n) {
  return filt16_n ? (filt16_n * 2u + 31u) / 32u * 4u : 4u << local_log2;
}
inline size_t server_smem_bytes(uint32_t local_log2, uint32_t n_cw, uint32_t ring_log2, uint32_t ev_log2,
                                uint32_t filt16_n = 0) {
  return (size_t)8 * rt_region_words(local_log2, filt16_n) + ((size_t)4 << ev_log2) + ((size_t)8 << queue_log2(n_cw)) +
         (((size_t)n_cw + 31) / 32 * 32) * 4 + 64 + (sizeof(CmSlot) << ring_log2);
}

// host-callable launchers (kernel.cu)
constexpr uint32_t kJvLog2 = 22;       // JVSTM global ATR entries

cudaError_t launch_fused(const KParams& p, uint32_t nslot, uint32_t grid, size_t smem,
                         cudaStream_t st);
cudaError_t launch_init_rings(uint64_t* rings, uint32_t nslot, const int32_t* init, uint64_t n,
                              uint32_t* gts, cudaStream_t st);
cudaError_t launch_gen_descs(GenParams g, uint64_t tx0, uint64_t n, uint32_t* out, cudaStream_t st);
// co-resident CTAs of the fused kernel for this configuration (server CTAs
// included; a multiple of the cluster size for a cluster server)
cudaError_t fused_capacity(const KParams& p, uint32_t nslot, size_t smem, int* ctas);
cudaError_t launch_init_kv(const KParams& p, uint32_t nslot, const uint32_t* keys, const uint32_t* vals,
                           const uint32_t* lru, const uint32_t* clocks, cudaStream_t st);
// Device preload of keys 0..n_keys-1 (kv_kernels.cuh) into the plain-word
// layout launch_init_kv installs (keys/vals/lru/clocks zeroed by the
// caller).  scratch: 3*T + n_keys words.  With cub_tmp == nullptr only sets
// *cub_bytes (the scan's temporary storage size).
cudaError_t launch_kv_preload(uint32_t n_keys, uint32_t T, uint32_t A, uint32_t* scratch, void* cub_tmp,
                              size_t* cub_bytes, uint32_t* keys, uint32_t* vals, uint32_t* lru, uint32_t* clocks,
                              cudaStream_t st);
cudaError_t launch_kv_newest(const KParams& p, uint32_t nslot, uint32_t* keys, uint32_t* vals, uint32_t* lru,
                             uint32_t* clocks, cudaStream_t st);
cudaError_t launch_gen_kv_descs(GenParams g, uint64_t tx0, uint64_t n, uint32_t* out, cudaStream_t st);

}  // namespace csmvd
