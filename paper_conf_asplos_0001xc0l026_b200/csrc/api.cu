// api.cu — the C ABI of include/bullet.h: handle, validation, per-step
// planning, kernel launches on the two phase streams, SM gating, perf model
// and split decision entry points, NCCL tensor parallelism.
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <set>
#include <string>
#include <vector>

#include "bullet.h"
#include "kernels.h"
#include "perfmodel.h"

using namespace bl;

namespace {

thread_local std::string g_err;

int set_err(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}

#define CK(x)                                                                           \
  do {                                                                                  \
    cudaError_t e_ = (x);                                                               \
    if (e_ != cudaSuccess)                                                              \
      return set_err(BULLET_ECUDA, "%s: %s (%s:%d)", #x, cudaGetErrorString(e_), __FILE__, \
                     __LINE__);                                                         \
  } while (0)

// ---------------------------------------------------------------- NCCL (dlopen)
struct Nccl {
  void* lib = nullptr;
  ncclResult_t (*getUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*commInitRankConfig)(ncclComm_t*, int, ncclUniqueId, int, ncclConfig_t*) = nullptr;
  ncclResult_t (*allReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
  const char* (*errStr)(ncclResult_t) = nullptr;
  bool load() {
    if (lib) return true;
    const char* env = getenv("BULLET_NCCL_LIB");
    lib = dlopen(env ? env : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!lib) return false;
    getUniqueId = (decltype(getUniqueId))dlsym(lib, "ncclGetUniqueId");
    commInitRankConfig = (decltype(commInitRankConfig))dlsym(lib, "ncclCommInitRankConfig");
    allReduce = (decltype(allReduce))dlsym(lib, "ncclAllReduce");
    commDestroy = (decltype(commDestroy))dlsym(lib, "ncclCommDestroy");
    errStr = (decltype(errStr))dlsym(lib, "ncclGetErrorString");
    return getUniqueId && commInitRankConfig && allReduce && commDestroy && errStr;
  }
} g_nccl;

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
EncodeTiledFn g_encode = nullptr;

int get_encode() {
  if (g_encode) return BULLET_OK;
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
  if (!fn || q != cudaDriverEntryPointSuccess)
    return set_err(BULLET_ECUDA, "cuTensorMapEncodeTiled unavailable");
  g_encode = (EncodeTiledFn)fn;
  return BULLET_OK;
}

// 2D bf16 K-major operand [rows][K], box {64, box_rows}, 128-byte swizzle.
int make_map(CUtensorMap* m, const void* ptr, int rows, int K, int box_rows) {
  cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)K * 2};
  cuuint32_t box[2] = {64, (cuuint32_t)box_rows};
  cuuint32_t es[2] = {1, 1};
  CUresult r = g_encode(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(ptr), dims,
                        strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                        CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_err(BULLET_ECUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return BULLET_OK;
}

struct PhaseWS {
  float* qkv = nullptr;
  void *q = nullptr, *o = nullptr, *h = nullptr, *act = nullptr;
  float* partials = nullptr;
  size_t partial_floats = 0;
  int* tile_sems = nullptr;        // [2][N_TILE_SEMS] stream-K counters, alternating slices per GEMM launch
  int sk_parity = 0;
  int* counters = nullptr;
  int n_counters = 0, next_ctr = 0;
  int2* tiles = nullptr;
  int* n_tiles = nullptr;
  TokInfo* tok = nullptr;          // per-token (position, KV slot), written by the plan kernel
  int max_tok = 0;
  int* rbc = nullptr;              // fused-norm row-block counters [n_rbc_slices][max_rb], zeroed per step
  int max_rb = 0, n_rbc_slices = 0, next_rbc = 0;
  int4* order = nullptr;           // decode rows in LPT order (plan kernel), valid this step if order_ok
  bool order_ok = false;
  float* kv_part = nullptr;        // decode phase, split-KV decode attention: partial softmax states
  int* kv_tick = nullptr;          //   and per-unit arrival tickets (contexts > one block window)
  int kv_cap = 1;                  //   KV chunks per unit the scratch holds
};

constexpr int GRAN = 2;            // split granularity: one TPC
const char* const SIGMA_DEFAULT = "sorted";   // order of sigma (BULLET_SIGMA; DESIGN.md §5 die probe)

// Symmetric region of the fused peer all-reduce (PEER mode, include/bullet.h):
// per phase two fp32 partial buffers, the fp32 hidden, ready counters
// [tp][max_rb], done counters [max_rb], expected-value bases [2][max_rb], an
// error word.  Offsets depend only on the model cfg: identical on every rank.
struct SymLayout {
  size_t part[2], hid, ready, done, base, err, end;
  int max_rb;
};
inline size_t al256(size_t x) { return (x + 255) & ~size_t(255); }
SymLayout sym_layout(const bullet_model_cfg& c, int phase) {
  SymLayout L{};
  size_t off = 0;
  for (int p = 0; p <= phase; ++p) {
    const size_t T = std::max(1, p == 0 ? c.max_prefill_tokens : c.max_decode_tokens);
    const size_t f = al256(T * c.d_model * sizeof(float));
    L.max_rb = (int)((T + 127) / 128);
    L.part[0] = off; L.part[1] = off + f; L.hid = off + 2 * f; L.ready = off + 3 * f;
    L.done = L.ready + al256((size_t)c.tp_size * L.max_rb * 8);
    L.base = L.done + al256((size_t)L.max_rb * 8);
    L.err = L.base + al256((size_t)2 * L.max_rb * 8);
    off = L.err + 256;
  }
  L.end = off;
  return L;
}
constexpr int N_TILE_SEMS = 2048;

}  // namespace

struct bullet_handle {
  bullet_model_cfg cfg;
  int dev = 0, n_sms = 0, elt = 2;
  std::vector<int> sigma;
  std::vector<int> die;              // die (0/1) of each smid from the die probe, -1 unknown
  std::vector<bullet_layer_weights> w;
  struct Packed { uint8_t *base = nullptr, *qkv = nullptr, *o = nullptr, *gu = nullptr, *down = nullptr; };
  std::vector<Packed> wp;            // bf16: pre-swizzled weight tiles (kernels.h)
  uint8_t* op_pack = nullptr;        // scratch for bullet_op_gemm with BULLET_GEMM_PACKED
  size_t op_pack_bytes = 0;
  std::vector<char> w_set;
  std::vector<void*> pk, pv;
  int n_blocks = 0, block_size = 0;
  float2* rope_cs = nullptr;
  PhaseWS ph[2];
  int* op_ctr = nullptr;
  int* gate_fallbacks = nullptr;     // launches whose last CTA worked off its SM range (gate_enter)
  Gate* d_gates = nullptr;           // BULLET_DEVICE_SPLIT: [2] (prefill, decode), written by bullet_set_split
  int32_t* log = nullptr;
  int log_cap = 0;
  int launch_seq = 0;
  PerfParams perf;
  ncclComm_t comm[2] = {nullptr, nullptr};
  // fused peer all-reduce (PEER mode): own symmetric region, every rank's base
  bool peer_mode = false, peer_connected = false;
  uint8_t* sym = nullptr;
  size_t sym_bytes = 0;
  std::vector<uint8_t*> peer_base;
  std::vector<void*> ipc_opened;
  cudaEvent_t ev_ts = nullptr;
  bool host_only = false;  // bullet_perf_create: perf model only
  // BULLET_PROFILE: events around every launch
  struct ProfRec { int kind, phase, layer; cudaEvent_t e0, e1; };
  std::vector<ProfRec> prof_recs;
  std::vector<cudaEvent_t> ev_pool;
  size_t ev_used = 0;
  long long n_launch = 0;
  // bullet_trace_enable: per-CTA timestamp records of the next launches
  unsigned long long* trace = nullptr;
  int trace_cap = 0, trace_n = 0;
  std::vector<int> trace_meta;   // [trace_cap][4]
};

namespace {

Gate gate_of(const bullet_handle* h, int lo, int hi) {
  Gate g;
  memset(&g, 0, sizeof g);
  for (int i = lo; i < hi; ++i) {
    const int s = h->sigma[i];
    g.m[s >> 5] |= 1u << (s & 31);
  }
  return g;
}

struct Ctx {  // one phase's launch context within a call
  bullet_handle* h;
  int phase;
  Gate gate;
  int m_sms;
  bool log;
  cudaStream_t st;
  bool op;     // op-level entry: counter = op_ctr, zeroed before each launch
  bool prof = false;
  int kind = 0, layer = -1;
  bool fuse_qkv = false;   // S3 in the QKV epilogue (EPI_QKV)
  bool fuse_norm = false;  // S6 / next S1 in the tail of the O-proj / down GEMM (NormFuse)
  const Gate* gdev = nullptr;   // BULLET_DEVICE_SPLIT: the phase's gate in device memory
};

constexpr size_t MAX_PROF = 1 << 16;

cudaEvent_t take_event(bullet_handle* h) {
  if (h->ev_used == h->ev_pool.size()) {
    cudaEvent_t e;
    if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
    h->ev_pool.push_back(e);
  }
  return h->ev_pool[h->ev_used++];
}

void prof_begin(Ctx& c) {
  bullet_handle* h = c.h;
  h->n_launch++;
  if (!c.prof || h->prof_recs.size() >= MAX_PROF) return;
  bullet_handle::ProfRec r{c.kind, c.phase, c.layer, take_event(h), take_event(h)};
  if (!r.e0 || !r.e1) return;
  cudaEventRecord(r.e0, c.st);
  h->prof_recs.push_back(r);
}

void prof_end(Ctx& c) {
  if (c.prof && !c.h->prof_recs.empty()) cudaEventRecord(c.h->prof_recs.back().e1, c.st);
}

#define LAUNCH(c, x)  \
  do {                \
    CK(x);            \
    prof_end(c);      \
  } while (0)

// Kernels with several CTAs per SM (the row grids, the fp32 SIMT kernels) are
// launched without PDL: launched early, their whole grid can fit on the SMs
// outside a small partition whose SMs the predecessor still holds, park
// there, and leave the gate's liveness fallback to run a unit off-range (seen
// with a 2-SM decode partition, test_smid_gating_invariants[146]).  The
// one-CTA-per-SM persistent kernels always leave CTAs queued for the
// partition's SMs (grid = SMs x occupancy).
static inline void no_pdl(Launch& L) { L.pdl = 0; }

int next_launch(Ctx& c, Launch* L) {
  prof_begin(c);
  memset(L, 0, sizeof *L);
  L->gate = c.gate;
  L->gdev = c.gdev;
  L->fallback = c.h->gate_fallbacks;
  L->log = c.log ? c.h->log : nullptr;
  L->log_cap = c.h->log_cap;
  L->launch_id = c.h->launch_seq++;
  L->phase = c.phase;
  // Programmatic dependent launch (common.cuh): a step kernel may launch in
  // its predecessor's tail, prologue and weight stream overlapping it.  Not
  // under BULLET_PROFILE (events between launches time each kernel alone),
  // not for op-level entries; BULLET_PDL=0 disables.  (A first version
  // triggered at kernel entry and let out-of-range CTAs leave at once: the
  // grid drained through the SMs the predecessor's gated-out CTAs had freed,
  // prefill layer 2.36 -> 102 ms — now triggers come in the tail and
  // out-of-range CTAs park until the predecessor completes.)
  static const bool pdl_on = !(getenv("BULLET_PDL") && !strcmp(getenv("BULLET_PDL"), "0"));
  // Not under tensor parallelism: a CTA parked on another partition's SM
  // (waiting for its own predecessor) could hold an SM that a kernel
  // spin-waiting on a peer rank (fused all-reduce, NCCL) needs — a cycle
  // (measured: the simulated-TP4 test hit the 20 s peer timeout).
  L->pdl = pdl_on && !c.op && !c.prof && c.h->cfg.tp_size == 1;
  if (c.h->trace && c.h->trace_n < c.h->trace_cap) {
    const int i = c.h->trace_n++;
    L->trace = c.h->trace + (size_t)i * BULLET_TRACE_CTAS * TRACE_SLOTS;
    int* m = c.h->trace_meta.data() + 4 * i;
    m[0] = c.kind; m[1] = c.phase; m[2] = c.layer; m[3] = 0;
  }
  if (c.op) {
    CK(cudaMemsetAsync(c.h->op_ctr, 0, 4 * sizeof(int), c.st));
    L->ctr = c.h->op_ctr;
    L->burn = c.h->op_ctr + 1;
  } else {
    PhaseWS& P = c.h->ph[c.phase];
    if (P.next_ctr + 2 > P.n_counters) return set_err(BULLET_ENOMEM, "work counters exhausted");
    L->ctr = P.counters + P.next_ctr++;
    L->burn = P.counters + P.next_ctr++;
  }
  return BULLET_OK;
}

// Grid of the one-CTA-per-SM persistent kernels.  CTAs that land on the
// other phase's SMs (free for a moment between its kernels) exit at once;
// with exactly one CTA per SM each such CTA would leave an SM of this phase
// without a worker for the whole kernel.  Spare CTAs (BULLET_GRID_MULT > 1)
// would take their place; measured: no gain (co-run 3.01-3.03 ms at x1 vs
// 3.09-3.24 at x2/x3, config 2), so the default is one CTA per SM.
int persist_grid(const Ctx& c, int per_sm) {
  static const int mult = [] {
    const char* e = getenv("BULLET_GRID_MULT");
    const int v = e ? atoi(e) : 1;
    return v >= 1 && v <= 8 ? v : 1;
  }();
  return c.h->n_sms * per_sm * (c.m_sms < c.h->n_sms ? mult : 1);
}

// Two-level accumulation policy (DESIGN R-4e).  Default: K chunks of
// KC_DEFAULT on the QKV and O-proj GEMMs when d_model >= 5120 — the GEMMs
// whose outputs are rounded (R2) or normalised and rounded (R4) inside the
// layer, where accumulation error turns into bf16 rounding flips that the
// rest of the layer amplifies.  Overrides (read once per process):
//   BULLET_GEMM_KCHUNK=kc (0 = off), BULLET_GEMM_KCHUNK_ONLY=list of
//   qkv,oproj,gate_up,down | all | attn (= qkv,oproj) | silu (= gate_up),
//   BULLET_GEMM_KCHUNK_MODE=splitk.
constexpr int KC_DEFAULT = 256;
constexpr unsigned KC_ALL = (1u << BULLET_K_QKV) | (1u << BULLET_K_OPROJ) | (1u << BULLET_K_GATE_UP) |
                            (1u << BULLET_K_DOWN);
struct KcPolicy { int kc_override; unsigned mask; bool splitk; };
const KcPolicy& kc_policy() {
  static const KcPolicy p = [] {
    KcPolicy r{-1, (1u << BULLET_K_QKV) | (1u << BULLET_K_OPROJ), false};
    if (const char* e = getenv("BULLET_GEMM_KCHUNK")) r.kc_override = atoi(e);
    if (const char* e = getenv("BULLET_GEMM_KCHUNK_MODE")) r.splitk = !strcmp(e, "splitk");
    if (const char* e = getenv("BULLET_GEMM_KCHUNK_ONLY")) {
      r.mask = 0;
      std::string s(e);
      size_t a = 0;
      while (a <= s.size()) {
        size_t b = s.find(',', a);
        if (b == std::string::npos) b = s.size();
        const std::string t = s.substr(a, b - a);
        if (t == "qkv") r.mask |= 1u << BULLET_K_QKV;
        else if (t == "oproj") r.mask |= 1u << BULLET_K_OPROJ;
        else if (t == "gate_up" || t == "silu") r.mask |= 1u << BULLET_K_GATE_UP;
        else if (t == "down") r.mask |= 1u << BULLET_K_DOWN;
        else if (t == "attn") r.mask |= (1u << BULLET_K_QKV) | (1u << BULLET_K_OPROJ);
        else if (t == "all") r.mask |= KC_ALL;
        a = b + 1;
      }
    }
    return r;
  }();
  return p;
}

struct QkvEpi {   // EPI_QKV destinations
  void* q; void* pk; void* pv;
};

int do_gemm(Ctx& c, int epi, const void* A, int M, int K, const void* B, int N, int silu_half,
            const void* bias, const float* resid, void* out, int ldo, const uint8_t* Bp = nullptr,
            const QkvEpi* qe = nullptr, const ArArgs* ar = nullptr, const void* norm_g = nullptr,
            void* norm_out = nullptr) {
  bullet_handle* h = c.h;
  if (M == 0) return BULLET_OK;
  GemmArgs a;
  memset(&a, 0, sizeof a);
  a.M = M; a.N = N; a.K = K; a.epi = epi; a.silu_half = silu_half; a.bias = bias;
  a.resid = resid; a.ldo = ldo;
  if (epi == EPI_SILU) a.out_t = out; else a.out_f32 = (float*)out;
  if (epi == EPI_QKV) {
    if (!qe || h->cfg.head_dim != 128 || h->cfg.dtype != BULLET_DTYPE_BF16)
      return set_err(BULLET_EUNSUPPORTED, "EPI_QKV: bf16, head_dim 128 only");
    a.q_out = qe->q; a.pool_k = qe->pk; a.pool_v = qe->pv; a.cs = h->rope_cs; a.tok = h->ph[c.phase].tok;
    a.H = h->cfg.n_heads; a.Hkv = h->cfg.n_kv_heads; a.kvB = h->block_size;
  }
  int rc = next_launch(c, &a.L);
  if (rc) return rc;
  if (norm_out) {   // fused RMSNorm in the GEMM tail: row-block counters + a row counter
    PhaseWS& P = h->ph[c.phase];
    if (c.op || epi != EPI_RESID || h->cfg.dtype != BULLET_DTYPE_BF16)
      return set_err(BULLET_EINVAL, "fused norm: bf16 step GEMMs with EPI_RESID only");
    if (P.next_ctr >= P.n_counters || P.next_rbc >= P.n_rbc_slices)
      return set_err(BULLET_ENOMEM, "work counters exhausted");
    a.nf.g = norm_g; a.nf.out = norm_out; a.nf.eps = h->cfg.rms_eps;
    {   // rows per claim: about one claim per SM of the partition, at most 4
      const int per = (M + c.m_sms - 1) / std::max(1, c.m_sms);
      a.nf.rows = per >= 4 ? 4 : per >= 2 ? 2 : 1;
    }
    a.nf.unit_ctr = P.counters + P.next_ctr++;
    a.nf.rb_ctr = P.rbc + (size_t)P.next_rbc++ * P.max_rb;
  }
  if (ar) {   // fused peer all-reduce (bf16 only, checked at create): its own unit counter
    PhaseWS& P = h->ph[c.phase];
    if (c.op || epi != EPI_F32) return set_err(BULLET_EINVAL, "fused all-reduce: step GEMMs with EPI_F32 only");
    if (P.next_ctr >= P.n_counters) return set_err(BULLET_ENOMEM, "work counters exhausted");
    a.ar = *ar;
    a.ar.ctr = P.counters + P.next_ctr++;
  }
  if (h->cfg.dtype == BULLET_DTYPE_FP32) {
    if (K % 16) return set_err(BULLET_EUNSUPPORTED, "fp32 GEMM needs K %% 16 == 0");
    a.bn = 64; a.mh = 1; a.n_full = 0; a.band = 1;
    no_pdl(a.L);
    LAUNCH(c, launch_gemm_simt<float>((const float*)A, (const float*)B, a, h->n_sms * 4, c.st));
    return BULLET_OK;
  }
  if (K % 64) return set_err(BULLET_EUNSUPPORTED, "GEMM needs K %% 64 == 0 (K=%d)", K);
  // packed B needs 64-row aligned halves: SiLU tiles of >= 128 rows
  auto fits = [&](int bn) {
    if (Bp && epi == EPI_SILU && bn < 128) return false;
    if (epi == EPI_QKV) return bn % 128 == 0 && N % bn == 0;   // tiles hold whole heads
    return epi == EPI_SILU ? ((N / 2) % (bn / 2) == 0 && N % 2 == 0) : (N % bn == 0);
  };
  // Plan (mh, bn, work split) on the phase's m SMs.  A k-block step of a
  // tile costs max(bytes streamed / per-SM copy bandwidth, MMA flops / per-SM
  // tensor rate); whole tiles fill full waves of the partition; the ragged
  // remainder (for decode-sized GEMMs: every tile) is either run as whole
  // tiles (a partly idle last wave) or streamed over K in m equal ranges
  // (stream-K: every SM streams the same k-blocks, partial tiles pay an fp32
  // partial round trip and a fixup that reads the tile's other segments
  // through one SM).  A single accumulator stage (mh * bn > 256 columns)
  // exposes the epilogue.  mh = 2 only for decode-sized M.  Rates: KI2 and
  // the per-CTA traces.
  // FL_SM: the per-SM bf16 rate a decode-sized tile sustains (9 TF/s: 256-row units at M = 256 measured
  // 7-9 % slower than two 128-row tiles, scripts/decode_gemm_plans.py, profiles/r02_decode_gemm_plans.log)
  constexpr double BW_SM = 110e9, FL_SM = 9.0e12, EPI_BW = 100e9, T0 = 0.6e-6;
  const int k_blocks = K / 64;
  const size_t pf = h->ph[c.phase].partial_floats;
  int mh = 1, bn = 0, n_full = 0, sk_tiles = 0, sk_chunks = 0;
  double best = 1e300;
  // mh = 1 is tried first and mh = 2 pays 5 %: with the warp-wide issue,
  // 128 x 256 tiles measured 10-13 % faster than the 256-row units the model
  // ranked equal or better at M = 256 (profiles/r02_decode_gemm_plans_v2.log)
  for (int cmh = 1; cmh <= ((M > 128 && M <= 512) ? 2 : 1); ++cmh) {
    const double pen = cmh == 2 ? 1.05 : 1.0;
    const int m_tiles = (M + 128 * cmh - 1) / (128 * cmh);
    for (int cand : {256, 128, 64}) {
      if (!fits(cand)) continue;
      const int tiles = m_tiles * (N / cand);
      const double out_b = 128.0 * cmh * cand * 4.0;
      const double t_kb = std::max((cmh * 16384.0 + cand * 128.0) / BW_SM, 2.0 * 128 * cmh * cand * 64 / FL_SM);
      const double t_tile = k_blocks * t_kb + (2 * cmh * cand > 512 ? out_b / EPI_BW : 0.0) + T0;
      const double cost_a = pen * std::ceil((double)tiles / c.m_sms) * t_tile;   // whole tiles only
      if (cost_a < best * 0.999) { best = cost_a; mh = cmh; bn = cand; n_full = tiles; sk_tiles = 0; sk_chunks = 0; }
      const int fw = tiles / c.m_sms, rem = tiles % c.m_sms;
      if (rem == 0) continue;
      const int chunks = std::min({c.m_sms, rem * k_blocks, 15 * rem});   // <= 16 segments per tile
      if ((size_t)2 * chunks * 128 * cmh * cand > pf || rem > N_TILE_SEMS) continue;
      // fixup phase (measured by the per-CTA traces): ~6 us to
      // store the partials and reach the phase, then ~4 us per round of
      // items (an item = 32 output columns x 128 rows of one streamed tile)
      const int items = rem * cmh * ((epi == EPI_QKV || epi == EPI_SILU) ? cand / 64 : cand / 32);
      const double cost_b = pen * (fw * t_tile + (double)rem * k_blocks / chunks * t_kb + T0 + 6e-6 +
                                   std::ceil((double)items / c.m_sms) * 4e-6);
      if (cost_b < best * 0.999) {
        best = cost_b; mh = cmh; bn = cand; n_full = fw * c.m_sms; sk_tiles = rem; sk_chunks = chunks;
      }
    }
  }
  if (!bn) return set_err(BULLET_EUNSUPPORTED, "GEMM N=%d not tileable", N);
  char kenv[32];   // per kernel kind (experiments): BULLET_GEMM_PLAN_K<kind>, prefill phase only: ..._K<kind>P
  const char* ov = nullptr;
  if (c.phase == 0) {
    snprintf(kenv, sizeof kenv, "BULLET_GEMM_PLAN_K%dP", c.kind);
    ov = getenv(kenv);
  }
  if (!ov) {
    snprintf(kenv, sizeof kenv, "BULLET_GEMM_PLAN_K%d", c.kind);
    ov = getenv(kenv);
  }
  if (!ov) ov = getenv("BULLET_GEMM_PLAN");
  if (ov) {   // experiments: "mh,bn,sk" (sk 1: stream the ragged remainder over K)
    int omh = 0, obn = 0, osk = 0;
    if (sscanf(ov, "%d,%d,%d", &omh, &obn, &osk) == 3 && fits(obn) && omh >= 1 && omh <= 2) {
      const int tiles = ((M + 128 * omh - 1) / (128 * omh)) * (N / obn), rem = tiles % c.m_sms;
      const int chunks = std::min({c.m_sms, rem * k_blocks, 15 * rem});
      if (!osk || !rem) { mh = omh; bn = obn; n_full = tiles; sk_tiles = 0; sk_chunks = 0; }
      else if ((size_t)2 * chunks * 128 * omh * obn <= pf && rem <= N_TILE_SEMS) {
        mh = omh; bn = obn; n_full = tiles - rem; sk_tiles = rem; sk_chunks = chunks;
      }
    }
  }
  int kcb = 0;
  {   // two-level accumulation (DESIGN R-4e): every tile's K range in chunks
      // of <= kc, each accumulated in TMEM, the chunks summed in IEEE fp32 in
      // a fixed order.  It brings the tcgen05 accumulation error (truncating,
      // 4.3e-6 relative per long-K GEMM) near IEEE fp32, which the layer needs
      // to stay under the north-star bar at d_model >= 5120 (R-4e).  Applied
      // by GEMM kind (kc_policy); on-chip (the epilogue sums the chunks in
      // registers, tile 128 x 128) unless BULLET_GEMM_KCHUNK_MODE=splitk
      // (chunks summed by the split-K fixup through global memory).
    const KcPolicy& kp = kc_policy();
    const int kc = kp.kc_override >= 0 ? kp.kc_override : (h->cfg.d_model >= 5120 ? KC_DEFAULT : 0);
    int kind = c.kind;
    if (c.op) kind = epi == EPI_QKV ? BULLET_K_QKV : epi == EPI_SILU ? BULLET_K_GATE_UP : -1;
    const bool sel = kind >= 0 ? ((kp.mask >> kind) & 1u) != 0 : kp.mask == KC_ALL;
    if (kc >= 64 && K > kc && sel) {
      bool done = false;
      const int kcb_ = std::max(1, kc / 64);
      if (kp.splitk) {   // every tile's K range streamed in ranges of <= kc, summed by the fixup
        const int tiles = ((M + 128 * mh - 1) / (128 * mh)) * (N / bn);
        const long long Ts = (long long)tiles * k_blocks;
        const int chunks = (int)((Ts + kcb_ - 1) / kcb_);
        // every range must get its own partial: when they do not fit
        // (prefill-sized M) fall through to the on-chip mode instead of
        // silently running fewer, longer ranges
        if ((size_t)2 * chunks * 128 * mh * bn <= h->ph[c.phase].partial_floats && tiles <= N_TILE_SEMS &&
            (k_blocks + kcb_ - 1) / kcb_ + 1 <= 16 && Ts * chunks < (1ll << 31)) {
          n_full = 0; sk_tiles = tiles; sk_chunks = chunks; done = true;
        }
      }
      if (!done && fits(128)) {
        mh = 1; bn = 128; sk_tiles = 0; sk_chunks = 0;
        n_full = ((M + 127) / 128) * (N / 128);
        kcb = kcb_;
      }
    }
  }
  if (getenv("BULLET_GEMM_DEBUG"))
    fprintf(stderr, "gemm M=%d N=%d K=%d m_sms=%d -> mh=%d bn=%d n_full=%d sk_tiles=%d sk_chunks=%d kcb=%d\n", M, N,
            K, c.m_sms, mh, bn, n_full, sk_tiles, sk_chunks, kcb);
  a.bn = bn; a.mh = mh; a.n_full = n_full; a.sk_tiles = sk_tiles; a.sk_chunks = sk_chunks; a.kcb = kcb;
  {   // second copy issuer for the weight tiles (BULLET_GEMM_SPLIT_B=0/1 overrides; default: on)
    static const int sb = getenv("BULLET_GEMM_SPLIT_B") ? atoi(getenv("BULLET_GEMM_SPLIT_B")) : 1;
    a.split_b = sb ? 1 : 0;
  }
  {  // rasterisation band: the activations of a band stay L2-resident (evict-last)
     // while every weight tile streams past them once per band: a band of
     // <= BULLET_GEMM_BAND_MB (default 64; co-run step vs 32 / 128 MB: config 2
     // 2.919 vs 2.968 / 2.922 ms, config 3 7.144 vs 7.201 / 7.272 ms) MB of activations
    static const double band_all =
        (getenv("BULLET_GEMM_BAND_MB") ? atof(getenv("BULLET_GEMM_BAND_MB")) : 64.0) * 1e6;
    char benv[40];   // per kernel kind (experiments): BULLET_GEMM_BAND_MB_K<kind>
    snprintf(benv, sizeof benv, "BULLET_GEMM_BAND_MB_K%d", c.kind);   // (one M tile in decode: no effect)
    const double band_bytes = getenv(benv) ? atof(getenv(benv)) * 1e6 : band_all;
    const int m_tiles = (M + 128 * mh - 1) / (128 * mh);
    const double a_tile = 128.0 * mh * K * 2;
    const int n_bands = std::max(1, (int)std::ceil(m_tiles * a_tile / band_bytes));
    a.band = std::max(1, (m_tiles + n_bands - 1) / n_bands);   // equal bands
  }
  a.b_packed = Bp;
  {   // epilogue-input L2 prefetch (BULLET_GEMM_EPI_PF=0 disables, A/B) and diagnostics
    static const int epf = getenv("BULLET_GEMM_EPI_PF") ? atoi(getenv("BULLET_GEMM_EPI_PF")) : 1;
    static const int edbg = getenv("BULLET_GEMM_EPI_DBG") ? atoi(getenv("BULLET_GEMM_EPI_DBG")) : 0;
    static const int ecoal = getenv("BULLET_GEMM_EPI_COAL") ? atoi(getenv("BULLET_GEMM_EPI_COAL")) : 1;
    a.epi_pf = epf; a.epi_dbg = edbg; a.epi_coal = ecoal;
  }
  {   // L2 prefetch distance of the weight stream (experiments; BULLET_GEMM_PF k-blocks)
    static const int pf = getenv("BULLET_GEMM_PF") ? atoi(getenv("BULLET_GEMM_PF")) : 0;
    a.b_pf = pf;
  }
  a.b_evict_first = ((M + 128 * mh - 1) / (128 * mh)) == 1;   // weights reused by no other M tile
  a.b_rows = N + (epi == EPI_SILU ? silu_half - N / 2 : 0);
  a.partials = h->ph[c.phase].partials;
  a.tile_sems = h->ph[c.phase].tile_sems;
  a.sk_parity = h->ph[c.phase].sk_parity;
  h->ph[c.phase].sk_parity ^= 1;   // every GEMM launch zeroes the slice the next one counts in
  if (sk_tiles) {   // the stream-K fixup phase's item counter
    if (c.op) {
      a.fix_ctr = h->op_ctr + 2;
    } else {
      PhaseWS& P = h->ph[c.phase];
      if (P.next_ctr >= P.n_counters) return set_err(BULLET_ENOMEM, "work counters exhausted");
      a.fix_ctr = P.counters + P.next_ctr++;
    }
  }
  CUtensorMap ma, mb;
  if ((rc = make_map(&ma, A, M, K, 128))) return rc;   // one 128-row half per TMA box
  if ((rc = make_map(&mb, B, N, K, bn / 2))) return rc;
  LAUNCH(c, launch_gemm_tc(ma, mb, a, persist_grid(c, 1), c.st));
  return BULLET_OK;
}

// Grid of the row-per-CTA kernels: all SMs (gated-out CTAs exit at once), at
// most 8 CTAs per SM and no more per SM than the partition has rows for —
// small decode batches would otherwise spend the kernel churning through
// CTAs that find no row left to claim.
int row_grid(const Ctx& c, int rows) {
  const int per_sm = std::max(1, std::min(8, (rows + c.m_sms - 1) / std::max(1, c.m_sms)));
  return c.h->n_sms * per_sm;
}

int do_rmsnorm(Ctx& c, const float* x, int n, const void* g, void* out) {
  if (n == 0) return BULLET_OK;
  NormArgs a;
  a.x = x; a.g = g; a.out = out; a.n = n; a.d = c.h->cfg.d_model; a.eps = c.h->cfg.rms_eps;
  int rc = next_launch(c, &a.L);
  if (rc) return rc;
  no_pdl(a.L);
  // one CTA per row (BULLET_NORM=warp: warp per row — measured slower, 9.6 -> 24 us
  // for 128 decode rows on 68 SMs: the per-warp row loads are latency-bound)
  static const bool warp = getenv("BULLET_NORM") && !strcmp(getenv("BULLET_NORM"), "warp");
  if (!warp) {
    if (c.h->cfg.dtype == BULLET_DTYPE_FP32) LAUNCH(c, launch_rmsnorm<float>(a, row_grid(c, n), c.st));
    else LAUNCH(c, launch_rmsnorm<__nv_bfloat16>(a, row_grid(c, n), c.st));
    return BULLET_OK;
  }
  const int per_sm = std::max(1, std::min(8, (n + 8 * c.m_sms - 1) / (8 * std::max(1, c.m_sms))));
  if (c.h->cfg.dtype == BULLET_DTYPE_FP32) LAUNCH(c, launch_rmsnorm_warp<float>(a, c.h->n_sms * per_sm, c.st));
  else LAUNCH(c, launch_rmsnorm_warp<__nv_bfloat16>(a, c.h->n_sms * per_sm, c.st));
  return BULLET_OK;
}

int do_rope(Ctx& c, const bullet_batch* b, int layer, const float* qkv, void* q) {
  bullet_handle* h = c.h;
  if (b->n_tokens == 0) return BULLET_OK;
  RopeArgs a;
  a.qkv = qkv; a.q_out = q; a.pool_k = h->pk[layer]; a.pool_v = h->pv[layer]; a.cs = h->rope_cs;
  a.cu = b->d_cu_seqlens; a.ctx = b->d_ctx_lens; a.bt = b->d_block_table;
  a.n_reqs = b->n_reqs; a.max_blocks = b->max_blocks_per_req; a.n_tok = b->n_tokens;
  a.H = h->cfg.n_heads; a.Hkv = h->cfg.n_kv_heads; a.hd = h->cfg.head_dim; a.B = h->block_size;
  a.max_pos = h->cfg.max_position;
  int rc = next_launch(c, &a.L);
  if (rc) return rc;
  no_pdl(a.L);
  if (h->cfg.dtype == BULLET_DTYPE_FP32) LAUNCH(c, launch_rope_kv<float>(a, row_grid(c, b->n_tokens), c.st));
  else LAUNCH(c, launch_rope_kv<__nv_bfloat16>(a, row_grid(c, b->n_tokens), c.st));
  return BULLET_OK;
}

int max_qlen(const bullet_batch* b) {
  int mq = 0;
  for (int r = 0; r < b->n_reqs; ++r) mq = std::max(mq, b->h_cu_seqlens[r + 1] - b->h_cu_seqlens[r]);
  return mq;
}

int max_kv(const bullet_batch* b) {
  int mk = 0;
  for (int r = 0; r < b->n_reqs; ++r)
    mk = std::max(mk, b->h_ctx_lens[r] + b->h_cu_seqlens[r + 1] - b->h_cu_seqlens[r]);
  return mk;
}

// Mixed (chunked-prefill hybrid) batch: leading requests with q > 1, then
// only requests with q <= 1.  Returns the number of leading requests (0 when
// the batch is not mixed) and their token count in *t0.
int mixed_split(const bullet_batch* b, int* t0) {
  int r0 = 0;
  while (r0 < b->n_reqs && b->h_cu_seqlens[r0 + 1] - b->h_cu_seqlens[r0] > 1) ++r0;
  if (r0 == 0 || r0 == b->n_reqs) return 0;
  for (int r = r0; r < b->n_reqs; ++r)
    if (b->h_cu_seqlens[r + 1] - b->h_cu_seqlens[r] > 1) return 0;
  *t0 = b->h_cu_seqlens[r0];
  return *t0 < b->n_tokens ? r0 : 0;
}

// TMA maps of the layer's K / V pool for the tcgen05 prefill attention: the
// pool [blocks][Hkv][16][128] bf16 viewed as [blocks * Hkv * 16][128], boxes
// of 16 rows (one block of one head) x 64 dims, 128-byte swizzle (the UMMA
// operand layout).  BULLET_PF5_TMA=0 keeps every tile on cp.async (A/B).
static int pf5_maps(bullet_handle* h, int layer, AttnArgs* a, CUtensorMap* mk, CUtensorMap* mv, CUtensorMap* mq) {
  static const int on = getenv("BULLET_PF5_TMA") ? atoi(getenv("BULLET_PF5_TMA")) : 1;
  memset(mk, 0, sizeof *mk);
  memset(mv, 0, sizeof *mv);
  memset(mq, 0, sizeof *mq);
  a->kv_tma = on && h->block_size == 16;
  if (!a->kv_tma) return BULLET_OK;
  const long long rows = (long long)h->n_blocks * h->cfg.n_kv_heads * 16;
  if (rows >= (1ll << 31)) { a->kv_tma = 0; return BULLET_OK; }
  int rc = make_map(mk, h->pk[layer], (int)rows, 128, 16);
  if (!rc) rc = make_map(mv, h->pv[layer], (int)rows, 128, 16);
  if (rc) return rc;
  // q [T][H][128] bf16: box {64 dims, 1 head, 128 tokens}
  cuuint64_t dims[3] = {128, (cuuint64_t)a->H, (cuuint64_t)a->n_tok};
  cuuint64_t strides[2] = {128 * 2, (cuuint64_t)a->H * 128 * 2};
  cuuint32_t box[3] = {64, 1, 128};
  cuuint32_t es[3] = {1, 1, 1};
  CUresult r = g_encode(mq, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void*>(a->q), dims, strides, box, es,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_err(BULLET_ECUDA, "cuTensorMapEncodeTiled (q) failed (%d)", (int)r);
  return BULLET_OK;
}

// K / V maps of the decode attention's stream (the same pool view and boxes as
// pf5_maps); BULLET_DEC_TMA=0 keeps the cp.async stream (A/B).
static int dec_maps(bullet_handle* h, int layer, AttnArgs* a, CUtensorMap* mk, CUtensorMap* mv, bool force = false) {
  static const int on = getenv("BULLET_DEC_TMA") ? atoi(getenv("BULLET_DEC_TMA")) : 1;
  memset(mk, 0, sizeof *mk);
  memset(mv, 0, sizeof *mv);
  a->kv_tma = (on || force) && h->block_size == 16;
  if (!a->kv_tma) return BULLET_OK;
  const long long rows = (long long)h->n_blocks * h->cfg.n_kv_heads * 16;
  if (rows >= (1ll << 31)) { a->kv_tma = 0; return BULLET_OK; }
  int rc = make_map(mk, h->pk[layer], (int)rows, 128, 16);
  return rc ? rc : make_map(mv, h->pv[layer], (int)rows, 128, 16);
}

// BULLET_DEC_KERNEL=5 selects the tcgen05 decode attention (attn_decode5.cu;
// bf16, head_dim 128, block 16, GQA groups <= 8) instead of the default
// mma.sync kernel (attn_decode.cu): parity-green but measured slower on
// partitions (its 64 KB stages are held through the whole
// S -> softmax -> PV chain, so fewer bytes stay in flight per SM).
static bool use_decode5(bullet_handle* h) {
  static const int k = getenv("BULLET_DEC_KERNEL") ? atoi(getenv("BULLET_DEC_KERNEL")) : 3;
  const int grp = h->cfg.n_heads / std::max(1, h->cfg.n_kv_heads);
  return k == 5 && h->cfg.dtype == BULLET_DTYPE_BF16 && h->cfg.head_dim == 128 && h->block_size == 16 && grp <= 8 &&
         (long long)h->n_blocks * h->cfg.n_kv_heads * 16 < (1ll << 31);
}

int do_attention(Ctx& c, const bullet_batch* b, int layer, const void* q, void* o, int kind) {
  bullet_handle* h = c.h;
  if (b->n_tokens == 0) return BULLET_OK;
  AttnArgs a;
  memset(&a, 0, sizeof a);
  a.kv_chunks = 1;
  static const int dec_pf = getenv("BULLET_DEC_PF") ? atoi(getenv("BULLET_DEC_PF")) : 0;
  a.dec_pf = dec_pf;
  a.q = q; a.o = o; a.pool_k = h->pk[layer]; a.pool_v = h->pv[layer];
  a.cu = b->d_cu_seqlens; a.ctx = b->d_ctx_lens; a.bt = b->d_block_table;
  a.n_reqs = b->n_reqs; a.max_blocks = b->max_blocks_per_req; a.n_tok = b->n_tokens;
  a.H = h->cfg.n_heads; a.Hkv = h->cfg.n_kv_heads; a.hd = h->cfg.head_dim; a.B = h->block_size;
  a.scale = (float)(1.0 / std::sqrt((double)a.hd));
  static const int dbg = getenv("BULLET_DBG") ? atoi(getenv("BULLET_DBG")) : 0;
  a.dbg = dbg;
  const bool bf16 = h->cfg.dtype == BULLET_DTYPE_BF16;
  int t0 = 0;
  const int r0 = (kind == 0 && !c.op && bf16 && a.hd == 128) ? mixed_split(b, &t0) : 0;
  if (r0) {   // hybrid batch: tcgen05 FA over the prefill chunks, decode kernel over the rest
    for (int r = r0; r < b->n_reqs; ++r)
      if (b->h_ctx_lens[r] + 1 > attn_decode_max_blocks() * h->block_size)
        return set_err(BULLET_EUNSUPPORTED, "hybrid batch: decode context too long");
    PhaseWS& P = h->ph[c.phase];
    a.tiles = P.tiles; a.n_tiles = P.n_tiles;   // the plan listed tiles of requests [0, r0) only
    CUtensorMap mk, mv, mq;
    int rc = pf5_maps(h, layer, &a, &mk, &mv, &mq);
    if (rc) return rc;
    if ((rc = next_launch(c, &a.L))) return rc;
    LAUNCH(c, launch_attn_prefill5(mk, mv, mq, a, persist_grid(c, attn_prefill5_ctas_per_sm(a.H, a.Hkv)), c.st));
    AttnArgs d = a;
    d.tok_base = t0;
    d.order = P.order_ok ? P.order : nullptr;
    const bool d5 = use_decode5(h);
    if ((rc = dec_maps(h, layer, &d, &mk, &mv, d5))) return rc;
    if ((rc = next_launch(c, &d.L))) return rc;
    if (d5) LAUNCH(c, launch_attn_decode5(mk, mv, d, persist_grid(c, 1), c.st));
    else LAUNCH(c, launch_attn_decode_tc(mk, mv, d, persist_grid(c, 1), c.m_sms <= 100 ? 4 : 1, c.st));
    return BULLET_OK;
  }
  if (kind == 0) kind = (bf16 && a.hd == 128) ? (max_qlen(b) > 1 ? 4 : 3) : 1;
  if (kind == 3 && use_decode5(h)) {   // tcgen05 decode attention (any context length: no KV chunks)
    CUtensorMap mk, mv;
    int rc = dec_maps(h, layer, &a, &mk, &mv, true);
    if (rc) return rc;
    if ((rc = next_launch(c, &a.L))) return rc;
    if (!c.op && h->ph[c.phase].order_ok) a.order = h->ph[c.phase].order;
    LAUNCH(c, launch_attn_decode5(mk, mv, a, persist_grid(c, 1), c.st));
    return BULLET_OK;
  }
  if (kind == 3) {
    if (!bf16 || a.hd != 128)
      return set_err(BULLET_EUNSUPPORTED, "tensor-core decode attention: bf16, hd 128 only");
    // contexts longer than one unit's block window are split over KV chunks
    // (partial softmax states merged in chunk order, attn_decode.cu)
    const int span = attn_decode_max_blocks() * h->block_size;
    a.kv_chunks = std::max(1, (max_kv(b) + span - 1) / span);
    if (a.kv_chunks > 1) {
      PhaseWS& P = h->ph[1];   // the decode phase owns the split scratch
      if (!P.kv_part || a.kv_chunks > P.kv_cap || b->n_tokens > P.max_tok)
        return set_err(BULLET_EUNSUPPORTED, "decode attention: context %d needs %d KV chunks (capacity %d, "
                       "from max_position)", max_kv(b), a.kv_chunks, P.kv_cap);
      a.kv_part = P.kv_part; a.kv_tick = P.kv_tick;
    }
    CUtensorMap mk, mv;
    int rc = dec_maps(h, layer, &a, &mk, &mv);
    if (rc) return rc;
    if ((rc = next_launch(c, &a.L))) return rc;
    // four consumer groups of 3 warps per SM on partitions (68 SMs: 78.6 vs
    // 72.3 GB/s/SM with two groups at 1k contexts), one on the full GPU (tail
    // balance) — scripts/attn_dec_bench.py, DESIGN.md §5
    if (!c.op && h->ph[c.phase].order_ok) a.order = h->ph[c.phase].order;
    LAUNCH(c, launch_attn_decode_tc(mk, mv, a, persist_grid(c, 1), c.m_sms <= 100 ? 4 : 1, c.st));
    return BULLET_OK;
  }
  if (kind == 2 || kind == 4) {
    if (!bf16 || a.hd != 128) return set_err(BULLET_EUNSUPPORTED, "tensor-core attention: bf16, hd 128 only");
    PhaseWS& P = h->ph[c.phase];
    a.tiles = P.tiles; a.n_tiles = P.n_tiles;
    if (c.op) {  // op-level: plan the tile list now
      PlanArgs pa{nullptr, 0, b->d_cu_seqlens, b->n_reqs, ATTN_TC_BQ, b->n_reqs, P.tiles, P.n_tiles,
                  nullptr, nullptr, nullptr, 0, 0, 0};
      prof_begin(c);
      LAUNCH(c, launch_plan(pa, c.st));
    }
    CUtensorMap mk, mv, mq;
    int rc = kind == 4 ? pf5_maps(h, layer, &a, &mk, &mv, &mq) : 0;
    if (rc) return rc;
    if ((rc = next_launch(c, &a.L))) return rc;
    if (kind == 4) LAUNCH(c, launch_attn_prefill5(mk, mv, mq, a, persist_grid(c, attn_prefill5_ctas_per_sm(a.H, a.Hkv)), c.st));
    else LAUNCH(c, launch_attn_prefill_tc(a, persist_grid(c, 2), c.st));
    return BULLET_OK;
  }
  int rc = next_launch(c, &a.L);
  if (rc) return rc;
  no_pdl(a.L);
  if (bf16) LAUNCH(c, launch_attn_simt<__nv_bfloat16>(a, h->n_sms * 4, c.st));
  else LAUNCH(c, launch_attn_simt<float>(a, h->n_sms * 4, c.st));
  return BULLET_OK;
}

int allreduce(Ctx& c, float* buf, size_t count) {
  bullet_handle* h = c.h;
  prof_begin(c);
  ncclResult_t r = g_nccl.allReduce(buf, buf, count, ncclFloat32, ncclSum, h->comm[c.phase], c.st);
  if (r != ncclSuccess) return set_err(BULLET_ENCCL, "ncclAllReduce: %s", g_nccl.errStr(r));
  prof_end(c);
  return BULLET_OK;
}

// All-reduce arguments of a phase's row-parallel GEMM: every rank's partial
// buffer `buf`, hidden and counters (PEER mode, connected).
ArArgs make_ar(const bullet_handle* h, int phase, int buf) {
  ArArgs r;
  memset(&r, 0, sizeof r);
  const SymLayout L = sym_layout(h->cfg, phase);
  r.n = h->cfg.tp_size; r.rank = h->cfg.tp_rank; r.max_rb = L.max_rb;
  for (int s = 0; s < r.n; ++s) {
    uint8_t* b = h->peer_base[s];
    r.part[s] = reinterpret_cast<float*>(b + L.part[buf]);
    r.hid[s] = reinterpret_cast<float*>(b + L.hid);
    r.ready[s] = reinterpret_cast<unsigned long long*>(b + L.ready);
    r.done[s] = reinterpret_cast<unsigned long long*>(b + L.done);
  }
  r.base = reinterpret_cast<unsigned long long*>(h->sym + L.base);
  r.err = reinterpret_cast<int*>(h->sym + L.err);
  return r;
}

// One decoder layer of one phase (DESIGN.md §2 steps S1-S9).
int run_layer(Ctx& c, const bullet_batch* b, int layer) {
  bullet_handle* h = c.h;
  PhaseWS& P = h->ph[c.phase];
  const bullet_layer_weights& w = h->w[layer];
  const bullet_model_cfg& cf = h->cfg;
  const int n = b->n_tokens, d = cf.d_model, H = cf.n_heads, Hkv = cf.n_kv_heads, hd = cf.head_dim;
  const int I = cf.d_ff, nq = (H + 2 * Hkv) * hd;
  const bool tp = cf.tp_size > 1, lead = cf.tp_rank == 0;
  int rc;
  c.layer = layer;
  c.kind = BULLET_K_RMSNORM1;
  // S1 — already done by the previous layer's down GEMM when the norm is fused
  if (!(c.fuse_norm && layer > b->layer_begin) && (rc = do_rmsnorm(c, b->d_hidden, n, w.g_attn, P.h)))
    return rc;
  c.kind = BULLET_K_QKV;
  const bullet_handle::Packed* wp = h->wp.empty() ? nullptr : &h->wp[layer];
  if (c.fuse_qkv) {   // S2 + S3: RoPE and the KV append in the QKV epilogue
    const QkvEpi qe{P.q, h->pk[layer], h->pv[layer]};
    if ((rc = do_gemm(c, EPI_QKV, P.h, n, d, w.w_qkv, nq, 0, w.b_qkv, nullptr, nullptr, nq,
                      wp ? wp->qkv : nullptr, &qe))) return rc;
  } else {
    if ((rc = do_gemm(c, EPI_F32, P.h, n, d, w.w_qkv, nq, 0, w.b_qkv, nullptr, P.qkv, nq,
                      wp ? wp->qkv : nullptr))) return rc;  // S2
    c.kind = BULLET_K_ROPE_KV;
    if ((rc = do_rope(c, b, layer, P.qkv, P.q))) return rc;                                  // S3
  }
  c.kind = BULLET_K_ATTN;
  if ((rc = do_attention(c, b, layer, P.q, P.o, 0))) return rc;                             // S4
  // S5: x1 = x + o W_o^T.  Under TP (NCCL) the non-lead ranks write their
  // partial into hidden and the fp32 all-reduce restores x + sum of partials
  // (S9); in PEER mode the GEMM writes its partial to the symmetric buffer
  // and reduces in the same kernel (NEXT-2).
  c.kind = BULLET_K_OPROJ;
  if (h->peer_mode) {
    const ArArgs ar = make_ar(h, c.phase, 0);
    if ((rc = do_gemm(c, EPI_F32, P.o, n, H * hd, w.w_o, d, 0, nullptr, nullptr, ar.part[ar.rank], d,
                      wp ? wp->o : nullptr, nullptr, &ar))) return rc;
  } else {
    const bool fn = c.fuse_norm && !tp;   // S5 + S6: RMSNorm in the O-proj GEMM's tail
    if ((rc = do_gemm(c, (!tp || lead) ? EPI_RESID : EPI_F32, P.o, n, H * hd, w.w_o, d, 0, nullptr,
                      b->d_hidden, b->d_hidden, d, wp ? wp->o : nullptr, nullptr, nullptr,
                      fn ? w.g_mlp : nullptr, fn ? P.h : nullptr))) return rc;
    c.kind = BULLET_K_ALLREDUCE;
    if (tp && (rc = allreduce(c, b->d_hidden, (size_t)n * d))) return rc;
  }
  c.kind = BULLET_K_RMSNORM2;
  if (!(c.fuse_norm && !tp && !h->peer_mode) && (rc = do_rmsnorm(c, b->d_hidden, n, w.g_mlp, P.h)))
    return rc;                                                                                // S6
  c.kind = BULLET_K_GATE_UP;
  if ((rc = do_gemm(c, EPI_SILU, P.h, n, d, w.w_gate_up, 2 * I, I, nullptr, nullptr, P.act, I,
                    wp ? wp->gu : nullptr))) return rc;  // S7
  c.kind = BULLET_K_DOWN;
  if (h->peer_mode) {   // S8 + S9 fused (partial buffer 1: consecutive all-reduces alternate)
    const ArArgs ar = make_ar(h, c.phase, 1);
    return do_gemm(c, EPI_F32, P.act, n, I, w.w_down, d, 0, nullptr, nullptr, ar.part[ar.rank], d,
                   wp ? wp->down : nullptr, nullptr, &ar);
  }
  // S8 (+ the next layer's S1 in the GEMM tail when the norm is fused)
  const bool fn = c.fuse_norm && !tp && layer + 1 < b->layer_end;
  if ((rc = do_gemm(c, (!tp || lead) ? EPI_RESID : EPI_F32, P.act, n, I, w.w_down, d, 0, nullptr,
                    b->d_hidden, b->d_hidden, d, wp ? wp->down : nullptr, nullptr, nullptr,
                    fn ? h->w[layer + 1].g_attn : nullptr, fn ? P.h : nullptr))) return rc;
  c.kind = BULLET_K_ALLREDUCE;
  if (tp && (rc = allreduce(c, b->d_hidden, (size_t)n * d))) return rc;
  return BULLET_OK;
}

int validate_batch(const bullet_handle* h, const bullet_batch* b, int phase) {
  const char* nm = phase == 0 ? "prefill" : "decode";
  if (b->n_reqs < 0 || b->n_tokens < 0) return set_err(BULLET_EINVAL, "%s: negative sizes", nm);
  if (b->n_tokens == 0) return BULLET_OK;
  if (!b->h_cu_seqlens || !b->h_ctx_lens || !b->d_cu_seqlens || !b->d_ctx_lens ||
      !b->d_block_table || !b->d_hidden)
    return set_err(BULLET_EINVAL, "%s: null pointer in batch", nm);
  if (b->h_cu_seqlens[0] != 0 || b->h_cu_seqlens[b->n_reqs] != b->n_tokens)
    return set_err(BULLET_EINVAL, "%s: cu_seqlens must run 0..n_tokens", nm);
  if (b->n_tokens > h->ph[phase].max_tok)
    return set_err(BULLET_ENOMEM, "%s: %d tokens > max %d", nm, b->n_tokens, h->ph[phase].max_tok);
  if (h->peer_mode) {
    if (!h->peer_connected) return set_err(BULLET_EINVAL, "PEER mode: bullet_tp_connect first");
    if ((const uint8_t*)b->d_hidden != h->sym + sym_layout(h->cfg, phase).hid)
      return set_err(BULLET_EINVAL, "%s: PEER mode needs the symmetric hidden (bullet_tp_hidden)", nm);
  }
  if (b->layer_begin < 0 || b->layer_end > h->cfg.n_layers || b->layer_begin > b->layer_end)
    return set_err(BULLET_EINVAL, "%s: layer range [%d,%d)", nm, b->layer_begin, b->layer_end);
  for (int l = b->layer_begin; l < b->layer_end; ++l)
    if (!h->w_set[l]) return set_err(BULLET_EINVAL, "%s: weights of layer %d not set", nm, l);
  if (b->max_blocks_per_req <= 0) return set_err(BULLET_EINVAL, "%s: max_blocks_per_req", nm);
  for (int r = 0; r < b->n_reqs; ++r) {
    const int q = b->h_cu_seqlens[r + 1] - b->h_cu_seqlens[r], cx = b->h_ctx_lens[r];
    if (q < 0 || cx < 0) return set_err(BULLET_EINVAL, "%s: request %d negative length", nm, r);
    if (q == 0) continue;
    if (cx + q > b->max_blocks_per_req * h->block_size)
      return set_err(BULLET_EKV, "%s: request %d needs %d tokens > block table %d", nm, r, cx + q,
                     b->max_blocks_per_req * h->block_size);
    if (cx + q > h->cfg.max_position)
      return set_err(BULLET_EINVAL, "%s: request %d position %d >= max_position", nm, r, cx + q - 1);
    if (b->h_block_table) {
      const int nb = (cx + q + h->block_size - 1) / h->block_size;
      for (int i = 0; i < nb; ++i) {
        const int blk = b->h_block_table[(size_t)r * b->max_blocks_per_req + i];
        if (blk < 0 || blk >= h->n_blocks)
          return set_err(BULLET_EKV, "%s: request %d block %d id %d out of [0,%d)", nm, r, i, blk, h->n_blocks);
      }
    }
  }
  return BULLET_OK;
}

int run_phase(Ctx& c, const bullet_batch* b) {
  PhaseWS& P = c.h->ph[c.phase];
  P.next_ctr = 0;
  P.next_rbc = 0;
  const bool tc_attn = c.h->cfg.dtype == BULLET_DTYPE_BF16 && c.h->cfg.head_dim == 128 && max_qlen(b) > 1;
  int t0 = 0;
  const int r0 = tc_attn ? mixed_split(b, &t0) : 0;
  PlanArgs pa{P.counters, P.n_counters, b->d_cu_seqlens, b->n_reqs, ATTN_TC_BQ, r0 ? r0 : b->n_reqs,
              tc_attn ? P.tiles : nullptr, P.n_tiles,
              c.fuse_qkv ? P.tok : nullptr, b->d_ctx_lens, b->d_block_table, b->max_blocks_per_req,
              c.h->block_size, b->n_tokens, P.rbc, P.n_rbc_slices * P.max_rb, nullptr, 0};
  // LPT order of the decode rows (pure decode batch, or the decode tail of a hybrid one)
  static const bool no_order = getenv("BULLET_DEC_ORDER") && !strcmp(getenv("BULLET_DEC_ORDER"), "0");
  P.order_ok = !no_order && c.h->cfg.dtype == BULLET_DTYPE_BF16 && c.h->cfg.head_dim == 128 &&
               (r0 > 0 || max_qlen(b) == 1) && b->n_tokens > 0;
  if (P.order_ok) { pa.order = P.order; pa.order_base = r0 ? t0 : 0; }
  c.kind = BULLET_K_PLAN;
  c.layer = -1;
  prof_begin(c);
  LAUNCH(c, launch_plan(pa, c.st));
  for (int l = b->layer_begin; l < b->layer_end; ++l) {
    int rc = run_layer(c, b, l);
    if (rc) return rc;
  }
  return BULLET_OK;
}

}  // namespace

// ================================================================== C ABI
extern "C" {

const char* bullet_last_error(void) { return g_err.c_str(); }

int bullet_nccl_unique_id(void* out128) {
  if (!out128) return set_err(BULLET_EINVAL, "null");
  if (!g_nccl.load()) return set_err(BULLET_ENCCL, "libnccl.so.2 not loadable: %s", dlerror());
  ncclUniqueId id;
  ncclResult_t r = g_nccl.getUniqueId(&id);
  if (r != ncclSuccess) return set_err(BULLET_ENCCL, "ncclGetUniqueId: %s", g_nccl.errStr(r));
  memcpy(out128, &id, sizeof id);
  return BULLET_OK;
}

int bullet_create(const bullet_model_cfg* cfg, const bullet_kv_pool* pool, const void* nccl_uids,
                  const char* perf_params_json, bullet_handle** out) {
  if (!cfg || !pool || !out) return set_err(BULLET_EINVAL, "null argument");
  *out = nullptr;
  const bullet_model_cfg& c = *cfg;
  if (c.n_layers <= 0 || c.d_model <= 0 || c.n_heads <= 0 || c.n_kv_heads <= 0 || c.head_dim <= 0 ||
      c.d_ff <= 0 || c.n_heads % c.n_kv_heads || c.max_position <= 0 || c.tp_size <= 0 ||
      c.tp_rank < 0 || c.tp_rank >= c.tp_size || c.max_prefill_tokens < 0 || c.max_decode_tokens < 0)
    return set_err(BULLET_EINVAL, "invalid model cfg");
  if (c.dtype != BULLET_DTYPE_BF16 && c.dtype != BULLET_DTYPE_FP32)
    return set_err(BULLET_EINVAL, "dtype");
  if (c.d_model % 64 || c.d_ff % 64 || (c.n_heads * c.head_dim) % 64 ||
      ((c.n_heads + 2 * c.n_kv_heads) * c.head_dim) % 64)
    return set_err(BULLET_EUNSUPPORTED, "dims must be multiples of 64");
  if (c.head_dim != 128 && c.head_dim != 64) return set_err(BULLET_EUNSUPPORTED, "head_dim 64/128");
  if (c.n_heads / c.n_kv_heads > 8) return set_err(BULLET_EUNSUPPORTED, "GQA group > 8");
  if (pool->block_size != 16) return set_err(BULLET_EUNSUPPORTED, "block_size must be 16");
  if (pool->n_blocks <= 0 || !pool->d_k || !pool->d_v) return set_err(BULLET_EINVAL, "kv pool");
  if (c.tp_size > 1 && !nccl_uids) {   // PEER mode: fused all-reduce over peer memory
    if (c.dtype != BULLET_DTYPE_BF16) return set_err(BULLET_EUNSUPPORTED, "fused all-reduce: bf16 only");
    if (c.tp_size > AR_MAX_RANKS) return set_err(BULLET_EUNSUPPORTED, "fused all-reduce: tp_size <= %d", AR_MAX_RANKS);
    if (c.d_model % (4 * c.tp_size)) return set_err(BULLET_EUNSUPPORTED, "fused all-reduce: d_model %% (4 tp) != 0");
  }

  int dev;
  CK(cudaGetDevice(&dev));
  cudaDeviceProp prop;
  CK(cudaGetDeviceProperties(&prop, dev));
  if (prop.major != 10) return set_err(BULLET_EUNSUPPORTED, "needs an sm_100 (Blackwell) GPU, got sm_%d%d", prop.major, prop.minor);
  int rc = get_encode();
  if (rc) return rc;
  for (auto pre : {preload_attn_decode, preload_attn_decode5, preload_attn_prefill5, preload_attn_tc, preload_attn_simt,
                   preload_elementwise, preload_gemm_tc, preload_stream}) {
    cudaError_t e = pre();
    if (e != cudaSuccess) return set_err(BULLET_ECUDA, "kernel preload: %s", cudaGetErrorString(e));
  }

  bullet_handle* h = new bullet_handle();
  h->cfg = c;
  h->dev = dev;
  h->n_sms = prop.multiProcessorCount;
  h->elt = c.dtype == BULLET_DTYPE_BF16 ? 2 : 4;
  h->w.resize(c.n_layers);
  h->w_set.assign(c.n_layers, 0);
  h->n_blocks = pool->n_blocks;
  h->block_size = pool->block_size;
  for (int l = 0; l < c.n_layers; ++l) {
    if (!pool->d_k[l] || !pool->d_v[l]) { delete h; return set_err(BULLET_EINVAL, "pool layer %d null", l); }
    h->pk.push_back(pool->d_k[l]);
    h->pv.push_back(pool->d_v[l]);
  }
  auto fail = [&](int code) { bullet_destroy(h); return code; };

  // ---- SM probe (KI1): the live %smid set, sorted (TPC pairs adjacent)
  {
    const int n = h->n_sms * 16;
    int* d_ids = nullptr;
    if (cudaMalloc(&d_ids, n * sizeof(int)) != cudaSuccess) return fail(set_err(BULLET_ENOMEM, "probe"));
    std::vector<int> ids(n);
    cudaError_t e = launch_probe(d_ids, n, 0);
    if (e == cudaSuccess) e = cudaMemcpy(ids.data(), d_ids, n * sizeof(int), cudaMemcpyDeviceToHost);
    cudaFree(d_ids);
    if (e != cudaSuccess) return fail(set_err(BULLET_ECUDA, "SM probe: %s", cudaGetErrorString(e)));
    std::set<int> s(ids.begin(), ids.end());
    h->sigma.assign(s.begin(), s.end());
    if ((int)h->sigma.size() != h->n_sms || h->sigma.back() >= 256)
      return fail(set_err(BULLET_ECUDA, "SM probe found %zu of %d SMs (max id %d)", h->sigma.size(),
                          h->n_sms, h->sigma.empty() ? -1 : h->sigma.back()));
  }
  // ---- die probe (KI1b) and the order of sigma (SURVEY §8a SG)
  {
    constexpr int NL = 64, STRIDE = 2048;   // lines 2 KB apart: the L2's die interleave grain
    void* lines = nullptr;
    uint32_t* d_lat = nullptr;
    std::vector<uint32_t> lat((size_t)256 * NL, 0);
    cudaError_t e = cudaMalloc(&lines, (size_t)NL * STRIDE);
    if (e == cudaSuccess) e = cudaMalloc(&d_lat, lat.size() * sizeof(uint32_t));
    if (e == cudaSuccess) e = cudaMemset(lines, 0, (size_t)NL * STRIDE);
    if (e == cudaSuccess) e = cudaMemset(d_lat, 0, lat.size() * sizeof(uint32_t));
    if (e == cudaSuccess) e = launch_die_probe(lines, NL, STRIDE, d_lat, h->n_sms * 4, 0);
    if (e == cudaSuccess) e = cudaMemcpy(lat.data(), d_lat, lat.size() * sizeof(uint32_t), cudaMemcpyDeviceToHost);
    cudaFree(lines); cudaFree(d_lat);
    if (e != cudaSuccess) return fail(set_err(BULLET_ECUDA, "die probe: %s", cudaGetErrorString(e)));
    h->die.assign(256, -1);
    // the lines near the first SM (below its median latency) vs the rest: an SM
    // on the same die sees the near set faster, one on the other die slower
    const int s0 = h->sigma[0];
    std::vector<uint32_t> l0(lat.begin() + (size_t)s0 * NL, lat.begin() + (size_t)(s0 + 1) * NL);
    std::vector<uint32_t> srt = l0;
    std::sort(srt.begin(), srt.end());
    const uint32_t med = srt[NL / 2];
    bool ok = srt[NL - 1] > srt[0];
    for (int sm : h->sigma) {
      double near = 0, far = 0;
      int nn = 0, nf = 0;
      for (int j = 0; j < NL; ++j) {
        const uint32_t v = lat[(size_t)sm * NL + j];
        if (!v) { ok = false; break; }
        if (l0[j] < med) { near += v; ++nn; } else { far += v; ++nf; }
      }
      if (!ok || !nn || !nf) { ok = false; break; }
      h->die[sm] = near / nn < far / nf ? 0 : 1;
    }
    if (!ok) std::fill(h->die.begin(), h->die.end(), -1);
    // order: BULLET_SIGMA=sorted (smid order) | die (die 0's TPCs, then die 1's:
    // a prefill range of <= 74 SMs stays on one die) | interleave (alternate
    // dies TPC by TPC: both ranges span both dies).  TPC pairs stay adjacent.
    const char* pol = getenv("BULLET_SIGMA");
    const std::string policy = pol ? pol : SIGMA_DEFAULT;
    if (ok && policy != "sorted") {
      std::vector<int> pairs[2];
      for (size_t i = 0; i + 1 < h->sigma.size(); i += 2) pairs[h->die[h->sigma[i]]].push_back((int)i);
      std::vector<int> order;
      if (policy == "die") {
        for (int d = 0; d < 2; ++d) for (int i : pairs[d]) order.push_back(i);
      } else {   // interleave
        for (size_t k = 0; k < std::max(pairs[0].size(), pairs[1].size()); ++k)
          for (int d = 0; d < 2; ++d) if (k < pairs[d].size()) order.push_back(pairs[d][k]);
      }
      std::vector<int> sig;
      for (int i : order) { sig.push_back(h->sigma[i]); sig.push_back(h->sigma[i + 1]); }
      if (h->sigma.size() % 2) sig.push_back(h->sigma.back());
      h->sigma = sig;
    }
  }

  // ---- RoPE (cos, sin) table, computed in fp64 then stored fp32
  {
    const int half = c.head_dim / 2;
    std::vector<double> inv(half);
    for (int i = 0; i < half; ++i) {
      double f = std::pow(c.rope_theta, -2.0 * i / c.head_dim);
      if (c.rope_llama3) {  // llama3 band rescaling (public Llama-3.1 config)
        const double L = c.rope_orig_max_pos, wl = 2.0 * M_PI / f;
        const double hi_w = L / c.rope_high_freq, lo_w = L / c.rope_low_freq;
        if (wl > lo_w) f /= c.rope_factor;
        else if (wl >= hi_w) {
          const double sm = (L / wl - c.rope_low_freq) / (c.rope_high_freq - c.rope_low_freq);
          f = (1.0 - sm) * f / c.rope_factor + sm * f;
        }
      }
      inv[i] = f;
    }
    std::vector<float2> cs((size_t)c.max_position * half);
    for (int p = 0; p < c.max_position; ++p)
      for (int i = 0; i < half; ++i) {
        const double t = (double)p * inv[i];
        cs[(size_t)p * half + i] = make_float2((float)std::cos(t), (float)std::sin(t));
      }
    if (cudaMalloc(&h->rope_cs, cs.size() * sizeof(float2)) != cudaSuccess ||
        cudaMemcpy(h->rope_cs, cs.data(), cs.size() * sizeof(float2), cudaMemcpyHostToDevice) != cudaSuccess)
      return fail(set_err(BULLET_ENOMEM, "rope table"));
  }

  // ---- per-phase workspace
  const int nq = (c.n_heads + 2 * c.n_kv_heads) * c.head_dim;
  for (int p = 0; p < 2; ++p) {
    PhaseWS& P = h->ph[p];
    P.max_tok = p == 0 ? c.max_prefill_tokens : c.max_decode_tokens;
    const size_t T = std::max(1, P.max_tok);
    P.n_counters = 32 * c.n_layers + 32;
    P.partial_floats = (size_t)2 * h->n_sms * 128 * 256;
    bool ok = cudaMalloc(&P.qkv, T * nq * sizeof(float)) == cudaSuccess &&
              cudaMalloc(&P.q, T * c.n_heads * c.head_dim * h->elt) == cudaSuccess &&
              cudaMalloc(&P.o, T * c.n_heads * c.head_dim * h->elt) == cudaSuccess &&
              cudaMalloc(&P.h, T * c.d_model * h->elt) == cudaSuccess &&
              cudaMalloc(&P.act, T * c.d_ff * h->elt) == cudaSuccess &&
              cudaMalloc(&P.partials, P.partial_floats * sizeof(float)) == cudaSuccess &&
              cudaMalloc(&P.tile_sems, 2 * N_TILE_SEMS * sizeof(int)) == cudaSuccess &&
              cudaMalloc(&P.counters, P.n_counters * sizeof(int)) == cudaSuccess &&
              cudaMalloc(&P.tiles, (T / ATTN_TC_BQ + T + 1) * sizeof(int2)) == cudaSuccess &&
              cudaMalloc(&P.n_tiles, sizeof(int)) == cudaSuccess &&
              cudaMalloc(&P.tok, T * sizeof(TokInfo)) == cudaSuccess &&
              cudaMalloc(&P.order, T * sizeof(int4)) == cudaSuccess &&
              cudaMalloc(&P.rbc, (size_t)(2 * c.n_layers + 2) * ((T + 127) / 128) * sizeof(int)) == cudaSuccess;
    P.max_rb = (int)((T + 127) / 128);
    P.n_rbc_slices = 2 * c.n_layers + 2;
    if (!ok) return fail(set_err(BULLET_ENOMEM, "workspace allocation (phase %d)", p));
    if (p == 1 && c.dtype == BULLET_DTYPE_BF16 && c.head_dim == 128) {   // split-KV decode attention scratch
      const int span = attn_decode_max_blocks() * pool->block_size;
      P.kv_cap = std::max(1, (c.max_position + span - 1) / span);
      if (P.kv_cap > 1) {
        const size_t units = T * c.n_kv_heads;
        if (cudaMalloc(&P.kv_part, units * P.kv_cap * 8 * 130 * sizeof(float)) != cudaSuccess ||
            cudaMalloc(&P.kv_tick, units * sizeof(int)) != cudaSuccess ||
            cudaMemset(P.kv_tick, 0, units * sizeof(int)) != cudaSuccess)
          return fail(set_err(BULLET_ENOMEM, "split-KV scratch"));
      }
    }
    cudaMemset(P.tile_sems, 0, 2 * N_TILE_SEMS * sizeof(int));
    cudaMemset(P.counters, 0, P.n_counters * sizeof(int));
  }
  if (cudaMalloc(&h->op_ctr, 4 * sizeof(int)) != cudaSuccess) return fail(set_err(BULLET_ENOMEM, "op ctr"));
  if (cudaMalloc(&h->gate_fallbacks, sizeof(int)) != cudaSuccess ||
      cudaMemset(h->gate_fallbacks, 0, sizeof(int)) != cudaSuccess)
    return fail(set_err(BULLET_ENOMEM, "gate fallback counter"));
  if (cudaMalloc(&h->d_gates, 2 * sizeof(Gate)) != cudaSuccess) return fail(set_err(BULLET_ENOMEM, "gates"));
  {   // default device split: everything to decode (bullet_set_split overwrites)
    const Gate all = gate_of(h, 0, h->n_sms);
    if (cudaMemcpy(h->d_gates, &all, sizeof all, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(h->d_gates + 1, &all, sizeof all, cudaMemcpyHostToDevice) != cudaSuccess)
      return fail(set_err(BULLET_ECUDA, "gates init"));
  }
  if (cudaEventCreateWithFlags(&h->ev_ts, cudaEventDisableTiming) != cudaSuccess)
    return fail(set_err(BULLET_ECUDA, "event"));
  if (cudaDeviceSynchronize() != cudaSuccess) return fail(set_err(BULLET_ECUDA, "init sync"));

  // ---- performance model parameters
  h->perf.set_default(h->n_sms);
  if (perf_params_json) {
    std::string err;
    if (!h->perf.parse(perf_params_json, &err)) return fail(set_err(BULLET_EINVAL, "%s", err.c_str()));
  }

  // ---- fused peer all-reduce: the symmetric region (zeroed counters)
  if (c.tp_size > 1 && !nccl_uids) {
    h->peer_mode = true;
    h->sym_bytes = sym_layout(c, 1).end;
    if (cudaMalloc(&h->sym, h->sym_bytes) != cudaSuccess) return fail(set_err(BULLET_ENOMEM, "symmetric region"));
    if (cudaMemset(h->sym, 0, h->sym_bytes) != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess)
      return fail(set_err(BULLET_ECUDA, "symmetric region init"));
  }
  // ---- tensor parallelism: one communicator per phase (concurrent streams)
  if (c.tp_size > 1 && nccl_uids) {
    if (!g_nccl.load()) return fail(set_err(BULLET_ENCCL, "libnccl.so.2 not loadable"));
    for (int p = 0; p < 2; ++p) {
      ncclUniqueId id;
      memcpy(&id, (const char*)nccl_uids + 128 * p, sizeof id);
      ncclConfig_t conf = NCCL_CONFIG_INITIALIZER;
      conf.maxCTAs = 16;  // NCCL kernels are not smid-gated: bound their footprint
      ncclResult_t r = g_nccl.commInitRankConfig(&h->comm[p], c.tp_size, id, c.tp_rank, &conf);
      if (r != ncclSuccess) return fail(set_err(BULLET_ENCCL, "ncclCommInitRankConfig: %s", g_nccl.errStr(r)));
    }
  }
  *out = h;
  return BULLET_OK;
}

int bullet_perf_create(const bullet_model_cfg* cfg, int n_sms, const char* json, bullet_handle** out) {
  if (!cfg || !out || n_sms <= 0 || n_sms > 256) return set_err(BULLET_EINVAL, "bad argument");
  if (cfg->n_heads <= 0 || cfg->n_kv_heads <= 0 || cfg->d_model <= 0 || cfg->head_dim <= 0 || cfg->d_ff <= 0)
    return set_err(BULLET_EINVAL, "invalid model cfg");
  bullet_handle* h = new bullet_handle();
  h->cfg = *cfg;
  h->host_only = true;
  h->n_sms = n_sms;
  h->elt = cfg->dtype == BULLET_DTYPE_BF16 ? 2 : 4;
  for (int i = 0; i < n_sms; ++i) h->sigma.push_back(i);
  h->perf.set_default(n_sms);
  if (json) {
    std::string err;
    if (!h->perf.parse(json, &err)) { delete h; return set_err(BULLET_EINVAL, "%s", err.c_str()); }
  }
  *out = h;
  return BULLET_OK;
}

int bullet_set_layer_weights(bullet_handle* h, int layer, const bullet_layer_weights* w) {
  if (!h || !w) return set_err(BULLET_EINVAL, "null");
  if (h->host_only) return set_err(BULLET_EUNSUPPORTED, "host-only handle");
  if (layer < 0 || layer >= h->cfg.n_layers) return set_err(BULLET_EINVAL, "layer %d", layer);
  if (!w->w_qkv || !w->w_o || !w->w_gate_up || !w->w_down || !w->g_attn || !w->g_mlp ||
      (h->cfg.qkv_bias && !w->b_qkv))
    return set_err(BULLET_EINVAL, "null weight pointer");
  h->w[layer] = *w;
  if (h->cfg.dtype == BULLET_DTYPE_BF16) {   // pack the B operands once (kernels.h layout)
    const bullet_model_cfg& c = h->cfg;
    const size_t nq = (size_t)(c.n_heads + 2 * c.n_kv_heads) * c.head_dim, d = c.d_model;
    const size_t hh = (size_t)c.n_heads * c.head_dim, I = c.d_ff;
    const size_t sz[4] = {nq * d * 2, d * hh * 2, 2 * I * d * 2, d * I * 2};
    if (h->wp.empty()) h->wp.resize(c.n_layers);
    bullet_handle::Packed& P = h->wp[layer];
    if (!P.base && cudaMalloc(&P.base, sz[0] + sz[1] + sz[2] + sz[3]) != cudaSuccess)
      return set_err(BULLET_ENOMEM, "packed weights of layer %d", layer);
    P.qkv = P.base; P.o = P.qkv + sz[0]; P.gu = P.o + sz[1]; P.down = P.gu + sz[2];
    CK(launch_pack_weight((const __nv_bfloat16*)w->w_qkv, (int)nq, (int)d, P.qkv, 0));
    CK(launch_pack_weight((const __nv_bfloat16*)w->w_o, (int)d, (int)hh, P.o, 0));
    CK(launch_pack_weight((const __nv_bfloat16*)w->w_gate_up, (int)(2 * I), (int)d, P.gu, 0));
    CK(launch_pack_weight((const __nv_bfloat16*)w->w_down, (int)d, (int)I, P.down, 0));
    CK(cudaStreamSynchronize(0));
  }
  if (!h->cfg.qkv_bias) h->w[layer].b_qkv = nullptr;
  h->w_set[layer] = 1;
  return BULLET_OK;
}

int bullet_num_sms(const bullet_handle* h, int* n, int* g) {
  if (!h) return set_err(BULLET_EINVAL, "null");
  if (n) *n = h->n_sms;
  if (g) *g = GRAN;
  return BULLET_OK;
}

int bullet_sm_order(const bullet_handle* h, int32_t* out, int cap) {
  if (!h || !out || cap < h->n_sms) return set_err(BULLET_EINVAL, "bad buffer");
  for (int i = 0; i < h->n_sms; ++i) out[i] = h->sigma[i];
  return BULLET_OK;
}

int bullet_sm_dies(const bullet_handle* h, int32_t* out, int cap) {
  if (!h || !out || cap < h->n_sms) return set_err(BULLET_EINVAL, "bad buffer");
  for (int i = 0; i < h->n_sms; ++i) out[i] = h->die.empty() ? -1 : h->die[h->sigma[i]];
  return BULLET_OK;
}

int bullet_gate_fallbacks(bullet_handle* h, long long* n) {
  if (!h || !n) return set_err(BULLET_EINVAL, "null");
  if (h->host_only) { *n = 0; return BULLET_OK; }
  int v = 0;
  CK(cudaMemcpy(&v, h->gate_fallbacks, sizeof v, cudaMemcpyDeviceToHost));
  *n = v;
  return BULLET_OK;
}

int bullet_set_smid_log(bullet_handle* h, int32_t* d_log, int capacity) {
  if (!h) return set_err(BULLET_EINVAL, "null");
  h->log = d_log;
  h->log_cap = d_log ? capacity : 0;
  return BULLET_OK;
}

// Shared body of bullet_step / bullet_step_ranges: prefill claims work on
// sigma[plo, phi), decode on sigma[dlo, dhi) (mode CORUN), else on all SMs.
static int step_impl(bullet_handle* h, const bullet_batch* pre, const bullet_batch* dec, int plo, int phi,
                     int dlo, int dhi, bool dec_paused, int flags, void* s_prefill, void* s_decode) {
  const int N = h->n_sms, mode = flags & 3;
  const bool has_pre = pre && pre->n_tokens > 0, has_dec = dec && dec->n_tokens > 0;
  int rc;
  if (pre && (rc = validate_batch(h, pre, 0))) return rc;
  if (dec && (rc = validate_batch(h, dec, 1))) return rc;
  if (mode == BULLET_CORUN && has_pre && phi <= plo)
    return set_err(BULLET_ESMRANGE, "prefill batch given with an empty prefill SM range");
  const bool run_dec = has_dec && !(mode == BULLET_CORUN && dec_paused);
  if (mode == BULLET_CORUN && run_dec && dhi <= dlo)
    return set_err(BULLET_ESMRANGE, "decode batch given with an empty decode SM range");
  if (h->log_cap == 0 && (flags & BULLET_SMID_LOG)) return set_err(BULLET_EINVAL, "SMID_LOG without a log buffer");
  if ((flags & BULLET_CHECK_KV) && has_pre && has_dec) {   // disjoint block sets
    if (!pre->h_block_table || !dec->h_block_table)
      return set_err(BULLET_EINVAL, "BULLET_CHECK_KV needs host block tables");
    std::vector<char> used(h->n_blocks, 0);
    auto mark = [&](const bullet_batch* b, bool check) -> int {
      for (int r = 0; r < b->n_reqs; ++r) {
        const int q = b->h_cu_seqlens[r + 1] - b->h_cu_seqlens[r];
        if (q == 0) continue;
        const int nb = (b->h_ctx_lens[r] + q + h->block_size - 1) / h->block_size;
        for (int i = 0; i < nb; ++i) {
          const int blk = b->h_block_table[(size_t)r * b->max_blocks_per_req + i];
          if (check && used[blk]) return blk;
          if (!check) used[blk] = 1;
        }
      }
      return -1;
    };
    mark(pre, false);
    const int clash = mark(dec, true);
    if (clash >= 0) return set_err(BULLET_EKV, "KV block %d is used by both a prefill and a decode request", clash);
  }
  const bool log = (flags & BULLET_SMID_LOG) != 0;
  cudaStream_t sp = (cudaStream_t)s_prefill, sd = (cudaStream_t)s_decode;
  const bool prof = (flags & BULLET_PROFILE) != 0;
  Ctx cp{h, 0, mode == BULLET_CORUN ? gate_of(h, plo, phi) : gate_of(h, 0, N),
         mode == BULLET_CORUN ? phi - plo : N, log, sp, false, prof};
  Ctx cd{h, 1, mode == BULLET_CORUN ? gate_of(h, dlo, dhi) : gate_of(h, 0, N),
         mode == BULLET_CORUN ? dhi - dlo : N, log, sd, false, prof};
  if (flags & BULLET_DEVICE_SPLIT) {   // SM sets from bullet_set_split (graph replay follows it)
    if (mode != BULLET_CORUN) return set_err(BULLET_EINVAL, "BULLET_DEVICE_SPLIT: CORUN only");
    cp.gdev = h->d_gates;
    cd.gdev = h->d_gates + 1;
  }
  cp.fuse_qkv = cd.fuse_qkv = !(flags & BULLET_UNFUSED) && h->cfg.dtype == BULLET_DTYPE_BF16 &&
                              h->cfg.head_dim == 128;
  // fused norm pays for decode-sized batches (the standalone kernel's launch
  // and drain dominate there: decode layer-step -1.6 % on 76 SMs); a prefill
  // GEMM's tail runs it with one CTA per SM where the standalone kernel packs
  // several (+0.7 % on a prefill layer) — so only up to 1024 rows
  // never under tensor parallelism: the row-parallel GEMMs' outputs are
  // partials until the all-reduce, so a norm in their tail would read them
  // (and S1 of the next layer would be skipped with nothing replacing it)
  const bool fn_ok = !(flags & BULLET_UNFUSED_NORM) && h->cfg.dtype == BULLET_DTYPE_BF16 && h->cfg.tp_size == 1 &&
                     h->cfg.d_model <= 8192;
  static const int fn_rows = getenv("BULLET_FUSED_NORM_MAX_ROWS") ? atoi(getenv("BULLET_FUSED_NORM_MAX_ROWS")) : 1024;
  cp.fuse_norm = fn_ok && pre && pre->n_tokens <= fn_rows;
  cd.fuse_norm = fn_ok && dec && dec->n_tokens <= fn_rows;
  if (has_pre && (rc = run_phase(cp, pre))) return rc;
  if (run_dec) {
    if (mode == BULLET_TIMESLICED && has_pre) {
      CK(cudaEventRecord(h->ev_ts, sp));
      CK(cudaStreamWaitEvent(sd, h->ev_ts, 0));
    }
    if ((rc = run_phase(cd, dec))) return rc;
  }
  return BULLET_OK;
}

int bullet_step(bullet_handle* h, const bullet_batch* pre, const bullet_batch* dec,
                int prefill_sm_count, int flags, void* s_prefill, void* s_decode) {
  if (!h) return set_err(BULLET_EINVAL, "null handle");
  if (h->host_only) return set_err(BULLET_EUNSUPPORTED, "host-only handle");
  const int N = h->n_sms, p = prefill_sm_count, mode = flags & 3;
  if (mode == 3) return set_err(BULLET_EINVAL, "flags: TIMESLICED and UNGATED are exclusive");
  if (p < 0 || p > N || (p % GRAN && p != N)) return set_err(BULLET_ESMRANGE, "prefill_sm_count %d not in [0,%d] step %d", p, N, GRAN);
  if (mode == BULLET_CORUN && pre && pre->n_tokens > 0 && p == 0)
    return set_err(BULLET_ESMRANGE, "prefill batch given with prefill_sm_count 0");
  return step_impl(h, pre, dec, 0, p, p, N, p == N, flags, s_prefill, s_decode);   // p = N: decode paused
}

int bullet_step_ranges(bullet_handle* h, const bullet_batch* pre, const bullet_batch* dec, int pre_lo, int pre_hi,
                       int dec_lo, int dec_hi, int flags, void* s_prefill, void* s_decode) {
  if (!h) return set_err(BULLET_EINVAL, "null handle");
  if (h->host_only) return set_err(BULLET_EUNSUPPORTED, "host-only handle");
  const int N = h->n_sms, mode = flags & 3;
  if (mode != BULLET_CORUN) return set_err(BULLET_EINVAL, "bullet_step_ranges: CORUN only");
  auto ok = [&](int x) { return x >= 0 && x <= N && (x % GRAN == 0 || x == N); };
  if (!ok(pre_lo) || !ok(pre_hi) || !ok(dec_lo) || !ok(dec_hi) || pre_lo > pre_hi || dec_lo > dec_hi)
    return set_err(BULLET_ESMRANGE, "ranges [%d,%d) [%d,%d) not within [0,%d] on step %d", pre_lo, pre_hi,
                   dec_lo, dec_hi, N, GRAN);
  return step_impl(h, pre, dec, pre_lo, pre_hi, dec_lo, dec_hi, false, flags, s_prefill, s_decode);
}

static PhaseShape model_shape(const bullet_handle* h) {
  PhaseShape s;
  s.d = h->cfg.d_model; s.H = h->cfg.n_heads; s.Hkv = h->cfg.n_kv_heads; s.hd = h->cfg.head_dim;
  s.I = h->cfg.d_ff; s.elt = h->elt;
  return s;
}

int bullet_model_predict(const bullet_handle* h, const bullet_batch_shape* shape, int sm_count,
                         int corun_sm_count, double* t_us) {
  if (!h || !shape || !t_us || shape->n_reqs < 0) return set_err(BULLET_EINVAL, "null");
  if (sm_count <= 0 || sm_count > h->n_sms || corun_sm_count < 0)
    return set_err(BULLET_ESMRANGE, "sm_count %d", sm_count);
  PhaseShape s = model_shape(h);
  for (int i = 0; i < shape->n_reqs; ++i) {
    s.q_lens.push_back(shape->q_lens[i]);
    s.ctx_lens.push_back(shape->ctx_lens[i]);
  }
  *t_us = layer_time(s, h->perf, sm_count, corun_sm_count) * 1e6;
  return BULLET_OK;
}

int bullet_choose_split(const bullet_handle* h, const bullet_sched_state* s, const bullet_slo* slo,
                        int* prefill_sm_count, int* decode_layer_steps) {
  if (!h || !s || !slo || !prefill_sm_count || !decode_layer_steps) return set_err(BULLET_EINVAL, "null");
  if (slo->v_min < 1 || slo->v_min > h->n_sms || slo->percentile <= 0 || slo->percentile > 1)
    return set_err(BULLET_EINVAL, "slo");
  SchedState S;
  S.layers_done = s->layers_done; S.total_layers = s->total_layers;
  for (int i = 0; i < s->n_prefill; ++i) { S.prefill_lens.push_back(s->prefill_lens[i]); S.prefill_waited_ms.push_back(s->prefill_waited_ms[i]); }
  for (int i = 0; i < s->n_pending; ++i) { S.pending_lens.push_back(s->pending_lens[i]); S.pending_waited_ms.push_back(s->pending_waited_ms[i]); }
  for (int i = 0; i < s->n_decode; ++i) { S.decode_tokens.push_back(s->decode_tokens[i]); S.decode_elapsed_ms.push_back(s->decode_elapsed_ms[i]); }
  S.decode_mean_ctx = s->decode_mean_ctx;
  S.u_k = s->u_k; S.v_k = s->v_k;
  if (slo->objective < 0 || slo->objective > 2) return set_err(BULLET_EINVAL, "slo objective");
  Slo sl{slo->ttft_norm_ms_per_tok, slo->tpot_ms, slo->w_max, slo->v_min, slo->percentile, slo->objective};
  PerfParams P = h->perf;
  P.M = h->n_sms;
  choose_split(P, model_shape(h), S, sl, GRAN, prefill_sm_count, decode_layer_steps);
  return BULLET_OK;
}

int bullet_get_colocation(const bullet_handle* h, double* p_c, double* p_b) {
  if (!h || !p_c || !p_b) return set_err(BULLET_EINVAL, "null");
  *p_c = h->perf.p_c; *p_b = h->perf.p_b;
  return BULLET_OK;
}

int bullet_get_phase_scale(const bullet_handle* h, double* pre, double* dec) {
  if (!h || !pre || !dec) return set_err(BULLET_EINVAL, "null");
  *pre = h->perf.scale_pre; *dec = h->perf.scale_dec;
  return BULLET_OK;
}

int bullet_set_phase_scale(bullet_handle* h, double pre, double dec) {
  if (!h || !(pre > 0.0) || !(dec > 0.0)) return set_err(BULLET_EINVAL, "phase scales must be > 0");
  h->perf.scale_pre = pre; h->perf.scale_dec = dec;
  return BULLET_OK;
}

int bullet_set_colocation(bullet_handle* h, double p_c, double p_b) {
  if (!h || !(p_c > 0.0) || !(p_b > 0.0)) return set_err(BULLET_EINVAL, "co-location factors must be > 0");
  h->perf.p_c = p_c; h->perf.p_b = p_b;
  return BULLET_OK;
}

int bullet_profile_read(bullet_handle* h, int32_t* kind, int32_t* phase, int32_t* layer, float* ms,
                        int cap, int* n) {
  if (!h || !n || cap < 0) return set_err(BULLET_EINVAL, "null");
  *n = 0;
  for (const auto& r : h->prof_recs) {
    if (*n >= cap) break;
    CK(cudaEventSynchronize(r.e1));
    float t = 0.f;
    CK(cudaEventElapsedTime(&t, r.e0, r.e1));
    if (kind) kind[*n] = r.kind;
    if (phase) phase[*n] = r.phase;
    if (layer) layer[*n] = r.layer;
    if (ms) ms[*n] = t;
    ++*n;
  }
  h->prof_recs.clear();
  h->ev_used = 0;
  return BULLET_OK;
}

int bullet_launch_count(const bullet_handle* h, long long* n) {
  if (!h || !n) return set_err(BULLET_EINVAL, "null");
  *n = h->n_launch;
  return BULLET_OK;
}

int bullet_trace_enable(bullet_handle* h, int max_launches) {
  if (!h || max_launches < 0) return set_err(BULLET_EINVAL, "bad argument");
  if (h->host_only) return set_err(BULLET_EUNSUPPORTED, "host-only handle");
  CK(cudaDeviceSynchronize());
  cudaFree(h->trace);
  h->trace = nullptr; h->trace_cap = h->trace_n = 0;
  h->trace_meta.clear();
  if (max_launches == 0) return BULLET_OK;
  const size_t bytes = (size_t)max_launches * BULLET_TRACE_CTAS * TRACE_SLOTS * sizeof(unsigned long long);
  if (cudaMalloc(&h->trace, bytes) != cudaSuccess) return set_err(BULLET_ENOMEM, "trace buffer (%zu bytes)", bytes);
  CK(cudaMemset(h->trace, 0, bytes));
  h->trace_cap = max_launches;
  h->trace_meta.assign((size_t)4 * max_launches, 0);
  return BULLET_OK;
}

int bullet_trace_read(bullet_handle* h, uint64_t* rec, int32_t* meta, int cap, int* n) {
  if (!h || !n || cap < 0 || (cap > 0 && (!rec || !meta))) return set_err(BULLET_EINVAL, "bad argument");
  *n = 0;
  if (!h->trace) return BULLET_OK;
  CK(cudaDeviceSynchronize());
  const int k = std::min(cap, h->trace_n);
  const size_t per = (size_t)BULLET_TRACE_CTAS * TRACE_SLOTS;
  CK(cudaMemcpy(rec, h->trace, (size_t)k * per * sizeof(unsigned long long), cudaMemcpyDeviceToHost));
  memcpy(meta, h->trace_meta.data(), (size_t)k * 4 * sizeof(int32_t));
  *n = k;
  CK(cudaMemset(h->trace, 0, (size_t)h->trace_cap * per * sizeof(unsigned long long)));
  h->trace_n = 0;
  return BULLET_OK;
}

int bullet_sync(bullet_handle* h) {
  if (!h) return set_err(BULLET_EINVAL, "null");
  if (h->host_only) return BULLET_OK;
  CK(cudaDeviceSynchronize());
  if (h->peer_mode)
    for (int p = 0; p < 2; ++p) {
      int e = 0;
      CK(cudaMemcpy(&e, h->sym + sym_layout(h->cfg, p).err, sizeof e, cudaMemcpyDeviceToHost));
      if (e) return set_err(BULLET_ENCCL, "fused all-reduce (phase %d): a peer did not arrive within 20 s", p);
    }
  return BULLET_OK;
}

void bullet_destroy(bullet_handle* h) {
  if (!h) return;
  if (h->host_only) { delete h; return; }
  cudaDeviceSynchronize();
  for (int p = 0; p < 2; ++p) {
    PhaseWS& P = h->ph[p];
    cudaFree(P.qkv); cudaFree(P.q); cudaFree(P.o); cudaFree(P.h); cudaFree(P.act);
    cudaFree(P.partials); cudaFree(P.tile_sems); cudaFree(P.counters); cudaFree(P.tiles);
    cudaFree(P.n_tiles); cudaFree(P.tok); cudaFree(P.rbc); cudaFree(P.order); cudaFree(P.kv_part); cudaFree(P.kv_tick);
    if (h->comm[p] && g_nccl.commDestroy) g_nccl.commDestroy(h->comm[p]);
  }
  for (void* p : h->ipc_opened) cudaIpcCloseMemHandle(p);
  cudaFree(h->sym);
  cudaFree(h->trace);
  cudaFree(h->rope_cs);
  for (auto& P : h->wp) cudaFree(P.base);
  cudaFree(h->op_pack);
  cudaFree(h->op_ctr);
  cudaFree(h->gate_fallbacks);
  cudaFree(h->d_gates);
  if (h->ev_ts) cudaEventDestroy(h->ev_ts);
  for (auto e : h->ev_pool) cudaEventDestroy(e);
  delete h;
}

int bullet_set_split(bullet_handle* h, int pre_lo, int pre_hi, int dec_lo, int dec_hi, void* stream) {
  if (!h) return set_err(BULLET_EINVAL, "null handle");
  if (h->host_only) return set_err(BULLET_EUNSUPPORTED, "host-only handle");
  const int N = h->n_sms;
  auto ok = [&](int x) { return x >= 0 && x <= N && (x % GRAN == 0 || x == N); };
  if (!ok(pre_lo) || !ok(pre_hi) || !ok(dec_lo) || !ok(dec_hi) || pre_lo > pre_hi || dec_lo > dec_hi)
    return set_err(BULLET_ESMRANGE, "ranges [%d,%d) [%d,%d) not within [0,%d] on step %d", pre_lo, pre_hi,
                   dec_lo, dec_hi, N, GRAN);
  CK(launch_set_gates(h->d_gates, gate_of(h, pre_lo, pre_hi), gate_of(h, dec_lo, dec_hi), (cudaStream_t)stream));
  return BULLET_OK;
}

// ------------------------------------------------ fused peer all-reduce setup
int bullet_tp_base(const bullet_handle* h, void** base) {
  if (!h || !base) return set_err(BULLET_EINVAL, "null");
  if (!h->peer_mode) return set_err(BULLET_EINVAL, "not in PEER mode (tp_size > 1, nccl_uids NULL)");
  *base = h->sym;
  return BULLET_OK;
}

int bullet_tp_ipc_handle(const bullet_handle* h, void* out64) {
  if (!h || !out64) return set_err(BULLET_EINVAL, "null");
  if (!h->peer_mode) return set_err(BULLET_EINVAL, "not in PEER mode");
  cudaIpcMemHandle_t m;
  CK(cudaIpcGetMemHandle(&m, h->sym));
  static_assert(sizeof m == 64, "cudaIpcMemHandle_t is 64 bytes");
  memcpy(out64, &m, sizeof m);
  return BULLET_OK;
}

int bullet_tp_connect(bullet_handle* h, void* const* bases) {
  if (!h || !bases) return set_err(BULLET_EINVAL, "null");
  if (!h->peer_mode) return set_err(BULLET_EINVAL, "not in PEER mode");
  const int n = h->cfg.tp_size;
  if (bases[h->cfg.tp_rank] != h->sym) return set_err(BULLET_EINVAL, "bases[tp_rank] is not this handle's region");
  for (int s = 0; s < n; ++s)
    if (!bases[s]) return set_err(BULLET_EINVAL, "null base of rank %d", s);
  h->peer_base.assign(n, nullptr);
  for (int s = 0; s < n; ++s) h->peer_base[s] = (uint8_t*)bases[s];
  h->peer_connected = true;
  return BULLET_OK;
}

int bullet_tp_connect_ipc(bullet_handle* h, const void* handles) {
  if (!h || !handles) return set_err(BULLET_EINVAL, "null");
  if (!h->peer_mode) return set_err(BULLET_EINVAL, "not in PEER mode");
  const int n = h->cfg.tp_size;
  std::vector<void*> bases(n, nullptr);
  for (int s = 0; s < n; ++s) {
    if (s == h->cfg.tp_rank) { bases[s] = h->sym; continue; }
    cudaIpcMemHandle_t m;
    memcpy(&m, (const char*)handles + 64 * s, sizeof m);
    void* p = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&p, m, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) return set_err(BULLET_ECUDA, "cudaIpcOpenMemHandle (rank %d): %s", s, cudaGetErrorString(e));
    h->ipc_opened.push_back(p);
    bases[s] = p;
  }
  return bullet_tp_connect(h, bases.data());
}

int bullet_tp_hidden(const bullet_handle* h, int phase, float** hidden) {
  if (!h || !hidden || phase < 0 || phase > 1) return set_err(BULLET_EINVAL, "bad argument");
  if (!h->peer_mode) return set_err(BULLET_EINVAL, "not in PEER mode");
  *hidden = reinterpret_cast<float*>(h->sym + sym_layout(h->cfg, phase).hid);
  return BULLET_OK;
}

// ---------------------------------------------------------- op-level entries
static int op_ctx(bullet_handle* h, int lo, int hi, void* stream, Ctx* c) {
  if (!h) return set_err(BULLET_EINVAL, "null handle");
  if (h->host_only) return set_err(BULLET_EUNSUPPORTED, "host-only handle");
  if (lo < 0 || hi > h->n_sms || lo >= hi) return set_err(BULLET_ESMRANGE, "range [%d,%d)", lo, hi);
  *c = Ctx{h, 0, gate_of(h, lo, hi), hi - lo, h->log_cap > 0, (cudaStream_t)stream, true};
  return BULLET_OK;
}

int bullet_op_gemm(bullet_handle* h, int epi, const void* A, int M, int K, const void* B, int N,
                   int silu_half, const void* bias, const float* resid, void* out, int lo, int hi,
                   void* stream) {
  Ctx c;
  int rc = op_ctx(h, lo, hi, stream, &c);
  if (rc) return rc;
  const bool packed = (epi & BULLET_GEMM_PACKED) != 0;
  epi &= ~BULLET_GEMM_PACKED;
  if (!A || !B || !out || M < 0 || K <= 0 || N <= 0 || epi < 0 || epi > 2) return set_err(BULLET_EINVAL, "gemm args");
  if (epi == EPI_RESID && !resid) return set_err(BULLET_EINVAL, "resid null");
  if (epi == EPI_SILU && (N % 2 || silu_half < N / 2)) return set_err(BULLET_EINVAL, "silu layout");
  const int ldo = epi == EPI_SILU ? N / 2 : N;
  const uint8_t* Bp = nullptr;
  if (packed) {   // pack B into scratch first (the layout bullet_step uses)
    if (h->cfg.dtype != BULLET_DTYPE_BF16) return set_err(BULLET_EUNSUPPORTED, "packed GEMM is bf16");
    const int rows = epi == EPI_SILU ? silu_half + N / 2 : N;
    const size_t need = (size_t)rows * K * 2;
    if (need > h->op_pack_bytes) {
      cudaFree(h->op_pack);
      h->op_pack = nullptr; h->op_pack_bytes = 0;
      if (cudaMalloc(&h->op_pack, need) != cudaSuccess) return set_err(BULLET_ENOMEM, "pack scratch");
      h->op_pack_bytes = need;
    }
    CK(launch_pack_weight((const __nv_bfloat16*)B, rows, K, h->op_pack, c.st));
    Bp = h->op_pack;
  }
  return do_gemm(c, epi, A, M, K, B, N, silu_half, bias, resid, out, ldo, Bp);
}

int bullet_op_stream(bullet_handle* h, const void* src, size_t bytes, int mode, int lo, int hi,
                     void* stream) {
  Ctx c;
  int rc = op_ctx(h, lo, hi, stream, &c);
  if (rc) return rc;
  if (!src || bytes == 0 || (mode & 0xff) > 8 || mode < 0) return set_err(BULLET_EINVAL, "stream args");
  StreamArgs a;
  memset(&a, 0, sizeof a);
  a.src = (const uint8_t*)src; a.bytes = bytes; a.mode = mode & 0xff; a.param = (mode >> 8) & 0xff;
  a.wrap = (mode >> 16) ? ((size_t)1 << (mode >> 16)) - 1 : ~(size_t)0;   // window 2^(mode >> 16) bytes
  a.sink = (uint32_t*)h->op_ctr;
  if ((rc = next_launch(c, &a.L))) return rc;
  LAUNCH(c, launch_stream(a, h->n_sms, c.st));
  return BULLET_OK;
}

int bullet_op_stream_mc(bullet_handle* h, const void* src, size_t bytes, int mc, int n_ctas, void* stream) {
  if (!h || !src || n_ctas < 2 || bytes == 0) return set_err(BULLET_EINVAL, "stream_mc args");
  if (h->host_only) return set_err(BULLET_EUNSUPPORTED, "host-only handle");
  CK(launch_stream_mc((const uint8_t*)src, bytes, mc, n_ctas, (uint32_t*)h->op_ctr, (cudaStream_t)stream));
  return BULLET_OK;
}

int bullet_op_rmsnorm(bullet_handle* h, const float* x, int n, const void* g, void* out, int lo,
                      int hi, void* stream) {
  Ctx c;
  int rc = op_ctx(h, lo, hi, stream, &c);
  if (rc) return rc;
  if (!x || !g || !out || n < 0) return set_err(BULLET_EINVAL, "rmsnorm args");
  return do_rmsnorm(c, x, n, g, out);
}

int bullet_op_rope_kv(bullet_handle* h, const bullet_batch* b, int layer, const float* qkv, void* q,
                      int lo, int hi, void* stream) {
  Ctx c;
  int rc = op_ctx(h, lo, hi, stream, &c);
  if (rc) return rc;
  if (!b || !qkv || !q || layer < 0 || layer >= h->cfg.n_layers) return set_err(BULLET_EINVAL, "rope args");
  bullet_batch bb = *b;
  bb.layer_begin = layer; bb.layer_end = layer;
  if ((rc = validate_batch(h, &bb, 0))) return rc;
  return do_rope(c, b, layer, qkv, q);
}

int bullet_op_attention(bullet_handle* h, const bullet_batch* b, int layer, const void* q, void* o,
                        int kind, int lo, int hi, void* stream) {
  Ctx c;
  int rc = op_ctx(h, lo, hi, stream, &c);
  if (rc) return rc;
  if (!b || !q || !o || layer < 0 || layer >= h->cfg.n_layers || kind < 0 || kind > 4)
    return set_err(BULLET_EINVAL, "attention args");
  bullet_batch bb = *b;
  bb.layer_begin = layer; bb.layer_end = layer;
  if ((rc = validate_batch(h, &bb, 0))) return rc;
  return do_attention(c, b, layer, q, o, kind);
}

}  // extern "C"
