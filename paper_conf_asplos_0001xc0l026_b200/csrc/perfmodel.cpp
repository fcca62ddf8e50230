// perfmodel.cpp — Bullet's performance estimator and SLO-aware split
// decision, host C++ (product code; the test oracle restates the same
// paper passages independently in oracle/perfmodel.py).
//
//   Eq. 1  s = 1 - g / (M ceil(g / M))
//   Eq. 2  t_i = max(c_i/C M/(m d_c p_c), b_i/B M/(m d_b p_b)) / (1 - s_i)
//   T_m = sum_i t_i
//   Alg. 1 + decode-SM search + decode pause
// Readings R-11..R-18 of DESIGN.md §3.
#include "perfmodel.h"

#include <algorithm>
#include <cctype>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <limits>
#include <map>
#include <string>
#include <vector>

namespace bl {

// ------------------------------------------------------------ tiny JSON
namespace {
struct JP {
  const char* p;
  std::map<std::string, std::vector<double>> out;
  void ws() { while (*p && isspace((unsigned char)*p)) ++p; }
  bool str(std::string& s) {
    ws();
    if (*p != '"') return false;
    ++p;
    s.clear();
    while (*p && *p != '"') s += *p++;
    if (*p != '"') return false;
    ++p;
    return true;
  }
  bool num(double& v) {
    ws();
    char* e = nullptr;
    v = strtod(p, &e);
    if (e == p) return false;
    p = e;
    return true;
  }
  // value at path `key` (dotted); objects recurse, arrays of numbers stored
  bool value(const std::string& key) {
    ws();
    if (*p == '{') {
      ++p;
      ws();
      if (*p == '}') { ++p; return true; }
      for (;;) {
        std::string k;
        if (!str(k)) return false;
        ws();
        if (*p != ':') return false;
        ++p;
        if (!value(key.empty() ? k : key + "." + k)) return false;
        ws();
        if (*p == ',') { ++p; continue; }
        if (*p == '}') { ++p; return true; }
        return false;
      }
    }
    if (*p == '[') {
      ++p;
      std::vector<double> v;
      ws();
      if (*p == ']') { ++p; out[key] = v; return true; }
      for (;;) {
        double d;
        if (!num(d)) return false;
        v.push_back(d);
        ws();
        if (*p == ',') { ++p; continue; }
        if (*p == ']') { ++p; break; }
        return false;
      }
      out[key] = v;
      return true;
    }
    if (*p == '"') { std::string s; return str(s); }
    double d;
    if (!num(d)) return false;
    out[key] = {d};
    return true;
  }
};
}  // namespace

bool PerfParams::parse(const char* json, std::string* err) {
  JP j{json, {}};
  if (!j.value("")) { if (err) *err = "perf params: malformed JSON"; return false; }
  auto get1 = [&](const char* k, double& dst) {
    auto it = j.out.find(k);
    if (it != j.out.end() && it->second.size() == 1) dst = it->second[0];
  };
  auto getv = [&](const char* k, std::vector<double>& dst) {
    auto it = j.out.find(k);
    if (it != j.out.end()) dst = it->second;
  };
  get1("M", M); get1("C_tflops", C_tflops); get1("B_gbs", B_gbs);
  {   // p_c / p_b: a number (constant over m) or a {"m": [...], "v": [...]} table
    double c = -1.0, b = -1.0;
    get1("p_c", c); get1("p_b", b);
    if (c > 0) { pc_m = {1.0, M}; pc_v = {c, c}; }
    if (b > 0) { pb_m = {1.0, M}; pb_v = {b, b}; }
    getv("p_c.m", pc_m); getv("p_c.v", pc_v); getv("p_b.m", pb_m); getv("p_b.v", pb_v);
    p_c = p_b = 1.0;
  }
  getv("d_c.m", dc_m); getv("d_c.v", dc_v); getv("d_b.m", db_m); getv("d_b.v", db_v);
  dca_m.clear(); dca_v.clear(); dba_m.clear(); dba_v.clear();
  getv("d_c_attn.m", dca_m); getv("d_c_attn.v", dca_v); getv("d_b_attn.m", dba_m); getv("d_b_attn.v", dba_v);
  if (dca_m.empty()) { dca_m = dc_m; dca_v = dc_v; }   // not given: the attention kernel shares d_c / d_b
  if (dba_m.empty()) { dba_m = db_m; dba_v = db_v; }
  get1("tiles.gemm_bm", gemm_bm); get1("tiles.gemm_bn", gemm_bn); get1("tiles.gemm_bk", gemm_bk);
  get1("tiles.min_k_blocks", min_k_blocks); get1("tiles.attn_bq", attn_bq);
  get1("tiles.rows_per_unit", rows_per_unit);
  get1("occ.gemm", occ_gemm); get1("occ.attn", occ_attn); get1("occ.elem", occ_elem);
  if (dc_m.size() != dc_v.size() || db_m.size() != db_v.size() || dc_m.empty() || db_m.empty() ||
      pc_m.size() != pc_v.size() || pb_m.size() != pb_v.size() || pc_m.empty() || pb_m.empty() ||
      dca_m.size() != dca_v.size() || dba_m.size() != dba_v.size()) {
    if (err) *err = "perf params: d_c / d_b / p_c / p_b tables malformed";
    return false;
  }
  return true;
}

void PerfParams::set_default(int n_sms) {
  M = n_sms;
  C_tflops = 1649.5; B_gbs = 6549.4;   // MEASURED_PEAKS.json (burst GEMM, copy)
  dc_m = {1.0, (double)n_sms}; dc_v = {1.0, 1.0};
  db_m = {1.0, (double)n_sms}; db_v = {1.0, 1.0};
  pc_m = {1.0, (double)n_sms}; pc_v = {1.0, 1.0};
  pb_m = {1.0, (double)n_sms}; pb_v = {1.0, 1.0};
  dca_m = dc_m; dca_v = dc_v; dba_m = db_m; dba_v = db_v;
  p_c = p_b = 1.0;
}

// Eq. 1
double wave_idle(double g, double M) {
  if (g <= 0 || M <= 0) return 0.0;
  const double w = std::ceil(g / M);
  return 1.0 - g / (M * w);
}

static double interp(const std::vector<double>& ms, const std::vector<double>& vs, double m) {
  if (m <= ms[0]) return vs[0];
  for (size_t i = 1; i < ms.size(); ++i)
    if (m <= ms[i]) return vs[i - 1] + (m - ms[i - 1]) / (ms[i] - ms[i - 1]) * (vs[i] - vs[i - 1]);
  return vs.back();
}

// Per-kernel (c_i, b_i, g_i, occupancy) of one layer of one phase.
std::vector<KernelCost> layer_kernels(const PhaseShape& s, const PerfParams& P, int m) {
  std::vector<KernelCost> ks;
  double n = 0, pairs = 0, keys = 0;
  int maxq = 0;
  for (size_t i = 0; i < s.q_lens.size(); ++i) {
    const double q = s.q_lens[i], c = s.ctx_lens[i];
    n += q;
    pairs += q * c + q * (q + 1) / 2;
    keys += c + q;
    maxq = std::max(maxq, s.q_lens[i]);
  }
  if (n == 0) return ks;
  const double d = s.d, H = s.H, Hkv = s.Hkv, hd = s.hd, I = s.I, e = s.elt;
  const double nq = (H + 2 * Hkv) * hd;
  const double rows = P.rows_per_unit;
  auto gemm = [&](const char* name, double K, double N, double extra) {
    const double tiles = std::ceil(n / P.gemm_bm) * std::ceil(N / P.gemm_bn);
    double splits = std::ceil(m * P.occ_gemm / tiles);
    splits = std::max(1.0, std::min(splits, std::floor(K / (P.gemm_bk * P.min_k_blocks))));
    ks.push_back({name, 2.0 * n * K * N, e * (K * N + n * K) + extra, tiles * splits, P.occ_gemm});
  };
  double attn_units = 0;
  if (maxq > 1) {
    for (int q : s.q_lens) attn_units += std::ceil(q / P.attn_bq);
    attn_units *= H;
  } else {
    attn_units = (double)s.q_lens.size() * Hkv;
  }
  ks.push_back({"rmsnorm1", 4.0 * n * d, 4 * n * d + e * n * d + e * d, std::ceil(n / rows), P.occ_elem});
  if (e == 2 && hd == 128) {   // bf16: RoPE + KV append fused into the QKV epilogue (bf16 q / k / v out)
    gemm("qkv", d, nq, e * n * nq);
    ks.back().c += 6.0 * n * (H + Hkv) * hd;
  } else {
    gemm("qkv", d, nq, 4 * n * nq);
    ks.push_back({"rope_kv", 6.0 * n * (H + Hkv) * hd, 4 * n * nq + e * n * nq, std::ceil(n / rows), P.occ_elem});
  }
  ks.push_back({"attn", 4.0 * hd * H * pairs, 2 * e * Hkv * hd * keys + 2 * e * n * H * hd, attn_units, P.occ_attn});
  gemm("o_proj", H * hd, d, 8 * n * d);
  ks.push_back({"rmsnorm2", 4.0 * n * d, 4 * n * d + e * n * d + e * d, std::ceil(n / rows), P.occ_elem});
  gemm("gate_up", d, 2 * I, e * n * I);
  gemm("down", I, d, 8 * n * d);
  return ks;
}

// T_m in seconds, Eq. 2 per kernel.
double layer_time(const PhaseShape& s, const PerfParams& P, int m, int corun_m) {
  if (m <= 0) return std::numeric_limits<double>::infinity();
  const double C = P.C_tflops * 1e12, B = P.B_gbs * 1e9, M = P.M;
  const double dc0 = interp(P.dc_m, P.dc_v, m), db0 = interp(P.db_m, P.db_v, m);
  const double dca = P.dca_m.empty() ? dc0 : interp(P.dca_m, P.dca_v, m);
  const double dba = P.dba_m.empty() ? db0 : interp(P.dba_m, P.dba_v, m);
  const double pc = corun_m > 0 ? interp(P.pc_m, P.pc_v, m) * P.p_c : 1.0;
  const double pb = corun_m > 0 ? interp(P.pb_m, P.pb_v, m) * P.p_b : 1.0;
  double total = 0;
  int maxq = 0;
  for (int q : s.q_lens) maxq = std::max(maxq, q);
  const double scale = maxq > 1 ? P.scale_pre : P.scale_dec;
  for (const auto& k : layer_kernels(s, P, m)) {
    const bool attn = !strcmp(k.name, "attn");
    const double dc = attn ? dca : dc0, db = attn ? dba : db0;
    const double sidle = wave_idle(k.g, (double)m * k.occ);
    const double tc = k.c / C * M / (m * dc * pc);
    const double tb = k.b / B * M / (m * db * pb);
    total += std::max(tc, tb) / (1.0 - sidle);
  }
  return total * scale;
}

static double p90(std::vector<double> v, double pct) {
  if (v.empty()) return 0.0;
  std::sort(v.begin(), v.end());
  long idx = (long)std::ceil(pct * (double)v.size()) - 1;
  if (idx < 0) idx = 0;
  return v[(size_t)idx];
}

struct Eval { double ttft, tpot, t_p; };

static Eval evaluate(const PerfParams& P, const PhaseShape& model, const SchedState& S,
                     const Slo& slo, int u, int v) {
  const int N = (int)P.M, L = S.total_layers;
  PhaseShape pre = model, dec = model;
  pre.q_lens = S.prefill_lens; pre.ctx_lens.assign(S.prefill_lens.size(), 0);
  const int mctx = (int)std::lround(S.decode_mean_ctx);
  dec.q_lens.assign(S.decode_tokens.size(), 1); dec.ctx_lens.assign(S.decode_tokens.size(), mctx);
  const double ms = 1e3;
  const double t_p = S.prefill_lens.empty() ? 0.0 : layer_time(pre, P, u, v) * ms;
  const double rem = t_p * (L - S.layers_done);                       // Alg. 1 l.3
  std::vector<double> ttft, tpot;
  for (size_t i = 0; i < S.prefill_lens.size(); ++i)                  // l.4-5
    ttft.push_back((rem + S.prefill_waited_ms[i]) / (slo.ttft_norm * S.prefill_lens[i]));
  for (size_t i = 0; i < S.pending_lens.size(); ++i) {                // l.6-7 (+ own prefill, R-15)
    PhaseShape one = model;
    one.q_lens = {S.pending_lens[i]}; one.ctx_lens = {0};
    const double own = layer_time(one, P, u, v) * ms * L;
    ttft.push_back((S.pending_waited_ms[i] + rem + own) / (slo.ttft_norm * S.pending_lens[i]));
  }
  if (!S.decode_tokens.empty()) {                                     // l.8-10 (R-14)
    double t_iter;
    if (v > 0) t_iter = layer_time(dec, P, v, u) * ms * L;
    else t_iter = layer_time(pre, P, N, 0) * ms + layer_time(dec, P, S.v_k, 0) * ms * L;
    for (size_t i = 0; i < S.decode_tokens.size(); ++i)
      tpot.push_back(((S.decode_elapsed_ms[i] + t_iter) / (S.decode_tokens[i] + 1)) / slo.tpot_ms);
  }
  return {p90(ttft, slo.percentile), p90(tpot, slo.percentile), t_p};
}

// R-23: gains within this fraction of the best are within the model's
// resolution (held-out MRE ~5 %); among them prefill is prioritised
constexpr double GAIN_TOL = 0.06;   // R-23: the fitted model's resolution (held-out MRE ~6 %)

void choose_split(const PerfParams& P, const PhaseShape& model, const SchedState& S,
                  const Slo& slo, int gran, int* prefill_sms, int* decode_steps) {
  const int N = (int)P.M, L = S.total_layers;
  const bool has_pre = !S.prefill_lens.empty() || !S.pending_lens.empty();
  if (S.decode_tokens.empty()) { *prefill_sms = N; *decode_steps = 0; return; }
  if (!has_pre) { *prefill_sms = 0; *decode_steps = L; return; }
  std::vector<int> cands;
  for (int v = slo.v_min; v <= N - gran; ++v)
    if (v % gran == 0 || v == slo.v_min) cands.push_back(v);
  if (cands.empty()) { *prefill_sms = N; *decode_steps = 0; return; }
  std::map<int, Eval> ev;
  for (int v : cands) ev[v] = evaluate(P, model, S, slo, N - v, v);
  int vk = cands[0];
  for (int v : cands)
    if (std::abs(v - S.v_k) < std::abs(vk - S.v_k)) vk = v;
  const bool ok_t = ev[vk].ttft <= 1.0, ok_d = ev[vk].tpot <= 1.0;

  auto reduce_decode = [&]() -> int {
    for (int v : cands)   // ascending: first feasible = smallest decode SM count
      if (v <= vk && ev[v].ttft <= 1.0 && ev[v].tpot <= 1.0) return v;
    const Eval pz = evaluate(P, model, S, slo, N, 0);
    if (pz.tpot <= 1.0) return 0;            // pause decode
    return cands.front();                    // v_min
  };
  auto reduce_prefill = [&]() -> int {
    for (int v : cands)
      if (v >= vk && ev[v].tpot <= 1.0) return v;
    int best = cands.front();
    for (int v : cands)
      if (ev[v].tpot < ev[best].tpot) best = v;
    return best;
  };
  auto balanced = [&]() -> int {
    int best = cands.front();
    for (int v : cands)
      if (std::max(ev[v].ttft, ev[v].tpot) < std::max(ev[best].ttft, ev[best].tpot)) best = v;
    return best;
  };
  // R-21 (objective 1): "meet stringent SLO requirements while maximizing
  // throughput" — among the splits that keep both SLOs, the one with
  // the most predicted tokens per ms: (prefill tokens + decode tokens x k) /
  // max(t_p, k t_d), k = round(t_p / t_d) >= 1; ties to the larger prefill
  // share.  None feasible: Alg. 1's rule.
  auto max_throughput = [&](double* best_tput) -> int {
    PhaseShape dec = model;
    const int mctx = (int)std::lround(S.decode_mean_ctx);
    dec.q_lens.assign(S.decode_tokens.size(), 1); dec.ctx_lens.assign(S.decode_tokens.size(), mctx);
    double n_pre = 0.0;
    for (int q : S.prefill_lens) n_pre += q;
    int best = -1;
    double best_t = -1.0;
    for (int v : cands) {
      if (ev[v].ttft > 1.0 || ev[v].tpot > 1.0) continue;
      const double t_p = ev[v].t_p, t_d = layer_time(dec, P, v, N - v) * 1e3;
      const int k = t_d > 0 ? std::max(1, (int)std::floor(t_p / t_d + 0.5)) : 1;
      const double cyc = std::max(t_p, k * t_d);
      const double tput = cyc > 0 ? (n_pre + (double)S.decode_tokens.size() * k) / cyc : 0.0;
      if (tput > best_t) { best_t = tput; best = v; }
    }
    if (best_tput) *best_tput = best_t;
    return best;
  };
  // R-22 (objective 1): the time-sliced cycle — one prefill layer, then k_ts
  // decode layer-steps, both alone on all N SMs, k_ts = round(t_p / t_d) —
  // is a candidate too, with its own TTFT / TPOT estimate (Alg. 1 l.3-10 on
  // the cycle time t_p + k_ts t_d); returns k_ts, or 0 when it misses an SLO
  auto timesliced = [&](double* tput) -> int {
    PhaseShape pre = model, dec = model;
    pre.q_lens = S.prefill_lens; pre.ctx_lens.assign(S.prefill_lens.size(), 0);
    const int mctx = (int)std::lround(S.decode_mean_ctx);
    dec.q_lens.assign(S.decode_tokens.size(), 1); dec.ctx_lens.assign(S.decode_tokens.size(), mctx);
    const double tp = S.prefill_lens.empty() ? 0.0 : layer_time(pre, P, N, 0) * 1e3;
    const double td = layer_time(dec, P, N, 0) * 1e3;
    if (tp <= 0.0 || td <= 0.0) return 0;
    const int k = std::max(1, (int)std::floor(tp / td + 0.5));
    const double cyc = tp + k * td, rem = cyc * (L - S.layers_done);
    std::vector<double> ttft, tpot;
    for (size_t i = 0; i < S.prefill_lens.size(); ++i)
      ttft.push_back((rem + S.prefill_waited_ms[i]) / (slo.ttft_norm * S.prefill_lens[i]));
    for (size_t i = 0; i < S.pending_lens.size(); ++i) {
      PhaseShape one = model;
      one.q_lens = {S.pending_lens[i]}; one.ctx_lens = {0};
      const double own = layer_time(one, P, N, 0) * 1e3 * L;
      ttft.push_back((S.pending_waited_ms[i] + rem + own) / (slo.ttft_norm * S.pending_lens[i]));
    }
    const double iter = cyc * L / k;
    for (size_t i = 0; i < S.decode_tokens.size(); ++i)
      tpot.push_back(((S.decode_elapsed_ms[i] + iter) / (S.decode_tokens[i] + 1)) / slo.tpot_ms);
    if (p90(ttft, slo.percentile) > 1.0 || p90(tpot, slo.percentile) > 1.0) return 0;
    double n_pre = 0.0;
    for (int q : S.prefill_lens) n_pre += q;
    *tput = (n_pre + (double)S.decode_tokens.size() * k) / cyc;
    return k;
  };
  // R-23 (objective 2): the split that makes co-running pay most — among
  // the SLO-feasible splits and k in {floor(r), ceil(r)} (r = t_p / t_d at
  // the split, k >= 1), the largest predicted co-location gain
  // G = (t_p(N) + k t_d(N)) / max(t_p(u), k t_d(v)): the time-sliced cycle
  // of the same work over the co-run cycle (north_star's target ratio, the
  // paper's co-run-vs-time-sliced axis, P:L7 / P:L155).  Ties: larger gain,
  // then the larger prefill share, then the smaller k.  Returns the gain.
  // Ties within the model's resolution (R-23: gains within GAIN_TOL of the
  // best) go to the larger prefill share ("prioritize prefill"), then
  // the larger gain, then the smaller k.  Returns the best gain.
  auto max_gain = [&](int* best_v, int* best_k) -> double {
    PhaseShape pre = model, dec = model;
    pre.q_lens = S.prefill_lens; pre.ctx_lens.assign(S.prefill_lens.size(), 0);
    const int mctx = (int)std::lround(S.decode_mean_ctx);
    dec.q_lens.assign(S.decode_tokens.size(), 1); dec.ctx_lens.assign(S.decode_tokens.size(), mctx);
    const double tpN = S.prefill_lens.empty() ? 0.0 : layer_time(pre, P, N, 0) * 1e3;
    const double tdN = layer_time(dec, P, N, 0) * 1e3;
    struct Cand { int v, k; double g; };
    std::vector<Cand> cs;
    double best_g = -1.0;
    for (int v : cands) {
      if (ev[v].ttft > 1.0 || ev[v].tpot > 1.0) continue;
      const double t_p = ev[v].t_p, t_d = layer_time(dec, P, v, N - v) * 1e3;
      if (t_d <= 0.0) continue;
      const int k0 = std::max(1, (int)std::floor(t_p / t_d));
      for (int k = k0; k <= k0 + 1; ++k) {
        const double g = (tpN + k * tdN) / std::max(t_p, k * t_d);
        cs.push_back({v, k, g});
        best_g = std::max(best_g, g);
      }
    }
    *best_v = -1; *best_k = 1;
    double pick_g = -1.0;
    for (const Cand& c : cs) {   // candidates in ascending v (cands order), k ascending
      if (c.g < (1.0 - GAIN_TOL) * best_g) continue;
      if (*best_v < 0 || c.v < *best_v || (c.v == *best_v && c.g > pick_g)) { *best_v = c.v; *best_k = c.k; pick_g = c.g; }
    }
    return best_g;
  };
  int v;
  if (ok_t && ok_d && slo.objective == 2) {
    int vb, kb;
    const double g = max_gain(&vb, &kb);
    if (vb >= 0 && g > 1.0) { *prefill_sms = N - vb; *decode_steps = kb; return; }
    double t_ts = -1.0;
    const int k_ts = timesliced(&t_ts);
    if (k_ts > 0) { *prefill_sms = N; *decode_steps = k_ts; return; }   // co-running does not pay
    if (vb >= 0) { *prefill_sms = N - vb; *decode_steps = kb; return; }
    v = reduce_decode();
  }
  else if (ok_t && ok_d && slo.objective == 1) {
    double t_co = -1.0, t_ts = -1.0;
    const int vb = max_throughput(&t_co);
    const int k_ts = timesliced(&t_ts);
    if (k_ts > 0 && t_ts > t_co) {   // time-sliced cycle: prefill_sms = N with k > 0
      *prefill_sms = N; *decode_steps = k_ts; return;
    }
    v = vb >= 0 ? vb : reduce_decode();
  }
  else if (ok_t && ok_d) v = reduce_decode();
  else if (!ok_t && !ok_d) v = balanced();
  else if (ok_t && !ok_d && (int)S.pending_lens.size() <= slo.w_max) v = reduce_prefill();
  else v = reduce_decode();
  if (v == 0) { *prefill_sms = N; *decode_steps = 0; return; }
  const int u = N - v;
  PhaseShape dec = model;
  const int mctx = (int)std::lround(S.decode_mean_ctx);
  dec.q_lens.assign(S.decode_tokens.size(), 1); dec.ctx_lens.assign(S.decode_tokens.size(), mctx);
  const double t_d = layer_time(dec, P, v, u) * 1e3;
  const double t_p = ev[v].t_p;
  *prefill_sms = u;
  *decode_steps = t_d > 0 ? std::max(1, (int)std::floor(t_p / t_d + 0.5)) : 1;
}

}  // namespace bl
