// perfmodel.h — host-side performance estimator (Eq. 1, Eq. 2, T_m) and the
// Alg. 1 split decision.  See perfmodel.cpp.
#pragma once
#include <string>
#include <vector>

namespace bl {

struct PerfParams {
  double M = 148, C_tflops = 1649.5, B_gbs = 6549.4;
  std::vector<double> dc_m{1, 148}, dc_v{1, 1}, db_m{1, 148}, db_v{1, 1};
  // the attention kernel's own d_c(m), d_b(m) (R-12b; default: the tables
  // above): its roofline efficiency differs from the GEMMs', so batches
  // with different KV / weight byte mixes need both
  std::vector<double> dca_m, dca_v, dba_m, dba_v;
  // co-location factors p_c(m), p_b(m): piecewise linear in the kernel's own
  // SM count m (a JSON number = constant), times the online scale (P:L195
  // estimator feedback, bullet_set_colocation)
  std::vector<double> pc_m{1, 148}, pc_v{1, 1}, pb_m{1, 148}, pb_v{1, 1};
  double p_c = 1, p_b = 1;   // scale
  // online level calibration per phase class (bullet_set_phase_scale): every
  // predicted layer time of a prefill-shaped (some q > 1) / decode-shaped
  // batch is multiplied by scale_pre / scale_dec (default 1)
  double scale_pre = 1, scale_dec = 1;
  double gemm_bm = 128, gemm_bn = 256, gemm_bk = 64, min_k_blocks = 4, attn_bq = 64, rows_per_unit = 8;
  double occ_gemm = 1, occ_attn = 1, occ_elem = 4;
  bool parse(const char* json, std::string* err);
  void set_default(int n_sms);
};

struct PhaseShape {
  int d, H, Hkv, hd, I, elt;
  std::vector<int> q_lens, ctx_lens;
};

struct KernelCost {
  const char* name;
  double c, b, g, occ;
};

struct SchedState {
  int layers_done, total_layers;
  std::vector<int> prefill_lens; std::vector<double> prefill_waited_ms;
  std::vector<int> pending_lens; std::vector<double> pending_waited_ms;
  std::vector<int> decode_tokens; std::vector<double> decode_elapsed_ms;
  double decode_mean_ctx;
  int u_k, v_k;
};

struct Slo {
  double ttft_norm, tpot_ms;
  int w_max, v_min;
  double percentile;
  int objective;   // 0: Alg. 1 as read (R-14..R-17); 1: + throughput among SLO-feasible splits (R-21, R-22);
                   // 2: + largest predicted co-location gain over time-slicing (R-23)
};

double wave_idle(double g, double M);
std::vector<KernelCost> layer_kernels(const PhaseShape& s, const PerfParams& P, int m);
double layer_time(const PhaseShape& s, const PerfParams& P, int m, int corun_m);
void choose_split(const PerfParams& P, const PhaseShape& model, const SchedState& S, const Slo& slo,
                  int gran, int* prefill_sms, int* decode_steps);

}  // namespace bl
