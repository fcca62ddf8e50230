"""Multi-step serving loop over bullet_step.

PAPER.md §3.3: every scheduling cycle the prefill batch
advances by a group of layers while the decode batch advances by k layer
steps on the other SMs; Alg. 1 re-decides (prefill SM count, k) each cycle
from the live request state (readings R-14..R-19); a request
that finishes prefill joins the decode batch copy-free (its KV blocks and
block-table row are kept).  Requests arrive by a seeded Poisson
process with ShareGPT-like prompt and output lengths (synthetic: the paper's
traces are out of scope).

This module is host orchestration only: request bookkeeping, a paged-block
allocator, the cycle state machine and the SLO metrics (TTFT, normalized
TTFT, TPOT, goodput).  All compute happens in the injected `step` callable —
on the GPU that is one bullet_step (scripts/serve.py); tests drive the same
loop with the host-only performance model.  Time is virtual: the clock
advances by each cycle's measured (or predicted) device time, so different
policies see the same arrival process.

Policies:
  bullet      co-run, (p, k) from Alg. 1 (bullet_choose_split)
  static      co-run at one fixed (prefill SMs, k) every cycle — the bench's
              tuned split; a diagnostic of the decision layer, not a policy
  bullet_tput the same with objective 1: when both SLOs hold, the split with
              the most predicted tokens/s among the SLO-feasible ones (R-21)
  bullet_gain the same with objective 2: when both SLOs hold, the split with
              the largest predicted gain of the co-run cycle over the same
              work time-sliced, or a time-sliced cycle when none gains (R-23)
  timesliced  same cycle structure, both phases on all SMs one after the
              other (BULLET_TIMESLICED), k from the model's full-GPU balance
  prefill_first  vLLM-style: while a prefill batch exists decode is paused
              (p = N); otherwise decode runs whole iterations on all SMs
  chunked     SARATHI / SGLang chunked prefill (the paper's comparison axis,
              P:L82-86): every iteration is ONE hybrid batch on
              all SMs — the decode members plus a chunk of the waiting
              prompts (token budget `chunk_tokens`, each chunk attending to
              the prompt's earlier chunks through the block table) — advanced
              k_full layers per cycle; a prompt's first token comes when its
              last chunk leaves the last layer
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np


@dataclass
class Request:
    rid: int
    arrival_ms: float
    prompt: int
    out_len: int                      # tokens to generate (first one comes from prefill)
    blocks: list = field(default_factory=list)
    first_token_ms: float | None = None
    finish_ms: float | None = None
    tokens: int = 0                   # tokens generated so far

    @property
    def ctx(self) -> int:
        """Cached positions before the token being decoded now."""
        return self.prompt + self.tokens - 1


def poisson_trace(rate_per_s: float, duration_s: float, seed: int = 0, prompt_mu=math.log(400),
                  prompt_sigma=0.8, prompt_clip=(32, 2048), out_mu=math.log(128), out_sigma=0.7,
                  out_clip=(8, 512)) -> list[Request]:
    """Seeded Poisson arrivals; prompt / output lengths lognormal, clipped
    (ShareGPT-like shapes)."""
    rng = np.random.default_rng(seed)
    t, reqs = 0.0, []
    while True:
        t += rng.exponential(1000.0 / rate_per_s)
        if t > duration_s * 1000.0:
            return reqs
        p = int(np.clip(round(rng.lognormal(prompt_mu, prompt_sigma)), *prompt_clip))
        o = int(np.clip(round(rng.lognormal(out_mu, out_sigma)), *out_clip))
        reqs.append(Request(len(reqs), t, p, o))


class BlockAllocator:
    """Free list of KV blocks (block ids index every layer's pool alike)."""

    def __init__(self, n_blocks: int, block_size: int = 16):
        self.free = list(range(n_blocks - 1, -1, -1))
        self.n_blocks, self.block_size = n_blocks, block_size

    def alloc(self, n_tokens: int):
        n = -(-n_tokens // self.block_size)
        if n > len(self.free):
            return None
        return [self.free.pop() for _ in range(n)]

    def release(self, blocks):
        self.free.extend(reversed(blocks))


@dataclass
class PhaseWork:
    """What one phase runs this cycle (consumed by the step callable)."""
    reqs: list
    q_lens: list
    ctx_lens: list
    layer_begin: int
    layer_end: int
    batch_id: int                     # changes when the batch membership changes


@dataclass
class Slo:
    ttft_norm_ms_per_tok: float = 3.0  # Table 2 ShareGPT row
    tpot_ms: float = 150.0
    w_max: int = 4
    v_min: int = 16
    percentile: float = 0.9
    objective: int = 0                 # 1: throughput among SLO-feasible splits (R-21, policy bullet_tput)

    def as_dict(self):
        return dict(ttft_norm_ms_per_tok=self.ttft_norm_ms_per_tok, tpot_ms=self.tpot_ms,
                    w_max=self.w_max, v_min=self.v_min, percentile=self.percentile, objective=self.objective)


class ServingLoop:
    """step(prefill: PhaseWork|None, decode: PhaseWork|None, p, flags_mode) -> device ms;
    choose(state dict, slo dict) -> (p, k)  [Alg. 1, used by the bullet policy];
    k_full: decode layer-steps per cycle for the time-sliced policy."""

    def __init__(self, n_layers: int, n_sms: int, step, choose, policy: str, allocator: BlockAllocator,
                 slo: Slo = Slo(), prefill_layers_per_cycle: int = 1, max_prefill_tokens: int = 8192,
                 max_decodes: int = 256, k_full: int = 4, chunk_tokens: int = 2048, feedback_model=None,
                 feedback_alpha: float = 0.2, static_split=(88, 6)):
        assert policy in ("bullet", "bullet_tput", "bullet_gain", "static", "timesliced", "prefill_first", "chunked")
        self.static_split = static_split   # policy "static": fixed (prefill SMs, decode layer-steps) co-run
        if policy in ("bullet_tput", "bullet_gain"):   # Alg. 1 with objective 1 (R-21 / R-22) or 2 (R-23)
            slo = Slo(**{**slo.__dict__, "objective": 1 if policy == "bullet_tput" else 2})
            policy = "bullet"
        self.L, self.N = n_layers, n_sms
        self.step, self.choose, self.policy = step, choose, policy
        self.alloc, self.slo = allocator, slo
        self.lp = prefill_layers_per_cycle
        self.max_prefill_tokens, self.max_decodes, self.k_full = max_prefill_tokens, max_decodes, k_full
        self.split = (n_sms // 2, n_sms - n_sms // 2)
        self.chunk_tokens = chunk_tokens
        self.log = []                 # per cycle: (now, p, k, prefill tokens, decodes, ms)
        self.unservable = []          # requests that can never be admitted (reported, loop ends)
        # online estimator feedback: after every co-run cycle the
        # ratio measured / predicted cycle time updates an EMA that rescales
        # the model's co-location factors p_c, p_b (bullet_set_colocation),
        # so the next decisions see the contention actually observed
        self.fb = feedback_model
        self.fb_alpha, self.fb_ratio = feedback_alpha, 1.0
        self.fb_base = feedback_model.colocation() if feedback_model is not None else None

    # ------------------------------------------------------------ helpers
    def _feedback(self, pw, dw, p, ms):
        """correlate the observed cycle time with the prediction."""
        n_pl, k = pw.layer_end - pw.layer_begin, dw.layer_end - dw.layer_begin
        t_p = self.fb.predict_us(pw.q_lens, pw.ctx_lens, p, self.N - p) / 1e3 * n_pl
        t_d = self.fb.predict_us(dw.q_lens, dw.ctx_lens, self.N - p, p) / 1e3 * k
        pred = max(t_p, t_d)
        if pred <= 0:
            return
        r = ms / pred * self.fb_ratio        # ratio to the uncorrected model
        r = min(2.0, max(0.5, r))
        self.fb_ratio = (1 - self.fb_alpha) * self.fb_ratio + self.fb_alpha * r
        self.fb.set_colocation(self.fb_base[0] / self.fb_ratio, self.fb_base[1] / self.fb_ratio)

    def _alg1_state(self, now, prefill, layers_done, pending, members):
        return dict(layers_done=layers_done if prefill else 0, total_layers=self.L,
                    prefill_lens=[r.prompt for r in prefill] if prefill else [],
                    prefill_waited_ms=[now - r.arrival_ms for r in prefill] if prefill else [],
                    pending_lens=[r.prompt for r in pending],
                    pending_waited_ms=[now - r.arrival_ms for r in pending],
                    decode_tokens=[r.tokens for r in members],
                    decode_elapsed_ms=[now - r.first_token_ms for r in members],
                    decode_mean_ctx=float(np.mean([r.ctx for r in members])) if members else 0.0,
                    u_k=self.split[0], v_k=self.split[1])

    # ------------------------------------------------------------ chunked prefill (baseline)
    def _run_chunked(self, trace, horizon, max_cycles):
        now, nxt = 0.0, 0
        pending, members, done = [], [], []
        filling = []                  # admitted prompts with tokens still to prefill: [req, tokens done]
        d_layer, it_id, hyb = 0, 0, None
        for _ in range(max_cycles):
            while nxt < len(trace) and trace[nxt].arrival_ms <= now:
                pending.append(trace[nxt]); nxt += 1
            if d_layer == 0:          # new iteration: admit prompts, cut this iteration's chunks
                while pending and len(members) + len(filling) < self.max_decodes:
                    blk = self.alloc.alloc(pending[0].prompt + pending[0].out_len)
                    if blk is None:
                        break
                    r = pending.pop(0); r.blocks = blk
                    filling.append([r, 0])
                budget = max(0, self.chunk_tokens - len(members))
                chunks = []
                for f in filling:
                    if budget <= 0:
                        break
                    c = min(budget, f[0].prompt - f[1])
                    if c > 0:
                        chunks.append((f, c)); budget -= c
                if not chunks and not members:
                    if nxt >= len(trace) and not pending and not filling:
                        break
                    if nxt < len(trace):
                        now = max(now, trace[nxt].arrival_ms)
                        continue
                it_id += 1
                # prefill chunks (q > 1 first), then the decodes: one hybrid batch
                order = sorted(chunks, key=lambda fc: fc[1] == 1)
                reqs = [f[0] for f, _ in order] + members
                q = [c for _, c in order] + [1] * len(members)
                ctx = [f[1] for f, _ in order] + [r.ctx for r in members]
                hyb = (order, list(members), reqs, q, ctx)
            if now >= horizon:
                break
            order, mem, reqs, q, ctx = hyb
            le = min(d_layer + self.k_full, self.L)
            pw = PhaseWork(reqs, q, ctx, d_layer, le, it_id)
            self.split = (self.N, 0)
            ms = self.step(pw, None, self.N, "timesliced")
            self.log.append((now, self.N, le - d_layer, sum(q) - len(mem), len(mem), ms))
            now += ms
            d_layer = le
            if d_layer < self.L:
                continue
            d_layer = 0               # iteration complete: chunks advance, decodes emit a token
            for f, c in order:
                f[1] += c
                if f[1] >= f[0].prompt:
                    r = f[0]
                    filling.remove(f)
                    r.first_token_ms, r.tokens = now, 1
                    if r.out_len <= 1:
                        r.finish_ms = now; self.alloc.release(r.blocks); done.append(r)
                    else:
                        members.append(r)
            still = []
            for r in mem:
                r.tokens += 1
                if r.tokens >= r.out_len:
                    r.finish_ms = now; self.alloc.release(r.blocks); done.append(r)
                else:
                    still.append(r)
            members = still + [r for r in members if r not in mem]
        return self.metrics(done, trace, now)

    # ------------------------------------------------------------ loop
    def run(self, trace: list[Request], horizon_ms: float | None = None, max_cycles: int = 10 ** 7):
        trace = sorted(trace, key=lambda r: r.arrival_ms)
        horizon = horizon_ms if horizon_ms is not None else float("inf")
        if self.policy == "chunked":
            return self._run_chunked(trace, horizon, max_cycles)
        now, nxt = 0.0, 0
        pending, ready, members = [], [], []
        prefill, layers_done, pre_id, dec_id = None, 0, 0, 0
        d_layer = 0                   # next decode layer of the current iteration
        done = []
        for _ in range(max_cycles):
            while nxt < len(trace) and trace[nxt].arrival_ms <= now:
                pending.append(trace[nxt]); nxt += 1
            # new prefill batch (FCFS while tokens and KV blocks last)
            if prefill is None and pending:
                batch, toks = [], 0
                while pending and toks + pending[0].prompt <= self.max_prefill_tokens:
                    r = pending[0]
                    blk = self.alloc.alloc(r.prompt + r.out_len)
                    if blk is None:
                        break
                    r.blocks = blk
                    batch.append(pending.pop(0)); toks += r.prompt
                if batch:
                    prefill, layers_done, pre_id = batch, 0, pre_id + 1
            # decode membership changes only between iterations
            if d_layer == 0:
                room = self.max_decodes - len(members)
                members += ready[:room]
                del ready[:room]
                dec_id += 1
            if prefill is None and not members:
                if nxt >= len(trace) and not pending and not ready:
                    break
                if nxt < len(trace):           # idle until the next arrival
                    now = max(now, trace[nxt].arrival_ms)
                    continue
                if not ready:                  # pending requests that can never be admitted
                    self.unservable = list(pending)   # (prompt > max_prefill_tokens or KV pool too small)
                    break
            if now >= horizon:
                break
            # ---- split decision
            if self.policy == "bullet":
                mode = "corun"
                if prefill and members:
                    p, k = self.choose(self._alg1_state(now, prefill, layers_done, pending, members),
                                       self.slo.as_dict())
                    if p >= self.N and k > 0:   # R-22: a time-sliced cycle (objective 1)
                        mode = "timesliced"
                elif prefill:
                    p, k = self.N, 0
                else:
                    p, k = 0, self.k_full
            elif self.policy == "static":      # the bench-tuned split every cycle (diagnostic)
                p, k = self.static_split if (prefill and members) else ((self.N, 0) if prefill else (0, self.k_full))
                mode = "corun"
            elif self.policy == "timesliced":
                p, k, mode = self.N, (self.k_full if members else 0), "timesliced"
            else:  # prefill_first
                p, k, mode = (self.N, 0, "corun") if prefill else (0, self.L, "corun")
            if p >= self.N:
                k = 0 if mode == "corun" else k   # decode paused
            if not members:
                k = 0
            pw = None
            if prefill and (p > 0 or mode == "timesliced"):
                le = min(layers_done + self.lp, self.L)
                pw = PhaseWork(prefill, [r.prompt for r in prefill], [0] * len(prefill), layers_done, le, pre_id)
            dw = None
            if k > 0:
                de = min(d_layer + k, self.L)
                dw = PhaseWork(members, [1] * len(members), [r.ctx for r in members], d_layer, de, dec_id)
            if pw is None and dw is None:     # e.g. p = 0 chosen while decode is empty
                if prefill is None:           # nothing runnable this cycle: stop, never build an empty batch
                    self.unservable = list(pending)
                    break
                p, k = self.N, 0
                le = min(layers_done + self.lp, self.L)
                pw = PhaseWork(prefill, [r.prompt for r in prefill], [0] * len(prefill), layers_done, le, pre_id)
            if mode == "corun" and pw is None:
                p = 0
            self.split = (p, self.N - p)
            ms = self.step(pw, dw, p, mode)
            self.log.append((now, p, k, sum(pw.q_lens) if pw else 0, len(members) if dw else 0, ms))
            if self.fb is not None and mode == "corun" and pw is not None and dw is not None and 0 < p < self.N:
                self._feedback(pw, dw, p, ms)
            now += ms
            # ---- advance the prefill batch
            if pw is not None:
                layers_done = pw.layer_end
                if layers_done >= self.L:
                    for r in prefill:
                        r.first_token_ms, r.tokens = now, 1
                        if r.out_len <= 1:
                            r.finish_ms = now
                            self.alloc.release(r.blocks)
                            done.append(r)
                        else:
                            ready.append(r)
                    prefill, layers_done = None, 0
            # ---- advance the decode iteration
            if dw is not None:
                d_layer = dw.layer_end
                if d_layer >= self.L:
                    d_layer = 0
                    still = []
                    for r in members:
                        r.tokens += 1
                        if r.tokens >= r.out_len:
                            r.finish_ms = now
                            self.alloc.release(r.blocks)
                            done.append(r)
                        else:
                            still.append(r)
                    members = still
        return self.metrics(done, trace, now)

    def metrics(self, done, trace, now):
        s = self.slo
        ttft = np.array([r.first_token_ms - r.arrival_ms for r in done]) if done else np.zeros(0)
        nttft = np.array([(r.first_token_ms - r.arrival_ms) / r.prompt for r in done]) if done else np.zeros(0)
        tpot = np.array([(r.finish_ms - r.first_token_ms) / (r.out_len - 1) for r in done if r.out_len > 1])
        ok = [((r.first_token_ms - r.arrival_ms) / r.prompt <= s.ttft_norm_ms_per_tok and
               (r.out_len <= 1 or (r.finish_ms - r.first_token_ms) / (r.out_len - 1) <= s.tpot_ms))
              for r in done]
        pct = lambda a, q: float(np.percentile(a, q)) if len(a) else None  # noqa: E731
        dur_s = max(now, 1e-9) / 1000.0
        return {"policy": self.policy, "requests": len(trace), "finished": len(done), "sim_ms": now,
                "cycles": len(self.log), "slo_attainment": float(np.mean(ok)) if ok else 0.0,
                "goodput_req_s": sum(ok) / dur_s, "throughput_tok_s": sum(r.prompt + r.out_len for r in done) / dur_s,
                "ttft_ms_p50": pct(ttft, 50), "ttft_ms_p90": pct(ttft, 90),
                "norm_ttft_ms_per_tok_p90": pct(nttft, 90), "tpot_ms_p50": pct(tpot, 50),
                "tpot_ms_p90": pct(tpot, 90), "unservable": len(self.unservable), "slo": s.as_dict()}
