"""Host logic of bench.py that the timing rules depend on (no GPU): the
clock / throttle summary the JSON line carries under "clocks"."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402


def test_clocks_summary_median_max_and_reason_union():
    c = bench.Clocks(0)
    c.nvml = object()   # rows as the NVML sampler records them
    c.rows = [(1965.0, 1965.0, set()), (1800.0, 1965.0, {"sw_power_cap"}), (1900.0, 1965.0, {"sw_power_cap"})]
    s = c.summary()
    assert s["sm_mhz"] == 1900.0 and s["sm_max_mhz"] == 1965.0
    assert s["reasons"] == ["sw_power_cap"] and s["samples"] == 3 and s["source"] == "nvml"


def test_clocks_summary_reports_rejecting_reasons():
    c = bench.Clocks(0)
    c.rows = [(1200.0, 1965.0, {"hw_thermal_slowdown"}), (1300.0, 1965.0, {"sw_thermal_slowdown", "hw_slowdown"})]
    assert c.summary()["reasons"] == ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"]


def test_clocks_unsampled_without_a_gpu():
    with bench.Clocks(0) as c:
        pass
    if not c.rows:   # no NVML / nvidia-smi here: the line says so instead of inventing clocks
        assert c.summary() == {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}


def test_default_config_follows_gpu_count():
    """--gpus N without --config: N = 1 runs BASELINE config 3 (the largest
    single-GPU config), 2 / 4 the Qwen2.5-14B TP configs, 8 Llama-70B TP8."""
    assert bench.DEFAULT_CONFIG == {1: "arxiv-8b", 2: "qwen14b-tp2", 4: "qwen14b-tp4", 8: "llama70b-tp8"}
    from workload import synth
    for n, name in bench.DEFAULT_CONFIG.items():
        assert synth.workload(name).tp == (n if n > 1 else 1)
        assert name in bench.SLO
    # Table 2: ShareGPT 3.0 ms / 150 ms, arXiv 1.5 ms / 175 ms
    assert bench.SLO["sharegpt-8b"]["ttft_norm_ms_per_tok"] == 3.0 and bench.SLO["sharegpt-8b"]["tpot_ms"] == 150.0
    assert bench.SLO["arxiv-8b"]["ttft_norm_ms_per_tok"] == 1.5 and bench.SLO["arxiv-8b"]["tpot_ms"] == 175.0


def _agree_rank(rank, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=2)
    try:
        t = bench.allreduce_max(1.0 + rank, 2)          # each rank's own "timing"
        d = bench.broadcast_obj((100 + rank, 7 + rank), 2)
        q.put((rank, t, d))
    finally:
        dist.destroy_process_group()


def test_rank_agreement_helpers_gloo():
    """Multi-rank bench: timings are max-reduced and the split is rank 0's on
    every rank, so all ranks take the same (p, k) decisions and enqueue the
    same step sequence (TP collectives pair up)."""
    import socket
    import torch.multiprocessing as mp
    s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_agree_rank, args=(r, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = sorted(q.get(timeout=120) for _ in ps)
    for p in ps:
        p.join(timeout=60)
    assert [o[1] for o in out] == [2.0, 2.0]
    assert [o[2] for o in out] == [(100, 7), (100, 7)]
