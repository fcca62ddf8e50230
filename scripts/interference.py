"""Where does the co-run slow the prefill phase?  Prefill layer of the bench
workload on sigma[0:p) timed (a) alone, (b) next to a pure HBM stream
(KI2 LDG kernel, no math) on the other SMs, (c) next to the real decode
phase (k layer-steps), (d) next to the decode phase with its attention in
stream-only mode is not available here (BULLET_DBG is process-wide).
Prints JSON lines (device ms of the prefill stream)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402


def main():
    p = int(sys.argv[1]) if len(sys.argv) > 1 else 80
    k = int(sys.argv[2]) if len(sys.argv) > 2 else 7
    torch.cuda.set_device(0)
    S = bench.Step("sharegpt-8b", k)
    B = S.B
    S.dec.layer_end = k
    buf = torch.empty(4 << 30, dtype=torch.uint8, device="cuda")
    side = torch.cuda.Stream()

    def prefill_ms(with_stream=False, with_decode=False, reps=10):
        out = []
        for _ in range(reps + 2):
            torch.cuda.synchronize()
            if with_stream:   # keep the other SMs streaming for longer than the prefill layer
                with torch.cuda.stream(side):
                    for _ in range(3):
                        S.bl.op_stream(buf, 0, p, S.N, stream=side)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(S.sp)
            S.bl.step(S.pre, S.dec if with_decode else None, p, B.CORUN, S.sp, S.sd)
            e1.record(S.sp)
            torch.cuda.synchronize()
            out.append(e0.elapsed_time(e1))
        out = sorted(out[2:])
        return out[len(out) // 2]

    for name, kw in (("alone", {}), ("hbm_stream_on_other_sms", {"with_stream": True}),
                     ("decode_on_other_sms", {"with_decode": True}), ("alone_again", {})):
        print(json.dumps({"p": p, "k": k, "prefill_next_to": name, "prefill_ms": round(prefill_ms(**kw), 4)}),
              flush=True)


if __name__ == "__main__":
    main()
