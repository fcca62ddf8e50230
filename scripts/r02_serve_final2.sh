#!/bin/bash
# Serving comparison on the final round-2 kernels (NEXT-1): all policies at 120 and 240 req/s.
set -u
O=gpurun_out/serve_final2; mkdir -p $O
for rate in 60 180; do
  timeout 1500 python scripts/serve.py --rate $rate --duration 3 --policies bullet_gain bullet timesliced prefill_first chunked > $O/serve_rate$rate.jsonl 2> $O/serve_rate$rate.err
  echo "rate $rate rc=$?"
done
echo done
