O=gpurun_out/r02; mkdir -p $O
for rate in 120 240; do
  timeout 1200 python scripts/serve.py --rate $rate --duration 3 --policies bullet_gain bullet timesliced prefill_first chunked > $O/s_serve_rate$rate.jsonl 2> $O/s_serve_rate$rate.err
done
echo done
