O=gpurun_out/r02; mkdir -p $O
bash scripts/capture_r02.sh 84 7 84 5 > $O/q_capture.log 2>&1
for rate in 120 240; do
  timeout 900 python scripts/serve.py --rate $rate --duration 3 --policies bullet_gain bullet timesliced prefill_first chunked --log-cycles $O/q_serve_cycles_$rate > $O/q_serve_rate$rate.jsonl 2> $O/q_serve_rate$rate.err
done
echo done
