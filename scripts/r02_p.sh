O=gpurun_out/r02; mkdir -p $O
( time timeout 1200 python bench.py > $O/p_bench3.json 2> $O/p_bench3.err ) 2> $O/p_bench3.time
timeout 900 python bench.py --config sharegpt-8b --no-cpu-baseline > $O/p_bench2.json 2> $O/p_bench2.err
( time timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > $O/p_ref3.json 2> $O/p_ref3.err ) 2> $O/p_ref3.time
echo done
