# R-4e precision sweep through the product path (step), full layer dims.
O=gpurun_out/r02; mkdir -p $O
run() { env "$@" timeout 900 python scripts/precision_layer.py llama3.1-70b qwen2.5-14b llama3.1-8b >> $O/prec.jsonl 2>>$O/prec.err; }
: > $O/prec.jsonl
run BULLET_GEMM_KCHUNK=0
run BULLET_GEMM_KCHUNK=512 BULLET_GEMM_KCHUNK_ONLY=attn
run BULLET_GEMM_KCHUNK=256 BULLET_GEMM_KCHUNK_ONLY=attn
run BULLET_GEMM_KCHUNK=128 BULLET_GEMM_KCHUNK_ONLY=attn
run BULLET_GEMM_KCHUNK=256 BULLET_GEMM_KCHUNK_ONLY=all
run BULLET_GEMM_KCHUNK=128 BULLET_GEMM_KCHUNK_ONLY=all
run BULLET_GEMM_KCHUNK=128 BULLET_GEMM_KCHUNK_ONLY=qkv
run BULLET_GEMM_KCHUNK=128 BULLET_GEMM_KCHUNK_ONLY=qkv,oproj,gate_up
# prefill-sized M (row-sampled oracle): default policy
timeout 900 python scripts/precision_layer.py qwen2.5-14b llama3.1-70b --pre 1024,512 --dec 2000,17 --sample 192 >> $O/prec.jsonl 2>>$O/prec.err
echo done
