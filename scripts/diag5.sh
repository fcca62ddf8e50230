cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
O=gpurun_out/d5_attn.jsonl; : > $O
for cfg in arxiv-8b sharegpt-8b; do
python scripts/attn_dec_bench.py --config $cfg --kind 3 --tag old >> $O 2>&1
for dbg in 0 1 2; do for nw in 16 12; do
BULLET_DBG=$dbg BULLET_DEC2_WARPS=$nw python scripts/attn_dec_bench.py --config $cfg --kind 5 --tag "dbg$dbg-w$nw" >> $O 2>&1
done; done; done
