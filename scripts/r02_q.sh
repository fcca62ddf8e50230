O=gpurun_out/r02; mkdir -p $O
KEEP_REP="r02_c3_attn_dec_p84 r02_c2_down_dec_p84" bash scripts/capture_r02.sh 84 7 84 5 > $O/q_capture.log 2>&1
du -sh gpurun_out/ncu2 >> $O/q_capture.log
echo done
