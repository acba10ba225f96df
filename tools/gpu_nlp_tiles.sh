# NLP / DIG / ASR dense-GEMM tile experiments: per-op times with the default tiles, BN capped at
# 128 / 64, and without CTA pairs.
mkdir -p gpurun_out
{
for cfg in "x:x" "128:1" "64:1" "x:0" "128:0" "64:0"; do
  bn=${cfg%%:*}; cp=${cfg##*:}
  for a in pos ner dig asr; do
    env $( [ $bn != x ] && echo DJINN_DENSE_BN=$bn ) $( [ $cp == 0 ] && echo DJINN_CTA_PAIR=0 ) TAG=bn$bn/cp$cp \
      timeout 300 python tools/op_times.py $a bf16 2>&1 | grep -E "gemm|total"
  done
done
} > gpurun_out/nlp_tiles.txt 2>&1
