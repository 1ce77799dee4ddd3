# resize + proxy in mini-batches of proxy_batch frames inside the 4500-frame device batch (the
# activations of a mini-batch stay in L2 between layers) vs one pass: C2 step time with the
# fused pack (pack_overlap 2, q = 0.7), 25 steps per point after a warm-up
mkdir -p gpurun_out
LOG=gpurun_out/${TAG:-proxy_batch}_ab.log
for pb in 0 1500 900 450 225 0; do
  echo "[pb=$pb] $(timeout 300 python scripts/e12_stage_time.py C2 2 0.7 $pb 2>&1 | tail -1)" >> $LOG
done
