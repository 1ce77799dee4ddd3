# ncu captures of the proxy kernels (scripts/prof_conv.py: two C2 steps, the second one's
# E1+E2, E3, E4, E5, D1 launches), serial and with the fused pack riding in E5 / D1, plus
# the launch list of one serial step; CSV exported on the box (the .ncu-rep stay there)
for ov in 0 2; do
  timeout 900 ncu -f --set full --clock-control none --import-source on -k regex:"conv_umma|e12s?_umma" -s 5 -c 5 \
    -o /tmp/conv_ov$ov python scripts/prof_conv.py --overlap $ov > gpurun_out/${TAG}_conv_ov$ov.log 2>&1
  ncu -i /tmp/conv_ov$ov.ncu-rep --page raw --csv > gpurun_out/${TAG}_conv_ov${ov}_raw.csv 2>> gpurun_out/${TAG}_conv_ov$ov.log
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"resize|umma|select|compact|slot|pack|ws_" -c 400 --csv \
  --log-file gpurun_out/${TAG}_launches.csv python scripts/prof_conv.py --overlap 0 > /dev/null 2>&1
