# ncu source-level view of the grouping kernel on the random-init proxy's C4b masks at the
# bench threshold (q = 0.7; every frame has > 64 components, so the work is in the second,
# full-slice launch: -s 1 -c 1), exported on the box
mkdir -p gpurun_out
WL=${WL:-C4b}
timeout 900 ncu -f --set full --import-source on --clock-control none -k regex:select_kernel -s ${SKIP:-1} -c 1 -o /tmp/sel \
  python scripts/e12_stage_time.py $WL 0 0.7 > gpurun_out/${TAG}_sel_prof.log 2>&1
ncu -i /tmp/sel.ncu-rep --page source --csv --print-source sass > gpurun_out/${TAG}_sel_source.csv 2>> gpurun_out/${TAG}_sel_prof.log
ncu -i /tmp/sel.ncu-rep --page details --csv > gpurun_out/${TAG}_sel_details.csv 2>> gpurun_out/${TAG}_sel_prof.log
ls -la gpurun_out/${TAG}_sel_* >> gpurun_out/${TAG}_sel_prof.log
