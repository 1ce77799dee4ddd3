# ncu --set full of resize / select / pack (scripts/prof_stages.py), exported on the box to
# CSV (the .ncu-rep itself is too large to bring back); summarise with scripts/ncu_stages.py
timeout 900 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "prof/" \
  -k regex:"resize_even|select_kernel|pack_kernel" -c 14 -o /tmp/r02_stages python scripts/prof_stages.py > gpurun_out/${TAG}_stages.log 2> gpurun_out/${TAG}_stages.err
grep '^{' gpurun_out/${TAG}_stages.log > gpurun_out/${TAG}_stages.json
ncu -i /tmp/r02_stages.ncu-rep --page raw --csv > gpurun_out/${TAG}_stages_raw.csv 2>> gpurun_out/${TAG}_stages.err
ncu -i /tmp/r02_stages.ncu-rep --page details --csv > gpurun_out/${TAG}_stages_details.csv 2>> gpurun_out/${TAG}_stages.err
