# ncu source-level view of the fused E1+E2 kernel (per-SASS stall reasons), exported on the box
# KREGEX: kernel name regex (default e12_umma); SCRIPT: the driver (default scripts/e12_time.py)
KREGEX=${KREGEX:-e12_umma}
SCRIPT=${SCRIPT:-scripts/e12_time.py}
timeout 900 ncu -f --set full --import-source on --clock-control none -k regex:$KREGEX -c 1 -o /tmp/e12 \
  python $SCRIPT > gpurun_out/${TAG}_e12_prof.log 2>&1
ncu -i /tmp/e12.ncu-rep --page source --csv --print-source cuda > gpurun_out/${TAG}_e12_source_cuda.csv 2>> gpurun_out/${TAG}_e12_prof.log
ncu -i /tmp/e12.ncu-rep --page source --csv --print-source sass > gpurun_out/${TAG}_e12_source.csv 2>> gpurun_out/${TAG}_e12_prof.log
ncu -i /tmp/e12.ncu-rep --page details --csv > gpurun_out/${TAG}_e12_details.csv 2>> gpurun_out/${TAG}_e12_prof.log
ncu -i /tmp/e12.ncu-rep --page raw --csv > gpurun_out/${TAG}_e12_raw.csv 2>> gpurun_out/${TAG}_e12_prof.log
ls -la gpurun_out/${TAG}_e12_* >> gpurun_out/${TAG}_e12_prof.log
