# compute-sanitizer over scripts/sanitize_run.py (C1-sized); logs under gpurun_out/ (summaries go to profiles/)
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 50 --error-exitcode 9 python scripts/sanitize_run.py \
    > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool exit=$?" >> gpurun_out/sanitize_summary.txt
done
