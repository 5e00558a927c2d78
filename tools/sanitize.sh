#!/bin/bash
# compute-sanitizer over small merged-execution cases (memcheck, racecheck, synccheck)
mkdir -p gpurun_out
CASES='tests/test_gpu_parity.py -k "cfg1_modes_vs_oracle and size0 or cfg2_tc_modes_vs_oracle and size0 or memo_counters"'
for tool in memcheck synccheck racecheck; do
  echo "== $tool"
  eval timeout 900 compute-sanitizer --tool $tool --print-limit 20 --target-processes all \
      python -m pytest $CASES -q -p no:cacheprovider > gpurun_out/sanitize_$tool.log 2>&1
  echo "rc=$?"; grep -E "ERROR SUMMARY|passed|failed|RACECHECK SUMMARY" gpurun_out/sanitize_$tool.log | tail -4
done
