cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q 2>&1 | tail -2
CASES='tests/test_gpu_gen.py -k "sw128_chain_grow or planes_3d or s2_1x1_proj or bottleneck_res"'
for tool in memcheck synccheck racecheck; do
  eval timeout 900 compute-sanitizer --tool $tool --print-limit 20 --target-processes all \
      python -m pytest $CASES -q -p no:cacheprovider > gpurun_out/r01c_sanitize_gen_$tool.log 2>&1
  echo "sanitize $tool rc=$?"; grep -E "ERROR SUMMARY|passed|failed|RACECHECK SUMMARY" gpurun_out/r01c_sanitize_gen_$tool.log | tail -3
done
timeout 300 python tools/memo_breakdown.py cfg1 cfg2 cfg5 2>&1 | tee gpurun_out/r01c_memo_breakdown.txt
timeout 900 python tools/sweep_fig10_11.py 2>&1 | tee gpurun_out/r01c_fig10_11.txt
