#!/bin/bash
# Round profiling (under gpurun): GPU tests, the bench line (all configurations), launch list of the bench command (cold,
# serialized), one full ncu capture of each hot kernel, ncu DRAM bytes merged vs layer-by-layer, compute-sanitizer.
# Usage: bash tools/profile_round.sh r02b
R=${1:-r02}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q 2>&1 | tail -3 | tee gpurun_out/${R}_pytest_gpu.txt
timeout 900 python bench.py > gpurun_out/${R}_bench.json 2> gpurun_out/${R}_bench.err; echo bench=$?
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv \
    --log-file gpurun_out/${R}_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-cudnn --no-extra > /dev/null 2>&1
echo launches=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:memo_pair -s 3 -c 1 \
    -o gpurun_out/${R}_memo_pair python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-cudnn --no-extra > /dev/null 2>&1
echo memo=$?
timeout 600 ncu --set full --clock-control none -k regex:brickify -s 2 -c 2 \
    -o gpurun_out/${R}_brickify python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-cudnn --no-extra > /dev/null 2>&1
echo brickify=$?
timeout 600 ncu --set full --clock-control none --import-source on -k gen_kernel -s 2 -c 1 \
    -o gpurun_out/${R}_gen_cfg5 python tools/run_subgraph.py cfg5 0 > /dev/null 2>&1
echo gen_cfg5=$?
timeout 600 ncu --set full --clock-control none -k gen_kernel -s 10 -c 1 \
    -o gpurun_out/${R}_gen_cfg4 python tools/run_subgraph.py cfg4 1 > /dev/null 2>&1
echo gen_cfg4=$?
for c in cfg3 cfg4 cfg5; do
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
      --log-file gpurun_out/${R}_launches_$c.csv python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline --no-cudnn > /dev/null 2>&1
  echo launches_$c=$?
done
for c in cfg2 cfg3 cfg4 cfg5; do   # merged-side DRAM bytes of one forward (the layer-by-layer side: tools/dram_bytes.py --impl lbl)
  timeout 600 ncu --nvtx --nvtx-include "fwd/" --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
      --csv --log-file gpurun_out/${R}_dram_${c}_merged.csv python tools/dram_bytes.py run --impl merged --config $c > /dev/null 2>&1
  echo dram_$c=$?
done
# (compute-sanitizer is closed on the GPU pool since round 2: the r02b-r02f sanitizer logs under profiles/ are the last)
